#!/bin/bash
# the -m gpu suite, C1/C2 per-batch times, the update-kernel timeline (debug build), a few bench lines
set -u
O=${O:-gpurun_out/state2}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/rc.txt
for c in C1 C2; do timeout 300 python tools/batch_times.py $c --steps 8 >> $O/bt.txt 2>&1; done
for c in C1 C2 C2-5050 C3; do GFSL_LIB=variants/libgfsl_dbg.so timeout 300 python tools/upd_timeline.py $c >> $O/timeline.txt 2>&1; done
for c in C1 C2 C2-5050 C3 INS-1M DEL-1M; do
  timeout 600 python bench.py --config $c --runs 3 --no-cpu-baseline --no-e2e >> $O/bench.jsonl 2>> $O/bench.err
done
