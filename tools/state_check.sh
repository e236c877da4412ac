#!/bin/bash
# One gpurun call: -m gpu tests, smoke, default bench (C5) and the small configs.
set -u
O=${O:-gpurun_out/state}; mkdir -p $O
nvidia-smi > $O/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/rc.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/rc.txt
timeout 900 python bench.py > $O/bench_default.jsonl 2> $O/bench_default.err; echo "bench rc=$?" >> $O/rc.txt
for c in ${CFGS:-C1 C2 C2-5050 INS-1M DEL-1M C3}; do
  timeout 600 python bench.py --config $c --runs 3 --no-cpu-baseline >> $O/bench_cfgs.jsonl 2>> $O/bench_cfgs.err
done
