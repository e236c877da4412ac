#!/bin/bash
# Round-2 diagnostics in one gpurun call: the -m gpu suite, then per-batch phase times
# (tools/batch_times.py, warm process) of the update-heavy configs.
set -u
O=${O:-gpurun_out/diag2}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
for c in ${CFGS:-INS-1M DEL-1M C1}; do for g in ${GROUPS_:-off on}; do
  timeout 300 python tools/batch_times.py $c --group $g --steps 8 >> $O/bt.txt 2>&1
done; done
for c in ${BENCH:-INS-1M DEL-1M C1 C2-5050}; do
  timeout 600 python bench.py --config $c --runs 3 --no-cpu-baseline --no-e2e >> $O/bench.jsonl 2>> $O/bench.err
done
