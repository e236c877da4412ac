#!/bin/bash
# R40 check + A/B in one gpurun call: the grouped-update tests, the -m gpu suite, then
# bench lines with grouping on / off on the update-heavy configs and the default.
set -u
O=${O:-gpurun_out/group}; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_group.py -x -q > $O/pytest_group.log 2>&1; echo "group tests rc=$?" >> $O/rc.txt
if [ -z "${NO_SUITE:-}" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
fi
for c in ${CFGS:-INS-1M DEL-1M C1 C2-5050 C2 C3}; do
  for g in on off; do
    timeout 600 python bench.py --config $c --runs ${RUNS:-3} --no-cpu-baseline --no-e2e --group $g >> $O/bench_ab.jsonl 2>> $O/bench_ab.err
  done
done
if [ -n "${C5:-}" ]; then
  for g in on off; do
    timeout 900 python bench.py --config C5 --runs 2 --no-cpu-baseline --no-e2e --group $g >> $O/bench_ab.jsonl 2>> $O/bench_ab.err
  done
fi
