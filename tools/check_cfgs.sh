#!/bin/bash
# the -m gpu suite + smoke, then bench lines of CFGS (RUNS runs each)
set -u
O=${O:-gpurun_out/check}; mkdir -p $O
if [ -z "${NO_SUITE:-}" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/rc.txt
fi
for c in ${CFGS:-C1 C2 C2-5050 C3 C5}; do
  timeout 900 python bench.py --config $c --runs ${RUNS:-3} --no-cpu-baseline --no-e2e --no-ubench > $O/tmp.json 2>>$O/bench.err
  tail -1 $O/tmp.json >> $O/bench.jsonl
  tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], d['value'], d['phase_ms_per_step'])" >> $O/summary.txt
done
