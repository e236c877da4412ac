#!/bin/bash
# the -m gpu suite; small-batch kernel on/off and the L2 min-key prefetch variant, A/B in one call
set -u
O=${O:-gpurun_out/small}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
run() {  # label env... -- bench args
  local label=$1; shift
  env "$@" timeout 900 python bench.py --no-cpu-baseline --no-e2e --no-ubench --runs ${RUNS:-3} $BARGS > $O/tmp.json 2>>$O/bench.err
  tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$label', d['config']['workload'], d['value'], d['phase_ms_per_step'])" >> $O/ab.txt
}
for c in C1 "custom --custom 10000:0:1250:8:100,0,0:perm:16" "custom --custom 100000:50000:12500:80:20,20,60:uniform:16" C2-5050; do
  for rep in 1 2; do
    BARGS="--config $c"; run small_on GFSL_SMALL_BATCH=16384
    BARGS="--config $c"; run small_off GFSL_SMALL_BATCH=0
  done
done
BARGS="--config C2-5050"; run small_128k GFSL_SMALL_BATCH=131072
BARGS="--config C2-5050"; run small_off GFSL_SMALL_BATCH=0
for c in C5 C4-16 C3 C2; do
  for rep in 1 2; do
    BARGS="--config $c"; run default GFSL_LIB=
    BARGS="--config $c"; run pfl2 GFSL_LIB=variants/libgfsl_pfl2.so
  done
done
