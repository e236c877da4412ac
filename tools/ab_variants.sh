#!/bin/bash
# A/B of library variants (variants/libgfsl_<v>.so, tools/build_variant.py) against the
# default build, interleaved, in one gpurun call.  VARIANTS="nopf ub6" CFGS="C2 C3"
set -u
O=${O:-gpurun_out/abv}; mkdir -p $O
if [ -z "${NO_SUITE:-}" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
fi
for c in ${CFGS:-C2 C3}; do
  for rep in 1 2; do
    for v in default ${VARIANTS:-}; do
      if [ $v = default ]; then L=""; else L=variants/libgfsl_$v.so; fi
      GFSL_LIB=$L timeout 900 python bench.py --config $c --runs ${RUNS:-3} --no-cpu-baseline --no-e2e --no-ubench > $O/tmp.json 2>>$O/bench.err
      tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', '$v', d['value'], d['phase_ms_per_step'])" >> $O/ab.txt
    done
  done
done
