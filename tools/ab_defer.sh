#!/bin/bash
# A/B of the deferred unlock (default build vs -DGFSL_NO_DEFER_UNLOCK) in one call, + suite
set -u
O=${O:-gpurun_out/abdefer}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
for c in ${CFGS:-C1 C2 C2-5050 C3 INS-1M}; do
  for v in default nodefer default nodefer; do
    if [ $v = default ]; then L=""; else L=variants/libgfsl_$v.so; fi
    GFSL_LIB=$L timeout 600 python bench.py --config $c --runs 3 --no-cpu-baseline --no-e2e --no-ubench > $O/tmp.json 2>>$O/bench.err
    tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', '$v', d['value'], d['phase_ms_per_step'])" >> $O/ab.txt
  done
done
for c in C2 C3; do GFSL_LIB=variants/libgfsl_dbg.so timeout 300 python tools/upd_timeline.py $c >> $O/timeline.txt 2>&1; done
if [ -n "${C5:-}" ]; then
  for v in default nodefer; do
    if [ $v = default ]; then L=""; else L=variants/libgfsl_$v.so; fi
    GFSL_LIB=$L timeout 900 python bench.py --config C5 --runs 2 --no-cpu-baseline --no-e2e --no-ubench > $O/tmp.json 2>>$O/bench.err
    tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C5', '$v', d['value'], d['phase_ms_per_step'])" >> $O/ab.txt
  done
fi
