#!/bin/bash
# the small-batch kernel (GFSL_SMALL_BATCH ops threshold) vs the two-kernel path on C2-size batches
set -u
O=${O:-gpurun_out/smallth}; mkdir -p $O
for c in C2 C2-2020 C2-5050 M1-1-98 C1; do
  for rep in 1 2; do
    for th in 0 1000000; do
      GFSL_SMALL_BATCH=$th timeout 600 python bench.py --config $c --runs 2 --no-cpu-baseline --no-e2e --no-ubench > $O/tmp.json 2>>$O/err
      tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', 'small=$th', d['value'], d['phase_ms_per_step'])" >> $O/ab.txt
    done
  done
done
