#!/bin/bash
# the -m gpu suite, then e2e with the Insert values zero-copy vs copied
set -u
O=${O:-gpurun_out/zc}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "suite rc=$?" >> $O/rc.txt
for c in C5 C3 C2 C4-16; do
  for zc in 1 0; do
    GFSL_ZC_VALUES=$zc timeout 900 python bench.py --config $c --runs 2 --no-cpu-baseline --no-ubench > $O/tmp.json 2>>$O/err
    tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['e2e']; print('$c', 'zc=$zc', d['value'], 'e2e', e['value'], e['h2d_bytes_per_step'], e.get('values'), e['runs_mops'])" >> $O/ab.txt
  done
done
