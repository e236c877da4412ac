#!/bin/bash
set -u
O=${O:-gpurun_out/zc2}; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_small.py tests/test_gpu_bench.py -x -q > $O/pytest.log 2>&1; echo "tests rc=$?" >> $O/rc.txt
for c in C4-16 C2-100 C5; do
  timeout 900 python bench.py --config $c --runs 2 --no-cpu-baseline --no-ubench > $O/tmp.json 2>>$O/err
  tail -1 $O/tmp.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['e2e']; print('$c', d['value'], 'e2e', e['value'], e['h2d_bytes_per_step'], e.get('values'))" >> $O/ab.txt
done
