#!/bin/bash
# Round-2 measurement pass (one gpurun call): every bench config (10 runs + CI, e2e, CPU
# oracle baseline), then the NEXT-4 sweep of tools/sweep_r2.py (key ranges 10K-100M x the
# paper's mixes, Contains-only, Insert-only from empty, Delete-only from full).
set -u
O=${O:-gpurun_out/final_r2}; mkdir -p $O
for c in ${CFGS:-C5 C5-S8 C5-S4 C5-S2 C2 C1 C2-100 C2-2020 C2-5050 C3 C3-zipf C3-zipf-raw C2-zipf-raw C4-16 C4-32 M1-1-98 M5-5-90 M20-20-60-10M INS-1M DEL-1M}; do
  timeout 1200 python bench.py --config $c ${BENCH_ARGS:-} >> $O/bench_all.jsonl 2>> $O/bench_all.err
  echo "$c rc=$?" >> $O/rc.txt
done
if [ -z "${NO_SWEEP:-}" ]; then
  timeout 3600 python tools/sweep_r2.py $O/sweep.jsonl --runs ${SWEEP_RUNS:-3} > $O/sweep.log 2>&1
  echo "sweep rc=$?" >> $O/rc.txt
fi
