#!/bin/bash
# the default bench line at HEAD (as the driver runs it), C2 / C3 / C4-16 / C5-S8 lines, then
# the launch list and per-config traffic (no full capture)
set -u
O=${O:-gpurun_out/final_head}; mkdir -p $O
timeout 900 python bench.py > $O/bench_default.jsonl 2> $O/bench_default.err; echo "default rc=$?" >> $O/rc.txt
for c in C2 C3 C4-16 C5-S8; do
  timeout 900 python bench.py --config $c >> $O/bench_cfgs.jsonl 2>> $O/bench_cfgs.err
done
NO_FULL=1 O=$O/prof bash tools/profile_r2.sh
