#!/bin/bash
# usage: tools/sweep.sh "C2:4 C2:8 C4-32:4" -- runs bench per config:team, prints a compact line
for ct in $1; do
  c=${ct%%:*}; rest=${ct#*:}; t=${rest%%:*}; n=${rest#*:}; [ "$n" = "$rest" ] && n=0
  timeout 600 python bench.py --config $c --team $t --chunk $n --no-e2e --no-ubench --no-cpu-baseline $EXTRA > /tmp/b.json 2>&1
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], 'N', d['config']['chunk_entries'], 'team', d['config']['contains_team'], 'Mops', d['value'], d['phase_ms_per_step'], 'frac', d['roofline']['frac'], 'gathers', d['search_gathers']['chunk_gathers_per_op'], d['search_gathers']['gather_GBps'])" || tail -5 /tmp/b.json
done
