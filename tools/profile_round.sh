#!/bin/bash
# One GPU call's profiling pass (run under gpurun from the repo root):
#  1. the launch list of the default bench command (ncu, gpu__time_duration only)
#  2. one `--set full` capture of one mid-run batch per config (tools/prof_step.py), with
#     --cache-control all: L2 is flushed before every replay pass, as bench.py flushes it
#     before every timed step
#  3. compute-sanitizer memcheck / synccheck on a small run (tools/sanitize_run.py)
# Outputs land in $O; tools/ncu_metrics.py summaries are written beside the reports.
set -u
O=${O:-gpurun_out/prof}; mkdir -p $O
CFGS=${CFGS:-"C2 C4-16"}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $O/launches_c2.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e \
  > $O/launches_c2_bench.log 2>&1
for c in $CFGS; do
  timeout 1200 ncu --profile-from-start off --set full --clock-control none --cache-control all \
    --import-source on -f -o $O/prof_$c python tools/prof_step.py $c > $O/prof_$c.log 2>&1
  python tools/ncu_metrics.py $O/prof_$c.ncu-rep > $O/ncu_$c.json 2>&1
done
timeout 600 compute-sanitizer --tool memcheck python tools/sanitize_run.py > $O/sanitizer_memcheck.log 2>&1
timeout 600 compute-sanitizer --tool synccheck python tools/sanitize_run.py > $O/sanitizer_synccheck.log 2>&1
