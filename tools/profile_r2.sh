#!/bin/bash
# Round-2 profiling pass (run under gpurun from the repo root; one GPU):
#  1. launch list (gpu__time_duration only, one pass, no replay) of the default bench (C5)
#  2. DRAM / L2 traffic of one mid-run batch per config: application replay (ncu reruns the
#     whole program per pass, so no 70-GB save/restore of the pool between passes),
#     --cache-control all (cold L2 per pass, as bench.py flushes L2 before each timed step)
#  3. one `--set full` capture of the C5 search and update kernels (application replay)
# The .ncu-rep reports stay on the box ($R, they exceed gpurun's 64-MiB copy-back); the
# summaries (tools/ncu_metrics.py JSON, raw/details/source CSV pages) go to $O.
set -u
O=${O:-gpurun_out/prof_r2}; mkdir -p $O
R=${R:-/tmp/prof_reps}; mkdir -p $R
CFGS=${CFGS:-"C5 C4-16 C3 C2"}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,lts__t_requests_srcunit_tex.sum,dram__sectors_read.sum
if [ -z "${NO_LAUNCHES:-}" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $O/launches_C5.csv python bench.py --runs 1 --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-ubench \
    > $O/launches_C5_bench.log 2>&1
  python tools/launch_summary.py $O/launches_C5.csv > $O/launch_summary_C5.txt 2>&1
fi
for c in $CFGS; do
  timeout 1200 ncu --replay-mode application --profile-from-start off --metrics $M --clock-control none \
    --cache-control all -f -o $R/traffic_$c python tools/prof_step.py $c > $O/traffic_$c.log 2>&1
  python tools/ncu_metrics.py $R/traffic_$c.ncu-rep > $O/ncu_$c.json 2>&1
done
if [ -z "${NO_FULL:-}" ]; then
  timeout 2400 ncu --replay-mode application --profile-from-start off --set full --import-source on \
    --clock-control none --cache-control all -k "regex:search_kernel|update_kernel" -f -o $R/full_C5 \
    python tools/prof_step.py C5 > $O/full_C5.log 2>&1
  python tools/ncu_metrics.py $R/full_C5.ncu-rep > $O/ncu_full_C5.json 2>&1
  ncu -i $R/full_C5.ncu-rep --page details --csv > $O/full_C5_details.csv 2>&1
  ncu -i $R/full_C5.ncu-rep --page raw --csv > $O/full_C5_raw.csv 2>&1
  ncu -i $R/full_C5.ncu-rep --page source --csv -k regex:update_kernel > $O/full_C5_update_source.csv 2>&1
  ncu -i $R/full_C5.ncu-rep --page source --csv -k regex:search_kernel > $O/full_C5_search_source.csv 2>&1
  ls -la $R > $O/reports_ls.txt
fi
du -sh $O
