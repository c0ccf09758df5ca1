#!/bin/bash
# Per-kernel launch list (cold, serialised: shares only) of a few trees of a workload:
#   tools/launch_list.sh C2 [trees] -> gpurun_out/launches_<wl>.csv + summary
wl=$1; trees=${2:-3}
out=gpurun_out; mkdir -p $out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_$wl.csv \
   python tools/prof_run.py $wl $trees > $out/launches_$wl.log 2>&1
python tools/launch_summary.py $out/launches_$wl.csv > $out/launches_${wl}_summary.txt 2>&1
