#!/bin/bash
# DRAM traffic of the bench's own histogram launches (roofline.traffic):
# ncu --set full on the first timed tree's D launches of `python bench.py` (warm-up W trees skipped),
# then tools/traffic_collect.py turns it into bytes per built row per level (profiles/hist_traffic.json).
#   gpurun -- 'bash tools/traffic_capture.sh r02 C5 5'
tag=${1:-r02}; wl=${2:-C5}; W=${3:-5}; D=${4:-8}
out=gpurun_out; mkdir -p $out
skip=$((W * D))
timeout 1800 ncu --set full --clock-control none -k regex:k_hist_smem -s $skip -c $D -o /tmp/${tag}_traffic_${wl} \
  python bench.py --workload $wl --steps 1 --warmup $W --no-e2e --no-cpu-baseline > $out/${tag}_traffic_${wl}_bench.log 2>&1
ncu -i /tmp/${tag}_traffic_${wl}.ncu-rep --page raw --csv > $out/${tag}_traffic_${wl}_raw.csv 2>/dev/null
python tools/ncu_summary.py /tmp/${tag}_traffic_${wl}.ncu-rep --sass 20 > $out/${tag}_ncu_hist_${wl}_timed.txt 2>&1
