#!/bin/bash
# A/B ncu of the histogram kernel on C5 (root launch + one deep launch) for library variants:
#   bash tools/ab_ncu.sh <tag> "<variant>=<command>" ...   (under gpurun; CSV summaries only)
tag=$1; shift
o=gpurun_out
for spec in "$@"; do
  v=${spec%%=*}; cmd=${spec#*=}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_hist_smem -s ${SKIP:-0} -c 1 \
      -o /tmp/${tag}_$v $cmd > $o/${tag}_$v.log 2>&1
  ncu -i /tmp/${tag}_$v.ncu-rep --page raw --csv > $o/${tag}_${v}_raw.csv 2>/dev/null
  ncu -i /tmp/${tag}_$v.ncu-rep --page source --csv --print-source sass > $o/${tag}_${v}_src.csv 2>/dev/null
done
