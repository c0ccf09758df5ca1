#!/bin/bash
# ncu evidence for the lower-fraction configs and the bench launch list:
#   gpurun -- 'bash tools/profile_r02.sh r02'
tag=${1:-r02}
out=gpurun_out; mkdir -p $out
for wl in C2 C3 C4; do
  D=$(python -c "from gen import gen; print(gen.WORKLOADS['$wl'].D)")
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_hist_(smem|diag)' -s $D -c $D \
     -o /tmp/${tag}_hist_$wl python tools/prof_run.py $wl 2 > $out/${tag}_ncu_hist_${wl}.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_find_split -s $D -c $D \
     -o /tmp/${tag}_fs_$wl python tools/prof_run.py $wl 2 > $out/${tag}_ncu_fs_${wl}.log 2>&1
  for k in hist fs; do
    python tools/ncu_summary.py /tmp/${tag}_${k}_$wl.ncu-rep --sass 20 > $out/${tag}_ncu_${k}_${wl}.txt 2>&1
  done
done
# launch list of the default bench command (cold, serialised per-launch times: shares only)
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/${tag}_launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
    > $out/${tag}_ncu_launches.log 2>&1
ls -la $out/${tag}_ncu_* | head -20
# the sort-and-segment small-node search on C2 forced to 768-row pairs (vs the histogram path)
SMALL_MAX_ROWS=768 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sort_search -s 13 -c 3 \
   -o /tmp/${tag}_small_C2 python tools/prof_run.py C2 2 > $out/${tag}_ncu_small_C2.log 2>&1
python tools/ncu_summary.py /tmp/${tag}_small_C2.ncu-rep --sass 25 > $out/${tag}_ncu_small_C2.txt 2>&1
