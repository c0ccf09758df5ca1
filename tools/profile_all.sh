#!/bin/bash
# Everything profiles/ is regenerated from (run under gpurun on one B200):
#   gpurun --timeout 3000 -- 'bash tools/profile_all.sh r01'
# Writes gpurun_out/<tag>_*; copy the summaries into profiles/ afterwards (tools/profile_collect.py).
set -x
tag=${1:-r01}
out=gpurun_out
mkdir -p $out
# 1. the bench line (default command) and every config / sweep as parity-size bench lines
timeout 900 python bench.py > $out/${tag}_bench_c5_n1.log 2>&1
for wl in C1 C2 C3 C4 S5 S10 S50 S100 S500; do
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 5 --warmup 3 > $out/${tag}_bench_$wl.log 2>&1
done
# 2. launch list of the bench command (per-launch device time; cold, serialised: shares only)
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/${tag}_launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
    > $out/${tag}_ncu_launches.log 2>&1
# 3. full ncu sets: one tree of histogram launches, and find_split launches (C5)
#    (reports stay in /tmp on the box: gpurun copies back <= 64 MiB; summaries + raw CSV come back)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_hist_smem -s 0 -c 8 \
    -o /tmp/${tag}_prof_hist_c5 python tools/prof_run.py C5 1 > $out/${tag}_ncu_hist.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_find_split -s 3 -c 3 \
    -o /tmp/${tag}_prof_fs_c5 python tools/prof_run.py C5 1 > $out/${tag}_ncu_fs.log 2>&1
for name in hist fs; do
  python tools/ncu_summary.py /tmp/${tag}_prof_${name}_c5.ncu-rep --sass 30 > $out/${tag}_ncu_${name}_c5.txt 2>&1
  ncu -i /tmp/${tag}_prof_${name}_c5.ncu-rep --page raw --csv > $out/${tag}_prof_${name}_c5_raw.csv 2>/dev/null
done
# 4. binning (once per dataset): warm timing and its launch list on C5
timeout 300 python tools/bin_probe.py C5 > $out/${tag}_bin_probe_c5.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/${tag}_launches_bin_c5.csv python tools/bin_probe.py C5 > $out/${tag}_ncu_bin.log 2>&1
# 5. micro-benchmarks of the on-chip accumulation pipes
./tools/microbench/atom_bench > $out/${tag}_atom_bench.txt 2>&1 || true
