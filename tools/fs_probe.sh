out=gpurun_out
for wl in C4 C3 S500; do for cg in 0 1; do
  FS_CG=$cg timeout 600 ncu --metrics gpu__time_duration.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none --csv -k regex:k_find_split python tools/prof_run.py $wl 2 > $out/fsprobe_${wl}_$cg.csv 2>&1
done; done
