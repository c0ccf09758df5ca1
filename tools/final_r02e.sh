#!/bin/bash
# Final bench lines of round 2 (all configs at the final code): gpurun_out/r02c_bench_*.log
out=gpurun_out; mkdir -p $out
timeout 900 python bench.py > $out/r02c_bench_c5_n1.log 2>&1
for wl in C1 C2 C3 C4 S5 S10 S50 S100 S500 S983; do
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > $out/r02c_bench_$wl.log 2>&1
done
timeout 600 python bench.py --workload C1 --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --graph > $out/r02c_bench_C1_graph.log 2>&1
timeout 900 python bench.py --predict --steps 5 --warmup 2 > $out/r02c_bench_predict_c5.log 2>&1
timeout 1200 python bench.py --impl reference > $out/r02c_bench_reference.log 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/r02c_launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
    > $out/r02c_ncu_launches.log 2>&1
for f in $out/r02c_bench_*.log; do echo "$f: $(grep '^{' $f | tail -1 | cut -c1-120)"; done
