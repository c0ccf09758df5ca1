#!/bin/bash
# Refresh of the bench lines whose kernels / table entries changed after tools/final_r02c.sh
# (work items per level; C2's small-node search): writes gpurun_out/r02c_bench_<wl>.log
out=gpurun_out; mkdir -p $out
for wl in C1 C2 C3 S5 S10 S50 S100; do
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > $out/r02c_bench_$wl.log 2>&1
done
timeout 600 python bench.py --workload C1 --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --graph > $out/r02c_bench_C1_graph.log 2>&1
for f in $out/r02c_bench_*.log; do echo "$f: $(grep '^{' $f | tail -1 | cut -c1-120)"; done
