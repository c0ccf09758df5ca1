# device time per tree, eager (host enqueues every launch) vs one CUDA graph per tree, same box
mkdir -p gpurun_out
for wl in C1 C2 C3 C4 S10; do
  for rep in 1 2; do
    timeout 300 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/gve_${wl}_eager_$rep.log 2>&1
    timeout 300 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --graph > gpurun_out/gve_${wl}_graph_$rep.log 2>&1
  done
done
