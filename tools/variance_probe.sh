# run-to-run variance of the device time per tree (fresh process each), per phase
mkdir -p gpurun_out
for rep in 1 2 3 4 5; do
  timeout 300 python bench.py --workload C3 --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/var_C3_$rep.log 2>&1
done
for rep in 1 2 3; do
  timeout 300 python bench.py --workload C4 --no-e2e --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/var_C4_$rep.log 2>&1
done
