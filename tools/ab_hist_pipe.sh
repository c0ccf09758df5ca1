# A/B of the histogram kernel's prefetch depth on C5 (per-level times and rows per level)
mkdir -p gpurun_out
rm -f gpurun_out/abw_all.jsonl
for rep in 1 2; do
for lib in def wd2 sb16; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  env $L timeout 400 python bench.py --workload C5 --no-e2e --no-cpu-baseline --steps 4 --warmup 3 > gpurun_out/abw_$lib.log 2>&1
  (echo -n "$lib "; tail -1 gpurun_out/abw_$lib.log) >> gpurun_out/abw_all.jsonl
done
done
