# per-item overhead probe: smaller maximum work items (rows per item) on C5
mkdir -p gpurun_out
rm -f gpurun_out/abq_all.jsonl
for lib in def c32k c16k; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  env $L timeout 400 python bench.py --workload C5 --no-e2e --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/abq_$lib.log 2>&1
  (echo -n "$lib "; tail -1 gpurun_out/abq_$lib.log) >> gpurun_out/abq_all.jsonl
done
