# A/B: split-search L2 prefetch distance (channels ahead) with the half-row kernel
mkdir -p gpurun_out
rm -f gpurun_out/abf_all.jsonl
for wl in C5 C4 S100; do
for lib in def pf0 pf4 pf8; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  st=10; [ $wl = C5 ] && st=4
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abf_${wl}_$lib.log 2>&1
  (echo -n "$lib "; tail -1 gpurun_out/abf_${wl}_$lib.log) >> gpurun_out/abf_all.jsonl
done
done
