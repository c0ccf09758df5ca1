# A/B of the histogram kernel's block size / q-prefetch depth (register pressure, spills)
mkdir -p gpurun_out
rm -f gpurun_out/abs_all.jsonl
for wl in C5 C3 C4 C2; do
for lib in t1024sb2 t768sb2 t768sb4 t640sb4; do
  L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"
  st=10; [ $wl = C5 ] && st=5
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abs_${wl}_$lib.log 2>&1
  (echo -n "$lib "; tail -1 gpurun_out/abs_${wl}_$lib.log) >> gpurun_out/abs_all.jsonl
done
done
