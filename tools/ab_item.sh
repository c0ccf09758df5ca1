# A/B: next-item prefetch before the flush + prologue loads before zeroing (current) vs previous
mkdir -p gpurun_out
rm -f gpurun_out/abi_all.jsonl
for rep in 1 2; do
for lib in head def; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  for wl in C5 C3; do
    st=10; [ $wl = C5 ] && st=5
    env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abi_${wl}_$lib.log 2>&1
    (echo -n "$lib "; tail -1 gpurun_out/abi_${wl}_$lib.log) >> gpurun_out/abi_all.jsonl
  done
done
done
