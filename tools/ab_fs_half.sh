# A/B: half-row split search (current build, min 3 blocks/SM) vs the 8-bin kernel (half0) and
# other residency targets; phase times from the bench JSON
mkdir -p gpurun_out
rm -f gpurun_out/abh_all.jsonl
for lib in half0 def hminb2 hminb4; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  for wl in C2 S100 C4 C5; do
    st=10; [ $wl = C5 ] && st=4
    env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abh_${wl}_$lib.log 2>&1
    (echo -n "$lib "; tail -1 gpurun_out/abh_${wl}_$lib.log) >> gpurun_out/abh_all.jsonl
  done
done
