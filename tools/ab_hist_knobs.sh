# A/B of histogram-kernel knobs after the spill fix (C5, C4)
mkdir -p gpurun_out
rm -f gpurun_out/abn_all.jsonl
for wl in C5 C4; do
for lib in def lcnt shfl pg8 pg2 sb1; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  st=10; [ $wl = C5 ] && st=5
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abn_${wl}_$lib.log 2>&1
  (echo -n "$lib "; tail -1 gpurun_out/abn_${wl}_$lib.log) >> gpurun_out/abn_all.jsonl
done
done
