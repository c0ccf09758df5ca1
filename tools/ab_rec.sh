# A/B: multi-block split records + separate gain kernel (current) vs previous build (build/ab/head)
mkdir -p gpurun_out
rm -f gpurun_out/abr_all.jsonl
for lib in head def; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  for wl in C2 S100 S500 C4; do
    env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/abr_${wl}_$lib.log 2>&1
    (echo -n "$lib "; tail -1 gpurun_out/abr_${wl}_$lib.log) >> gpurun_out/abr_all.jsonl
  done
done
