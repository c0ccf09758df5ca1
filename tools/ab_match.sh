# A/B: count atomics combined across lanes with MATCH.ANY (build/ab/match) vs default
mkdir -p gpurun_out
rm -f gpurun_out/abm_all.jsonl
for rep in 1 2; do
for lib in def match; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  for wl in C5 C3; do
    st=10; [ $wl = C5 ] && st=5
    env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/abm_${wl}_$lib.log 2>&1
    (echo -n "$lib "; tail -1 gpurun_out/abm_${wl}_$lib.log) >> gpurun_out/abm_all.jsonl
  done
done
done
