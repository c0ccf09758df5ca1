# A/B: compacted deep levels (default) vs gathered (--no-compact), same build
mkdir -p gpurun_out
rm -f gpurun_out/abk_all.jsonl
for rep in 1 2; do
for mode in gather compact; do
  F=""; [ $mode = gather ] && F="--no-compact"
  for wl in C5 C3 C4; do
    st=10; [ $wl = C5 ] && st=5
    timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 $F > gpurun_out/abk_${wl}_$mode.log 2>&1
    (echo -n "$mode "; tail -1 gpurun_out/abk_${wl}_$mode.log) >> gpurun_out/abk_all.jsonl
  done
done
done
