# A/B: cached root counts vs accumulated every tree (bench --no-root-cache), same build
mkdir -p gpurun_out
rm -f gpurun_out/abc_all.jsonl
for rep in 1 2; do
for mode in nocache cache; do
  F=""; [ $mode = nocache ] && F="--no-root-cache"
  for wl in C5 C3 C4 C2; do
    st=10; [ $wl = C5 ] && st=5
    timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 $F > gpurun_out/abc_${wl}_$mode.log 2>&1
    (echo -n "$mode "; tail -1 gpurun_out/abc_${wl}_$mode.log) >> gpurun_out/abc_all.jsonl
  done
done
done
