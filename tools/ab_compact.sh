# A/B: compaction of gathered levels from level L (bench --compact-from L; 0 = gather everywhere)
mkdir -p gpurun_out
rm -f gpurun_out/abk_all.jsonl
for wl in C5 C3 C4; do
for cf in 0 1 3 5; do
  st=10; [ $wl = C5 ] && st=5
  timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 --compact-from $cf > gpurun_out/abk_${wl}_$cf.log 2>&1
  (echo -n "$cf "; tail -1 gpurun_out/abk_${wl}_$cf.log) >> gpurun_out/abk_all.jsonl
done
done
