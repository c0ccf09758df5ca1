mkdir -p gpurun_out
for wl in C5 C4 C2 C3; do
for lib in pf0 def pf4; do
  if [ $lib = def ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/abfs_${wl}_${lib}.log 2>&1
done
done
