#!/bin/bash
# Round-2 measurement set (1 B200): the driver's default bench line, every config / sweep point, the
# inference line and the reference arm.  Writes gpurun_out/r02f_*.
out=gpurun_out; mkdir -p $out
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $out/r02f_bench_c5_n1.log 2>&1
for wl in C1 C2 C3 C4 S5 S10 S50 S100 S500; do
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > $out/r02f_bench_$wl.log 2>&1
done
timeout 600 python bench.py --workload C1 --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --graph > $out/r02f_bench_C1_graph.log 2>&1
timeout 900 python bench.py --predict --steps 5 --warmup 2 > $out/r02f_bench_predict_c5.log 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $out/r02f_bench_reference.log 2>&1
for f in $out/r02f_*.log; do echo "$f: $(grep '^{' $f | tail -1 | cut -c1-200)"; done
