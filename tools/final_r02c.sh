#!/bin/bash
# Round-2 final measurement set (1 B200), session 2: writes gpurun_out/r02c_*; collect with
#   python tools/profile_collect.py r02c
out=gpurun_out; mkdir -p $out
python -m pytest tests -m gpu -q > $out/r02c_pytest_gpu.log 2>&1; echo "rc=$?" >> $out/r02c_pytest_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $out/r02c_bench_c5_n1.log 2>&1
for wl in C1 C2 C3 C4 S5 S10 S50 S100 S500 S983; do
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > $out/r02c_bench_$wl.log 2>&1
done
timeout 600 python bench.py --workload C1 --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --graph > $out/r02c_bench_C1_graph.log 2>&1
timeout 900 python bench.py --predict --steps 5 --warmup 2 > $out/r02c_bench_predict_c5.log 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $out/r02c_bench_reference.log 2>&1
# launch list of the bench command (cold, serialised: shares only)
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/r02c_launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
    > $out/r02c_ncu_launches.log 2>&1
# the channel-split split search (new this session): one tree of find_split launches on C4 and S500
for wl in C4 S500; do
  D=$(python -c "from gen import gen; w = gen.sweep(500) if '$wl' == 'S500' else gen.WORKLOADS['$wl']; print(w.D)")
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_find_split -s $D -c $D \
     -o /tmp/r02c_fs_$wl python tools/prof_run.py $wl 2 > $out/r02c_ncu_fs_$wl.log 2>&1
  python tools/ncu_summary.py /tmp/r02c_fs_$wl.ncu-rep --sass 20 > $out/r02c_ncu_fs_$wl.txt 2>&1
done
for f in $out/r02c_bench_*.log; do echo "$f: $(grep '^{' $f | tail -1 | cut -c1-160)"; done
