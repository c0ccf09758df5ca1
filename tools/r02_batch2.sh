#!/bin/bash
# round-2 batch: small-node search G-variant parity, deep trees, re-calibration of the variant table
mkdir -p gpurun_out
python -m pytest tests/test_gpu_parity.py tests/test_gpu_hparams.py -q -p no:cacheprovider -k "small or trees_and or deep or grid" > gpurun_out/pytest_r02h.log 2>&1
tail -4 gpurun_out/pytest_r02h.log
cp paper_conf_icpp_liupw25_b200/hist_variant_table.json gpurun_out/hist_variant_table_before.json
timeout 1500 python tools/calibrate_hist.py C2 S5 S10 S50 C1 > gpurun_out/calibrate_r02.log 2>&1
tail -6 gpurun_out/calibrate_r02.log | cut -c1-400
for wl in C2 S10 S50 C1; do
  timeout 300 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/bench_r02h_$wl.json
  python -c "import json; b=json.load(open('gpurun_out/bench_r02h_$wl.json')); print('$wl', b['ms_per_step'], b['phase_ms_per_tree'])"
done
