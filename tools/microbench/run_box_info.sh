#!/bin/bash
# Box facts + on-chip accumulation micro-benchmarks (run under gpurun).
mkdir -p gpurun_out
{
  echo "== nproc"; nproc; echo "== free -g"; free -g; echo "== lscpu"; lscpu | head -20
  echo "== nvidia-smi"; nvidia-smi; nvidia-smi -q | grep -iE "clocks|MHz|Power Limit" | head -40
  echo "== python"; python -c "import torch; print(torch.__version__, torch.cuda.get_device_name(0), torch.cuda.get_device_properties(0)); import torch.cuda.nccl as n; print('nccl', n.version())"
} > gpurun_out/box_info.txt 2>&1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/mb_clocks.csv &
SMI=$!
./tools/microbench/atom_bench > gpurun_out/atom_bench.txt 2>&1
kill $SMI
