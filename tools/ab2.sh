for v in shfl lcnt lcntshfl; do
  GBDTMO_LIB=build/ab/$v/libgbdtmo.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "packed or (trees and C5s) or (trees and C2s)" > gpurun_out/ab2_${v}_pytest.log 2>&1
  echo "$v pytest rc=$?" >> gpurun_out/ab2_summary.txt
done
HK=0 timeout 300 python tools/hk_probe.py C5 C3 > gpurun_out/ab2_base_probe.log 2>&1
for v in shfl lcnt lcntshfl; do
  GBDTMO_LIB=build/ab/$v/libgbdtmo.so HK=0 timeout 300 python tools/hk_probe.py C5 C3 > gpurun_out/ab2_${v}_probe.log 2>&1
done
bash tools/ab_ncu.sh ab2 "shfl=env GBDTMO_LIB=build/ab/shfl/libgbdtmo.so python tools/prof_run.py C5 1" "lcnt=env GBDTMO_LIB=build/ab/lcnt/libgbdtmo.so python tools/prof_run.py C5 1"
