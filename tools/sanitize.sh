#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the library's kernels:
# every histogram variant on small C1 / C3s / C2s trees, graph replay, inference, and the
# 2-process peer exchange.  Logs: gpurun_out/<tag>_sanitize_*.log, summary: <tag>_sanitize_summary.txt
#   gpurun -- 'bash tools/sanitize.sh r02'
tag=${1:-r02}
out=gpurun_out; mkdir -p $out
S="compute-sanitizer --print-limit 50 --kernel-name kns=gbdtmo --error-exitcode 9"
sum=$out/${tag}_sanitize_summary.txt
: > $sum
run() {   # tool case variant
  local log=$out/${tag}_sanitize_$1_$2_$3.log
  timeout 900 $S --tool $1 python tools/sanitize_run.py $2 $3 > $log 2>&1
  local rc=$?
  echo "$1 $2 $3 rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $log | tr '\n' ' ')" >> $sum
}
for tool in memcheck racecheck synccheck; do
  for v in k0 k1 k2 gmem small; do run $tool C1 $v; run $tool C3s $v; done
  run $tool C2s k1; run $tool C2s sparse; run $tool C2s small; run $tool C1 graph; run $tool C3s predict; run $tool C3s binhost; run $tool C3s packed
done
# initcheck on the default path (uninitialised device reads)
run initcheck C3s k0; run initcheck C2s k1
# 2-process peer exchange (both ranks under memcheck / racecheck)
for tool in memcheck racecheck; do
  log=$out/${tag}_sanitize_${tool}_peer.log
  timeout 1200 $S --tool $tool --target-processes all python -m pytest tests/test_gpu_multiproc.py -q -p no:cacheprovider \
     -k "peer and not expiry" > $log 2>&1
  echo "$tool peer rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|passed|failed' $log | tr '\n' ' ')" >> $sum
done
cat $sum
