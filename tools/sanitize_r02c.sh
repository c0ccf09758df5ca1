#!/bin/bash
# compute-sanitizer over the kernels new in round 2 session 2: the run-parallel small-node search
# (k_seg_search) and the channel-split split search (k_find_split_c), softmax and MSE.
tag=${1:-r02c}
out=gpurun_out; mkdir -p $out
S="compute-sanitizer --print-limit 50 --kernel-name kns=gbdtmo --error-exitcode 9"
sum=$out/${tag}_sanitize_summary.txt
: > $sum
run() {
  local log=$out/${tag}_sanitize_$1_$2_$3.log
  timeout 900 $S --tool $1 python tools/sanitize_run.py $2 $3 > $log 2>&1
  echo "$1 $2 $3 rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $log | tr '\n' ' ')" >> $sum
}
for tool in memcheck racecheck synccheck; do
  run $tool C2s small; run $tool C3s small; run $tool C1 small; run $tool C3s cg8; run $tool C2s cg2; run $tool C2s k1
done
run initcheck C2s small; run initcheck C3s cg8
cat $sum
