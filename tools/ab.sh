#!/bin/bash
# Generic A/B of library builds on bench workloads (measurement only):
#   tools/ab.sh <tag> "<lib names: default or build/ab/<name>>" "<workloads>" [steps] [extra bench args]
# writes gpurun_out/ab_<tag>.jsonl: ms/tree and phase split per (lib, workload), libs interleaved
tag=$1; libs=$2; wls=$3; steps=${4:-10}; extra=$5
mkdir -p gpurun_out
out=gpurun_out/ab_$tag.jsonl; : > $out
for rep in 1 2; do
for wl in $wls; do
for lib in $libs; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  log=gpurun_out/ab_${tag}_${wl}_${lib}_$rep.log
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $steps --warmup 3 $extra > $log 2>&1
  python - "$lib" "$wl" "$rep" $log >> $out <<'PY'
import json, sys
lib, wl, rep, path = sys.argv[1:5]
try:
    b = json.loads([l for l in open(path) if l.startswith("{")][-1])
    print(json.dumps({"lib": lib, "wl": wl, "rep": int(rep), "ms": b["ms_per_step"], "phases": b["phase_ms_per_tree"],
                      "rows_built": b.get("work", {}).get("rows_built_per_tree")}))
except Exception as ex:
    print(json.dumps({"lib": lib, "wl": wl, "rep": int(rep), "error": repr(ex)}))
PY
done
done
done
cat $out
