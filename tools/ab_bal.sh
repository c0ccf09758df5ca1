#!/bin/bash
# A/B: balanced last round of histogram batches (GBDTMO_HIST_BAL) on vs off
mkdir -p gpurun_out
out=gpurun_out/ab_bal.jsonl; : > $out
for wl in C5 C3 C4 S10 S50 S100 C1; do
for lib in default bal0; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/ab_bal_${wl}_$lib.log 2>&1
  python - "$lib" "$wl" gpurun_out/ab_bal_${wl}_$lib.log >> $out <<'PY'
import json, sys
lib, wl, path = sys.argv[1:4]
try:
    b = json.loads([l for l in open(path) if l.startswith("{")][-1])
    print(json.dumps({"lib": lib, "wl": wl, "ms": b["ms_per_step"], "hist_ms_by_level": b["hist_ms_by_level"]}))
except Exception as ex:
    print(json.dumps({"lib": lib, "wl": wl, "error": repr(ex)}))
PY
done
done
cat $out
