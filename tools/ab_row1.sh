#!/bin/bash
# A/B: phase-2 lane map of the K = 16 histogram kernel (row pair per instruction vs one row)
mkdir -p gpurun_out
out=gpurun_out/ab_row1.jsonl; : > $out
for wl in C5 C3 C4; do
for lib in row0 row1sb2 default row1sb8; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  st=10; [ $wl = C5 ] && st=8
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/ab_row1_${wl}_$lib.log 2>&1
  python - "$lib" "$wl" gpurun_out/ab_row1_${wl}_$lib.log >> $out <<'PY'
import json, sys
lib, wl, path = sys.argv[1:4]
try:
    b = json.loads([l for l in open(path) if l.startswith("{")][-1])
    print(json.dumps({"lib": lib, "wl": wl, "ms": b["ms_per_step"], "hist_ns_row": b["work"]["hist_ns_per_built_row"],
                      "hist_ms_by_level": b["hist_ms_by_level"], "frac": b["roofline"]["frac"]}))
except Exception as ex:
    print(json.dumps({"lib": lib, "wl": wl, "error": repr(ex)}))
PY
done
done
cat $out
