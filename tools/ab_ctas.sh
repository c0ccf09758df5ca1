#!/bin/bash
# A/B: 1 histogram CTA per SM (1024 threads, 6-feature tiles) vs 2 CTAs (512 threads, 3-feature tiles)
mkdir -p gpurun_out
out=gpurun_out/ab_ctas.jsonl; : > $out
for wl in C5 C3 C4; do
for lib in default ctas2_t512; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  st=10; [ $wl = C5 ] && st=8
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/ab_ctas_${wl}_$lib.log 2>&1
  python - "$lib" "$wl" gpurun_out/ab_ctas_${wl}_$lib.log >> $out <<'PY'
import json, sys
lib, wl, path = sys.argv[1:4]
try:
    b = json.loads([l for l in open(path) if l.startswith("{")][-1])
    print(json.dumps({"lib": lib, "wl": wl, "ms": b["ms_per_step"], "hist_ms_by_level": b["hist_ms_by_level"],
                      "rows": b["rows_built_by_level"], "ns_row": b["work"]["hist_ns_per_built_row"]}))
except Exception as ex:
    print(json.dumps({"lib": lib, "wl": wl, "error": repr(ex)}))
PY
done
done
cat $out
