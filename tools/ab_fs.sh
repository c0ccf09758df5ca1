#!/bin/bash
# A/B: split search TMA-fed (default) vs register-fed half-row kernel
mkdir -p gpurun_out
out=gpurun_out/ab_fs_minb4.jsonl; : > $out
for wl in C5 C4 C3; do
for lib in default fs_minb4; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  st=10; [ $wl = C5 ] && st=8
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps $st --warmup 3 > gpurun_out/ab_fs_${wl}_$lib.log 2>&1
  python - "$lib" "$wl" gpurun_out/ab_fs_${wl}_$lib.log >> $out <<'PY'
import json, sys
lib, wl, path = sys.argv[1:4]
try:
    b = json.loads([l for l in open(path) if l.startswith("{")][-1])
    print(json.dumps({"lib": lib, "wl": wl, "ms": b["ms_per_step"], "phases": b["phase_ms_per_tree"]}))
except Exception as ex:
    print(json.dumps({"lib": lib, "wl": wl, "error": repr(ex)}))
PY
done
done
cat $out
