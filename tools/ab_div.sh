#!/bin/bash
# A/B: softmax Eq. (3) child terms with one fp64 division (default) vs two
mkdir -p gpurun_out
out=gpurun_out/ab_div.jsonl; : > $out
for wl in C2 S100 S500; do
for lib in default div2; do
  if [ $lib = default ]; then L=""; else L="GBDTMO_LIB=build/ab/$lib/libgbdtmo.so"; fi
  env $L timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/ab_div_${wl}_$lib.log 2>&1
  python - "$lib" "$wl" gpurun_out/ab_div_${wl}_$lib.log >> $out <<'PY'
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
