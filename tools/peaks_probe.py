"""Print the shared-atomic microbenchmark modes of tools/microbench/peaks.cu (one GPU)."""
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
L = C.CDLL(os.path.join(ROOT, "tools", "microbench", "libgbdtmo_peaks.so"))
L.peaks_atoms.argtypes = [C.c_int, C.c_int, C.c_int] + [C.POINTER(C.c_double)] * 3
for mode in (0, 1, 2):
    a, b, c = C.c_double(), C.c_double(), C.c_double()
    rc = L.peaks_atoms(0, mode, int(sys.argv[1]) if len(sys.argv) > 1 else 80000, C.byref(a), C.byref(b), C.byref(c))
    print(json.dumps({"mode": mode, "rc": rc, "lane_ops_per_clk_sm": a.value, "T_lane_ops_per_s": b.value / 1e12,
                      "clk_mhz": c.value}))
