"""Time gbdtmo_bin (bin_features) on a workload's matrix generated in HBM: first call and warm calls.

  python tools/bin_probe.py C5
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from gen import gen  # noqa: E402


def main():
    w = gen.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "C5"]
    m = int(sys.argv[2]) if len(sys.argv) > 2 else w.m
    ctx = pkg.Context(0)
    X = torch.empty((w.n, m), dtype=torch.float32, device="cuda")
    gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, m, w.m, X.data_ptr(), m,
                    torch.cuda.current_stream().cuda_stream)
    out = []
    for it in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ds = pkg.bin_features(ctx, X, w.B)
        e1.record()
        torch.cuda.synchronize()
        out.append(round(e0.elapsed_time(e1), 2))
        del ds
    print(json.dumps({"workload": w.name, "n": w.n, "m": m, "bin_features_ms": out,
                      "x_gb": w.n * m * 4 / 1e9}))


if __name__ == "__main__":
    main()
