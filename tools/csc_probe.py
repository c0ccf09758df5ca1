"""A sparse workload trained from CSC with the CSC-driven histograms (gbdtmo_build_hist_csc, all
levels or levels < k) vs the dense-bin kernels: ms per tree and phase split, trees checked equal.

    python tools/csc_probe.py [C2|C3] [warm=3] [timed=10] [keep=1.0]

keep < 1 zeroes each entry of X with probability 1 - keep (targets from the original X)."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_liupw25_b200 as pkg     # noqa: E402
from gen import gen                             # noqa: E402


def csc(X):
    nz = X != 0
    col_ptr = np.zeros(X.shape[1] + 1, np.int64)
    col_ptr[1:] = np.cumsum(nz.sum(0))
    rows, cols = np.nonzero(nz.T)           # column-major order
    return X.T[nz.T].astype(np.float32), cols.astype(np.int32), col_ptr


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C2"
    warm = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    timed = int(sys.argv[3]) if len(sys.argv) > 3 else 10
    keep = float(sys.argv[4]) if len(sys.argv) > 4 else 1.0
    w = gen.WORKLOADS[wl]
    X = gen.features_host(w)
    Y = torch.from_numpy(gen.targets_host(w, X)).cuda()
    if keep < 1.0:
        u = gen.uniform_host(w.seed, 91, 0, X.size).reshape(X.shape)
        X = np.where(u < keep, X, 0.0).astype(np.float32)
    ctx = pkg.Context(0)
    vals, rows, cp = csc(X)
    ds = pkg.bin_features_csc(ctx, torch.from_numpy(vals).cuda(), torch.from_numpy(rows).cuda(), torch.from_numpy(cp),
                              w.n, w.B)
    out = {"wl": w.name, "nnz": int(cp[-1]), "density": float(cp[-1]) / (w.n * w.m)}
    ref = None
    for mode in ("dense", "csc", "csc2", "csc1"):
        P = pkg.Params(loss=w.loss, T=warm + timed, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
        lv = int(mode[3:]) if mode.startswith("csc") and len(mode) > 3 else None
        b = pkg.Booster(ctx, ds, Y, P, csc_hist=mode.startswith("csc"), csc_levels=lv)
        for _ in range(warm):
            b.step()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(timed):
            b.step(time_hist=True)
        e1.record()
        torch.cuda.synchronize()
        st = np.stack([t["node_state"].cpu().numpy() for t in b.trees])
        ft = np.stack([t["feature"].cpu().numpy() for t in b.trees])
        out[mode] = {"ms_per_tree": round(e0.elapsed_time(e1) / timed, 3),
                     "phase_ms": {k: round(v / timed, 3) for k, v in b.phase_ms(timed).items()}}
        if ref is None:
            ref = (st, ft)
        else:
            out["same_trees_" + mode] = bool(np.array_equal(st, ref[0]) and np.array_equal(ft[st == 1], ref[1][st == 1]))
    print(json.dumps(out))


if __name__ == "__main__":
    main()
