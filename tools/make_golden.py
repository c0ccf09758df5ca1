"""Write the free-running parity goldens tests/golden/<cfg>_T<T>.npz — ORACLE ONLY.

Every stored value comes from oracle/ (the plain fp64 C oracle) on inputs from gen/ (the seeded
generators, no method arithmetic); nothing here imports the product package or touches a GPU.
The goldens exist because the oracle needs minutes to hours for T trees of the full-size configs
("the free-running 10-tree golden predictions for C4-C5 may be precomputed on
the CPU-only dev box ... per-tree split records, plus yhat for a fixed 65,536-row sample and
per-output fp64 sums"); tests/test_gpu_golden.py compares the CUDA path with them.

Contents (heap-indexed trees, NH = 2^(D+1) - 1 nodes, Algorithm 1):
  state, feat, bin, nrows, n_left  int  [T][NH]     tree records (0 none, 1 split, 2 leaf)
  gain                             f64  [T][NH]     Eq. (3) at the chosen split
  leaf                             f64  [T][NH][d]  v = -lr G/(H + lambda), 0 elsewhere
  sample_rows                      i64  [S]         rows i * n // S
  pred_sample                      f64  [S][d]      yhat after T trees at those rows
  pred_sum, pred_sumsq             f64  [d]         per-output sum / sum of squares of yhat, all rows
  nbins, cuts_digest               binning summary (nbins per feature, sha256 of the cuts bytes)
  src_sha                          sha256 of oracle.c, oracle.h, gen.py, gen.c, gen_rng.h (a test
                                   checks the goldens are not stale)
  leaf_scale                       f64  [T][NH][d]  AG_k / (H_k + lambda) per leaf and output, AG_k = sum
                                   |g_k| over the leaf's rows: the scale of the leaf-value error metric
                                   (leaves inherit the histogram's |x - x*| / AG metric)

usage: python tools/make_golden.py C3 [C4 C5 C2] [--T 10] [--threads N]
"""
from __future__ import annotations

import argparse
import hashlib
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from gen import gen  # noqa: E402

SAMPLE = {"C1": 2000, "C2": 8192, "C3": 8192, "C4": 1024, "C5": 65536}
SRC = ["oracle/oracle.c", "oracle/oracle.h", "gen/gen.py", "gen/gen.c", "gen/gen_rng.h"]


def src_sha() -> str:
    h = hashlib.sha256()
    for f in SRC:
        h.update(open(os.path.join(ROOT, f), "rb").read())
    return h.hexdigest()


def golden_path(name: str, T: int) -> str:
    return os.path.join(ROOT, "tests", "golden", f"{name}_T{T}.npz")


def oracle_bins(w, strip: int = 256):
    """Oracle binning (reading R14) of the workload's X, column strip by column strip (binning is
    per column), so C5's 32.8 GB X is never held: bins u16 [m][n]."""
    from oracle import oracle
    bins = np.empty((w.m, w.n), np.uint16)
    cuts = np.empty((w.m, w.B - 1), np.float32)
    nbins = np.empty(w.m, np.int32)
    for c0 in range(0, w.m, strip):
        nc = min(strip, w.m - c0)
        X = gen.features_host(w, c0=c0, nc=nc)
        c, nb, b = oracle.bin_matrix(X, w.B)
        bins[c0:c0 + nc], cuts[c0:c0 + nc], nbins[c0:c0 + nc] = b, c, nb
    return cuts, nbins, bins


def make(name: str, T: int) -> str:
    from oracle import oracle
    w = gen.WORKLOADS[name]
    t0 = time.time()
    cuts, nbins, bins = oracle_bins(w)
    t1 = time.time()
    X = gen.features_host(w) if w.index == 2 else None          # C2 labels need all columns
    Y = gen.targets_host(w, X)
    del X
    ref = oracle.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=T, D=w.D, lam=w.lam,
                       gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    t2 = time.time()
    S = min(SAMPLE[name], w.n)
    rows = (np.arange(S, dtype=np.int64) * w.n) // S
    pred = ref["pred"]
    out = golden_path(name, T)
    np.savez_compressed(
        out, state=ref["state"], feat=ref["feat"], bin=ref["bin"], nrows=ref["nrows"], n_left=ref["n_left"],
        gain=ref["gain"], leaf=ref["leaf"], sample_rows=rows, pred_sample=pred[rows],
        pred_sum=pred.sum(axis=0), pred_sumsq=(pred * pred).sum(axis=0), nbins=nbins,
        cuts_digest=np.frombuffer(hashlib.sha256(cuts.tobytes()).digest(), np.uint8),
        src_sha=np.array(src_sha()), workload=np.array(repr(w)), T=np.array(T),
        oracle_threads=np.array(oracle.num_threads()), seconds=np.array([t1 - t0, t2 - t1]))
    print(f"{name}: T={T} bin {t1 - t0:.1f}s train {t2 - t1:.1f}s ({oracle.num_threads()} threads) -> {out}",
          flush=True)
    add_leaf_scale(name, T, bins=bins, Y=Y)
    return out


def add_leaf_scale(name: str, T: int, bins=None, Y=None) -> None:
    """Replays the golden's own trees with oracle functions only (oracle_grad at the prediction
    before each tree, oracle_partition along the recorded splits, oracle_update_pred with the
    recorded leaves) to get every leaf's rows, and stores leaf_scale = AG_k / (H_k + lambda)."""
    from oracle import oracle
    w = gen.WORKLOADS[name]
    path = golden_path(name, T)
    g = dict(np.load(path))
    if bins is None:
        _, _, bins = oracle_bins(w)
    if Y is None:
        X = gen.features_host(w) if w.index == 2 else None
        Y = gen.targets_host(w, X)
        del X
    y = Y.astype(np.float64)
    NH = g["state"].shape[1]
    pred = np.zeros((w.n, w.d))
    scale = np.zeros((T, NH, w.d))
    for t in range(T):
        gr, hs = oracle.grad(w.loss, y, pred)
        rows = {0: np.arange(w.n, dtype=np.int32)}
        st = g["state"][t]
        for h in range(NH):
            if h not in rows:
                continue
            r = rows[h]
            if st[h] == 1:
                left, right = oracle.partition(bins, r, int(g["feat"][t][h]), int(g["bin"][t][h]))
                rows[2 * h + 1], rows[2 * h + 2] = left, right
            elif st[h] == 2:
                AG = np.abs(gr[r]).sum(0)
                H = hs[r].sum(0)
                scale[t, h] = AG / (H + w.lam)
                oracle.update_pred(pred, r, g["leaf"][t][h])
    err = float(np.max(np.abs(pred[g["sample_rows"]] - g["pred_sample"])))
    assert err < 1e-9, f"replay of the golden's trees does not reproduce its prediction ({err})"
    g["leaf_scale"] = scale
    np.savez_compressed(path, **g)
    print(f"{name}: leaf_scale added (replay matches the golden prediction to {err:.1e})", flush=True)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--T", type=int, default=10)
    ap.add_argument("--leaf-scale-only", action="store_true", help="add leaf_scale to existing goldens")
    a = ap.parse_args()
    for c in a.configs:
        if a.leaf_scale_only:
            add_leaf_scale(c, a.T)
        else:
            make(c, a.T)
