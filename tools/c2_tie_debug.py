"""Debug a non-tie split difference in the C2 100-tree report: replay tie-locked to tree T0, then compare
the GPU's level histograms of heap node H (feature F) with the oracle's direct histogram of the same rows.
  python tools/c2_tie_debug.py T0 H F"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from gen import gen  # noqa: E402
from oracle import oracle as orc  # noqa: E402
from tests.gpu_helpers import tie_locked_oracle, to_np  # noqa: E402
from tests.test_gpu_golden import _device_inputs, _replay_pred  # noqa: E402
from tools.make_golden import oracle_bins  # noqa: E402


def main():
    T0, H, F = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
    w = gen.WORKLOADS["C2"]
    g = dict(np.load(os.path.join(ROOT, "tests", "golden", "C2_T10.npz")))
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    P = pkg.Params(loss=w.loss, T=T0 + 1, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    for _ in range(T0):
        b.step()
    torch.cuda.synchronize()
    pred_gpu_before = b.pred.cpu().numpy().copy()
    # tree T0 level by level up to H's level
    lvl_h = int(np.floor(np.log2(H + 1)))
    b._apply_options()
    ctx.gbdtmo_grad(b.p, b.y, b.pred, b.q, b.scales, b.state, b.gh)
    for lvl in range(lvl_h + 1):
        b._level(lvl)
    torch.cuda.synchronize()
    V, B, m, d = b.p.V, w.B, w.m, w.d
    slot = H - ((1 << lvl_h) - 1)
    LN = 1 << lvl_h
    last = lvl_h == w.D - 1
    hs = slot >> 1 if last else slot
    LS = LN // 2 if last else LN
    Hh = b.hist[lvl_h % 2][: LS * m * V * B].view(LS, m, V, B)[hs, F].cpu().numpy().astype(np.float64)   # [V][B]
    Cn = b.cnt[lvl_h % 2][: LS * m * B].view(LS, m, B)[hs, F].cpu().numpy()
    sc = b.scales.cpu().numpy().astype(np.float64)
    key = int(b.keys[slot].item()) if not False else 0
    # the oracle, tie-locked on the GPU's trees 0..T0-1 (which it replays), then its own g/h at tree T0
    trees = [to_np(x) for x in b.trees]
    _, nbins, bins = oracle_bins(w)
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    pred0 = _replay_pred(orc, bins, g, 7, w)
    pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, pred0, trees, 7, T0, w.D, w.lam, w.gamma, w.lr,
                                   w.min_node)
    gr, hh = orc.grad(1, y, pred)
    # rows of node H in tree T0 along the GPU's tree T0 (splits above H)
    nid = torch.empty(w.n, dtype=torch.int32, device="cuda")
    ctx.gbdtmo_rows_export(b.p, b.state, lvl_h, None, nid, None, None)
    torch.cuda.synchronize()
    rows = np.nonzero(nid.cpu().numpy() == H)[0].astype(np.int32)
    HG, HH, CNT = orc.build_hist(bins, B, gr, hh, rows)
    gpu_g = Hh[:d].T * sc[None, :d]
    gpu_h = Hh[d:].T * sc[None, d:]
    out = {"rows": len(rows), "pred_max_abs_diff_before": float(np.max(np.abs(pred_gpu_before - pred))),
           "cnt_equal": bool(np.array_equal(Cn, CNT[F])), "G_max_abs_err": float(np.max(np.abs(gpu_g - HG[F]))),
           "H_max_abs_err": float(np.max(np.abs(gpu_h - HH[F]))), "G_scale": float(np.max(np.abs(HG[F]))),
           "H_scale": float(np.max(HH[F])), "scales": sc.tolist(), "ties": [str(t) for t in ties][:10],
           "h_min_pos": float(hh[rows][hh[rows] > 0].min()) if np.any(hh[rows] > 0) else 0.0,
           "h_zero_frac": float(np.mean(hh[rows] == 0)), "key": key}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
