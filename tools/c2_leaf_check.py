"""Debug: along the GPU's own C2 trees, recompute every leaf with the oracle (oracle_grad at the GPU's
own pre-tree prediction, rows by oracle_partition along the GPU's splits, oracle_leaf_value) and report
the first tree whose leaves or whose prediction disagree.   python tools/c2_leaf_check.py T"""
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
from tests.gpu_helpers import to_np  # noqa: E402
from tests.test_gpu_golden import _device_inputs  # noqa: E402
from tools.make_golden import oracle_bins  # noqa: E402


def main():
    T = int(sys.argv[1])
    w = gen.WORKLOADS["C2"]
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    P = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    preds = []
    for _ in range(T):
        preds.append(b.pred.cpu().numpy().copy())
        b.step()
    torch.cuda.synchronize()
    preds.append(b.pred.cpu().numpy().copy())
    trees = [to_np(x) for x in b.trees]
    _, nbins, bins = oracle_bins(w)
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    report = []
    pred = np.zeros((w.n, w.d))
    for t in range(T):
        gr, hh = orc.grad(1, y, preds[t])
        rows = {0: np.arange(w.n, dtype=np.int32)}
        worst = 0.0
        worst_info = None
        for h in range(len(trees[t]["node_state"])):
            if h not in rows:
                continue
            r = rows[h]
            st = trees[t]["node_state"][h]
            if st == 1:
                rows[2 * h + 1], rows[2 * h + 2] = orc.partition(bins, r, int(trees[t]["feature"][h]),
                                                                 int(trees[t]["bin"][h]))
            elif st == 2:
                v = orc.leaf_value(gr[r].sum(0), hh[r].sum(0), w.lam, w.lr)
                e = float(np.max(np.abs(v - trees[t]["leaf"][h])))
                if e > worst:
                    worst, worst_info = e, (h, len(r), float(np.max(np.abs(v))), float(hh[r].sum(0).max()))
                orc.update_pred(pred, r, trees[t]["leaf"][h])
        pd = float(np.max(np.abs(pred - preds[t + 1])))
        report.append({"tree": t, "leaf_max_abs_err": worst, "worst": worst_info, "pred_walk_vs_gpu": pd,
                       "pred_max_abs": float(np.max(np.abs(preds[t + 1])))})
    print(json.dumps(report))


if __name__ == "__main__":
    main()
