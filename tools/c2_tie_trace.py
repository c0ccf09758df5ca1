"""Debug: tree-by-tree tie-locked oracle vs the GPU's predictions on C2 (where do they diverge?)."""
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
    T = int(sys.argv[1])
    w = gen.WORKLOADS["C2"]
    g = dict(np.load(os.path.join(ROOT, "tests", "golden", "C2_T10.npz")))
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    P = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    preds = [b.pred.cpu().numpy().copy()]
    for _ in range(T):
        b.step()
        preds.append(b.pred.cpu().numpy().copy())
    trees = [to_np(x) for x in b.trees]
    _, nbins, bins = oracle_bins(w)
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    pred = _replay_pred(orc, bins, g, 7, w)
    print(json.dumps({"tree": 6, "diff": float(np.max(np.abs(pred - preds[7])))}), flush=True)
    for t in range(7, T):
        before = pred.copy()
        pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, pred, trees, t, t + 1, w.D, w.lam, w.gamma,
                                       w.lr, w.min_node)
        dgpu = preds[t + 1] - preds[t]
        dorc = pred - before
        diff = float(np.max(np.abs(pred - preds[t + 1])))
        i = int(np.argmax(np.max(np.abs(dgpu - dorc), axis=1)))
        print(json.dumps({"tree": t, "diff": diff, "ties": [str(x) for x in ties],
                          "worst_row": i, "gpu_delta": dgpu[i].tolist()[:10], "orc_delta": dorc[i].tolist()[:10]}),
              flush=True)
        if diff > 1e-3:
            break


if __name__ == "__main__":
    main()
