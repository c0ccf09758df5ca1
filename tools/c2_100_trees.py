"""C2 (MNIST-shaped softmax) at its configured 100 trees: the CUDA path vs the oracle (SURVEY §8(c)-4:
"For C2 (T = 100) the gate applies at tree 10; report tree 100 too").  The GPU trains 100 trees
free-running; the oracle replays the golden's trees (tests/golden/C2_T10.npz) up to the first
difference and continues tie-locked (tests/gpu_helpers.tie_locked_oracle: every differing split must
be a tie within 1e-6 of the oracle's own best).  Prints one JSON line: ties, max |yhat - oracle| after
10 and 100 trees.   python tools/c2_100_trees.py   (on a B200; ~5 minutes of host oracle work)"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from gen import gen  # noqa: E402
from oracle import oracle as orc  # noqa: E402
from tests.gpu_helpers import compare_trees, tie_locked_oracle, to_np  # noqa: E402
from tests.test_gpu_golden import _device_inputs, _replay_pred  # noqa: E402
from tools.make_golden import oracle_bins  # noqa: E402


def main():
    w = gen.WORKLOADS["C2"]
    T = 100
    g = dict(np.load(os.path.join(ROOT, "tests", "golden", "C2_T10.npz")))
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    P = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P, keep_model=True)
    pred10 = None
    for t in range(T):
        b.step()
        if t == 9:
            torch.cuda.synchronize()
            pred10 = b.pred.cpu().numpy().copy()
    torch.cuda.synchronize()
    trees = [to_np(x) for x in b.trees]
    def differs(t):
        try:
            return bool(compare_trees(trees[t], g["state"][t], g["feat"][t], g["bin"][t], g["nrows"][t]))
        except AssertionError:
            return True
    t0 = next((t for t in range(10) if differs(t)), 10)
    _, nbins, bins = oracle_bins(w)
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    pred = _replay_pred(orc, bins, g, t0, w)
    t_start = time.time()
    p10, ties10 = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, pred, trees, t0, 10, w.D, w.lam, w.gamma, w.lr,
                                    w.min_node)
    p100, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, p10, trees, 10, T, w.D, w.lam, w.gamma, w.lr,
                                   w.min_node)
    out = {"workload": w.name, "trees": T, "first_difference_tree": t0,
           "ties": [list(map(lambda v: v if not isinstance(v, np.generic) else v.item(), x)) for x in ties10 + ties],
           "max_abs_pred_diff_after_10": float(np.max(np.abs(pred10 - p10))),
           "max_abs_pred_diff_after_100": float(np.max(np.abs(b.pred.cpu().numpy() - p100))),
           "oracle_seconds": time.time() - t_start, "oracle_threads": orc.num_threads()}
    print(json.dumps(out, default=str))


if __name__ == "__main__":
    main()
