"""Where does the CUDA path's free-running model first differ from an oracle golden, and is it a tie?

On the GPU box:   python tools/tie_probe.py gpu C2      -> gpurun_out/tie_probe_C2.npz (the GPU's trees)
Here (CPU):       python tools/tie_probe.py check C2    -> first differing node; the oracle's gain at the
                  GPU's (feature, bin) vs its best at that node (north star: splits may differ only where
                  gains tie within 1e-6 relative), with the oracle replaying the golden's own trees."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from gen import gen  # noqa: E402


def gpu(name):
    import torch
    import paper_conf_icpp_liupw25_b200 as pkg
    from tests.test_gpu_golden import _device_inputs
    w = gen.WORKLOADS[name]
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    P = pkg.Params(loss=w.loss, T=10, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    b.fit()
    torch.cuda.synchronize()
    out = {k: np.stack([t[k].cpu().numpy() for t in b.trees]) for k in b.trees[0]}
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    np.savez(os.path.join(ROOT, "gpurun_out", f"tie_probe_{name}.npz"), **out)


def check(name):
    from oracle import oracle
    from tools.make_golden import oracle_bins
    w = gen.WORKLOADS[name]
    g = dict(np.load(os.path.join(ROOT, "tests", "golden", f"{name}_T10.npz")))
    G = dict(np.load(os.path.join(ROOT, "gpurun_out", f"tie_probe_{name}.npz")))
    first = None
    for t in range(10):
        for h in range(g["state"].shape[1]):
            if g["state"][t][h] == 1 and (G["feature"][t][h] != g["feat"][t][h] or G["bin"][t][h] != g["bin"][t][h]):
                first = (t, h)
                break
            if g["state"][t][h] != G["node_state"][t][h]:
                first = (t, h)
                break
        if first:
            break
    print("first difference:", first)
    if not first:
        return
    t, hd = first
    _, nbins, bins = oracle_bins(w)
    X = gen.features_host(w) if w.index == 2 else None
    y = gen.targets_host(w, X).astype(np.float64)
    pred = np.zeros((w.n, w.d))
    for tt in range(t + 1):
        gr, hs = oracle.grad(w.loss, y, pred)
        rows = {0: np.arange(w.n, dtype=np.int32)}
        for h in range(g["state"].shape[1]):
            if h not in rows:
                continue
            r = rows[h]
            if tt == t and h == hd:
                HG, HH, CNT = oracle.build_hist(bins, w.B, gr, hs, r)
                sp = oracle.find_split(HG, HH, CNT, nbins, gr[r].sum(0), hs[r].sum(0), len(r), w.lam, w.min_node,
                                       want_all=True)
                ag = sp["all_gains"]
                gf, gb = int(G["feature"][t][h]), int(G["bin"][t][h])
                print(f"tree {t} node {h} rows {len(r)}: oracle best (f={sp['feature']}, b={sp['bin']}) gain "
                      f"{sp['gain']!r}; GPU (f={gf}, b={gb}) oracle gain {ag[gf, gb]!r} (GPU's own {G['gain'][t][h]!r}); "
                      f"relative gap {(sp['gain'] - ag[gf, gb]) / sp['gain']:.3e}; GPU state {G['node_state'][t][h]}")
                return
            if g["state"][tt][h] == 1:
                left, right = oracle.partition(bins, r, int(g["feat"][tt][h]), int(g["bin"][tt][h]))
                rows[2 * h + 1], rows[2 * h + 2] = left, right
            elif g["state"][tt][h] == 2:
                oracle.update_pred(pred, r, g["leaf"][tt][h])


if __name__ == "__main__":
    {"gpu": gpu, "check": check}[sys.argv[1]](sys.argv[2])
