"""One or two training trees through the C ABI for compute-sanitizer (tools/sanitize.sh).

  python tools/sanitize_run.py <case> <variant>
case: C1 | C3s | C2s;  variant: k0 (row-pair smem), k1 (diagonal), k2 (TMA-staged), gmem (global
atomics for every node), small (sort-and-segment small nodes), sparse (default-bin skip), graph
(CUDA-graph replay), predict (gbdtmo_predict), binhost (train() from a pinned host matrix:
gbdtmo_bin_host strip uploads on the context's copy stream), packed (tile-packed bins), cg2 / cg8
(channel-split split search forced to 2 / 8 warp pairs).  Prints
the max |pred - oracle| (parity still holds under the tool)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from gen import gen  # noqa: E402
from oracle import oracle  # noqa: E402

CASES = {"C1": gen.WORKLOADS["C1"].scaled(T=2),
         "C3s": gen.WORKLOADS["C3"].scaled(n=12_000, m=20, T=2, D=5),
         "C2s": gen.WORKLOADS["C2"].scaled(n=6_000, m=40, T=2, D=5)}


def main():
    case, var = sys.argv[1], sys.argv[2]
    w = CASES[case]
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ctx = pkg.Context(0)
    kw = dict(k0=dict(hist_kernel=0, gmem_max_rows=0, small_max_rows=0),
              k1=dict(hist_kernel=1, gmem_max_rows=0, small_max_rows=0),
              k2=dict(hist_kernel=2, gmem_max_rows=0, small_max_rows=0),
              gmem=dict(gmem_max_rows=1 << 30, small_max_rows=0),
              small=dict(small_max_rows=4000, gmem_max_rows=0),
              sparse=dict(sparse_default=True, hist_kernel=0),
              graph=dict(), predict=dict(), binhost=dict(), packed=dict(packed_bins=True, hist_kernel=0),
              cg8=dict(fs_channel_groups=8), cg2=dict(fs_channel_groups=2))[var]
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    if var == "binhost":
        b = pkg.train(torch.from_numpy(X).pin_memory(), torch.from_numpy(Y), P, ctx=ctx)
    else:
        b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P,
                        **kw)
    if var == "binhost":
        pass
    elif var == "graph":
        b.capture()
        for _ in range(w.T):
            b.step_graph()
    else:
        b.fit()
    if var == "predict":
        p = pkg.predict(ctx, b.trees, torch.from_numpy(X).cuda(), w.D, w.d)
        assert torch.equal(p, b.pred)
    torch.cuda.synchronize()
    cuts, nbins, bins = oracle.bin_matrix(X, w.B)
    ref = oracle.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                       lr=w.lr, min_node=w.min_node)
    err = float(np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])))
    print(f"sanitize_run {case} {var}: {ctx.gbdtmo_launch_count()} launches, max |pred - oracle| = {err:.3e}")
    assert err <= 1e-4


if __name__ == "__main__":
    main()
