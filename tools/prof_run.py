"""Minimal driver for ncu captures: set up one workload in HBM and run a few trees.

  ncu --set full -k regex:k_hist_smem -s 1 -c 1 -o gpurun_out/prof python tools/prof_run.py C5 2
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from gen import gen  # noqa: E402


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C5"
    trees = int(sys.argv[2]) if len(sys.argv) > 2 else 2
    w = gen.sweep(int(wl[1:])) if wl.startswith("S") else gen.WORKLOADS[wl]
    dev = torch.device("cuda:0")
    ctx = pkg.Context(0)
    X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
    gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                    torch.cuda.current_stream().cuda_stream)
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    Y = torch.from_numpy(gen.targets_host(w)).to(dev)
    P = pkg.Params(loss=w.loss, T=trees, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    kw = {}
    if os.environ.get("PACKED") is not None:       # A/B: PACKED=0 row-major bins, PACKED=1 tile-packed
        kw["packed_bins"] = os.environ["PACKED"] == "1"
    if os.environ.get("SMALL_MAX_ROWS") is not None:
        kw["small_max_rows"] = int(os.environ["SMALL_MAX_ROWS"])
    if os.environ.get("FS_CG") is not None:         # A/B: GBDTMO_OPT_FS_CHANNEL_GROUPS
        kw["fs_channel_groups"] = int(os.environ["FS_CG"])
    b = pkg.Booster(ctx, ds, Y, P, **kw)
    for _ in range(trees):
        b.step()
    torch.cuda.synchronize()
    print("done", wl, trees, "launches", ctx.gbdtmo_launch_count())


if __name__ == "__main__":
    main()
