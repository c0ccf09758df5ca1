"""Deep trees at full size (histogram memory): C5 (2 M x 4,096 x 16) at depth D,
T trees; prints ms per tree, rows built per level and the peak device memory.

    python tools/depth_probe.py [D=10] [T=3]
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_liupw25_b200 as pkg     # noqa: E402
from gen import gen                             # noqa: E402


def main():
    D = int(sys.argv[1]) if len(sys.argv) > 1 else 10
    T = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    w = gen.WORKLOADS["C5"].scaled(D=D)
    dev = torch.device("cuda:0")
    ctx = pkg.Context(0)
    X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
    gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                    torch.cuda.current_stream().cuda_stream)
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    torch.cuda.empty_cache()
    Y = torch.from_numpy(gen.targets_host(w)).to(dev)
    P = pkg.Params(loss=w.loss, T=T + 1, D=D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    b.step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(T):
        b.step()
    e1.record()
    torch.cuda.synchronize()
    st = b.trees[-1]["node_state"].cpu()
    splits_by_level = [int((st[(1 << l) - 1:(1 << (l + 1)) - 1] == 1).sum()) for l in range(D)]
    hist_gb = sum(h.numel() * 8 for h in b.hist if h is not None) / 1e9 if b.hist[0] is not b.hist[1] else b.hist[0].numel() * 8 / 1e9
    print(json.dumps({"workload": w.name, "D": D, "trees_timed": T, "ms_per_tree": e0.elapsed_time(e1) / T,
                      "splits_by_level_last_tree": splits_by_level, "hist_buffers_gb": hist_gb,
                      "max_memory_allocated_gb": torch.cuda.max_memory_allocated() / 1e9,
                      "device_total_gb": torch.cuda.get_device_properties(0).total_memory / 1e9}))


if __name__ == "__main__":
    main()
