"""Where the end-to-end (bench.py `e2e`) time goes on one GPU: pinned host X -> train() phases.

    python tools/e2e_probe.py [C5] [trees=20]

Times (CUDA events on the current stream, synchronised per phase, so phases do not overlap here):
bin_features_host (strip H2D + binning), Booster construction, every tree of fit(), D2H of yhat.
"""
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_liupw25_b200 as pkg     # noqa: E402
from paper_conf_icpp_liupw25_b200.booster import bin_features_host, Booster   # noqa: E402
from gen import gen                             # noqa: E402
import bench                                    # noqa: E402


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C5"
    T = int(sys.argv[2]) if len(sys.argv) > 2 else 20
    w = gen.WORKLOADS[wl]
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    Xh = torch.empty((w.n, w.m), dtype=torch.float32, pin_memory=True)
    gen.matrix_host(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, out=Xh.numpy())
    Yh = torch.from_numpy(bench.host_targets(w)).pin_memory()
    ctx = pkg.Context(0)
    P = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    out = {"workload": w.name, "trees": T}

    def span(name, fn):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = fn()
        e1.record()
        torch.cuda.synchronize()
        out[name] = {"event_ms": round(e0.elapsed_time(e1), 2), "wall_ms": round(1e3 * (time.perf_counter() - t0), 2)}
        return r

    for rep in range(2):                           # rep 0: first call in the process (cold), rep 1: warm
        tag = f"r{rep}_"
        Yd = span(tag + "y_h2d", lambda: Yh.to(dev, non_blocking=True).contiguous().float())
        ds = span(tag + "bin_features_host", lambda: bin_features_host(ctx, Xh, w.B, dev))
        b = span(tag + "booster_init", lambda: Booster(ctx, ds, Yd, P))
        tree_ms = []
        for t in range(T):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            b.step()
            e1.record()
            torch.cuda.synchronize()
            tree_ms.append(round(e0.elapsed_time(e1), 2))
        out[tag + "tree_ms"] = tree_ms
        pred_h = torch.empty((w.n, w.d), dtype=torch.float64, pin_memory=True)
        span(tag + "pred_d2h", lambda: pred_h.copy_(b.pred, non_blocking=True))
        print(json.dumps(out), flush=True)
        del b, ds, Yd
        torch.cuda.empty_cache()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
