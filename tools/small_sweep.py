"""Sort-and-segment threshold sweep: ms per tree and phase split vs GBDTMO_OPT_SMALL_MAX_ROWS.

    python tools/small_sweep.py C2 0,128,256,512,1024,2048 [warm=3] [timed=10]

Every threshold trains the same trees (checked against the first threshold's split records).
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_liupw25_b200 as pkg     # noqa: E402
from gen import gen                             # noqa: E402
import bench                                    # noqa: E402


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C2"
    ths = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "0,128,512,2048").split(",")]
    warm = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    timed = int(sys.argv[4]) if len(sys.argv) > 4 else 10
    w = gen.WORKLOADS[wl] if wl in gen.WORKLOADS else gen.sweep(int(wl[1:]))
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    ctx = pkg.Context(0)
    X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
    if w.classes_sweep:
        X.copy_(torch.from_numpy(gen.features_host(w, 0, w.n, 0, w.m)))
    else:
        gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                        torch.cuda.current_stream().cuda_stream)
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    Y = torch.from_numpy(bench.host_targets(w)).to(dev)
    P = pkg.Params(loss=w.loss, T=warm + timed, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr,
                   min_node=w.min_node)
    ref = None
    for t in ths:
        b = pkg.Booster(ctx, ds, Y, P, small_max_rows=t)
        for _ in range(warm):
            b.step()
        torch.cuda.synchronize()
        b.phase_marks = []
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(timed):
            b.step(time_hist=True)
        e1.record()
        torch.cuda.synchronize()
        recs = [(tr["feature"].cpu(), tr["bin"].cpu(), tr["node_state"].cpu()) for tr in b.trees]
        if ref is None:
            ref = recs
        same = all(torch.equal(a[0], c[0]) and torch.equal(a[1], c[1]) and torch.equal(a[2], c[2])
                   for a, c in zip(ref, recs))
        ph = {k: round(v / timed, 3) for k, v in b.phase_ms(timed).items()}
        print(json.dumps({"wl": wl, "small_max_rows": t, "ms_per_tree": round(e0.elapsed_time(e1) / timed, 3),
                          "phase_ms": ph, "same_trees": same}), flush=True)
        del b
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
