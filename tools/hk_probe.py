"""A/B of the two shared-memory histogram lane mappings on a full workload shape (ms per tree).

  python tools/hk_probe.py C5 [C2 ...]        (on a B200)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from calibrate_hist import time_trees  # noqa: E402
from gen import gen  # noqa: E402


def main():
    ctx = pkg.Context(0)
    for name in sys.argv[1:] or ["C5"]:
        w = gen.WORKLOADS[name] if name in gen.WORKLOADS else gen.sweep(int(name[1:]))
        if w.classes_sweep:
            X = torch.from_numpy(gen.features_host(w)).cuda()
        else:
            X = torch.empty((w.n, w.m), dtype=torch.float32, device="cuda")
            gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                            torch.cuda.current_stream().cuda_stream)
        ds = pkg.bin_features(ctx, X, w.B)
        del X
        torch.cuda.empty_cache()
        Y = torch.from_numpy(gen.targets_host(w)).cuda()
        V = w.d * (2 if w.loss == gen.LOSS_SOFTMAX else 1)
        gm = pkg.booster.variant_threshold(V, w.m, "gmem_max_rows", n=w.n)
        sm = pkg.booster.variant_threshold(V, w.m, "small_max_rows", n=w.n)
        kernels = [int(k) for k in os.environ.get("HK", "0,1").split(",")]
        res = {}
        for hk in kernels + kernels:
            res.setdefault(hk, []).append(round(time_trees(ctx, ds, Y, w, gm, sm, warm=2, timed=3, hk=hk), 3))
        print(json.dumps({"workload": w.name, "gmem": gm, "small": sm, "ms_per_tree_by_hist_kernel": res}), flush=True)
        del ds, Y
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
