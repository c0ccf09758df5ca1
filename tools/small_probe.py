"""Time whole trees at a few small-node thresholds (quick A/B for the sort-and-segment search).

  python tools/small_probe.py C2 0 512 1024        (on a B200)
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
    name = sys.argv[1]
    w = gen.WORKLOADS[name] if name in gen.WORKLOADS else gen.sweep(int(name[1:]))
    thr = [int(x) for x in sys.argv[2:]] or [0, 1024]
    ctx = pkg.Context(0)
    X = torch.from_numpy(gen.features_host(w)).cuda()
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    Y = torch.from_numpy(gen.targets_host(w)).cuda()
    gm = pkg.booster.variant_threshold(w.d * (2 if w.loss == gen.LOSS_SOFTMAX else 1), w.m, "gmem_max_rows")
    res = {t: round(time_trees(ctx, ds, Y, w, gm, t, warm=2, timed=5), 4) for t in thr}
    print(json.dumps({"workload": w.name, "gmem_max_rows": gm, "ms_per_tree_by_small": res}))


if __name__ == "__main__":
    main()
