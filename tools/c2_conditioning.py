"""Conditioning of the C2 (MNIST-shaped softmax, lr = 1, lambda = 1) boosting trajectory, oracle only:
two fp64 oracle runs whose initial predictions differ by 1e-13 (far below any arithmetic difference
between implementations), compared tree by tree.  With lr = 1 the softmax Newton leaves reach
thousands and the map from one tree's prediction to the next amplifies differences by ~2x per tree,
so free-running agreement beyond ~20 trees is not a property any two correct implementations share.
  python tools/c2_conditioning.py [T]  -> profiles/r02_c2_conditioning.json"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from gen import gen  # noqa: E402
from oracle import oracle as orc  # noqa: E402


def main():
    T = int(sys.argv[1]) if len(sys.argv) > 1 else 40
    w = gen.WORKLOADS["C2"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    eps = 1e-13 * (gen.uniform_host(w.seed, 99, 0, w.n * w.d).reshape(w.n, w.d) - 0.5)
    pa, pb = np.zeros((w.n, w.d)), eps.copy()
    rows = []
    for t in range(T):
        ra = orc.train(bins, nbins, w.B, y, loss=1, T=1, D=w.D, pred=pa)
        rb = orc.train(bins, nbins, w.B, y, loss=1, T=1, D=w.D, pred=pb)
        pa, pb = ra["pred"], rb["pred"]
        same = bool(np.array_equal(ra["state"], rb["state"]) and np.array_equal(ra["feat"], rb["feat"]) and
                    np.array_equal(ra["bin"], rb["bin"]))
        rows.append({"tree": t, "max_abs_pred_diff": float(np.max(np.abs(pa - pb))), "same_tree": same,
                     "max_abs_pred": float(np.max(np.abs(pa)))})
        print(json.dumps(rows[-1]), flush=True)
    json.dump({"workload": w.name, "perturbation": "initial prediction +- 5e-14 (uniform)", "trees": rows},
              open(os.path.join(ROOT, "profiles", "r02_c2_conditioning.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
