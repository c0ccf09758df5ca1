import sys, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_icpp_liupw25_b200 as pkg
from gen import gen
w = gen.WORKLOADS["C3"].scaled(n=5000, m=24, T=1, D=3)
X = gen.features_host(w); Y = gen.targets_host(w, X)
ctx = pkg.Context(0)
ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
P = pkg.Params(loss=w.loss, T=1, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
b = pkg.Booster(ctx, ds, torch.from_numpy(Y).cuda(), P, hist_kernel=2, gmem_max_rows=0, small_max_rows=0)
b.fit(1); torch.cuda.synchronize(); print("ok")
