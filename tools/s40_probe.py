import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_icpp_liupw25_b200 as pkg
from gen import gen
from oracle import oracle as orc
w = gen.sweep(40, n=4_000, m=16, T=2, D=4)
X = gen.features_host(w); Y = gen.targets_host(w, X)
cuts, nbins, bins = orc.bin_matrix(X, w.B)
ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
ctx = pkg.Context(0)
for small in (0, 2000):
  for cg in (0, 1):
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P, small_max_rows=small, fs_channel_groups=cg)
    b.fit(); torch.cuda.synchronize()
    for t in range(w.T):
        st = b.trees[t]['node_state'].cpu().numpy(); ft = b.trees[t]['feature'].cpu().numpy(); bt = b.trees[t]['bin'].cpu().numpy()
        diff = [h for h in range(len(st)) if st[h]==1 and ref['state'][t][h]==1 and (ft[h]!=ref['feat'][t][h] or bt[h]!=ref['bin'][t][h])]
        print('small', small, 'cg', cg, 'tree', t, 'diff nodes', diff[:5], [(ft[h],bt[h],ref['feat'][t][h],ref['bin'][t][h], b.trees[t]['gain'].cpu().numpy()[h], ref['gain'][t][h]) for h in diff[:2]])
