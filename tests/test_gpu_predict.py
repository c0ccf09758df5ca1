"""Inference for unseen rows through gbdtmo_predict."""
import numpy as np
import pytest
import torch

from gen import gen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("case", ["C1", "C3s", "C2s"])
def test_predict_train_rows_equals_training_prediction_and_oracle_on_unseen(orc, case):
    import paper_conf_icpp_liupw25_b200 as pkg
    w = {"C1": gen.WORKLOADS["C1"], "C3s": gen.WORKLOADS["C3"].scaled(n=50_000, m=20, T=3, D=6),
         "C2s": gen.WORKLOADS["C2"].scaled(n=20_000, m=64, T=3, D=5)}[case]
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ctx = pkg.Context(0)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P)
    b.fit()
    # training rows: the instance-parallel walk reproduces the incremental training prediction exactly
    pt = pkg.predict(ctx, b.trees, torch.from_numpy(X).cuda(), w.D, w.d)
    torch.cuda.synchronize()
    assert torch.equal(pt, b.pred)
    # unseen rows (next row range of the same generator) vs the oracle's trees walked on the host
    Xu = gen.features_host(w, r0=w.n, nr=7_000)
    pu = pkg.predict(ctx, b.trees, torch.from_numpy(Xu).cuda(), w.D, w.d).cpu().numpy()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    hu = orc.predict(Xu, cuts, nbins, w.B, ref, w.D)                 # oracle walk
    assert np.max(np.abs(pu - hu)) <= 1e-4
    # and the exported thresholds are the oracle's cut values
    for t in range(w.T):
        st = b.trees[t]["node_state"].cpu().numpy()
        thr = b.trees[t]["threshold"].cpu().numpy()
        sp = st == 1
        np.testing.assert_array_equal(thr[sp], cuts[ref["feat"][t][sp], ref["bin"][t][sp]])


@pytest.mark.parametrize("n,m,T,D", [(3000, 3000, 4, 5),      # 8-row tiles staged in shared memory
                                     (700, 50_000, 3, 4),      # rows too wide to stage: global reads
                                     (2500, 12, 300, 2)])      # > 256 trees: tree chunks
def test_predict_shapes_vs_oracle_walk(orc, n, m, T, D):
    """gbdtmo_predict on wide rows, unstaged rows and multi-chunk forests: the GPU's exported trees
    walked by the oracle (oracle_predict) on the GPU trees' own (feature, bin) and
    the oracle's cuts of the same training columns; training rows reproduce the training pred."""
    import paper_conf_icpp_liupw25_b200 as pkg
    w = gen.WORKLOADS["C3"].scaled(n=n, m=m, T=T, D=D)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ctx = pkg.Context(0)
    P = pkg.Params(loss=0, T=T, D=D, B=w.B, lr=0.3, min_node=5)
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P)
    b.fit()
    pt = pkg.predict(ctx, b.trees, torch.from_numpy(X).cuda(), D, w.d)
    torch.cuda.synchronize()
    assert torch.equal(pt, b.pred)
    Xu = gen.features_host(w, r0=n, nr=1111) * 1.5
    pu = pkg.predict(ctx, b.trees, torch.from_numpy(Xu).cuda(), D, w.d).cpu().numpy()
    cuts, nbins, _ = orc.bin_matrix(X, w.B)
    trees = {k: np.stack([t[kk].cpu().numpy() for t in b.trees]) for k, kk in
             (("state", "node_state"), ("feat", "feature"), ("bin", "bin"), ("leaf", "leaf"))}
    ref = orc.predict(Xu, cuts, nbins, w.B, trees, D)
    np.testing.assert_allclose(pu, ref, rtol=0, atol=1e-12)
