"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

C2, C3, C4: the oracle still finishes one full tree in seconds, so whole trees are compared.
C5 (2,000,000 x 4,096 x 16): inputs are generated in HBM exactly as bench.py does; the oracle
checks sampled outputs it can compute one by one (binning of sampled columns, the root
histogram of sampled features, Eq. (3) at the GPU's winning split, the root partition), plus
properties that hold at any size.
"""
import numpy as np
import pytest
import torch

from gen import gen
from tests.gpu_helpers import compare_trees, to_np

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_icpp_liupw25_b200 as pkg
    pkg.lib()
    return pkg


def _params(pkg, w, T):
    return pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)


@pytest.mark.parametrize("name,T", [("C2", 2), ("C3", 1), ("C4", 1)])
def test_full_size_trees_vs_oracle(orc, pkg, name, T):
    w = gen.WORKLOADS[name]
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ctx = pkg.Context(0)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).cuda(), _params(pkg, w, T))
    b.fit()
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    del X
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    for t in range(T):
        gt = to_np(b.trees[t])
        diffs = compare_trees(gt, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
        assert not diffs, (t, diffs)
        leaves = gt["node_state"] == 2
        np.testing.assert_allclose(gt["leaf"][leaves], ref["leaf"][t][leaves], rtol=1e-5, atol=1e-6)
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4


def test_c5_full_size_sampled(orc, pkg):
    w = gen.WORKLOADS["C5"]
    dev = torch.device("cuda:0")
    ctx = pkg.Context(0)
    X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
    gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                    torch.cuda.current_stream().cuda_stream)
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    torch.cuda.empty_cache()
    Y = gen.targets_host(w)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(dev), _params(pkg, w, 1), gmem_max_rows=0, small_max_rows=0)
    # --- sampled columns on the host (bit-identical generator) -> oracle binning
    sample = np.array([0, 1, 777, 2048, 4095], np.int64)
    Xs = np.stack([gen.matrix_host(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, int(c), 1, w.m)[:, 0] for c in sample], 1)
    cuts, nbins, bins = orc.bin_matrix(Xs, w.B)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy()[sample], nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy()[sample], cuts)
    gb = ds.bins[: w.n * ds.ld_bins].view(w.n, ds.ld_bins)
    for j, c in enumerate(sample):
        np.testing.assert_array_equal(gb[:, int(c)].cpu().numpy(), bins[j])
    # --- level 0 through the ABI, then the root histogram of the sampled features
    b._apply_options()
    ctx.gbdtmo_grad(b.p, b.y, b.pred, b.q, b.scales, b.state)
    b._level(0)
    torch.cuda.synchronize()
    sc = b.scales.cpu().numpy().astype(np.float64)
    V, B, m = b.p.V, w.B, w.m
    H = b.hist[0][: m * V * B].view(m, V, B)
    CN = b.cnt[0][: m * B].view(m, B)
    g, h = orc.grad(0, Y.astype(np.float64), np.zeros(Y.shape))
    rows = np.arange(w.n, dtype=np.int32)
    HG, HH, CNT = orc.build_hist(bins, B, g, h, rows)
    for j, c in enumerate(sample):
        np.testing.assert_array_equal(CN[int(c)].cpu().numpy(), CNT[j])
        gpu = H[int(c)].transpose(0, 1).cpu().numpy() * sc[None, :]
        assert np.array_equal(gpu, HG[j]), c          # dyadic targets, tree 1: bit-exact
    # --- the GPU's root split: Eq. (3) by the oracle at that split, and it beats every sampled feature
    keys = b.keys.cpu().numpy()
    from paper_conf_icpp_liupw25_b200.parallel import unpack_key
    fg, bb, gkey = unpack_key(int(keys[0]), B)
    Xf = gen.matrix_host(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, fg, 1, w.m)
    cf, nf, bf = orc.bin_matrix(Xf, w.B)
    HGf, HHf, CNTf = orc.build_hist(bf, B, g, h, rows)
    G, Hs = g.sum(0), h.sum(0)
    spf = orc.find_split(HGf, HHf, CNTf, nf, G, Hs, w.n, w.lam, w.min_node, want_all=True)
    gain_at = spf["all_gains"][0, bb]
    assert abs(gain_at - gkey) <= 1e-8 * abs(gain_at)
    sps = orc.find_split(HG, HH, CNT, nbins, G, Hs, w.n, w.lam, w.min_node)
    assert sps["gain"] <= gain_at * (1 + 1e-6)
    # --- root partition: the left child holds exactly the rows with bin <= b
    nid = torch.empty(w.n, dtype=torch.int32, device=dev)
    ctx.gbdtmo_rows_export(b.p, b.state, 1, None, nid, None, None)
    torch.cuda.synchronize()
    left = nid.cpu().numpy() == 1
    np.testing.assert_array_equal(left, bf[0] <= bb)
