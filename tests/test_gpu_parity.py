"""CUDA path (through the C ABI) vs the CPU oracle on the same seeded inputs.

Tolerances:
  bins, cuts, counts, tree structure, partitions  bit-exact (ties: oracle gain at the GPU's
      choice within 1e-6 relative of the oracle's best, R22)
  histograms   |gpu - oracle| <= 1e-5 * max(|oracle|, sum|g| of the bin)  (exact on dyadic tree-1 inputs)
  leaf values / predictions after T trees      <= 1e-4 absolute (north star)
"""
import numpy as np
import pytest
import torch

from gen import gen
from tests.gpu_helpers import compare_trees, node_rows, to_np

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_icpp_liupw25_b200 as pkg
    pkg.lib()
    return pkg


@pytest.fixture(scope="module")
def ctx(pkg):
    return pkg.Context(0)


def _params(pkg, w, T=None, D=None):
    return pkg.Params(loss=w.loss, T=T or w.T, D=D or w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr,
                      min_node=w.min_node)


def _inputs(w):
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    return X, Y


CASES = {
    "C1": gen.WORKLOADS["C1"],
    "C2s": gen.WORKLOADS["C2"].scaled(n=20_000, m=64, T=3, D=6),
    "C3s": gen.WORKLOADS["C3"].scaled(n=100_000, m=24, T=3, D=6),
    "C4s": gen.WORKLOADS["C4"].scaled(n=20_000, m=20, T=2, D=4),
    "C5s": gen.WORKLOADS["C5"].scaled(n=50_000, m=70, T=2, D=5),
    "S300s": gen.sweep(300, n=6_000, m=24, T=2, D=3),        # NEXT-2 class sweep, d = 300 softmax
    "S6s": gen.sweep(6, n=8_000, m=30, T=2, D=5),             # d = 6 softmax: 4 features per small-search warp
}


# ---------------------------------------------------------------------------- binning

@pytest.mark.parametrize("case", ["C1", "C2s", "C3s", "C4s"])
def test_bin_matches_oracle(orc, pkg, ctx, case):
    w = CASES[case]
    X = gen.features_host(w)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
    gb = ds.bins[: w.n * ds.ld_bins].view(w.n, ds.ld_bins)[:, : w.m].cpu().numpy()
    np.testing.assert_array_equal(gb.T, bins)


@pytest.mark.parametrize("case,strip", [("C1", 5), ("C3s", 8), ("C2s", 7)])
def test_bin_host_strips_match_oracle(orc, pkg, ctx, case, strip):
    """bin_features_host (column strips uploaded on a copy stream while the previous strip is
    binned) gives the oracle's bins, cuts and nbins; ragged last strip."""
    w = CASES[case]
    X = gen.features_host(w)
    Xh = torch.from_numpy(np.ascontiguousarray(X)).pin_memory()
    ds = pkg.bin_features_host(ctx, Xh, w.B, DEV, strip=strip)
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
    gb = ds.bins[: w.n * ds.ld_bins].view(w.n, ds.ld_bins)[:, : w.m].cpu().numpy()
    np.testing.assert_array_equal(gb.T, bins)


def test_bin_edge_cases(orc, pkg, ctx):
    rng = np.random.default_rng(0)
    n = 9000
    X = np.stack([
        np.zeros(n), np.full(n, -3.5), rng.integers(0, 3, n), rng.normal(size=n),
        np.where(rng.random(n) < 0.5, -0.0, 0.0), rng.integers(0, 300, n),
        np.concatenate([np.zeros(n - 5), rng.normal(size=5)]), np.arange(n)[::-1],
    ], axis=1).astype(np.float32)
    for B in (2, 16, 256):
        ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), B)
        torch.cuda.synchronize()
        cuts, nbins, bins = orc.bin_matrix(X, B)
        np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
        np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
        gb = ds.bins[: n * ds.ld_bins].view(n, ds.ld_bins)[:, : X.shape[1]].cpu().numpy()
        np.testing.assert_array_equal(gb.T, bins)


@pytest.mark.parametrize("n", [1, 2, 3, 7, 257, 8193, 20011])
def test_bin_selection_edge_cases(orc, pkg, ctx, n):
    """Exact order statistics by digit selection: ragged n, exactly B / B+1 distinct values,
    duplicates straddling target ranks, mixed signs, denormals and huge magnitudes."""
    rng = np.random.default_rng(n)
    cols = [
        rng.integers(0, 256, n), rng.integers(0, 257, n),                        # B and B+1 distinct
        np.repeat(rng.normal(size=(n + 9) // 10), 10)[:n],                        # runs of 10 equal values
        rng.normal(size=n) * np.float32(1e-40), rng.normal(size=n) * 1e30,        # denormal / huge
        np.where(rng.random(n) < 0.9, 0.0, rng.normal(size=n)),                   # 90 % zeros
        -np.abs(rng.standard_cauchy(n)), rng.random(n).astype(np.float32) + 1.0,  # heavy tail; one exponent
    ] + [rng.normal(size=n) for _ in range(60)]                                   # > 64 columns: two tiles
    X = np.stack(cols, axis=1).astype(np.float32)
    for B in (2, 255, 256):
        ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), B)
        torch.cuda.synchronize()
        cuts, nbins, bins = orc.bin_matrix(X, B)
        np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
        np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
        gb = ds.bins[: n * ds.ld_bins].view(n, ds.ld_bins)[:, : X.shape[1]].cpu().numpy()
        np.testing.assert_array_equal(gb.T, bins)


# ------------------------------------------------------------ CSC input

def _csc_check(orc, pkg, ctx, X, B):
    values, row_idx, col_ptr = orc.csc_from_dense(X)
    n = X.shape[0]
    ds = pkg.bin_features_csc(ctx, torch.from_numpy(values).to(DEV), torch.from_numpy(row_idx).to(DEV),
                              torch.from_numpy(col_ptr), n, B)
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, B)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
    gb = ds.bins[: n * ds.ld_bins].view(n, ds.ld_bins)[:, : X.shape[1]].cpu().numpy()
    np.testing.assert_array_equal(gb.T, bins)
    return ds


def test_bin_csc_paper_example(orc, pkg, ctx):
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "csc_example.json")))
    for B in (2, 4, 256):
        _csc_check(orc, pkg, ctx, np.array(g["dense"], np.float32), B)


@pytest.mark.parametrize("n,density", [(1, 0.5), (7, 0.3), (5000, 0.19), (40001, 0.05), (40001, 0.9)])
def test_bin_csc_equals_dense(orc, pkg, ctx, n, density):
    rng = np.random.default_rng(n)
    m = 70                                                           # two column tiles
    X = np.where(rng.random((n, m)) < density, rng.normal(size=(n, m)), 0.0).astype(np.float32)
    X[:, 3] = 0.0                                                    # empty column
    X[:, 4] = rng.normal(size=n)                                     # fully dense column
    X[:, 5] = np.where(rng.random(n) < density, -np.abs(rng.normal(size=n)), 0.0)   # zero is the maximum
    X[:, 6] = np.where(rng.random(n) < density, rng.integers(1, 300, n), 0)         # few / many distinct
    for B in (16, 256):
        _csc_check(orc, pkg, ctx, X, B)


def test_bin_csc_explicit_zeros(orc, pkg, ctx):
    # stored 0.0 / -0.0 entries are ordinary values equal to the implicit zeros
    rng = np.random.default_rng(11)
    n, m = 3000, 9
    X = np.where(rng.random((n, m)) < 0.3, rng.normal(size=(n, m)), 0.0).astype(np.float32)
    vals, rows, ptr = [], [], [0]
    for j in range(m):
        keep = np.nonzero((X[:, j] != 0) | (rng.random(n) < 0.2))[0]     # some zeros stored explicitly
        v = X[keep, j].copy()
        v[(v == 0) & (rng.random(len(v)) < 0.5)] = -0.0
        vals.append(v); rows.append(keep.astype(np.int32)); ptr.append(ptr[-1] + len(keep))
    ds = pkg.bin_features_csc(ctx, torch.from_numpy(np.concatenate(vals)).to(DEV),
                              torch.from_numpy(np.concatenate(rows)).to(DEV), torch.tensor(ptr, dtype=torch.int64), n, 256)
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, 256)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), nbins)
    np.testing.assert_array_equal(ds.cuts.cpu().numpy(), cuts)
    gb = ds.bins[: n * ds.ld_bins].view(n, ds.ld_bins)[:, :m].cpu().numpy()
    np.testing.assert_array_equal(gb.T, bins)


def test_bin_csc_mnist_shaped(orc, pkg, ctx):
    w = CASES["C2s"]
    X = gen.features_host(w)
    _csc_check(orc, pkg, ctx, X, w.B)


# ------------------------------------------------------------------------- gradients

@pytest.mark.parametrize("case", ["C1", "C2s"])
def test_grad_matches_oracle(orc, pkg, ctx, case):
    w = CASES[case]
    X, Y = _inputs(w)
    rng = np.random.default_rng(1)
    pred = rng.normal(scale=0.3, size=Y.shape)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), _params(pkg, w), pred=torch.from_numpy(pred).to(DEV))
    ctx.gbdtmo_set_stream(torch.cuda.current_stream().cuda_stream)
    ctx.gbdtmo_grad(b.p, b.y, b.pred, b.q, b.scales, b.state, b.gh)
    torch.cuda.synchronize()
    q = b.q.cpu().numpy().astype(np.float64)
    gh = b.gh.cpu().numpy()
    sc = b.scales.cpu().numpy().astype(np.float64)
    assert np.all(np.log2(sc) == np.round(np.log2(sc)))           # powers of two
    g, h = orc.grad(w.loss, Y.astype(np.float64), pred)
    d = w.d
    gq = q[:, :d] * sc[:d]
    # fp32 arithmetic (2^-23 relative) + fixed-point quantisation (2^-31 P)
    # fp64 arithmetic (~1e-15) + fixed-point quantisation (half a unit of 2^-30 P)
    tol = 1e-14 * np.maximum(np.abs(g), 1.0) + sc[:d] * 0.5
    assert np.all(np.abs(gq - g) <= tol)
    if w.loss == 1:
        hq = q[:, d:] * sc[d:]
        assert np.all(np.abs(hq - h) <= 1e-14 + sc[d:] * 0.5)
    assert np.all(np.abs(q) <= 2 ** 30)
    # the fp64 g (and h) kept for the leaf sums: the oracle's values to fp64 rounding
    np.testing.assert_allclose(gh[:, :d], g, rtol=1e-14, atol=1e-15)
    if w.loss == 1:
        np.testing.assert_allclose(gh[:, d:], h, rtol=1e-14, atol=1e-15)


# ------------------------------------------------------------------------ histograms

@pytest.mark.parametrize("case,hk", [(c, k) for k in (0, 1) for c in ("C1", "C3s", "C5s", "C2s", "C4s")] +
                         [(c, 2) for c in ("C3s", "C5s", "C2s", "C4s")])
def test_histograms_per_level_vs_oracle(orc, pkg, ctx, case, hk):
    """Every level's histograms (built and derived by subtraction) vs the oracle's direct
    per-node histograms over the oracle's node rows; exact on tree-1 dyadic MSE inputs."""
    w = CASES[case]
    X, Y = _inputs(w)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=1, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    rows = node_rows(bins, ref["state"][0], ref["feat"][0], ref["bin"][0], w.n)
    g, h = orc.grad(w.loss, Y.astype(np.float64), np.zeros(Y.shape))
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), _params(pkg, w, T=1), sparse_default=(hk == 0),
                    gmem_max_rows=0, small_max_rows=0, hist_kernel=hk)
    b._apply_options()
    ctx.gbdtmo_grad(b.p, b.y, b.pred, b.q, b.scales, b.state)
    sc = None
    V, B, m, d = b.p.V, w.B, w.m, w.d
    checked = 0
    for lvl in range(w.D):
        b._level(lvl)
        torch.cuda.synchronize()
        if sc is None:
            sc = b.scales.cpu().numpy().astype(np.float64)
        last = lvl == w.D - 1 and lvl > 0      # derived histograms of the last level are never materialised:
        LN = 1 << lvl                          # there only the BUILT child (the smaller, tie -> left) is checked
        LS = LN // 2 if last else LN                      # last level: pair (2s, 2s+1) stored at slot s
        H = b.hist[lvl % 2][: LS * m * V * B].view(LS, m, V, B).transpose(2, 3).cpu().numpy()
        CN = b.cnt[lvl % 2][: LS * m * B].view(LS, m, B).cpu().numpy()
        for slot in range(LN):
            hid = LN - 1 + slot
            if ref["state"][0][hid] != 1:         # only nodes that were searched and split
                continue
            if last:
                par = (hid - 1) // 2
                nl, nr = ref["n_left"][0][par], ref["nrows"][0][par] - ref["n_left"][0][par]
                built_left = nl <= nr
                if (hid == 2 * par + 1) != built_left:
                    continue
            r = rows[hid]
            HG, HH, CNT = orc.build_hist(bins, B, g, h, r)
            hs = slot >> 1 if last else slot
            np.testing.assert_array_equal(CN[hs], CNT)
            gpu_g = H[hs][:, :, :d] * sc[:d]
            AG = np.zeros((m, B, d))
            np.add.at(AG, (np.arange(m)[:, None], bins[:, r]), np.abs(g[r])[None, :, :].repeat(m, 0))
            err = np.abs(gpu_g - HG) / np.maximum(np.maximum(np.abs(HG), AG), 1e-300)
            assert err.max() <= 1e-5, (lvl, slot, err.max())
            if w.loss == 0 and w.index in (1, 3, 5):
                assert np.array_equal(gpu_g, HG), (lvl, slot)      # dyadic tree 1: bit-exact
            if w.loss == 1:
                gpu_h = H[hs][:, :, d:] * sc[d:]
                assert np.all(np.abs(gpu_h - HH) <= 1e-5 * HH + CNT[:, :, None] * 2.0 ** -32)
            checked += 1
    assert checked > 0


# ------------------------------------------------------------------- whole trees

@pytest.mark.parametrize("case,sparse,gmem,small,hk", [
    ("C1", False, 0, 0, 0), ("C2s", False, 0, 0, 0), ("C2s", True, 0, 0, 0), ("C3s", False, 0, 0, 0),
    ("C4s", False, 0, 0, 0), ("C5s", False, 0, 0, 0), ("S300s", False, 0, 0, 0),
    ("C3s", False, 1 << 30, 0, 0), ("C2s", True, 3000, 0, 0), ("C5s", False, 5000, 0, 0),   # global-atomic variant
    ("C1", False, 0, 2000, 0), ("C2s", False, 0, 4000, 0), ("C2s", True, 256, 2500, 0),     # sort-and-segment small nodes
    ("C3s", False, 0, 9000, 0), ("C5s", False, 0, 6000, 0), ("S6s", False, 0, 3000, 0), ("S6s", False, 0, 0, 0),
    ("C1", False, 0, 0, 1), ("C2s", False, 0, 0, 1), ("C3s", False, 0, 0, 1), ("C4s", False, 0, 0, 1),  # diagonal
    ("C5s", False, 0, 0, 1), ("S300s", False, 0, 0, 1), ("C2s", False, 3000, 128, 1),
    ("C2s", False, 0, 0, 2), ("C3s", False, 0, 0, 2), ("C4s", False, 0, 0, 2), ("C5s", False, 0, 0, 2),  # TMA-staged
    ("S300s", False, 0, 0, 2), ("C5s", False, 5000, 0, 2), ("C3s", False, 0, 9000, 2)])
def test_trees_and_predictions_vs_oracle(orc, pkg, ctx, case, sparse, gmem, small, hk):
    w = CASES[case]
    X, Y = _inputs(w)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), _params(pkg, w), sparse_default=sparse, gmem_max_rows=gmem,
                    small_max_rows=small, hist_kernel=hk)
    assert (b.dflt is not None) == (sparse and w.index == 2)     # only the MNIST-shaped data has dominant bins
    b.fit()
    torch.cuda.synchronize()
    for t in range(w.T):
        gt = to_np(b.trees[t])
        diffs = compare_trees(gt, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
        assert not diffs, (t, diffs)
        leaves = gt["node_state"] == 2
        np.testing.assert_allclose(gt["leaf"][leaves], ref["leaf"][t][leaves], rtol=1e-5, atol=1e-6)
        split = gt["node_state"] == 1
        np.testing.assert_allclose(gt["gain"][split], ref["gain"][t][split], rtol=1e-6)
    err = np.max(np.abs(b.pred.cpu().numpy() - ref["pred"]))
    assert err <= 1e-4, err


def test_partition_rows_are_stable_and_complete(orc, pkg, ctx):
    """After each level the row list of every node equals the oracle's stable partition."""
    w = CASES["C3s"]
    X, Y = _inputs(w)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=1, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    rows = node_rows(bins, ref["state"][0], ref["feat"][0], ref["bin"][0], w.n)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), _params(pkg, w, T=1))
    b.step()
    torch.cuda.synchronize()
    NH = b.NH
    rl_t = torch.empty(w.n, dtype=torch.int32, device=DEV)
    nid_t = torch.empty(w.n, dtype=torch.int32, device=DEV)
    beg_t = torch.empty(NH, dtype=torch.int32, device=DEV)
    end_t = torch.empty(NH, dtype=torch.int32, device=DEV)
    ctx.gbdtmo_rows_export(b.p, b.state, w.D, rl_t, nid_t, beg_t, end_t)
    torch.cuda.synchronize()
    rl, nid, begin, end = (x.cpu().numpy() for x in (rl_t, nid_t, beg_t, end_t))
    for hid, r in rows.items():
        if ref["state"][0][hid] == 2:
            np.testing.assert_array_equal(rl[begin[hid]:end[hid]], r)
            assert np.all(nid[r] == hid)


def test_two_shards_equal_one(orc, pkg, ctx):
    """Feature partitioning emulated on one GPU: two shards exchange through
    MAX(keys) and SUM(xchg) exactly as the NCCL path does; trees and predictions must equal the
    single-shard run bit for bit, and the fp64 oracle's trees (exact splits, predictions <= 1e-4)."""
    w = CASES["C3s"]
    X, Y = _inputs(w)
    Yd = torch.from_numpy(Y).to(DEV)
    P = _params(pkg, w, T=2)
    full = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B), Yd.clone(), P,
                       gmem_max_rows=0, small_max_rows=0)
    full.fit()
    half = w.m // 2 + 3
    shards = []
    for f0, f1 in ((0, half), (half, w.m)):
        ds = pkg.bin_features(ctx, torch.from_numpy(np.ascontiguousarray(X[:, f0:f1])).to(DEV), w.B,
                              f_begin=f0, m_global=w.m)
        shards.append(pkg.Booster(ctx, ds, Yd.clone(), P, gmem_max_rows=0, small_max_rows=0))
    for t in range(P.T):
        for s in shards:
            s._apply_options()
            ctx.gbdtmo_grad(s.p, s.y, s.pred, s.q, s.scales, s.state, s.gh)
        for lvl in range(P.D):
            cur, par = lvl % 2, (lvl - 1) % 2
            for s in shards:
                ph = s.hist[par] if lvl else None
                pc = s.cnt[par] if lvl else None
                ctx.gbdtmo_build_hist(s.p, lvl, s.ds.bins, s.dflt, s.q, s.state, s.hist[cur], s.cnt[cur])
                ctx.gbdtmo_find_split(s.p, lvl, s.ds.nbins, s.dflt, s.scales, s.state, s.hist[cur], s.cnt[cur], ph, pc,
                                      s.keys)
            kmax = torch.maximum(shards[0].keys, shards[1].keys)
            for s in shards:
                s.keys.copy_(kmax)
                ph = s.hist[par] if lvl else None
                pc = s.cnt[par] if lvl else None
                ctx.gbdtmo_split_record(s.p, lvl, s.ds.bins, s.dflt, s.q, s.scales, s.state, s.hist[cur], s.cnt[cur], ph, pc,
                                        s.keys, s.xchg)
            xs = shards[0].xchg + shards[1].xchg
            for s in shards:
                s.xchg.copy_(xs)
                ctx.gbdtmo_partition(s.p, lvl, s.state, s.xchg)
        for s in shards:
            ctx.gbdtmo_leaf_values(s.p, s.scales, s.state, s.leaf, s.gh)
            ctx.gbdtmo_update_pred(s.p, s.state, s.leaf, s.pred)
            s.trees.append(s.export())
    torch.cuda.synchronize()
    for t in range(P.T):
        a = to_np(full.trees[t])
        for s in shards:
            bb = to_np(s.trees[t])
            for k in ("node_state", "feature", "bin", "n_rows", "n_left"):
                np.testing.assert_array_equal(a[k], bb[k])
            np.testing.assert_array_equal(a["leaf"], bb["leaf"])
    for s in shards:
        assert torch.equal(full.pred, s.pred)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=P.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    for t in range(P.T):
        assert not compare_trees(to_np(shards[0].trees[t]), ref["state"][t], ref["feat"][t], ref["bin"][t],
                                 ref["nrows"][t])
    assert np.max(np.abs(shards[1].pred.cpu().numpy() - ref["pred"])) <= 1e-4


def test_graph_replay_equals_eager(pkg, ctx):
    w = CASES["C1"]
    X, Y = _inputs(w)
    P = _params(pkg, w, T=3)
    a = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B), torch.from_numpy(Y).to(DEV), P)
    a.fit()
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B), torch.from_numpy(Y).to(DEV), P)
    b.capture()          # captures one tree; its warm-up tree runs outside the graph and is not kept
    assert not b.trees and not bool(b.pred.any())       # (the warm-up leaves pred untouched)
    for _ in range(3):
        b.step_graph()
    torch.cuda.synchronize()
    assert torch.equal(a.pred, b.pred)
    for ta, tb in zip(a.trees, b.trees):          # records exported after each replay
        for k in ("node_state", "feature", "bin", "n_rows", "n_left", "leaf", "threshold"):
            assert torch.equal(ta[k], tb[k]), k


@pytest.mark.parametrize("case", ["C1", "C3s", "C2s"])
def test_public_train_from_host_matches_oracle(orc, pkg, ctx, case):
    """The public entry point bench.py's e2e leg times: pkg.train() from pinned HOST X / Y (strip
    upload overlapped with binning, then the trees): trees equal the oracle's, predictions within
    the north star's 1e-4."""
    w = CASES[case]
    X, Y = _inputs(w)
    Xh = torch.from_numpy(np.ascontiguousarray(X)).pin_memory()
    Yh = torch.from_numpy(np.ascontiguousarray(Y)).pin_memory()
    P = _params(pkg, w)
    b = pkg.train(Xh, Yh, P, device=DEV, ctx=ctx)
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    for t in range(w.T):
        st = b.trees[t]["node_state"].cpu().numpy()
        assert np.array_equal(st, ref["state"][t]), t
        split = st == 1
        assert np.array_equal(b.trees[t]["feature"].cpu().numpy()[split], ref["feat"][t][split])
        assert np.array_equal(b.trees[t]["bin"].cpu().numpy()[split], ref["bin"][t][split])
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) < 1e-4


@pytest.mark.parametrize("case,sparse,kernel", [("C3s", False, None), ("C2s", True, None), ("C2s", False, 1),
                                               ("C1", False, None)])
def test_cached_root_counts_equal_accumulated(pkg, ctx, case, sparse, kernel):
    """gbdtmo_set_root_counts: trees 2.. take the root's count histogram from the cache instead of
    accumulating it; trees, leaves and predictions are identical (both shared-memory variants and
    the sparsity-aware path, where find_split completes the cached default-bin counts)."""
    w = CASES[case]
    X, Y = _inputs(w)
    P = _params(pkg, w, T=3)
    out = []
    for cache in (False, True):
        ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
        b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), P, sparse_default=sparse, hist_kernel=kernel,
                        cache_root_counts=cache)
        b.fit()
        torch.cuda.synchronize()
        assert (b.root_cnt is not None) == cache
        out.append(b)
    a, c = out
    assert torch.equal(a.pred, c.pred)
    for ta, tc in zip(a.trees, c.trees):
        for k in ("node_state", "feature", "bin", "n_rows", "n_left", "leaf"):
            assert torch.equal(ta[k], tc[k]), k


@pytest.mark.parametrize("case,sparse", [("C3s", False), ("C5s", False), ("C2s", True), ("C4s", False)])
def test_packed_bins_layout_and_equivalence(orc, pkg, ctx, case, sparse):
    """gbdtmo_pack_bins writes the documented [tile][row][8] layout (checked against a numpy
    re-layout of the oracle's bins), and training from the packed copy gives exactly the trees and
    predictions of the row-major path (integer histograms: bit-equal), which equal the oracle's."""
    w = CASES[case]
    X, Y = _inputs(w)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)          # bins [m][n]
    ds = pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B)
    yd = torch.from_numpy(Y).to(DEV)
    kw = dict(sparse_default=sparse, gmem_max_rows=0, small_max_rows=0, hist_kernel=0)
    bp = pkg.Booster(ctx, ds, yd, _params(pkg, w), packed_bins=True, **kw)
    torch.cuda.synchronize()
    n, m, k = w.n, w.m, 6                                # K = 16 tiles of 6 features at B = 256 (hist_config)
    nt = (m + k - 1) // k
    ng = (nt + 3) // 4                                   # groups of 4 tiles per row
    assert bp.packed.numel() == ng * n * 4 * 8
    want = np.zeros((ng, n, 4, 8), dtype=np.uint8)
    for f in range(m):
        t = f // k
        want[t // 4, :, t % 4, f % k] = bins[f]
    np.testing.assert_array_equal(bp.packed.view(ng, n, 4, 8).cpu().numpy(), want)
    br = pkg.Booster(ctx, ds, yd, _params(pkg, w), packed_bins=False, **kw)
    bp.fit()
    br.fit()
    torch.cuda.synchronize()
    assert torch.equal(bp.pred, br.pred)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    for t in range(w.T):
        a, b = to_np(bp.trees[t]), to_np(br.trees[t])
        for key in ("node_state", "feature", "bin", "n_rows"):
            np.testing.assert_array_equal(a[key], b[key])
        assert not compare_trees(a, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
    assert np.max(np.abs(bp.pred.cpu().numpy() - ref["pred"])) <= 1e-4


@pytest.mark.parametrize("case", ["C2s", "C3s", "S300s"])
def test_leaf_values_fp64_exact_vs_fixed_point(orc, pkg, ctx, case):
    """gbdtmo_leaf_values with gh sums g, h in fp64 over each leaf's rows (R17): the leaves equal
    the oracle's to fp64 rounding (rtol 1e-10 + 1e-13), also for confident softmax leaves whose tiny G
    sits at the fixed point's resolution floor n_leaf 2^-31 (R29); the fixed-point path
    (gh = NULL) stays within that floor of them."""
    w = CASES[case].scaled(T=4)
    X, Y = _inputs(w)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).to(DEV), w.B), torch.from_numpy(Y).to(DEV),
                    _params(pkg, w))
    for t in range(w.T):
        b._tree()                                    # leaf values from fp64 row sums (the default)
        torch.cuda.synchronize()
        fixed = torch.empty_like(b.leaf)
        # (the prediction has been updated: recompute the fixed-point leaves from the same state)
        ctx.gbdtmo_leaf_values(b.p, b.scales, b.state, fixed)
        torch.cuda.synchronize()
        rec = to_np(b.export())
        assert not compare_trees(rec, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
        lv = rec["node_state"] == 2
        np.testing.assert_allclose(rec["leaf"][lv], ref["leaf"][t][lv], rtol=1e-10, atol=1e-13)
        # |dG| <= n P_g 2^-31, |dH| <= n P_h 2^-31 (softmax P_g = 1, P_h = 1/4; MSE H is exact) ->
        # |dv| <= (|dG| + |v| |dH|) / lambda
        pg = 1.0 if w.loss == 1 else 64.0
        floor = rec["n_rows"][lv][:, None] * 2.0 ** -31 * (pg + np.abs(rec["leaf"][lv])) / w.lam * 2
        assert np.all(np.abs(fixed.cpu().numpy()[lv] - rec["leaf"][lv]) <= floor + 1e-9 * np.abs(rec["leaf"][lv]))
