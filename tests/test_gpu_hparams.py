"""Hyper-parameter grid on the GPU path vs the oracle (VERDICT r1 "Hyper-parameter coverage"):
lambda (R1) in {0, 0.5, 2.5}, gamma (Alg. 1 "threshold for valid splits",
PAPER.md:122; R2/R3) in {0, 0.3 x the root's best gain}, learning rate (R9) in
{0.1, 1}, minimum instances per node (R4) in {1, 5, 100}, d = 1 (GBDT-SO as a
special case), softmax with d = 2, and B in {2, 16} bins.  Trees must equal the
oracle's (exact states, row counts, (f, b)), leaves rtol 1e-5, predictions within 1e-4 after T
trees, for the default and the diagonal histogram kernels."""
import dataclasses

import numpy as np
import pytest
import torch

from gen import gen
from tests.gpu_helpers import compare_trees, tie_locked_oracle, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_icpp_liupw25_b200 as pkg
    pkg.lib()
    return pkg


@pytest.fixture(scope="module")
def ctx(pkg):
    return pkg.Context(0)


BASE = {
    "C1": gen.WORKLOADS["C1"],
    "C3s": gen.WORKLOADS["C3"].scaled(n=60_000, m=24, T=3, D=6),
    "C2s": gen.WORKLOADS["C2"].scaled(n=16_000, m=48, T=3, D=5),
}


def _inputs(case, d=None, B=None):
    w = BASE[case]
    if B is not None:
        w = dataclasses.replace(w, B=B)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    if d is not None and d != w.d:
        if w.loss == 1:                  # softmax with d classes: fold the labels (label mod d)
            lab = np.argmax(Y, axis=1) % d
            Y = np.eye(d, dtype=np.float32)[lab]
        else:                            # MSE: the first d outputs
            Y = np.ascontiguousarray(Y[:, :d])
        w = dataclasses.replace(w, d=d)
    return w, X, Y


def _run(orc, pkg, ctx, w, X, Y, lam, gamma_frac, lr, min_node, hk, **kw):
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    gamma = 0.0
    if gamma_frac:
        r0 = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=1, D=1, lam=lam, gamma=0.0, lr=lr,
                       min_node=min_node)
        gamma = gamma_frac * r0["gain"][0][0]
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=lam, gamma=gamma, lr=lr,
                    min_node=min_node)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=lam, gamma=gamma, lr=lr, min_node=min_node)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(np.ascontiguousarray(Y)).cuda(), P, hist_kernel=hk, **kw)
    b.fit()
    torch.cuda.synchronize()
    n_leaf_gamma = 0
    for t in range(w.T):
        gt = to_np(b.trees[t])
        diffs = compare_trees(gt, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
        assert not diffs, (t, diffs)
        lv = gt["node_state"] == 2
        np.testing.assert_allclose(gt["leaf"][lv], ref["leaf"][t][lv], rtol=1e-5, atol=1e-7)
        sp = gt["node_state"] == 1
        np.testing.assert_allclose(gt["gain"][sp], ref["gain"][t][sp], rtol=1e-6)
        assert np.all(gt["gain"][sp] > gamma)
        n_leaf_gamma += int(lv.sum())
    err = np.max(np.abs(b.pred.cpu().numpy() - ref["pred"]))
    assert err <= 1e-4, err
    return ref


def _differs(tree, ref, t):
    """True where tree t differs from the oracle's (a different split moves rows: compare_trees asserts)."""
    try:
        return bool(compare_trees(tree, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t]))
    except AssertionError:
        return True


GRID = [
    # case, d, B, lambda, gamma_frac, lr, min_node
    ("C1", None, None, 0.0, 0.0, 1.0, 20),
    ("C1", None, None, 0.5, 0.0, 0.1, 5),
    ("C1", None, None, 2.5, 0.3, 1.0, 1),
    ("C1", 1, None, 1.0, 0.0, 1.0, 20),          # d = 1: single-output GBDT
    ("C1", 1, 2, 0.0, 0.0, 0.1, 5),              # d = 1, two bins
    ("C1", None, 16, 1.0, 0.3, 0.1, 100),
    ("C1", None, 2, 2.5, 0.0, 1.0, 1),
    ("C3s", None, None, 0.0, 0.0, 0.1, 100),
    ("C3s", None, None, 2.5, 0.3, 1.0, 5),
    ("C3s", None, 16, 0.5, 0.0, 1.0, 1),
    ("C3s", 1, None, 1.0, 0.3, 0.1, 20),
    ("C3s", None, 2, 1.0, 0.0, 1.0, 20),
    ("C2s", None, None, 0.5, 0.0, 0.1, 5),       # softmax
    ("C2s", None, None, 2.5, 0.3, 1.0, 100),
    ("C2s", 2, None, 1.0, 0.0, 1.0, 20),         # softmax, d = 2 (binary)
    ("C2s", 2, 16, 0.5, 0.3, 0.1, 1),
    ("C2s", None, 2, 1.0, 0.0, 1.0, 5),
]


@pytest.mark.parametrize("hk", [0, 1])
@pytest.mark.parametrize("case,d,B,lam,gfrac,lr,mn", GRID)
def test_hparam_grid_vs_oracle(orc, pkg, ctx, case, d, B, lam, gfrac, lr, mn, hk):
    w, X, Y = _inputs(case, d, B)
    _run(orc, pkg, ctx, w, X, Y, lam, gfrac, lr, mn, hk)


@pytest.mark.parametrize("cg", [1, 2, 4, 8])
@pytest.mark.parametrize("case,d,lam,gfrac,mn", [("C3s", None, 1.0, 0.0, 20), ("C3s", 3, 0.5, 0.3, 5),
                                                   ("C2s", None, 1.0, 0.0, 20), ("C2s", 2, 2.5, 0.0, 1),
                                                   ("C1", None, 0.0, 0.3, 5)])
def test_channel_split_search_vs_oracle(orc, pkg, ctx, case, d, lam, gfrac, mn, cg):
    """GBDTMO_OPT_FS_CHANNEL_GROUPS forced to 1 (half-row kernel), 2 and 4 (k_find_split_c: the
    Eq. (3) sum over outputs split over warp pairs, CG > d clamped): trees, gains, leaves
    and predictions equal the oracle's at every level, incl. derived children and the last level."""
    w, X, Y = _inputs(case, d)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    y = Y.astype(np.float64)
    gamma = 0.0
    if gfrac:
        r0 = orc.train(bins, nbins, w.B, y, loss=w.loss, T=1, D=1, lam=lam, gamma=0.0, lr=1.0, min_node=mn)
        gamma = gfrac * r0["gain"][0][0]
    ref = orc.train(bins, nbins, w.B, y, loss=w.loss, T=w.T, D=w.D, lam=lam, gamma=gamma, lr=1.0, min_node=mn)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=lam, gamma=gamma, lr=1.0, min_node=mn)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
    b = pkg.Booster(ctx, ds, torch.from_numpy(np.ascontiguousarray(Y)).cuda(), P, fs_channel_groups=cg)
    b.fit()
    torch.cuda.synchronize()
    trees = [to_np(t) for t in b.trees]
    for t in range(w.T):
        if _differs(trees[t], ref, t):
            # a near-tie (min_node 1, binary softmax: symmetric candidates): the tie-locked oracle
            # (R30) adopts the GPU's choice where the gains tie within 1e-6 and must agree elsewhere
            pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, np.zeros_like(y), trees, 0, w.T,
                                           w.D, lam, gamma, 1.0, mn)
            assert ties
            assert np.max(np.abs(b.pred.cpu().numpy() - pred)) <= 1e-4
            return
        sp = trees[t]["node_state"] == 1
        np.testing.assert_allclose(trees[t]["gain"][sp], ref["gain"][t][sp], rtol=1e-6)
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4


def test_gamma_makes_leaves_where_oracle_does(orc, pkg, ctx):
    """gamma between the gains of the tree's splits: some nodes that split at gamma = 0 become
    leaves, on both sides identically (the strict 'gain > gamma' rule, R2/R3)."""
    w, X, Y = _inputs("C3s")
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    r0 = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=0, T=1, D=w.D)
    gains = np.sort(r0["gain"][0][r0["state"][0] == 1])
    gfrac = gains[len(gains) // 2] / r0["gain"][0][0]          # the median split gain
    ref = _run(orc, pkg, ctx, dataclasses.replace(w, T=2), X, Y, 1.0, gfrac, 1.0, 20, 0)
    assert (ref["state"][0] == 1).sum() < (r0["state"][0] == 1).sum()


def test_near_tie_duplicate_features(orc, pkg, ctx):
    """Exact ties (duplicated columns: every candidate of the copy ties with the original) resolve
    to the smallest feature on the GPU as in the oracle (R16), through the packed-key argmax, for
    every histogram kernel and the sort-and-segment small-node search."""
    w, X, Y = _inputs("C3s")
    X = X.copy()
    X[:, 9] = X[:, 0]
    X[:, 17] = X[:, 3]
    X[:, 23] = X[:, 1]
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=0, T=w.T, D=w.D)
    used = ref["feat"][ref["state"] == 1]
    assert np.any(np.isin(used, [0, 1, 3])) and not np.any(np.isin(used, [9, 17, 23]))
    P = pkg.Params(loss=0, T=w.T, D=w.D, B=w.B)
    for kw in (dict(hist_kernel=0), dict(hist_kernel=1), dict(hist_kernel=2), dict(small_max_rows=6000),
               dict(gmem_max_rows=1 << 30)):
        ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
        b = pkg.Booster(ctx, ds, torch.from_numpy(Y).cuda(), P, **kw)
        b.fit()
        torch.cuda.synchronize()
        for t in range(w.T):
            assert not compare_trees(to_np(b.trees[t]), ref["state"][t], ref["feat"][t], ref["bin"][t],
                                     ref["nrows"][t]), (kw, t)


@pytest.mark.parametrize("case,D", [("C3s", 10), ("C1", 9)])
def test_deep_trees_vs_oracle(orc, pkg, ctx, case, D):
    """Depth 10 (the last level keeps one histogram slot per sibling pair, R31): trees and
    predictions equal the oracle's; min_node 5 so the deep levels really split."""
    w = dataclasses.replace(BASE[case], D=D, T=2)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ref = _run(orc, pkg, ctx, w, X, Y, 1.0, 0.0, 1.0, 5, 0)
    assert np.any(ref["state"][:, (1 << (D - 1)) - 1:(1 << D) - 1] == 1)      # splits at the last level


def test_small_option_ignored_beyond_64_channels(orc, pkg, ctx):
    """GBDTMO_OPT_SMALL_MAX_ROWS on a softmax problem with 2 x 40 channels: the small-node path (its
    split records cover at most 64 channels) must stay off, and the trees equal the oracle's."""
    w = gen.sweep(40, n=4_000, m=16, T=2, D=4)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P,
                    small_max_rows=2000)
    b.fit()
    torch.cuda.synchronize()
    trees = [to_np(t) for t in b.trees]
    if any(_differs(trees[t], ref, t) for t in range(w.T)):
        # near-ties among 40 classes' Eq. (3) sums: the tie-locked oracle (R30) must accept every difference
        y = Y.astype(np.float64)
        pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, np.zeros_like(y), trees, 0, w.T, w.D,
                                       w.lam, w.gamma, w.lr, w.min_node)
        assert ties
        assert np.max(np.abs(b.pred.cpu().numpy() - pred)) <= 1e-4
        return
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4
