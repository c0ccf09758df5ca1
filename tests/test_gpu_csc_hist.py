"""NEXT-1: histograms built from the CSC non-zeros (gbdtmo_build_hist_csc, §3.2)
vs the oracle.  The zero bin of every feature is recovered from the node totals by the split
search (reading R25), so the trees must equal the oracle's dense-bin trees: exact states, row
counts and (f, b), leaves and predictions to the usual bars; exact ties resolved tie-locked (R30)."""
import dataclasses

import numpy as np
import pytest
import torch

from gen import gen
from tests.gpu_helpers import compare_trees, tie_locked_oracle, to_np

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_icpp_liupw25_b200 as pkg
    pkg.lib()
    return pkg


@pytest.fixture(scope="module")
def ctx(pkg):
    return pkg.Context(0)


def _sparse_inputs(case):
    if case == "C2s":      # MNIST-shaped pixels: 81% zeros, softmax
        w = gen.WORKLOADS["C2"].scaled(n=20_000, m=64, T=3, D=6)
        X = gen.features_host(w)
        Y = gen.targets_host(w, X)
    elif case == "C3s":    # regression features with 70% of the entries zeroed, MSE
        w = gen.WORKLOADS["C3"].scaled(n=40_000, m=24, T=3, D=6)
        X = gen.features_host(w)
        Y = gen.targets_host(w, X)
        keep = gen.uniform_host(w.seed, 77, 0, X.size).reshape(X.shape) < 0.3
        X = np.where(keep, X, 0.0).astype(np.float32)
    else:                  # d = 1, B = 16, small nodes searched from rows on top
        w = dataclasses.replace(gen.WORKLOADS["C1"], B=16, T=3)
        X = gen.features_host(w)
        Y = gen.targets_host(w, X)
        X = np.where(np.abs(X) < 0.6, 0.0, X).astype(np.float32)
        Y = np.ascontiguousarray(Y[:, :1])
        w = dataclasses.replace(w, d=1)
    return w, X, Y


@pytest.mark.parametrize("case,small,levels", [("C2s", 0, None), ("C2s", 512, None), ("C2s", 512, 3), ("C3s", 0, None),
                                               ("C3s", 0, 2), ("C1", 0, None), ("C1", 300, None)])
def test_csc_histogram_trees_vs_oracle(orc, pkg, ctx, case, small, levels):
    w, X, Y = _sparse_inputs(case)
    assert (X == 0).mean() > 0.2
    values, row_idx, col_ptr = orc.csc_from_dense(X)
    ds = pkg.bin_features_csc(ctx, torch.from_numpy(values).to(DEV), torch.from_numpy(row_idx).to(DEV),
                              torch.from_numpy(col_ptr), X.shape[0], w.B)
    assert ds.csc_nnz == len(values)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    zb = ds.csc_zbin.cpu().numpy()
    np.testing.assert_array_equal(zb, [int(np.sum(cuts[f] <= 0.0)) for f in range(X.shape[1])])
    y = Y.astype(np.float64)
    ref = orc.train(bins, nbins, w.B, y, loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma, lr=w.lr,
                    min_node=w.min_node)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, torch.from_numpy(np.ascontiguousarray(Y)).to(DEV), P, csc_hist=True, small_max_rows=small,
                    csc_levels=levels)
    b.fit()
    torch.cuda.synchronize()
    trees = [to_np(t) for t in b.trees]
    for t in range(w.T):
        try:
            differs = bool(compare_trees(trees[t], ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t]))
        except AssertionError:          # a different split moved rows
            differs = True
        if differs:
            pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, np.zeros_like(y), trees, 0, w.T, w.D,
                                           w.lam, w.gamma, w.lr, w.min_node)
            assert ties
            assert np.max(np.abs(b.pred.cpu().numpy() - pred)) <= 1e-4
            return
        lv = trees[t]["node_state"] == 2
        np.testing.assert_allclose(trees[t]["leaf"][lv], ref["leaf"][t][lv], rtol=1e-5, atol=1e-7)
        sp = trees[t]["node_state"] == 1
        np.testing.assert_allclose(trees[t]["gain"][sp], ref["gain"][t][sp], rtol=1e-6)
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4


def test_csc_histogram_edge_cases(orc, pkg, ctx):
    """No stored entries at all (every feature constant 0: the root stays a leaf, as in the oracle),
    and one column holding every row (no implicit zeros) next to empty columns."""
    w = dataclasses.replace(gen.WORKLOADS["C1"], B=16, T=2, D=3)
    X0 = gen.features_host(w)
    Y = gen.targets_host(w, X0)
    for X in (np.zeros_like(X0), np.concatenate([X0[:, :1] + 10.0, np.zeros_like(X0[:, 1:])], axis=1)):
        values, row_idx, col_ptr = orc.csc_from_dense(X)
        ds = pkg.bin_features_csc(ctx, torch.from_numpy(values).to(DEV), torch.from_numpy(row_idx).to(DEV),
                                  torch.from_numpy(col_ptr), X.shape[0], w.B)
        cuts, nbins, bins = orc.bin_matrix(X, w.B)
        ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                        lr=w.lr, min_node=w.min_node)
        P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
        b = pkg.Booster(ctx, ds, torch.from_numpy(Y).to(DEV), P, csc_hist=True)
        b.fit()
        torch.cuda.synchronize()
        for t in range(w.T):
            assert not compare_trees(to_np(b.trees[t]), ref["state"][t], ref["feat"][t], ref["bin"][t],
                                     ref["nrows"][t])
        assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4
