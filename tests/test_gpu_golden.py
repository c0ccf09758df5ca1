"""North-star free-running gate at BASELINE.json's full sizes: T = 10 trees trained independently by
the CUDA path (through the C ABI, in the launch configuration bench.py times: measured variant
table, cached root counts, packed bins) and by the fp64 oracle, from the same seeded inputs.

  - every tree: node states, row counts (exact), split (feature, bin) (exact), gains rtol 1e-5,
    leaf values rtol 1e-5 (Algorithm 1; Eq. 3);
  - yhat after 10 trees within 1e-4 absolute (north star) on the golden's row sample, and the
    per-output sums over all n rows within n * 1e-4;
  - binning: nbins and a digest of the cuts equal the oracle's.

C2-C5 compare with tests/golden/<cfg>_T10.npz, written by tools/make_golden.py from oracle/ only
(the oracle needs minutes to hours per config).  C1 runs the oracle in the test.
"""
import hashlib
import os

import numpy as np
import pytest
import torch

from gen import gen
from tests.gpu_helpers import compare_trees, to_np

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_icpp_liupw25_b200 as pkg
    pkg.lib()
    return pkg


def _golden(name, T=10):
    path = os.path.join(GOLDEN, f"{name}_T{T}.npz")
    if not os.path.exists(path):
        pytest.skip(f"{path} not generated (tools/make_golden.py {name})")
    return dict(np.load(path))


def _device_inputs(pkg, ctx, w):
    """The workload in HBM exactly as bench.py builds it (C5: X generated on the device)."""
    dev = torch.device("cuda:0")
    if w.index == 5:
        X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
        gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                        torch.cuda.current_stream().cuda_stream)
        Y = gen.targets_host(w)
    else:
        Xh = gen.features_host(w)
        Y = gen.targets_host(w, Xh)
        X = torch.from_numpy(Xh).to(dev)
        del Xh
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    torch.cuda.empty_cache()
    return ds, torch.from_numpy(Y).to(dev)


def _first_diff(trees, ref, T):
    """First tree whose structure differs from the oracle's (None: all equal)."""
    for t in range(T):
        gt = to_np(trees[t])
        try:
            if compare_trees(gt, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t]):
                return t
        except AssertionError:
            return t
    return None


def _check_trees(trees, ref, T, leaf_rtol=1e-5):
    for t in range(T):
        gt = to_np(trees[t])
        diffs = compare_trees(gt, ref["state"][t], ref["feat"][t], ref["bin"][t], ref["nrows"][t])
        assert not diffs, f"tree {t}: splits differ from the oracle at heap nodes {diffs}"
        split = gt["node_state"] == 1
        np.testing.assert_array_equal(gt["n_left"][split], ref["n_left"][t][split])
        # gains are differences of Eq. (3) terms computed from histograms held to 1e-5: after the
        # first softmax trees (tiny hessians, P_h = 1/4 quantisation) they drift by ~2.5e-6
        # relative, the split choice itself staying exact (R28)
        np.testing.assert_allclose(gt["gain"][split], ref["gain"][t][split], rtol=1e-5)
        leaves = gt["node_state"] == 2
        if "leaf_scale" in ref:
            # leaves inherit the histogram metric, |v - v*| <= 1e-5 max(|v*|, AG / (H + lambda))
            # (AG = sum |g| over the leaf's rows: softmax leaf sums G cancel, the quantisation error does not)
            v, vr, sc = gt["leaf"][leaves], ref["leaf"][t][leaves], ref["leaf_scale"][t][leaves]
            err = np.abs(v - vr) / np.maximum(np.abs(vr), sc)
            assert err.max() <= leaf_rtol, (t, float(err.max()))
        else:
            np.testing.assert_allclose(gt["leaf"][leaves], ref["leaf"][t][leaves], rtol=leaf_rtol, atol=1e-7)


# configs whose oracle is cheap enough to re-run tie-locked from the first tie on the GPU box
TIE_LOCK = {"C2", "C3", "C4"}


@pytest.mark.parametrize("name", ["C2", "C3", "C4", "C5"])
def test_ten_trees_full_size_vs_oracle_golden(orc, pkg, name):
    g = _golden(name)
    w = gen.WORKLOADS[name]
    T = int(g["T"])
    ctx = pkg.Context(0)
    ds, Y = _device_inputs(pkg, ctx, w)
    np.testing.assert_array_equal(ds.nbins.cpu().numpy(), g["nbins"])
    assert hashlib.sha256(ds.cuts.cpu().numpy().tobytes()).digest() == g["cuts_digest"].tobytes()
    P = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, P)
    b.fit()
    torch.cuda.synchronize()
    t0 = _first_diff(b.trees, g, T)
    if t0 is not None:
        # a near-tie (north star: splits may differ where gains tie within 1e-6 relative): the oracle
        # replays trees 0..t0-1 from the golden and runs on tie-locked
        assert name in TIE_LOCK, f"{name}: tree {t0} differs from the golden; no tie-locked re-run for this size"
        from tests.gpu_helpers import tie_locked_oracle
        from tools.make_golden import oracle_bins
        _check_trees(b.trees, g, t0)
        _, nbins, bins = oracle_bins(w)
        X = gen.features_host(w) if w.index == 2 else None
        y = gen.targets_host(w, X).astype(np.float64)
        pred0 = _replay_pred(orc, bins, g, t0, w)
        pred, ties = tie_locked_oracle(orc, bins, nbins, w.B, y, w.loss, pred0, [to_np(x) for x in b.trees], t0, T,
                                       w.D, w.lam, w.gamma, w.lr, w.min_node)
        print(f"{name}: ties (tree, node, gpu, oracle, rel gap): {ties}")
        assert ties, "trees differ but no tie was found"
        err = np.max(np.abs(b.pred.cpu().numpy() - pred))
        assert err <= 1e-4, f"max |yhat - tie-locked oracle| after {T} trees = {err:.3e}"
        return
    _check_trees(b.trees, g, T)
    rows = torch.from_numpy(g["sample_rows"]).cuda()
    ps = b.pred[rows].cpu().numpy()
    err = np.max(np.abs(ps - g["pred_sample"]))
    assert err <= 1e-4, f"max |yhat - oracle| on {len(rows)} sampled rows after {T} trees = {err:.3e}"
    s = b.pred.sum(0).cpu().numpy()
    assert np.all(np.abs(s - g["pred_sum"]) <= w.n * 1e-4)
    s2 = (b.pred * b.pred).sum(0).cpu().numpy()
    assert np.all(np.abs(s2 - g["pred_sumsq"]) <= 1e-6 * np.abs(g["pred_sumsq"]) + w.n * 1e-4)


def _replay_pred(orc, bins, g, t_end, w):
    """yhat before tree t_end from the golden's own trees (oracle_partition + oracle_update_pred)."""
    pred = np.zeros((w.n, w.d))
    for t in range(t_end):
        rows = {0: np.arange(w.n, dtype=np.int32)}
        for h in range(g["state"].shape[1]):
            if h not in rows:
                continue
            if g["state"][t][h] == 1:
                rows[2 * h + 1], rows[2 * h + 2] = orc.partition(bins, rows[h], int(g["feat"][t][h]), int(g["bin"][t][h]))
            elif g["state"][t][h] == 2:
                orc.update_pred(pred, rows[h], g["leaf"][t][h])
    return pred


def test_ten_trees_c1_vs_oracle(orc, pkg):
    """C1 at 10 trees (its config says 5; the gate is at 10), oracle in the test."""
    w = gen.WORKLOADS["C1"].scaled(T=10)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    ctx = pkg.Context(0)
    ds = pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B)
    P = pkg.Params(loss=w.loss, T=10, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).cuda(), P)
    b.fit()
    torch.cuda.synchronize()
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=10, D=w.D, lam=w.lam, gamma=w.gamma,
                    lr=w.lr, min_node=w.min_node)
    _check_trees(b.trees, ref, 10)
    assert np.max(np.abs(b.pred.cpu().numpy() - ref["pred"])) <= 1e-4
