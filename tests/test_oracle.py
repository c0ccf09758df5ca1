"""Pins of the CPU oracle against things other than itself (no GPU needed).

Each test names the PAPER.md passage / DESIGN.md reading it pins and the independent
evidence used: closed forms, finite differences, invariants, brute force with a
different algorithm, numerical minimisation of Eq. (2), or a library special case
(scikit-learn CART boosting for MSE, Python's stable sort for the partition).
"""
import numpy as np
import pytest
from scipy.optimize import minimize

from gen import gen


# ------------------------------------------------------------------ binning (R14)

def test_bin_permutation_closed_form(orc):
    # x a permutation of 0..n-1 with B | n, n > B: bin(x) = floor(x * B / n)   (R14 rule ii)
    n, B = 1024, 64
    rng = np.random.default_rng(0)
    X = rng.permutation(n).astype(np.float32).reshape(n, 1)
    cuts, nbins, bins = orc.bin_matrix(X, B)
    assert nbins[0] == B
    np.testing.assert_array_equal(bins[0], (X[:, 0].astype(np.int64) * B) // n)


def test_bin_few_distinct_is_rank(orc):
    # <= B distinct values: one bin per distinct value, bin = rank among distinct values (R14 rule i)
    rng = np.random.default_rng(1)
    vals = np.sort(rng.normal(size=40)).astype(np.float32)
    X = rng.choice(vals, size=(3000, 1)).astype(np.float32)
    cuts, nbins, bins = orc.bin_matrix(X, 64)
    distinct = np.unique(X[:, 0])
    assert nbins[0] == len(distinct)
    np.testing.assert_array_equal(bins[0], np.searchsorted(distinct, X[:, 0]))


def test_bin_properties_random(orc):
    rng = np.random.default_rng(2)
    n, m, B = 5000, 6, 32
    X = rng.normal(size=(n, m)).astype(np.float32)
    X[:, 3] = np.round(X[:, 3] * 3)           # ties
    X[:, 4] = 7.0                             # constant column -> 1 bin
    cuts, nbins, bins = orc.bin_matrix(X, B)
    assert nbins[4] == 1 and np.all(bins[4] == 0)
    for f in range(m):
        assert 1 <= nbins[f] <= B
        order = np.argsort(X[:, f], kind="stable")
        assert np.all(np.diff(bins[f][order].astype(int)) >= 0)          # monotone in x
        assert bins[f].max() == nbins[f] - 1
        c = cuts[f][: nbins[f] - 1]
        assert np.all(np.diff(c) > 0) and np.all(np.isinf(cuts[f][nbins[f] - 1:]))
        # bin(x) = #{cuts <= x}, checked with numpy's searchsorted (right side)
        np.testing.assert_array_equal(bins[f], np.searchsorted(c, X[:, f], side="right"))
    # distinct continuous values: every bin holds >= floor(n/B) rows
    counts = np.bincount(bins[0], minlength=nbins[0])
    assert counts.min() >= n // B


def test_bin_mnist_shaped_column(orc):
    # C2 column shape: 81% zeros, rest integers 1..255 -> rule (i), 256 bins, hot bin 0 (DESIGN.md Inputs)
    w = gen.WORKLOADS["C2"]
    X = gen.features_host(w, 0, 60000, 0, 2)
    cuts, nbins, bins = orc.bin_matrix(X, 256)
    assert list(nbins) == [256, 256]
    frac0 = np.mean(bins[0] == 0)
    assert 0.79 < frac0 < 0.83


# ------------------------------------------------------- CSC storage

def _golden(name):
    import json
    import os
    return json.load(open(os.path.join(os.path.dirname(__file__), "golden", name)))


def test_csc_matches_paper_worked_example(orc):
    # PAPER.md:181-201 prints the dense rows of x0..x4 and their CSC arrays (tests/golden/csc_example.json)
    g = _golden("csc_example.json")
    X = np.array(g["dense"], np.float32)
    values, row_idx, col_ptr = orc.csc_from_dense(X)
    assert values.tolist() == g["values"]
    assert row_idx.tolist() == g["row_indices"]
    assert col_ptr.tolist() == g["col_pointers"]
    back = orc.dense_from_csc(np.array(g["values"]), np.array(g["row_indices"]), np.array(g["col_pointers"]), 5)
    np.testing.assert_array_equal(back, X)


def test_csc_round_trip_and_scipy(orc):
    # independent library special case: scipy.sparse's CSC of the same matrix
    import scipy.sparse as sp
    rng = np.random.default_rng(3)
    X = np.where(rng.random((300, 17)) < 0.8, 0.0, rng.normal(size=(300, 17))).astype(np.float32)
    X[:, 5] = 0.0                                        # an empty column
    values, row_idx, col_ptr = orc.csc_from_dense(X)
    ref = sp.csc_matrix(X)
    ref.sort_indices()
    np.testing.assert_array_equal(col_ptr, ref.indptr)
    np.testing.assert_array_equal(row_idx, ref.indices)
    np.testing.assert_array_equal(values, ref.data)
    np.testing.assert_array_equal(orc.dense_from_csc(values, row_idx, col_ptr, 300), X)


# ------------------------------------------------------------------- gradients

def _mse_loss(y, p):
    return np.sum((p - y) ** 2)


def _ce_loss(y, p):
    z = p - p.max()
    return -np.sum(y * (z - np.log(np.sum(np.exp(z)))))


@pytest.mark.parametrize("loss", [0, 1])
def test_grad_finite_differences(orc, loss):
    # g = dl/dyhat, h = d2l/dyhat_k^2, checked by central differences of the loss itself
    rng = np.random.default_rng(3)
    n, d = 7, 5
    if loss == 0:
        y = rng.normal(size=(n, d)); f = _mse_loss
    else:
        y = np.eye(d)[rng.integers(0, d, n)]; f = _ce_loss
    p = rng.normal(size=(n, d))
    g, h = orc.grad(loss, y, p)
    eps = 1e-4
    for i in range(n):
        for k in range(d):
            e = np.zeros(d); e[k] = eps
            fp, f0, fm = f(y[i], p[i] + e), f(y[i], p[i]), f(y[i], p[i] - e)
            assert abs((fp - fm) / (2 * eps) - g[i, k]) < 1e-7 * max(1, abs(g[i, k]))
            assert abs((fp - 2 * f0 + fm) / eps ** 2 - h[i, k]) < 2e-4


def test_softmax_invariants(orc):
    rng = np.random.default_rng(4)
    n, d = 500, 10
    y = np.eye(d)[rng.integers(0, d, n)]
    p = rng.normal(scale=3, size=(n, d))
    g, h = orc.grad(1, y, p)
    assert np.max(np.abs(g.sum(axis=1))) < 1e-14            # sum_k (p_k - y_k) = 0
    assert np.all(h > 0) and np.all(h <= 0.25)


# ------------------------------------------------------------------ histograms

def _tiny(seed, n=300, m=5, d=3, B=16, loss=1):
    rng = np.random.default_rng(seed)
    X = rng.normal(size=(n, m)).astype(np.float32)
    X[:, 1] = rng.integers(0, 6, n)
    cuts, nbins, bins = oracle_bin_cache(X, B)
    if loss == 1:
        y = np.eye(d)[rng.integers(0, d, n)]
    else:
        y = rng.normal(size=(n, d))
    p = rng.normal(size=(n, d))
    return X, bins, nbins, y, p


def oracle_bin_cache(X, B):
    from oracle import oracle
    return oracle.bin_matrix(X, B)


def test_hist_matches_numpy_scatter_and_invariants(orc):
    X, bins, nbins, y, p = _tiny(5)
    g, h = orc.grad(1, y, p)
    rows = np.random.default_rng(6).permutation(len(X))[:211].astype(np.int32)
    HG, HH, CNT = orc.build_hist(bins, 16, g, h, rows)
    m, B, d = HG.shape
    for f in range(m):
        ref = np.zeros((B, d)); np.add.at(ref, bins[f][rows], g[rows])       # library scatter-add
        np.testing.assert_allclose(HG[f], ref, rtol=0, atol=1e-12)
        np.testing.assert_array_equal(CNT[f], np.bincount(bins[f][rows], minlength=B))
        np.testing.assert_allclose(HG[f].sum(0), g[rows].sum(0), atol=1e-12)  # sum over bins = node G
        np.testing.assert_allclose(HH[f].sum(0), h[rows].sum(0), atol=1e-12)
        assert CNT[f].sum() == len(rows)
        # softmax: sum_k HG[f][b][k] = 0 for every bin
        assert np.max(np.abs(HG[f].sum(1))) < 1e-12


def test_hist_parent_equals_children_exactly_dyadic(orc):
    # North-star invariant parent = left + right, bit-exact on dyadic inputs (R24)
    rng = np.random.default_rng(7)
    n, m, d, B = 4000, 4, 3, 32
    X = rng.normal(size=(n, m)).astype(np.float32)
    cuts, nbins, bins = orc.bin_matrix(X, B)
    y = np.round(rng.normal(size=(n, d)) * 65536) / 65536
    g, h = orc.grad(0, y, np.zeros((n, d)))
    rows = np.arange(n, dtype=np.int32)
    P = orc.build_hist(bins, B, g, h, rows)
    left, right = orc.partition(bins, rows, 2, 13)
    L = orc.build_hist(bins, B, g, h, left)
    R = orc.build_hist(bins, B, g, h, right)
    for a, b, c in zip(P, L, R):
        assert np.array_equal(a, b + c)
    np.testing.assert_array_equal(P[1], 2.0 * P[2][:, :, None].repeat(d, 2))   # MSE: HH = 2 CNT


# ---------------------------------------------------------------- split search

def _exhaustive_best(X, g, h, rows, lam, min_node):
    """Raw-threshold enumeration: every distinct value v of every feature, left = {x < v},
    sums straight from the rows, objective from Eq. (2) minimised numerically per side."""
    best = None
    for f in range(X.shape[1]):
        xs = X[rows, f]
        for v in np.unique(xs)[1:]:
            L = rows[xs < v]; R = rows[xs >= v]
            if len(L) < min_node or len(R) < min_node:
                continue
            gain = _objective(g[rows], h[rows], lam) - _objective(g[L], h[L], lam) - _objective(g[R], h[R], lam)
            if best is None or gain > best[0] + 1e-9 * abs(best[0]):
                best = (gain, f, v)
    return best


def _objective(g, h, lam):
    """L*(v) of Eq. (2) with diagonal H, by numerical minimisation."""
    G, H = g.sum(0), h.sum(0)
    fun = lambda v: float(G @ v + 0.5 * np.sum(H * v * v) + 0.5 * lam * v @ v)
    jac = lambda v: G + H * v + lam * v
    r = minimize(fun, np.zeros(len(G)), jac=jac, method="BFGS", options={"gtol": 1e-13, "maxiter": 500})
    return r.fun


@pytest.mark.parametrize("seed,loss", [(10, 1), (11, 0), (12, 1)])
def test_split_vs_exhaustive_enumeration(orc, seed, loss):
    X, bins, nbins, y, p = _tiny(seed, n=150, m=4, d=3, B=256, loss=loss)   # B > n: bins = distinct values
    g, h = orc.grad(loss, y, p)
    rows = np.arange(len(X), dtype=np.int32)
    lam, min_node = 1.0, 5
    HG, HH, CNT = orc.build_hist(bins, 256, g, h, rows)
    sp = orc.find_split(HG, HH, CNT, nbins, g.sum(0), h.sum(0), len(rows), lam, min_node, want_all=True)
    gain, f, v = _exhaustive_best(X, g, h, rows, lam, min_node)
    assert sp["valid"]
    assert abs(sp["gain"] - gain) <= 1e-7 * abs(gain)
    # the oracle's winner is the same raw threshold (or ties within the 1e-6 band)
    cuts, _, _ = orc.bin_matrix(X, 256)
    thr = cuts[sp["feature"]][sp["bin"]]
    if (sp["feature"], thr) != (f, v):
        assert abs(sp["gain"] - gain) <= 1e-6 * abs(gain)
    # Eq. (3) closed form at every candidate equals the numerically minimised objective difference
    allg = sp["all_gains"]
    fb = [(ff, bb) for ff in range(allg.shape[0]) for bb in range(allg.shape[1]) if np.isfinite(allg[ff, bb])]
    for ff, bb in fb[:: max(1, len(fb) // 12)]:
        L = rows[bins[ff][rows] <= bb]; R = rows[bins[ff][rows] > bb]
        ref = _objective(g, h, lam) - _objective(g[L], h[L], lam) - _objective(g[R], h[R], lam)
        assert abs(allg[ff, bb] - ref) <= 1e-8 * max(1.0, abs(ref))


def test_single_output_reduces_to_textbook_gain(orc):
    # d = 1: GBDT-SO is a special case of GBDT-MO; XGBoost-style gain
    # 1/2 [GL^2/(HL+l) + GR^2/(HR+l) - G^2/(H+l)] -- compare against the d-output gain of a
    # problem whose d outputs are identical copies: gain_d = d * gain_1.
    rng = np.random.default_rng(13)
    GL, HL, G, H = rng.normal(), rng.uniform(1, 5), rng.normal(), rng.uniform(6, 9)
    g1 = orc.gain([GL], [HL], [G], [H], 1.0)
    g4 = orc.gain([GL] * 4, [HL] * 4, [G] * 4, [H] * 4, 1.0)
    assert abs(g4 - 4 * g1) < 1e-12 * abs(g4)


def test_mse_lambda0_gain_is_sse_reduction(orc):
    # MSE, lambda = 0: Eq. (3) = sum_k SSE reduction (multi-output CART criterion)
    rng = np.random.default_rng(14)
    r = rng.normal(size=(60, 3)); mask = rng.random(60) < 0.4
    g = -2 * r; h = 2 * np.ones_like(r)
    gain = orc.gain(g[mask].sum(0), h[mask].sum(0), g.sum(0), h.sum(0), 0.0)
    sse = lambda a: np.sum((a - a.mean(0)) ** 2)
    assert abs(gain - (sse(r) - sse(r[mask]) - sse(r[~mask]))) < 1e-10 * sse(r)


def test_leaf_value_minimises_eq2(orc):
    rng = np.random.default_rng(15)
    g = rng.normal(size=(30, 4)); h = rng.uniform(0.1, 1, size=(30, 4)); lam = 0.7
    v = orc.leaf_value(g.sum(0), h.sum(0), lam, 1.0)
    G, H = g.sum(0), h.sum(0)
    r = minimize(lambda x: float(G @ x + 0.5 * np.sum(H * x * x) + 0.5 * lam * x @ x), np.zeros(4),
                 jac=lambda x: G + H * x + lam * x, method="BFGS", options={"gtol": 1e-14})
    np.testing.assert_allclose(v, r.x, rtol=1e-7, atol=1e-9)


def test_partition_is_stable_sort(orc):
    X, bins, nbins, y, p = _tiny(16)
    rows = np.random.default_rng(17).permutation(len(X))[:200].astype(np.int32)
    left, right = orc.partition(bins, rows, 0, 5)
    key = (bins[0][rows] > 5).astype(int)
    ref = rows[np.argsort(key, kind="stable")]                 # library stable sort
    np.testing.assert_array_equal(np.concatenate([left, right]), ref)
    assert np.all(bins[0][left] <= 5) and np.all(bins[0][right] > 5)


# ------------------------------------------------ whole model: sklearn special case

@pytest.mark.parametrize("D,T", [(4, 5), (3, 3)])
def test_mse_model_equals_sklearn_residual_trees(orc, D, T):
    """MSE, lambda = gamma = 0, lr = 1, base 0, min_node 20: T trees of Algorithm 1 =
    T multi-output CART regressors (max_depth D, min_samples_leaf 20) fitted to residuals
    on the bin matrix (R1, R2, R4, R9, R10, R11)."""
    from sklearn.tree import DecisionTreeRegressor
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    res = orc.train(bins, nbins, w.B, y, loss=0, T=T, D=D, lam=0.0, gamma=0.0, lr=1.0, min_node=20)
    Xb = bins.T.astype(np.float64)
    pred = np.zeros_like(y)
    for t in range(T):
        tree = DecisionTreeRegressor(max_depth=D, min_samples_leaf=20, random_state=0).fit(Xb, y - pred)
        pred += tree.predict(Xb)
        root_f = tree.tree_.feature[0]
        assert res["state"][t][0] == 1 and res["feat"][t][0] == root_f
        assert res["bin"][t][0] == int(np.floor(tree.tree_.threshold[0]))
    assert np.max(np.abs(res["pred"] - pred)) < 1e-9


@pytest.mark.parametrize("T,D,lam,lr", [(5, 4, 1.0, 0.5), (4, 3, 0.5, 0.7), (3, 5, 2.5, 0.3)])
def test_softmax_two_class_model_equals_sklearn_hgb(orc, T, D, lam, lr):
    """Whole softmax model pinned through its 2-class special case.  With d = 2, softmax CE with
    the diagonal Hessian (R12, R13) gives g_1 = -g_0 = p_1 - y_1 and h_0 = h_1 = p_1 (1 - p_1),
    p_1 = sigmoid(z_1 - z_0); Eq. (3) summed over k is then 2 G^2 / (H + lambda), so every split
    is the binary-logistic split, and the margin z_1 - z_0 moves by 2 x (-lr G / (H + lambda))
    per leaf.  That is scikit-learn's HistGradientBoostingClassifier (binary log
    loss, same g/h) at learning_rate 2 lr, l2 = lambda, max_depth D, min_samples_leaf 20,
    unlimited leaves (level-wise = leaf-wise here, R6), baseline log-odds 0 (balanced labels,
    R10), fitted on the bin matrix (R14: integer bins bin to themselves).  sklearn keeps g/h
    in float32, hence the 1e-6 tolerance; lambda stays >= 0.5 because with lambda -> 0 pure
    nodes drive p to 0/1, where sklearn's float32 hessians underflow and its fixed
    min_hessian_to_split = 1e-3 (not a model parameter of the paper) starts to bind."""
    from sklearn.ensemble import HistGradientBoostingClassifier
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    n = X.shape[0]
    score = np.tanh(1.3 * X[:, 0] - X[:, 3]) + 0.5 * X[:, 5] * X[:, 2] + 0.3 * X[:, 7]
    lab = np.zeros(n, np.int64)
    lab[np.argsort(score, kind="stable")[n // 2:]] = 1          # exactly n/2 positives
    Y = np.stack([1.0 - lab, lab.astype(np.float64)], 1)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    assert all(len(np.unique(bins[f])) == nbins[f] for f in range(w.m))   # every bin present
    res = orc.train(bins, nbins, w.B, Y, loss=1, T=T, D=D, lam=lam, gamma=0.0, lr=lr, min_node=20)
    Xb = bins.T.astype(np.float64)
    clf = HistGradientBoostingClassifier(learning_rate=2 * lr, max_iter=T, max_leaf_nodes=None, max_depth=D,
                                         min_samples_leaf=20, l2_regularization=lam, early_stopping=False,
                                         max_bins=255).fit(Xb, lab)
    raw = clf._raw_predict(Xb)[:, 0]
    margin = res["pred"][:, 1] - res["pred"][:, 0]
    assert np.max(np.abs(raw - margin)) < 1e-6 * max(1.0, np.max(np.abs(margin)))
    np.testing.assert_allclose(res["pred"][:, 0], -res["pred"][:, 1], rtol=0, atol=1e-12)
    for t in range(T):
        nodes = clf._predictors[t][0].nodes
        assert int(res["feat"][t][0]) == int(nodes[0]["feature_idx"])
        assert int(res["bin"][t][0]) == int(nodes[0]["bin_threshold"])
        assert int((res["state"][t] == 2).sum()) == int(nodes["is_leaf"].sum())


def test_train_softmax_invariants(orc):
    # softmax model, d > 2: structural invariants (the model as a whole is pinned at d = 2 above;
    # the per-step pins cover general d)
    w = gen.WORKLOADS["C2"].scaled(n=3000, m=20, T=3, D=3)
    X = gen.features_host(w, 0, w.n, 0, w.m)
    y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    res = orc.train(bins, nbins, w.B, y, loss=1, T=3, D=3, lam=1.0, gamma=0.0, lr=1.0, min_node=20)
    for t in range(3):
        st, nr, nl = res["state"][t], res["nrows"][t], res["n_left"][t]
        assert st[0] != 0 and nr[0] == w.n
        for i in range(len(st)):
            if st[i] == 1:
                assert nr[2 * i + 1] == nl[i] and nr[2 * i + 2] == nr[i] - nl[i]
                assert nl[i] >= 20 and nr[i] - nl[i] >= 20
        leaves = st == 2
        assert nr[leaves].sum() == w.n
        # softmax leaf values sum to ~0 over classes (sum_k G_k = 0, h symmetric-ish not required) -> finite
        assert np.all(np.isfinite(res["leaf"][t][leaves]))
    # training reduces the loss
    p0 = np.zeros_like(y)
    def ce(p):
        z = p - p.max(1, keepdims=True)
        return -np.mean(np.sum(y * (z - np.log(np.exp(z).sum(1, keepdims=True))), 1))
    assert ce(res["pred"]) < ce(p0)


# ------------------------------------------------ tie-break (R16) and the split rule gamma (R2, R3)

def _gap_column_problem(n_per=30):
    """Column 0: integers 0..39 (n_per rows each), rows with x in 15..24 removed from the node, so
    bins 15..24 are EMPTY in the node; targets depend on x >= 20.  Column 1: noise.  Column 2: an
    exact copy of column 0 (same bins, same gains at every candidate)."""
    rng = np.random.default_rng(21)
    x = np.repeat(np.arange(40), n_per).astype(np.float32)
    X = np.stack([x, rng.normal(size=len(x)).astype(np.float32), x], 1)
    y = np.where(x >= 20, 1.0, -1.0)[:, None] + 0.01 * rng.normal(size=(len(x), 1))
    rows = np.nonzero((x < 15) | (x > 24))[0].astype(np.int32)
    return X, y, rows


def test_tie_break_smallest_feature_then_smallest_bin(orc):
    """R16: max gain, then smallest feature, then smallest bin.  The best partition of the node
    ({x <= 14} vs {x >= 25}) is produced by candidates b = 14..24 of column 0 (bins 15..24 are
    empty in the node: bit-identical gains) and by the same 11 candidates of its copy, column 2.
    The rule must pick (0, 14); a '>=' slip in the scan picks (2, 24), a feature-only slip (0, 24)."""
    X, y, rows = _gap_column_problem()
    cuts, nbins, bins = orc.bin_matrix(X, 64)
    assert nbins[0] == 40 and nbins[2] == 40
    g, h = orc.grad(0, y, np.zeros_like(y))
    HG, HH, CNT = orc.build_hist(bins, 64, g, h, rows)
    assert np.all(CNT[0][15:25] == 0)
    sp = orc.find_split(HG, HH, CNT, nbins, g[rows].sum(0), h[rows].sum(0), len(rows), 1.0, 5, want_all=True)
    allg = sp["all_gains"]
    assert len(set(allg[0, 14:25].tolist())) == 1 and np.array_equal(allg[0], allg[2])   # the 22-way tie
    assert np.max(allg[np.isfinite(allg)]) == allg[0, 14]                              # it is the maximum
    assert (sp["feature"], sp["bin"]) == (0, 14)
    # independent check of the tie's partition: raw-threshold enumeration (no histograms)
    gain, f, v = _exhaustive_best(X, g, h, rows, 1.0, 5)
    assert f == 0 and v == 25.0 and abs(gain - sp["gain"]) <= 1e-7 * abs(gain)


def test_tie_break_in_whole_model_prefers_lower_duplicate(orc):
    """R16 through Algorithm 1: with columns 3 and 7 exact copies of columns 0 and 2, no split of
    any tree may use column 3 or 7 (each of their candidates ties with the copy's lower index)."""
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    X = X.copy()
    X[:, 3] = X[:, 0]
    X[:, 7] = X[:, 2]
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    res = orc.train(bins, nbins, w.B, y, loss=0, T=5, D=4, lam=1.0, gamma=0.0, lr=1.0, min_node=20)
    used = res["feat"][res["state"] == 1]
    assert np.any(np.isin(used, [0, 2]))           # the informative originals are used ...
    assert not np.any(np.isin(used, [3, 7]))       # ... never their later copies


def test_gamma_split_rule_strict(orc):
    """R2/R3 (Alg. 1 lines 14-17, gamma = 'threshold for valid splits',
    PAPER.md:122): a node splits iff its best gain > gamma.  gamma = the root's best gain exactly
    -> the root is a leaf; gamma one ulp below -> it splits."""
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    r0 = orc.train(bins, nbins, w.B, y, T=1, D=3, gamma=0.0)
    best = r0["gain"][0][0]
    assert r0["state"][0][0] == 1 and best > 0
    r_eq = orc.train(bins, nbins, w.B, y, T=1, D=3, gamma=best)
    assert r_eq["state"][0][0] == 2 and np.all(r_eq["state"][0][1:] == 0)
    r_lo = orc.train(bins, nbins, w.B, y, T=1, D=3, gamma=np.nextafter(best, 0.0))
    assert r_lo["state"][0][0] == 1


def test_gamma_infinite_gives_root_leaves_closed_form(orc):
    """gamma larger than any gain: every tree is one root leaf, so for MSE (g = 2(yhat - y), h = 2)
    yhat_{t+1} = yhat_t - lr * 2 sum(yhat_t - y) / (2 n + lambda) for every row:
    a closed-form recursion computed here in numpy."""
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64) + 0.75          # off-centre, so leaves are non-zero
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    lam, lr, T = 3.0, 0.4, 4
    res = orc.train(bins, nbins, w.B, y, T=T, D=4, lam=lam, lr=lr, gamma=1e300)
    c = np.zeros(w.d)
    for t in range(T):
        assert res["state"][t][0] == 2 and np.all(res["state"][t][1:] == 0)
        c = c - lr * 2.0 * (w.n * c - y.sum(0)) / (2.0 * w.n + lam)
    np.testing.assert_allclose(res["pred"], np.broadcast_to(c, y.shape), rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("frac", [0.05, 0.1, 0.3])
def test_gamma_every_node_by_exhaustive_enumeration(orc, frac):
    """gamma > 0 against raw-threshold enumeration (no histograms): every split node's gain exceeds
    gamma, and every leaf that could have split (depth < D, >= 2 min_node rows) has no raw
    threshold with gain > gamma (up to 1e-9 relative)."""
    X, bins, nbins, y, p = _tiny(31, n=240, m=3, d=2, B=256, loss=0)
    y = y + 0.2 * X[:, :1].astype(np.float64)
    g0, h0 = orc.grad(0, y, np.zeros_like(y))
    root_best = _exhaustive_best(X, g0, h0, np.arange(len(X), dtype=np.int32), 1.0, 10)[0]
    gamma, D, mn = frac * root_best, 4, 10
    res = orc.train(bins, nbins, 256, y, T=1, D=D, lam=1.0, gamma=gamma, min_node=mn)
    from tests.gpu_helpers import node_rows
    rows = node_rows(bins, res["state"][0], res["feat"][0], res["bin"][0], len(X))
    n_leaf_checked = 0
    for hid, r in rows.items():
        st = res["state"][0][hid]
        depth = int(np.floor(np.log2(hid + 1)))
        if st == 1:
            assert res["gain"][0][hid] > gamma
        elif st == 2 and depth < D and len(r) >= 2 * mn:
            best = _exhaustive_best(X, g0, h0, r.astype(np.int32), 1.0, mn)
            assert best is None or best[0] <= gamma * (1 + 1e-9)
            n_leaf_checked += 1
    assert n_leaf_checked > 0 and np.any(res["state"][0] == 1)


# ------------------------------------------------------------------ inference

def test_predict_walk_equals_incremental_training_prediction(orc):
    """oracle_predict walks every tree from the root on RAW feature values; on the training rows it
    must reproduce oracle_train's prediction, which never walks a tree (rows carry their leaf,
    PAPER.md:164) -- two different computations of the same model output."""
    for w, loss in ((gen.WORKLOADS["C1"].scaled(T=6), 0), (gen.WORKLOADS["C2"].scaled(n=3000, m=30, T=3, D=4), 1)):
        X = gen.features_host(w)
        y = gen.targets_host(w, X).astype(np.float64)
        cuts, nbins, bins = orc.bin_matrix(X, w.B)
        res = orc.train(bins, nbins, w.B, y, loss=loss, T=w.T, D=w.D, lr=0.7)
        p = orc.predict(X, cuts, nbins, w.B, res, w.D)
        np.testing.assert_allclose(p, res["pred"], rtol=0, atol=1e-12)


def test_predict_unseen_rows_equals_sklearn_tree_predict(orc):
    """MSE, lambda = 0, lr = 1: each oracle tree is a CART regressor on the bin matrix (pinned above);
    on UNSEEN rows the oracle walk over raw values must equal sklearn's tree.predict on the rows'
    bins (bin(x) from searchsorted on the training cuts)."""
    from sklearn.tree import DecisionTreeRegressor
    w = gen.WORKLOADS["C1"]
    X = gen.features_host(w)
    y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    T, D = 4, 4
    res = orc.train(bins, nbins, w.B, y, loss=0, T=T, D=D, lam=0.0, lr=1.0, min_node=20)
    Xu = gen.features_host(gen.WORKLOADS["C1"].scaled(n=5000), r0=2000, nr=3000)      # rows never trained on
    Xu = Xu * 1.3 + 0.1                                                               # incl. out-of-range values
    Bu = np.stack([np.searchsorted(cuts[f][: nbins[f] - 1], Xu[:, f], side="right") for f in range(w.m)], 1)
    Xb = bins.T.astype(np.float64)
    pred_tr = np.zeros_like(y)
    pred_u = np.zeros((len(Xu), w.d))
    for t in range(T):
        tree = DecisionTreeRegressor(max_depth=D, min_samples_leaf=20, random_state=0).fit(Xb, y - pred_tr)
        pred_tr += tree.predict(Xb)
        pred_u += tree.predict(Bu.astype(np.float64))
    p = orc.predict(Xu, cuts, nbins, w.B, res, D)
    np.testing.assert_allclose(p, pred_u, rtol=0, atol=1e-9)
