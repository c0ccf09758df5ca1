"""ctypes wrapper of the plain C fp64 oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  The product package never imports this module.
Every function forwards to the C function of the same name; see oracle.h for the
PAPER.md passage each one follows.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

LOSS_MSE, LOSS_SOFTMAX = 0, 1


class Split(C.Structure):
    _fields_ = [("valid", C.c_int32), ("feature", C.c_int32), ("bin", C.c_int32),
                ("pad", C.c_int32), ("gain", C.c_double), ("n_left", C.c_int64)]


class Params(C.Structure):
    _fields_ = [("loss", C.c_int32), ("T", C.c_int32), ("D", C.c_int32), ("min_node", C.c_int32),
                ("lambda_", C.c_double), ("gamma", C.c_double), ("lr", C.c_double)]


def build(force: bool = False) -> str:
    so = os.path.join(_HERE, "liboracle.so")
    src = os.path.join(_HERE, "oracle.c")
    hdr = os.path.join(_HERE, "oracle.h")
    if force or not os.path.exists(so) or os.path.getmtime(so) < max(os.path.getmtime(src), os.path.getmtime(hdr)):
        cmd = f"gcc -O2 -fopenmp -fPIC -shared -ffp-contract=off -o {so} {src} -lm"
        if os.system(cmd) != 0:
            raise RuntimeError("oracle build failed: " + cmd)
    return so


def lib():
    global _LIB
    if _LIB is None:
        # ORACLE_LIB: an instrumented build of the same source (tools/oracle_asan.sh), test infrastructure only
        _LIB = C.CDLL(os.environ.get("ORACLE_LIB") or build())
        P = C.c_void_p
        i32, i64, f64 = C.c_int32, C.c_int64, C.c_double
        _LIB.oracle_bin.argtypes = [P, i64, i32, i64, i32, P, P, P]
        _LIB.oracle_csc_from_dense.argtypes = [P, i64, i32, i64, P, P, P]
        _LIB.oracle_dense_from_csc.argtypes = [P, P, P, i64, i32, i64, P]
        _LIB.oracle_grad.argtypes = [i32, P, P, i64, i32, P, P]
        _LIB.oracle_build_hist.argtypes = [P, i64, i32, i32, P, P, i32, P, i64, P, P, P]
        _LIB.oracle_gain.argtypes = [P, P, P, P, i32, f64]
        _LIB.oracle_gain.restype = f64
        _LIB.oracle_find_split.argtypes = [P, P, P, i32, P, i32, i32, P, P, i64, f64, i64, C.POINTER(Split), P]
        _LIB.oracle_partition.argtypes = [P, i64, P, i64, i32, i32, P, P, C.POINTER(i64)]
        _LIB.oracle_leaf_value.argtypes = [P, P, i32, f64, f64, P]
        _LIB.oracle_update_pred.argtypes = [P, i32, P, i64, P]
        _LIB.oracle_train.argtypes = [P, i64, i32, P, i32, P, i32, C.POINTER(Params), P,
                                      P, P, P, P, P, P, P]
        _LIB.oracle_predict.argtypes = [P, i64, i64, P, P, i32, i32, i32, i32, P, P, P, P, P]
        _LIB.oracle_num_threads.restype = i32
    return _LIB


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def bin_matrix(X, B):
    """X float32 [n][m] -> (cuts f32 [m][B-1], nbins i32 [m], bins_cm u16 [m][n])."""
    X = _c(X, np.float32)
    n, m = X.shape
    cuts = np.empty((m, B - 1), np.float32)
    nbins = np.empty(m, np.int32)
    bins = np.empty((m, n), np.uint16)
    lib().oracle_bin(_p(X), n, m, m, B, _p(cuts), _p(nbins), _p(bins))
    return cuts, nbins, bins


def csc_from_dense(X):
    """X float32 [n][m] -> (values f32 [nnz], row_idx i32 [nnz], col_ptr i64 [m+1])."""
    X = _c(X, np.float32)
    n, m = X.shape
    col_ptr = np.empty(m + 1, np.int64)
    lib().oracle_csc_from_dense(_p(X), n, m, m, None, None, _p(col_ptr))
    nnz = int(col_ptr[m])
    values = np.empty(nnz, np.float32)
    row_idx = np.empty(nnz, np.int32)
    lib().oracle_csc_from_dense(_p(X), n, m, m, _p(values), _p(row_idx), _p(col_ptr))
    return values, row_idx, col_ptr


def dense_from_csc(values, row_idx, col_ptr, n):
    values = _c(values, np.float32); row_idx = _c(row_idx, np.int32); col_ptr = _c(col_ptr, np.int64)
    m = len(col_ptr) - 1
    X = np.empty((n, m), np.float32)
    lib().oracle_dense_from_csc(_p(values), _p(row_idx), _p(col_ptr), n, m, m, _p(X))
    return X


def grad(loss, y, pred):
    y = _c(y, np.float64); pred = _c(pred, np.float64)
    n, d = y.shape
    g = np.empty((n, d)); h = np.empty((n, d))
    lib().oracle_grad(loss, _p(y), _p(pred), n, d, _p(g), _p(h))
    return g, h


def build_hist(bins_cm, B, g, h, rows):
    bins_cm = _c(bins_cm, np.uint16); g = _c(g, np.float64); h = _c(h, np.float64)
    rows = _c(rows, np.int32)
    m, n = bins_cm.shape
    d = g.shape[1]
    HG = np.empty((m, B, d)); HH = np.empty((m, B, d)); CNT = np.empty((m, B), np.int64)
    lib().oracle_build_hist(_p(bins_cm), n, m, B, _p(g), _p(h), d, _p(rows), len(rows),
                            _p(HG), _p(HH), _p(CNT))
    return HG, HH, CNT


def gain(GL, HL, G, H, lam):
    a = [_c(v, np.float64) for v in (GL, HL, G, H)]
    return float(lib().oracle_gain(*[_p(v) for v in a], len(a[0]), lam))


def find_split(HG, HH, CNT, nbins, G, H, cnt, lam, min_node, want_all=False):
    HG = _c(HG, np.float64); HH = _c(HH, np.float64); CNT = _c(CNT, np.int64)
    nbins = _c(nbins, np.int32); G = _c(G, np.float64); H = _c(H, np.float64)
    m, B, d = HG.shape
    out = Split()
    allg = np.empty((m, B)) if want_all else None
    lib().oracle_find_split(_p(HG), _p(HH), _p(CNT), m, _p(nbins), B, d, _p(G), _p(H), int(cnt),
                            lam, int(min_node), C.byref(out), _p(allg))
    res = dict(valid=bool(out.valid), feature=out.feature, bin=out.bin, gain=out.gain, n_left=out.n_left)
    if want_all:
        res["all_gains"] = allg
    return res


def partition(bins_cm, rows, f, b):
    bins_cm = _c(bins_cm, np.uint16); rows = _c(rows, np.int32)
    m, n = bins_cm.shape
    left = np.empty(len(rows), np.int32); right = np.empty(len(rows), np.int32)
    nl = C.c_int64(0)
    lib().oracle_partition(_p(bins_cm), n, _p(rows), len(rows), f, b, _p(left), _p(right), C.byref(nl))
    return left[:nl.value].copy(), right[:len(rows) - nl.value].copy()


def leaf_value(G, H, lam, lr):
    G = _c(G, np.float64); H = _c(H, np.float64)
    v = np.empty(len(G))
    lib().oracle_leaf_value(_p(G), _p(H), len(G), lam, lr, _p(v))
    return v


def update_pred(pred, rows, v):
    assert pred.dtype == np.float64 and pred.flags.c_contiguous
    rows = _c(rows, np.int32); v = _c(v, np.float64)
    lib().oracle_update_pred(_p(pred), pred.shape[1], _p(rows), len(rows), _p(v))


def train(bins_cm, nbins, B, y, loss=LOSS_MSE, T=5, D=4, lam=1.0, gamma=0.0, lr=1.0, min_node=20,
          pred=None):
    """Algorithm 1.  Returns dict of pred and per-tree heap arrays."""
    bins_cm = _c(bins_cm, np.uint16); nbins = _c(nbins, np.int32); y = _c(y, np.float64)
    m, n = bins_cm.shape
    d = y.shape[1]
    slots = (1 << (D + 1)) - 1
    pred = np.zeros((n, d)) if pred is None else _c(pred, np.float64).copy()
    state = np.zeros((T, slots), np.int32)
    feat = np.full((T, slots), -1, np.int32)
    binv = np.full((T, slots), -1, np.int32)
    gain_ = np.zeros((T, slots))
    n_left = np.zeros((T, slots), np.int64)
    nrows = np.zeros((T, slots), np.int64)
    leaf = np.zeros((T, slots, d))
    prm = Params(loss, T, D, min_node, lam, gamma, lr)
    lib().oracle_train(_p(bins_cm), n, m, _p(nbins), B, _p(y), d, C.byref(prm), _p(pred),
                       _p(state), _p(feat), _p(binv), _p(gain_), _p(n_left), _p(nrows), _p(leaf))
    return dict(pred=pred, state=state, feat=feat, bin=binv, gain=gain_, n_left=n_left,
                nrows=nrows, leaf=leaf)


def predict(X, cuts, nbins, B, ref, D, T=None, pred=None):
    """Tree walk over raw features (oracle_predict) with the trees of an
    oracle.train result `ref` (its first T trees); returns pred [n][d] fp64."""
    X = _c(X, np.float32); cuts = _c(cuts, np.float32); nbins = _c(nbins, np.int32)
    n = X.shape[0]
    T = ref["state"].shape[0] if T is None else T
    d = ref["leaf"].shape[2]
    st = _c(ref["state"][:T], np.int32); ft = _c(ref["feat"][:T], np.int32); bt = _c(ref["bin"][:T], np.int32)
    lf = _c(ref["leaf"][:T], np.float64)
    pred = np.zeros((n, d)) if pred is None else _c(pred, np.float64).copy()
    lib().oracle_predict(_p(X), n, X.shape[1], _p(cuts), _p(nbins), B, T, D, d, _p(st), _p(ft), _p(bt), _p(lf),
                         _p(pred))
    return pred
