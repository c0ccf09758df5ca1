"""Seeded synthetic inputs shared by tests/ and bench.py (no method arithmetic here).

Counter-based (gen_rng.h): element (i, c) of stream s under seed S depends only on
(S, s, i*ncols_total + c), so any row/column slice is reproducible on its own, and the
host build (libgbdtgen.so) and device build (libgbdtgen_cuda.so) are bit-identical.

Workload recipes follow the shapes of BASELINE.json configs and
the flavour of the paper's datasets:
  C1 tiny regression, C2 MNIST-shaped softmax, C3 multi-output regression,
  C4 Delicious/NUS-WIDE-shaped multi-label, C5 high-dimensional regression.
"""
from __future__ import annotations

import ctypes as C
import dataclasses
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_HOST = None
_CUDA = None

KIND_NORMAL, KIND_PIXEL = 0, 1
STREAM_X, STREAM_NOISE, STREAM_W, STREAM_LABEL = 1, 2, 3, 4
PIXEL_ZERO_Q24 = int(round(0.81 * (1 << 24)))   # MNIST-like zero fraction (DESIGN.md Inputs)
LOSS_MSE, LOSS_SOFTMAX = 0, 1


def build_host(force=False):
    so = os.path.join(_HERE, "libgbdtgen.so")
    srcs = [os.path.join(_HERE, f) for f in ("gen.c", "gen_rng.h")]
    if force or not os.path.exists(so) or os.path.getmtime(so) < max(map(os.path.getmtime, srcs)):
        cmd = f"gcc -O2 -fopenmp -fPIC -shared -ffp-contract=off -o {so} {srcs[0]}"
        if os.system(cmd) != 0:
            raise RuntimeError("gen build failed: " + cmd)
    return so


def build_cuda(force=False, nvcc="nvcc"):
    so = os.path.join(_HERE, "libgbdtgen_cuda.so")
    srcs = [os.path.join(_HERE, f) for f in ("gen_cuda.cu", "gen_rng.h")]
    if force or not os.path.exists(so) or os.path.getmtime(so) < max(map(os.path.getmtime, srcs)):
        cmd = (f"{nvcc} -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -Xcompiler -fPIC -shared "
               f"-o {so} {srcs[0]}")
        if os.system(cmd) != 0:
            raise RuntimeError("gen cuda build failed: " + cmd)
    return so


def _host():
    global _HOST
    if _HOST is None:
        _HOST = C.CDLL(build_host())
        P, i32, i64, u64, u32 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_uint32
        _HOST.gen_matrix_f32.argtypes = [u64, u64, i32, u32, i64, i64, i64, i64, i64, P, i64]
        _HOST.gen_uniform_f64_array.argtypes = [u64, u64, i64, i64, P]
    return _HOST


def _cuda():
    global _CUDA
    if _CUDA is None:
        _CUDA = C.CDLL(build_cuda())
        P, i32, i64, u64, u32 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_uint32
        _CUDA.gen_matrix_f32_cuda.argtypes = [u64, u64, i32, u32, i64, i64, i64, i64, i64, P, i64, P]
        _CUDA.gen_matrix_f32_cuda.restype = C.c_int
    return _CUDA


def matrix_host(seed, stream, kind, r0, nr, c0, nc, ncols_total, out=None):
    out = np.empty((nr, nc), np.float32) if out is None else out
    assert out.dtype == np.float32 and out.flags.c_contiguous
    _host().gen_matrix_f32(seed, stream, kind, PIXEL_ZERO_Q24, r0, nr, c0, nc, ncols_total,
                           out.ctypes.data_as(C.c_void_p), out.shape[1])
    return out


def matrix_cuda(seed, stream, kind, r0, nr, c0, nc, ncols_total, out_ptr, ld_out, cuda_stream=0):
    rc = _cuda().gen_matrix_f32_cuda(seed, stream, kind, PIXEL_ZERO_Q24, r0, nr, c0, nc, ncols_total,
                                     out_ptr, ld_out, cuda_stream)
    if rc != 0:
        raise RuntimeError(f"gen_matrix_f32_cuda failed: cuda error {rc}")


def uniform_host(seed, stream, i0, count):
    out = np.empty(count, np.float64)
    _host().gen_uniform_f64_array(seed, stream, i0, count, out.ctypes.data_as(C.c_void_p))
    return out


def normal_host(seed, stream, shape):
    n = int(np.prod(shape))
    return matrix_host(seed, stream, KIND_NORMAL, 0, 1, 0, n, n).reshape(shape).astype(np.float64)


@dataclasses.dataclass(frozen=True)
class Workload:
    name: str
    index: int          # 1..5 (BASELINE.json configs[index-1])
    n: int
    m: int
    d: int
    B: int
    D: int
    T: int
    loss: int
    x_kind: int
    lam: float = 1.0
    gamma: float = 0.0
    lr: float = 1.0
    min_node: int = 20
    classes_sweep: bool = False      # NEXT-2 (Fig. 6b): sklearn-style multi-class, features depend on labels

    @property
    def seed(self):
        return 1234 + self.index

    def scaled(self, n=None, m=None, T=None, D=None):
        return dataclasses.replace(self, n=n or self.n, m=m or self.m, T=T or self.T, D=D or self.D)


WORKLOADS = {
    "C1": Workload("C1-tiny-regression", 1, 2_000, 16, 4, 64, 4, 5, LOSS_MSE, KIND_NORMAL),
    "C2": Workload("C2-mnist-shaped-softmax", 2, 60_000, 784, 10, 256, 8, 100, LOSS_SOFTMAX, KIND_PIXEL),
    "C3": Workload("C3-multi-output-regression", 3, 1_000_000, 100, 32, 256, 8, 10, LOSS_MSE, KIND_NORMAL),
    "C4": Workload("C4-multilabel-delicious-nuswide", 4, 200_000, 500, 256, 256, 6, 10, LOSS_MSE, KIND_NORMAL),
    "C5": Workload("C5-high-dim-feature-partitioned", 5, 2_000_000, 4096, 16, 256, 8, 10, LOSS_MSE, KIND_NORMAL),
}


def sweep(d: int, n: int = 100_000, m: int = 100, T: int = 100, D: int = 6) -> Workload:
    """NEXT-2 class-count sweep (Fig. 6b: 100 trees of depth 6 on scikit-learn-style
    multi-class data, 5..500 classes; DESIGN.md Inputs: n = 100k, m = 100, 20 informative features)."""
    return Workload(f"S{d}-class-sweep", 100 + d, n, m, d, 256, D, T, LOSS_SOFTMAX, KIND_NORMAL, classes_sweep=True)


def _sweep_labels(w: Workload, r0: int, nr: int):
    return (np.floor(uniform_host(w.seed, STREAM_LABEL, r0, nr) * w.d)).astype(np.int64)


def _sweep_centroids(w: Workload):
    return 1.5 * normal_host(w.seed, STREAM_W, (w.d, 20))


def informative_columns(w: Workload):
    """Columns the targets depend on (DESIGN.md Inputs)."""
    if w.index == 5:
        k = min(64, w.m)
        return np.array([(j * w.m) // k for j in range(k)], np.int64)
    k = {1: 6, 3: 16, 4: 32}.get(w.index, 0)
    return np.arange(min(k, w.m), dtype=np.int64)


def features_host(w: Workload, r0=0, nr=None, c0=0, nc=None):
    nr = w.n - r0 if nr is None else nr
    nc = w.m - c0 if nc is None else nc
    X = matrix_host(w.seed, STREAM_X, w.x_kind, r0, nr, c0, nc, w.m)
    if w.classes_sweep:            # class centroid shift on the 20 informative columns
        lab = _sweep_labels(w, r0, nr)
        cen = _sweep_centroids(w)
        lo, hi = max(c0, 0), min(c0 + nc, 20)
        if lo < hi:
            X[:, lo - c0:hi - c0] += cen[lab][:, lo:hi].astype(np.float32)
    return X


def _columns_host(w: Workload, cols):
    out = np.empty((w.n, len(cols)), np.float64)
    for j, c in enumerate(cols):
        out[:, j] = matrix_host(w.seed, STREAM_X, w.x_kind, 0, w.n, int(c), 1, w.m)[:, 0]
    return out


def targets_host(w: Workload, X=None):
    """Targets y [n][d] float32 (fp64-computed, rounded as stated in DESIGN.md Inputs)."""
    n, d = w.n, w.d
    if w.classes_sweep:
        y = np.zeros((n, d), np.float32)
        y[np.arange(n), _sweep_labels(w, 0, n)] = 1.0
        return y
    if w.index == 2:   # MNIST-shaped: label = argmax(X V / 255 + Gumbel); one-hot
        Xf = X if X is not None else features_host(w)
        V = normal_host(w.seed, STREAM_W, (w.m, d))
        mask = uniform_host(w.seed, STREAM_W + 16, 0, w.m * d).reshape(w.m, d) < 0.1
        logits = (Xf.astype(np.float64) @ (V * mask)) / 255.0
        u = uniform_host(w.seed, STREAM_LABEL, 0, n * d).reshape(n, d)
        logits += -np.log(-np.log(np.clip(u, 1e-300, 1.0 - 1e-16)))
        y = np.zeros((n, d), np.float32)
        y[np.arange(n), np.argmax(logits, axis=1)] = 1.0
        return y
    cols = informative_columns(w)
    XS = (X[:, cols].astype(np.float64) if X is not None else _columns_host(w, cols))
    k = XS.shape[1]
    if w.index == 4:   # multi-label {0,1}, ~2% positives
        A = normal_host(w.seed, STREAM_W, (k, d)) / np.sqrt(k)
        u = uniform_host(w.seed, STREAM_NOISE, 0, n * d).reshape(n, d)
        logistic = np.log(np.clip(u, 1e-300, None)) - np.log1p(-np.minimum(u, 1.0 - 1e-16))
        return ((XS @ A - 4.25 + logistic) > 0).astype(np.float32)
    hidden = 8 if w.index == 1 else 32
    W1 = normal_host(w.seed, STREAM_W, (k, hidden)) / np.sqrt(k)
    W2 = normal_host(w.seed, STREAM_W + 32, (hidden, d)) / np.sqrt(hidden)
    eps = normal_host(w.seed, STREAM_NOISE, (n, d))
    y = np.tanh(XS @ W1) @ W2 + 0.1 * eps
    y -= y.mean(axis=0, keepdims=True)
    y = np.round(y * 65536.0) / 65536.0           # dyadic grid 2^-16
    return y.astype(np.float32)
