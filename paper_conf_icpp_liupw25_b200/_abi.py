"""Thin ctypes binding of libgbdtmo.so (include/gbdtmo.h): argument marshalling only.

Every function has the C name and forwards plain integers / pointers; tensors are passed by
their data pointer (``t.data_ptr()``).  A non-OK status raises ``GbdtmoError`` with the
library's message.  There is no fallback: if the library is missing this module raises on
import of :func:`lib`.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# GBDTMO_LIB overrides the library path (A/B builds of the same sources; see tools/ab_build.sh)
LIB_PATH = os.environ.get("GBDTMO_LIB") or os.path.join(_HERE, "libgbdtmo.so")

OK, EINVAL, ECUDA, ENOMEM, EUNSUPPORTED = 0, 1, 2, 3, 5
LOSS_MSE, LOSS_SOFTMAX = 0, 1
NODE_NONE, NODE_SPLIT, NODE_LEAF, NODE_ACTIVE = 0, 1, 2, 3

# Every symbol include/gbdtmo.h declares (checked by tests/test_abi_load.py).
SYMBOLS = (
    "gbdtmo_abi_version", "gbdtmo_create", "gbdtmo_destroy", "gbdtmo_set_stream", "gbdtmo_last_error",
    "gbdtmo_launch_count", "gbdtmo_bins_bytes", "gbdtmo_bin_workspace_bytes", "gbdtmo_state_bytes",
    "gbdtmo_hist_bytes", "gbdtmo_xchg_count", "gbdtmo_bin", "gbdtmo_grad", "gbdtmo_build_hist",
    "gbdtmo_find_split", "gbdtmo_split_record", "gbdtmo_partition", "gbdtmo_leaf_values",
    "gbdtmo_update_pred", "gbdtmo_tree_export", "gbdtmo_rows_export", "gbdtmo_default_bins", "gbdtmo_predict",
    "gbdtmo_set_option", "gbdtmo_search_small", "gbdtmo_bin_csc", "gbdtmo_packed_bins_bytes", "gbdtmo_pack_bins",
    "gbdtmo_build_hist_packed", "gbdtmo_csc_nz_bins", "gbdtmo_build_hist_csc", "gbdtmo_peer_window_bytes", "gbdtmo_peer_open", "gbdtmo_peer_connect",
    "gbdtmo_peer_buffers", "gbdtmo_peer_status", "gbdtmo_peer_close", "gbdtmo_split_record_peer",
    "gbdtmo_partition_peer", "gbdtmo_set_root_counts", "gbdtmo_peer_status_async", "gbdtmo_bin_host",
    "gbdtmo_bin_host_workspace_bytes",
)
(OPT_GMEM_MAX_ROWS, OPT_SMALL_MAX_ROWS, OPT_HIST_KERNEL, OPT_PEER_TIMEOUT_MS, OPT_FS_CHANNEL_GROUPS,
 OPT_HIST_WAVES) = 1, 2, 3, 4, 5, 6
PEER_HANDLE_BYTES = 64


class GbdtmoError(RuntimeError):
    pass


class Problem(C.Structure):
    """gbdtmo_problem (include/gbdtmo.h)."""
    _fields_ = [("n", C.c_int64), ("m", C.c_int32), ("f_begin", C.c_int32), ("m_global", C.c_int32),
                ("d", C.c_int32), ("B", C.c_int32), ("D", C.c_int32), ("loss", C.c_int32),
                ("min_node", C.c_int32), ("lambda_", C.c_double), ("gamma", C.c_double), ("lr", C.c_double),
                ("ld_bins", C.c_int64)]

    @property
    def V(self):
        return 2 * self.d if self.loss == LOSS_SOFTMAX else self.d


_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise GbdtmoError(f"{LIB_PATH} not built: run `make` or __graft_entry__.build()")
        L = C.CDLL(LIB_PATH)
        P, i32, i64, f64, sz = C.c_void_p, C.c_int32, C.c_int64, C.c_double, C.c_size_t
        PP = C.POINTER(Problem)
        sig = {
            "gbdtmo_abi_version": ([], C.c_int),
            "gbdtmo_create": ([C.c_int, C.POINTER(P)], C.c_int),
            "gbdtmo_destroy": ([P], C.c_int),
            "gbdtmo_set_stream": ([P, P], C.c_int),
            "gbdtmo_last_error": ([P], C.c_char_p),
            "gbdtmo_set_option": ([P, i32, i64], C.c_int),
            "gbdtmo_launch_count": ([P], i64),
            "gbdtmo_bins_bytes": ([i64, i64], sz),
            "gbdtmo_bin_workspace_bytes": ([i64, i32, i32], sz),
            "gbdtmo_state_bytes": ([PP, C.POINTER(sz)], C.c_int),
            "gbdtmo_hist_bytes": ([PP, i32, C.POINTER(sz), C.POINTER(sz)], C.c_int),
            "gbdtmo_xchg_count": ([PP, C.POINTER(i64)], C.c_int),
            "gbdtmo_bin": ([P, P, i64, i32, i64, i32, P, i64, P, P, P, sz], C.c_int),
            "gbdtmo_bin_csc": ([P, P, P, P, P, i64, i32, i32, P, i64, P, P, P, sz], C.c_int),
            "gbdtmo_bin_host": ([P, P, i64, i32, i64, i32, P, i64, P, P, P, sz, i32], C.c_int),
            "gbdtmo_bin_host_workspace_bytes": ([i64, i32, i32, i32], sz),
            "gbdtmo_grad": ([P, PP, P, P, P, P, P, P], C.c_int),
            "gbdtmo_default_bins": ([P, P, i64, i32, i64, i32, i64, P], C.c_int),
            "gbdtmo_build_hist": ([P, PP, i32, P, P, P, P, P, P], C.c_int),
            "gbdtmo_build_hist_packed": ([P, PP, i32, P, P, P, P, P, P, P], C.c_int),
            "gbdtmo_csc_nz_bins": ([P, i32, i32, P, P, P, i64, P, P, P], C.c_int),
            "gbdtmo_build_hist_csc": ([P, PP, i32, P, P, P, i64, P, P, P, P, P], C.c_int),
            "gbdtmo_packed_bins_bytes": ([PP], sz),
            "gbdtmo_pack_bins": ([P, PP, P, P], C.c_int),
            "gbdtmo_find_split": ([P, PP, i32, P, P, P, P, P, P, P, P, P], C.c_int),
            "gbdtmo_split_record": ([P, PP, i32, P, P, P, P, P, P, P, P, P, P, P], C.c_int),
            "gbdtmo_search_small": ([P, PP, i32, P, P, P, P, P, P], C.c_int),
            "gbdtmo_partition": ([P, PP, i32, P, P], C.c_int),
            "gbdtmo_leaf_values": ([P, PP, P, P, P, P], C.c_int),
            "gbdtmo_update_pred": ([P, PP, P, P, P], C.c_int),
            "gbdtmo_tree_export": ([P, PP, P, P, P, P, P, P, P, P, P], C.c_int),
            "gbdtmo_predict": ([P, P, i64, i32, i64, i32, i32, i32, P, P, P, P, P], C.c_int),
            "gbdtmo_rows_export": ([P, PP, P, i32, P, P, P, P], C.c_int),
            "gbdtmo_set_root_counts": ([P, P], C.c_int),
            "gbdtmo_peer_window_bytes": ([PP], sz),
            "gbdtmo_peer_open": ([P, PP, i32, i32, P], C.c_int),
            "gbdtmo_peer_connect": ([P, P], C.c_int),
            "gbdtmo_peer_buffers": ([P, PP, i32, C.POINTER(P), C.POINTER(P)], C.c_int),
            "gbdtmo_peer_status": ([P, C.POINTER(i64), C.POINTER(i64)], C.c_int),
            "gbdtmo_peer_close": ([P], C.c_int),
            "gbdtmo_peer_status_async": ([P, P], C.c_int),
            "gbdtmo_split_record_peer": ([P, PP, i32, P, P, P, P, P, P, P, P, P, P], C.c_int),
            "gbdtmo_partition_peer": ([P, PP, i32, P, P], C.c_int),
        }
        for name, (args, res) in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _LIB = L
    return _LIB


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


class Context:
    """Owns one gbdtmo_ctx; methods mirror the C calls (same names without the prefix)."""

    def __init__(self, device: int = 0):
        self._h = C.c_void_p()
        st = lib().gbdtmo_create(device, C.byref(self._h))
        if st != OK:
            raise GbdtmoError(f"gbdtmo_create(device={device}) failed with status {st}")

    def close(self):
        if self._h:
            lib().gbdtmo_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, st, name):
        if st != OK:
            msg = lib().gbdtmo_last_error(self._h)
            raise GbdtmoError(f"{name}: status {st}: {msg.decode() if msg else ''}")

    # lifecycle -------------------------------------------------------------
    def gbdtmo_set_stream(self, stream_handle: int):
        self._check(lib().gbdtmo_set_stream(self._h, C.c_void_p(stream_handle)), "gbdtmo_set_stream")

    def gbdtmo_set_option(self, option: int, value: int):
        self._check(lib().gbdtmo_set_option(self._h, option, value), "gbdtmo_set_option")

    def gbdtmo_set_root_counts(self, root_cnt):
        self._check(lib().gbdtmo_set_root_counts(self._h, _ptr(root_cnt)), "gbdtmo_set_root_counts")

    def gbdtmo_launch_count(self) -> int:
        return int(lib().gbdtmo_launch_count(self._h))

    # sizes (host) ------------------------------------------------------------
    @staticmethod
    def gbdtmo_bins_bytes(n, ld_bins) -> int:
        return int(lib().gbdtmo_bins_bytes(n, ld_bins))

    @staticmethod
    def gbdtmo_bin_workspace_bytes(n, m, B) -> int:
        return int(lib().gbdtmo_bin_workspace_bytes(n, m, B))

    @staticmethod
    def gbdtmo_state_bytes(p: Problem) -> int:
        v = C.c_size_t()
        if lib().gbdtmo_state_bytes(C.byref(p), C.byref(v)) != OK:
            raise GbdtmoError("gbdtmo_state_bytes: invalid problem")
        return int(v.value)

    @staticmethod
    def gbdtmo_hist_bytes(p: Problem, level: int):
        h, c = C.c_size_t(), C.c_size_t()
        if lib().gbdtmo_hist_bytes(C.byref(p), level, C.byref(h), C.byref(c)) != OK:
            raise GbdtmoError("gbdtmo_hist_bytes: invalid problem or level")
        return int(h.value), int(c.value)

    @staticmethod
    def gbdtmo_xchg_count(p: Problem) -> int:
        v = C.c_int64()
        if lib().gbdtmo_xchg_count(C.byref(p), C.byref(v)) != OK:
            raise GbdtmoError("gbdtmo_xchg_count: invalid problem")
        return int(v.value)

    # the hot-path calls --------------------------------------------------------
    def gbdtmo_bin_csc(self, values, row_idx, col_ptr, col_ptr_host, n, m, B, bins, ld_bins, cuts, nbins, ws,
                       ws_bytes):
        self._check(lib().gbdtmo_bin_csc(self._h, _ptr(values), _ptr(row_idx), _ptr(col_ptr), _ptr(col_ptr_host), n,
                                         m, B, _ptr(bins), ld_bins, _ptr(cuts), _ptr(nbins), _ptr(ws), ws_bytes),
                    "gbdtmo_bin_csc")

    @staticmethod
    def gbdtmo_bin_host_workspace_bytes(n, m, B, strip) -> int:
        return int(lib().gbdtmo_bin_host_workspace_bytes(n, m, B, strip))

    def gbdtmo_bin_host(self, X_host, n, m, ld_x, B, bins, ld_bins, cuts, nbins, ws, ws_bytes, strip):
        self._check(lib().gbdtmo_bin_host(self._h, _ptr(X_host), n, m, ld_x, B, _ptr(bins), ld_bins, _ptr(cuts),
                                          _ptr(nbins), _ptr(ws), ws_bytes, strip), "gbdtmo_bin_host")

    def gbdtmo_bin(self, X, n, m, ld_x, B, bins, ld_bins, cuts, nbins, ws, ws_bytes):
        self._check(lib().gbdtmo_bin(self._h, _ptr(X), n, m, ld_x, B, _ptr(bins), ld_bins, _ptr(cuts),
                                     _ptr(nbins), _ptr(ws), ws_bytes), "gbdtmo_bin")

    def gbdtmo_grad(self, p, y, pred, q, scales, state, gh=None):
        self._check(lib().gbdtmo_grad(self._h, C.byref(p), _ptr(y), _ptr(pred), _ptr(q), _ptr(scales),
                                      _ptr(state), _ptr(gh)), "gbdtmo_grad")

    def gbdtmo_default_bins(self, bins, n, m, ld_bins, B, min_count, dflt):
        self._check(lib().gbdtmo_default_bins(self._h, _ptr(bins), n, m, ld_bins, B, min_count, _ptr(dflt)),
                    "gbdtmo_default_bins")

    def gbdtmo_build_hist(self, p, level, bins, dflt, q, state, hist, cnt):
        self._check(lib().gbdtmo_build_hist(self._h, C.byref(p), level, _ptr(bins), _ptr(dflt), _ptr(q),
                                            _ptr(state), _ptr(hist), _ptr(cnt)), "gbdtmo_build_hist")

    def gbdtmo_build_hist_packed(self, p, level, bins, packed, dflt, q, state, hist, cnt):
        self._check(lib().gbdtmo_build_hist_packed(self._h, C.byref(p), level, _ptr(bins), _ptr(packed), _ptr(dflt),
                                                   _ptr(q), _ptr(state), _ptr(hist), _ptr(cnt)),
                    "gbdtmo_build_hist_packed")

    def gbdtmo_csc_nz_bins(self, m, B, col_ptr, row_idx, bins, ld_bins, cuts, nz_bins, zbin):
        self._check(lib().gbdtmo_csc_nz_bins(self._h, m, B, _ptr(col_ptr), _ptr(row_idx), _ptr(bins), ld_bins,
                                             _ptr(cuts), _ptr(nz_bins), _ptr(zbin)), "gbdtmo_csc_nz_bins")

    def gbdtmo_build_hist_csc(self, p, level, col_ptr, row_idx, nz_bins, nnz, zbin, q, state, hist, cnt):
        self._check(lib().gbdtmo_build_hist_csc(self._h, C.byref(p), level, _ptr(col_ptr), _ptr(row_idx),
                                                _ptr(nz_bins), nnz, _ptr(zbin), _ptr(q), _ptr(state), _ptr(hist),
                                                _ptr(cnt)), "gbdtmo_build_hist_csc")

    @staticmethod
    def gbdtmo_packed_bins_bytes(p) -> int:
        return int(lib().gbdtmo_packed_bins_bytes(C.byref(p)))

    def gbdtmo_pack_bins(self, p, bins, packed):
        self._check(lib().gbdtmo_pack_bins(self._h, C.byref(p), _ptr(bins), _ptr(packed)), "gbdtmo_pack_bins")

    def gbdtmo_find_split(self, p, level, nbins, dflt, scales, state, hist, cnt, parent_hist, parent_cnt, keys):
        self._check(lib().gbdtmo_find_split(self._h, C.byref(p), level, _ptr(nbins), _ptr(dflt), _ptr(scales),
                                            _ptr(state), _ptr(hist), _ptr(cnt), _ptr(parent_hist), _ptr(parent_cnt),
                                            _ptr(keys)), "gbdtmo_find_split")

    def gbdtmo_search_small(self, p, level, bins, q, nbins, scales, state, keys):
        self._check(lib().gbdtmo_search_small(self._h, C.byref(p), level, _ptr(bins), _ptr(q), _ptr(nbins),
                                              _ptr(scales), _ptr(state), _ptr(keys)), "gbdtmo_search_small")

    def gbdtmo_split_record(self, p, level, bins, dflt, q, scales, state, hist, cnt, parent_hist, parent_cnt, keys,
                            xchg):
        self._check(lib().gbdtmo_split_record(self._h, C.byref(p), level, _ptr(bins), _ptr(dflt), _ptr(q),
                                              _ptr(scales), _ptr(state),
                                              _ptr(hist), _ptr(cnt), _ptr(parent_hist), _ptr(parent_cnt),
                                              _ptr(keys), _ptr(xchg)), "gbdtmo_split_record")

    def gbdtmo_partition(self, p, level, state, xchg):
        self._check(lib().gbdtmo_partition(self._h, C.byref(p), level, _ptr(state), _ptr(xchg)),
                    "gbdtmo_partition")

    def gbdtmo_leaf_values(self, p, scales, state, leaf, gh=None):
        self._check(lib().gbdtmo_leaf_values(self._h, C.byref(p), _ptr(scales), _ptr(state), _ptr(gh), _ptr(leaf)),
                    "gbdtmo_leaf_values")

    def gbdtmo_update_pred(self, p, state, leaf, pred):
        self._check(lib().gbdtmo_update_pred(self._h, C.byref(p), _ptr(state), _ptr(leaf), _ptr(pred)),
                    "gbdtmo_update_pred")

    def gbdtmo_tree_export(self, p, state, node_state=None, feature=None, bin=None, gain=None, n_rows=None,
                           n_left=None, cuts=None, threshold=None):
        self._check(lib().gbdtmo_tree_export(self._h, C.byref(p), _ptr(state), _ptr(node_state), _ptr(feature),
                                             _ptr(bin), _ptr(gain), _ptr(n_rows), _ptr(n_left), _ptr(cuts),
                                             _ptr(threshold)), "gbdtmo_tree_export")

    def gbdtmo_predict(self, X, n, m, ld_x, T, D, d, node_state, feature, threshold, leaf, pred):
        self._check(lib().gbdtmo_predict(self._h, _ptr(X), n, m, ld_x, T, D, d, _ptr(node_state), _ptr(feature),
                                         _ptr(threshold), _ptr(leaf), _ptr(pred)), "gbdtmo_predict")

    def gbdtmo_rows_export(self, p, state, level, rows=None, node_of_row=None, node_begin=None, node_end=None):
        self._check(lib().gbdtmo_rows_export(self._h, C.byref(p), _ptr(state), level, _ptr(rows), _ptr(node_of_row),
                                             _ptr(node_begin), _ptr(node_end)), "gbdtmo_rows_export")

    # NEXT-4: fused peer-memory exchange ------------------------------------------
    @staticmethod
    def gbdtmo_peer_window_bytes(p) -> int:
        return int(lib().gbdtmo_peer_window_bytes(C.byref(p)))

    def gbdtmo_peer_open(self, p, rank: int, world: int) -> bytes:
        h = (C.c_uint8 * PEER_HANDLE_BYTES)()
        self._check(lib().gbdtmo_peer_open(self._h, C.byref(p), rank, world, h), "gbdtmo_peer_open")
        return bytes(h)

    def gbdtmo_peer_connect(self, handles: bytes):
        buf = (C.c_uint8 * len(handles)).from_buffer_copy(handles)
        self._check(lib().gbdtmo_peer_connect(self._h, buf), "gbdtmo_peer_connect")

    def gbdtmo_peer_buffers(self, p, level: int):
        k, x = C.c_void_p(), C.c_void_p()
        self._check(lib().gbdtmo_peer_buffers(self._h, C.byref(p), level, C.byref(k), C.byref(x)),
                    "gbdtmo_peer_buffers")
        return int(k.value), int(x.value)

    def gbdtmo_peer_status(self):
        e, r = C.c_int64(), C.c_int64()
        self._check(lib().gbdtmo_peer_status(self._h, C.byref(e), C.byref(r)), "gbdtmo_peer_status")
        return int(e.value), int(r.value)

    def gbdtmo_peer_status_async(self, out):
        self._check(lib().gbdtmo_peer_status_async(self._h, _ptr(out)), "gbdtmo_peer_status_async")

    def gbdtmo_peer_close(self):
        self._check(lib().gbdtmo_peer_close(self._h), "gbdtmo_peer_close")

    def gbdtmo_split_record_peer(self, p, level, bins, dflt, q, scales, state, hist, cnt, parent_hist, parent_cnt,
                                 keys_merged):
        self._check(lib().gbdtmo_split_record_peer(self._h, C.byref(p), level, _ptr(bins), _ptr(dflt), _ptr(q),
                                                   _ptr(scales), _ptr(state), _ptr(hist), _ptr(cnt),
                                                   _ptr(parent_hist), _ptr(parent_cnt), _ptr(keys_merged)),
                    "gbdtmo_split_record_peer")

    def gbdtmo_partition_peer(self, p, level, state, xchg_merged):
        self._check(lib().gbdtmo_partition_peer(self._h, C.byref(p), level, _ptr(state), _ptr(xchg_merged)),
                    "gbdtmo_partition_peer")
