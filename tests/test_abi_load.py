"""The C-ABI library loads on a CPU-only host and exports every symbol include/gbdtmo.h declares
(no compute calls without a GPU); the host-side size queries and argument validation work."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "gbdtmo.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gbdtmo_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    from paper_conf_icpp_liupw25_b200 import _abi
    L = _abi.lib()
    names = _declared()
    assert len(names) >= 20
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(_abi.SYMBOLS)
    assert L.gbdtmo_abi_version() == 2


def test_sizes_and_validation_on_host():
    from paper_conf_icpp_liupw25_b200 import _abi
    P = _abi.Problem(n=2_000_000, m=4096, f_begin=0, m_global=4096, d=16, B=256, D=8, loss=0, min_node=20,
                     lambda_=1.0, gamma=0.0, lr=1.0, ld_bins=4096)
    h, c = _abi.Context.gbdtmo_hist_bytes(P, 6)
    assert h == 64 * 4096 * 256 * 16 * 8 and c == 64 * 4096 * 256 * 4
    h, c = _abi.Context.gbdtmo_hist_bytes(P, 7)            # last level: only the built child of each pair
    assert h == 64 * 4096 * 256 * 16 * 8 and c == 64 * 4096 * 256 * 4
    assert _abi.Context.gbdtmo_xchg_count(P) == 128 * 20 + (2_000_000 + 63) // 64
    assert _abi.Context.gbdtmo_state_bytes(P) > 3 * 4 * 2_000_000
    bad = _abi.Problem(n=10, m=4, f_begin=0, m_global=4, d=2, B=300, D=3, loss=0, min_node=1, lambda_=1.0,
                       gamma=0.0, lr=1.0, ld_bins=8)
    with pytest.raises(_abi.GbdtmoError):
        _abi.Context.gbdtmo_state_bytes(bad)
    assert _abi.Context.gbdtmo_bins_bytes(10, 16) == 10 * 16 + 32
    # peer window (NEXT-4): header + per-level keys + per-level exchange buffers
    xc = _abi.Context.gbdtmo_xchg_count(P)
    wb = _abi.Context.gbdtmo_peer_window_bytes(P)
    assert wb >= 512 + 8 * 8 * 128 + 8 * 8 * xc and wb < 512 + 8 * 8 * 128 + 8 * 8 * (xc + 32) + 256
    assert _abi.Context.gbdtmo_peer_window_bytes(bad) == 0


def test_create_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_icpp_liupw25_b200 import _abi
    with pytest.raises(_abi.GbdtmoError):
        _abi.Context(0)
