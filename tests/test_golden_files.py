"""The oracle-only goldens of the full-size free-running gate (tests/golden/<cfg>_T10.npz, written
by tools/make_golden.py) are not stale and are internally consistent (no GPU needed)."""
import glob
import os

import numpy as np
import pytest

from gen import gen

HERE = os.path.dirname(os.path.abspath(__file__))
FILES = sorted(glob.glob(os.path.join(HERE, "golden", "C*_T*.npz")))


def test_goldens_exist():
    names = {os.path.basename(f).split("_")[0] for f in FILES}
    assert {"C2", "C3", "C4"} <= names, names


@pytest.mark.parametrize("path", FILES, ids=[os.path.basename(f) for f in FILES])
def test_golden_matches_current_oracle_sources_and_is_consistent(path):
    import sys
    sys.path.insert(0, os.path.dirname(HERE))
    from tools.make_golden import src_sha
    g = dict(np.load(path))
    assert str(g["src_sha"]) == src_sha(), "oracle/gen sources changed since the golden was written: regenerate"
    name = os.path.basename(path).split("_")[0]
    w = gen.WORKLOADS[name]
    assert str(g["workload"]) == repr(w)
    T = int(g["T"])
    for t in range(T):
        st, nr, nl = g["state"][t], g["nrows"][t], g["n_left"][t]
        assert nr[0] == w.n and st[0] in (1, 2)
        assert nr[st == 2].sum() == w.n                                 # leaves partition the rows
        for h in np.nonzero(st == 1)[0]:
            assert nr[2 * h + 1] == nl[h] and nr[2 * h + 2] == nr[h] - nl[h]
            assert min(nl[h], nr[h] - nl[h]) >= w.min_node
            assert g["gain"][t][h] > w.gamma
    assert g["pred_sample"].shape == (len(g["sample_rows"]), w.d)
    assert np.all(np.isfinite(g["pred_sample"]))
