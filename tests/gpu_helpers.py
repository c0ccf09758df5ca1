"""Shared helpers of the GPU parity tests (test harness only)."""
import numpy as np


def node_rows(bins_cm, state, feat, binv, n):
    """Rows of every heap node of one oracle tree, in order (stable partition by the recorded
    splits; the definition of SplitNode)."""
    out = {0: np.arange(n, dtype=np.int32)}
    for h in range(len(state)):
        if state[h] == 1 and h in out:
            r = out[h]
            go_left = bins_cm[feat[h]][r] <= binv[h]
            out[2 * h + 1] = r[go_left]
            out[2 * h + 2] = r[~go_left]
    return out


def compare_trees(gpu, ref_state, ref_feat, ref_bin, ref_nrows, gains_at=None):
    """Tree-record equality; returns the list of heap nodes whose split differs (ties)."""
    st = gpu["node_state"]
    diffs = []
    for h in range(len(st)):
        if ref_state[h] == 0 and st[h] == 0:
            continue
        assert st[h] == ref_state[h], (h, st[h], ref_state[h])
        assert gpu["n_rows"][h] == ref_nrows[h], (h, gpu["n_rows"][h], ref_nrows[h])
        if st[h] == 1 and (gpu["feature"][h] != ref_feat[h] or gpu["bin"][h] != ref_bin[h]):
            diffs.append(h)
    return diffs


def to_np(rec):
    return {k: v.cpu().numpy() for k, v in rec.items()}
