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


def tie_locked_oracle(orc, bins, nbins, B, y, loss, pred0, gpu_trees, t0, T, D, lam, gamma, lr, min_node,
                      rel=1e-6):
    """SURVEY §8(c)-4 "tie-locked" oracle (test harness over oracle step functions only): Algorithm 1
    from tree t0 with the prediction pred0, node by node (oracle_build_hist + oracle_find_split at every
    searchable node), compared with the GPU's trees.  Where the GPU's (feature, bin)
    differs from the oracle's argmax, the oracle's own Eq. (3) gain at the GPU's choice must be within
    `rel` of the oracle's best (north star: ties within 1e-6 relative; R22) -- then the oracle adopts the
    GPU's choice and goes on; any other difference fails.  Returns (pred after tree T-1, list of ties)."""
    import numpy as np
    pred = pred0.copy()
    ties = []
    n = y.shape[0]
    for t in range(t0, T):
        gt = gpu_trees[t]
        g, h = orc.grad(loss, y, pred)
        rows = {0: np.arange(n, dtype=np.int32)}
        for hid in range(len(gt["node_state"])):
            if hid not in rows:
                continue
            r = rows[hid]
            depth = int(np.floor(np.log2(hid + 1)))
            G, H = g[r].sum(0), h[r].sum(0)
            st_g = int(gt["node_state"][hid])
            split = None
            if depth < D and len(r) >= 2 * min_node:
                HG, HH, CNT = orc.build_hist(bins, B, g, h, r)
                sp = orc.find_split(HG, HH, CNT, nbins, G, H, len(r), lam, min_node, want_all=True)
                o_split = sp["valid"] and sp["gain"] > gamma
                if st_g == 1:
                    fg, bg = int(gt["feature"][hid]), int(gt["bin"][hid])
                    at = sp["all_gains"][fg, bg]
                    assert np.isfinite(at), (t, hid, "GPU split is not a valid candidate", fg, bg)
                    if (fg, bg) != (sp["feature"], sp["bin"]) or not o_split:
                        best = max(sp["gain"], gamma) if sp["valid"] else gamma
                        assert at >= best - rel * abs(best), (t, hid, "not a tie", at, best, fg, bg, sp)
                        ties.append((t, hid, (fg, bg), (sp["feature"], sp["bin"]), float((best - at) / abs(best))))
                    split = (fg, bg)
                else:
                    assert not o_split or sp["gain"] <= gamma + rel * abs(gamma if gamma else sp["gain"]), \
                        (t, hid, "GPU leaf where the oracle splits", sp)
                    if o_split:
                        ties.append((t, hid, None, (sp["feature"], sp["bin"]), None))
            else:
                assert st_g != 1, (t, hid, "GPU split at a node the oracle cannot split")
            if split is not None:
                left, right = orc.partition(bins, r, split[0], split[1])
                rows[2 * hid + 1], rows[2 * hid + 2] = left, right
            else:
                v = orc.leaf_value(G, H, lam, lr)
                orc.update_pred(pred, r, v)
    return pred, ties
