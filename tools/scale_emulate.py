"""Emulated strong scaling of the feature-partitioned scheme on ONE GPU.

This run has one B200, so N-GPU tree times cannot be measured directly.  This tool runs the
N ranks' work of a tree for real, rank after rank on the one GPU, in the same lockstep order the
multi-GPU run follows, and times every rank's kernels of every phase with CUDA events:

    phase grad             (replicated)          -> every rank
    per level: hist+search (feature shard)       -> rank r's shard only
               [key exchange]
               split_record (owner writes)       -> every rank
               [record exchange]
               partition    (replicated)         -> every rank
    leaf values + prediction update (replicated)

On N GPUs the ranks run a phase concurrently, each on its own full GPU, and meet at the exchange,
so the emulated tree time is  sum over phases of max over ranks (phase time)  plus the exchange
cost, which is reported separately (not measurable here).  The exchanges are done between the
phases by the host with torch ops (max of the keys, sum of the records): plumbing, not timed.
Trees must equal the single-rank run's bit for bit (checked).

    python tools/scale_emulate.py [C5] [trees=3] [N list=1,2,4,8]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_liupw25_b200 as pkg           # noqa: E402
from paper_conf_icpp_liupw25_b200.parallel import shard_range   # noqa: E402
from gen import gen                                   # noqa: E402
import bench                                          # noqa: E402  (host_targets)


class Timer:
    def __init__(self):
        self.ev = []

    def span(self):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        self.ev.append((e0, e1))
        return e0, e1


def make_ranks(w, N, Y, dev):
    ranks = []
    for r in range(N):
        f0, f1 = shard_range(w.m, r, N)
        X = torch.empty((w.n, f1 - f0), dtype=torch.float32, device=dev)
        gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, f0, f1 - f0, w.m, X.data_ptr(), f1 - f0,
                        torch.cuda.current_stream().cuda_stream)
        ctx = pkg.Context(0)
        ds = pkg.bin_features(ctx, X, w.B, f_begin=f0, m_global=w.m)
        del X
        P = pkg.Params(loss=w.loss, T=1000, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
        b = pkg.Booster(ctx, ds, Y, P, keep_model=False)
        ranks.append(b)
        torch.cuda.empty_cache()
    return ranks


def tree(ranks, D):
    """One tree, lockstep; returns (per-phase list of per-rank ms)."""
    phases = []

    def run(fn, name):
        spans = []
        for b in ranks:
            b._apply_options()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn(b)
            e1.record()
            spans.append((e0, e1))
        phases.append((name, spans))

    run(lambda b: b.ctx.gbdtmo_grad(b.p, b.y, b.pred, b.q, b.scales, b.state, b.gh), "grad")
    for lvl in range(D):
        cur, par = lvl % 2, (lvl - 1) % 2

        def hs(b, lvl=lvl, cur=cur, par=par):
            ph = b.hist[par] if lvl > 0 else None
            pc = b.cnt[par] if lvl > 0 else None
            if b.packed is not None:
                b.ctx.gbdtmo_build_hist_packed(b.p, lvl, b.ds.bins, b.packed, b.dflt, b.q, b.state, b.hist[cur],
                                               b.cnt[cur])
            else:
                b.ctx.gbdtmo_build_hist(b.p, lvl, b.ds.bins, b.dflt, b.q, b.state, b.hist[cur], b.cnt[cur])
            b.ctx.gbdtmo_find_split(b.p, lvl, b.ds.nbins, b.dflt, b.scales, b.state, b.hist[cur], b.cnt[cur], ph, pc,
                                    b.keys)
            if b.small_max_rows > 0:
                b.ctx.gbdtmo_search_small(b.p, lvl, b.ds.bins, b.q, b.ds.nbins, b.scales, b.state, b.keys)
        run(hs, f"L{lvl} hist+search")
        LN = 1 << lvl
        k = torch.stack([b.keys[:LN] for b in ranks]).max(0).values        # (exchange: MAX)
        for b in ranks:
            b.keys[:LN].copy_(k)

        def rec(b, lvl=lvl, cur=cur, par=par):
            ph = b.hist[par] if lvl > 0 else None
            pc = b.cnt[par] if lvl > 0 else None
            b.ctx.gbdtmo_split_record(b.p, lvl, b.ds.bins, b.dflt, b.q, b.scales, b.state, b.hist[cur], b.cnt[cur],
                                      ph, pc, b.keys, b.xchg)
        run(rec, f"L{lvl} split_record")
        x = torch.stack([b.xchg for b in ranks]).sum(0)                     # (exchange: SUM)
        for b in ranks:
            b.xchg.copy_(x)
        run(lambda b, lvl=lvl: b.ctx.gbdtmo_partition(b.p, lvl, b.state, b.xchg), f"L{lvl} partition")

    def fin(b):
        b.ctx.gbdtmo_leaf_values(b.p, b.scales, b.state, b.leaf, b.gh)
        b.ctx.gbdtmo_update_pred(b.p, b.state, b.leaf, b.pred)
    run(fin, "leaf+update")
    return phases


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C5"
    T = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    Ns = [int(x) for x in (sys.argv[3] if len(sys.argv) > 3 else "1,2,4,8").split(",")]
    w = gen.WORKLOADS[wl]
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    Y = torch.from_numpy(bench.host_targets(w)).to(dev)
    ref_pred = None
    out = {"workload": w.name, "trees_timed": T - 1, "gpus": {}}
    for N in Ns:
        ranks = make_ranks(w, N, Y, dev)
        per_tree = []
        for t in range(T):
            ph = tree(ranks, w.D)
            torch.cuda.synchronize()
            if t == 0:
                continue                          # first tree: warm-up (attributes, first touch)
            rows = []
            for name, spans in ph:
                ms = [e0.elapsed_time(e1) for e0, e1 in spans]
                rows.append((name, max(ms), sum(ms) / len(ms)))
            per_tree.append(rows)
        tree_ms = [sum(r[1] for r in rows) for rows in per_tree]
        hist_ms = [sum(r[1] for r in rows if "hist" in r[0]) for rows in per_tree]
        repl_ms = [sum(r[1] for r in rows if "hist" not in r[0]) for rows in per_tree]
        pred = ranks[0].pred.clone()
        for b in ranks[1:]:
            assert torch.equal(b.pred, pred), "ranks diverged"
        if ref_pred is None:
            ref_pred = pred
        same = bool(torch.equal(pred, ref_pred))
        out["gpus"][N] = {"ms_per_tree": float(np.median(tree_ms)), "hist_search_ms": float(np.median(hist_ms)),
                          "replicated_ms": float(np.median(repl_ms)), "exchanges_per_tree": 2 * w.D,
                          "pred_equals_1_rank": same,
                          "phases_ms_max_over_ranks": [(n, round(mx, 3)) for n, mx, _ in per_tree[-1]]}
        print(json.dumps({"N": N, **{k: v for k, v in out["gpus"][N].items() if k != "phases_ms_max_over_ranks"}}),
              flush=True)
        del ranks
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
    t1 = out["gpus"][Ns[0]]["ms_per_tree"] if Ns[0] == 1 else None
    if t1:
        out["speedup_excl_exchange"] = {N: t1 / v["ms_per_tree"] for N, v in out["gpus"].items()}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
