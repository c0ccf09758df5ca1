"""The Booster's multi-rank path (feature shards) run as two processes sharing cuda:0:
trees and predictions must equal the single-process run bit for bit, for both exchanges —
"collective" (torch.distributed all-reduces over a gloo group; NCCL needs one GPU per rank, the
exchange code is the same) and "peer" (NEXT-4: the fused peer-memory exchange; the two processes'
windows are mapped with CUDA IPC on the one device, the waits inside the kernels progress under
the driver's time slicing between the two contexts).  The peer run also replays CUDA graphs."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _case():
    from gen import gen
    return gen.WORKLOADS["C3"].scaled(n=60_000, m=30, T=2, D=5)


def _worker(rank, world, port, out, exchange="collective", graph=False, timeout_ms=None, delay_rank1=0.0):
    import sys
    sys.path.insert(0, ROOT)
    if timeout_ms is not None:
        os.environ["GBDTMO_PEER_TIMEOUT_MS"] = str(timeout_ms)
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_icpp_liupw25_b200 as pkg
    from paper_conf_icpp_liupw25_b200.parallel import shard_range
    from gen import gen
    w = _case()
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    f0, f1 = shard_range(w.m, rank, world)
    ctx = pkg.Context(0)
    ds = pkg.bin_features(ctx, torch.from_numpy(np.ascontiguousarray(X[:, f0:f1])).cuda(), w.B, f_begin=f0,
                          m_global=w.m)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, torch.from_numpy(Y).cuda(), P, group=dist.group.WORLD, exchange=exchange)
    if exchange == "peer" and timeout_ms is None:
        ctx.gbdtmo_set_option(pkg._abi.OPT_PEER_TIMEOUT_MS, 120_000)
    raised = None
    if delay_rank1 and rank == 1:
        import time
        time.sleep(delay_rank1)       # rank 0's first bounded wait must expire
    try:
        if graph:                     # trees replayed from one captured CUDA graph
            b.capture()               # (its warm-up tree runs outside the graph and is not kept)
            b.trees.clear()
            for _ in range(w.T):
                b.step_graph()
            b.check_peer(block=True)
        else:
            b.fit()
    except pkg.PeerExchangeError as ex:
        raised = str(ex)
    torch.cuda.synchronize()
    status = b.peer_status() if exchange == "peer" else (0, 0)
    out[rank] = ([{k: v.cpu().numpy() for k, v in t.items()} for t in b.trees], b.pred.cpu().numpy(), status, raised)
    dist.destroy_process_group()


@pytest.mark.parametrize("exchange,graph", [("collective", False), ("peer", False), ("peer", True)])
def test_two_rank_booster_equals_single_rank_and_oracle(orc, exchange, graph):
    """Each rank's trees (feature shards) equal the fp64 oracle's trees of the whole
    feature set (exact (f, b), n_rows, leaves rtol 1e-5, predictions <= 1e-4), and the 1-rank run
    bit for bit."""
    import sys
    sys.path.insert(0, ROOT)
    import paper_conf_icpp_liupw25_b200 as pkg
    from gen import gen
    from tests.gpu_helpers import compare_trees
    w = _case()
    X = gen.features_host(w)
    Y = gen.targets_host(w, X)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    oref = orc.train(bins, nbins, w.B, Y.astype(np.float64), loss=w.loss, T=w.T, D=w.D, lam=w.lam, gamma=w.gamma,
                     lr=w.lr, min_node=w.min_node)
    ctx = pkg.Context(0)
    P = pkg.Params(loss=w.loss, T=w.T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    ref = pkg.Booster(ctx, pkg.bin_features(ctx, torch.from_numpy(X).cuda(), w.B), torch.from_numpy(Y).cuda(), P)
    ref.fit()
    torch.cuda.synchronize()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.start_processes(_worker, args=(2, _free_port(), out, exchange, graph), nprocs=2, join=True, start_method="spawn")
    for rank in range(2):
        trees, pred, (epoch, err), raised = out[rank]
        assert err == 0 and raised is None, f"peer exchange error word {err:#x}: {raised}"
        if exchange == "peer":
            assert epoch == (w.T + graph) * w.D          # one exchange per level (+ the capture warm-up tree)
        for t in range(w.T):
            a = {k: v.cpu().numpy() for k, v in ref.trees[t].items()}
            for k in ("node_state", "feature", "bin", "n_rows", "n_left", "leaf"):
                np.testing.assert_array_equal(trees[t][k], a[k])
            assert not compare_trees(trees[t], oref["state"][t], oref["feat"][t], oref["bin"][t], oref["nrows"][t])
            lv = trees[t]["node_state"] == 2
            np.testing.assert_allclose(trees[t]["leaf"][lv], oref["leaf"][t][lv], rtol=1e-5, atol=1e-6)
        np.testing.assert_array_equal(pred, ref.pred.cpu().numpy())
        assert np.max(np.abs(pred - oref["pred"])) <= 1e-4


def test_peer_wait_expiry_is_safe_and_raises():
    """Waits bounded at 1 ms while rank 1 starts 3 s late, so rank 0's first wait expires: the run
    must finish without a fault, the expired wait is recorded in the error word, every level after
    it ends its nodes as leaves (no partition from partial records), and Booster.fit raises
    PeerExchangeError on every rank whose error word is set (never a silent degenerate model)."""
    w = _case()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.start_processes(_worker, args=(2, _free_port(), out, "peer", False, 1, 3.0), nprocs=2, join=True,
                       start_method="spawn")
    _, _, (_, err0), raised0 = out[0]
    assert err0 != 0 and raised0 is not None and "expired" in raised0
    for rank in range(2):
        trees, pred, (epoch, err), raised = out[rank]
        assert np.all(np.isfinite(pred))
        assert (raised is not None) == (err != 0)
        for t in trees:
            st = t["node_state"]
            assert set(np.unique(st)) <= {0, 1, 2}
            assert t["n_rows"][0] == w.n and int(t["n_rows"][st == 2].sum()) == w.n   # leaves cover all rows
        if err:
            assert (err & 0xFF) in (1, 2)
