"""Feature-partitioned multi-process protocol on CPU with the gloo backend.

Two processes each own half of the features, search splits only on their shard with the CPU
oracle, and exchange exactly what the GPU path exchanges (paper_conf_icpp_liupw25_b200.parallel):
a MAX all-reduce of packed split keys and a SUM all-reduce of the owner's split record + row
bitmap.  The trees both ranks grow must equal the single-process oracle tree.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _sharded_tree(rank, world, loss, port, out):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from gen import gen
    from oracle import oracle
    from paper_conf_icpp_liupw25_b200 import parallel
    w = gen.WORKLOADS["C1"] if loss == 0 else gen.WORKLOADS["C2"].scaled(n=3000, m=24, D=4)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X).astype(np.float64)
    f0, f1 = parallel.shard_range(w.m, rank, world)
    cuts, nbins, bins = oracle.bin_matrix(np.ascontiguousarray(X[:, f0:f1]), w.B)
    g, h = oracle.grad(loss, Y, np.zeros_like(Y))
    n, D, B = w.n, w.D, w.B
    NH = (1 << (D + 1)) - 1
    state = np.zeros(NH, np.int32)
    feat = np.full(NH, -1, np.int32)
    binv = np.full(NH, -1, np.int32)
    nleft = np.zeros(NH, np.int64)
    rows = {0: np.arange(n, dtype=np.int32)}
    words = (n + 63) // 64
    for lvl in range(D):
        LN = 1 << lvl
        first = LN - 1
        keys = torch.zeros(LN, dtype=torch.int64)
        for i in range(LN):
            hid = first + i
            if hid not in rows:
                continue
            r = rows[hid]
            if len(r) < 2 * w.min_node:
                state[hid] = 2
                continue
            HG, HH, CNT = oracle.build_hist(bins, B, g, h, r)
            sp = oracle.find_split(HG, HH, CNT, nbins, g[r].sum(0), h[r].sum(0), len(r), w.lam, w.min_node)
            if sp["valid"] and sp["gain"] > w.gamma:
                keys[i] = parallel.pack_key(sp["gain"], f0 + sp["feature"], sp["bin"], B)
        parallel.exchange_keys(keys)
        rec = torch.zeros(LN * 3 + words, dtype=torch.int64)      # (f+1, b, n_left) per slot, then bitmap
        for i in range(LN):
            hid = first + i
            if hid not in rows or state[hid] == 2:
                continue
            dec = parallel.unpack_key(int(keys[i]), B)
            if dec is None:
                continue
            fg, b, _ = dec
            if f0 <= fg < f1:
                r = rows[hid]
                left = r[bins[fg - f0][r] <= b]
                rec[3 * i] = fg + 1
                rec[3 * i + 1] = b
                rec[3 * i + 2] = len(left)
                bm = np.zeros(words * 64, bool)
                bm[left] = True
                packed = np.packbits(bm, bitorder="little").view(np.uint64)
                rec[3 * LN:] += torch.from_numpy(packed.astype(np.int64))
        parallel.exchange_records(rec)
        bitmap = rec[3 * LN:].numpy().view(np.uint64)
        bits = np.unpackbits(bitmap.view(np.uint8), bitorder="little").astype(bool)[: n]
        for i in range(LN):
            hid = first + i
            if hid not in rows or state[hid] == 2:
                continue
            if int(rec[3 * i]) == 0:
                state[hid] = 2
                continue
            r = rows[hid]
            go = bits[r]
            state[hid] = 1
            feat[hid], binv[hid], nleft[hid] = int(rec[3 * i]) - 1, int(rec[3 * i + 1]), int(rec[3 * i + 2])
            assert go.sum() == nleft[hid]
            rows[2 * hid + 1] = r[go]
            rows[2 * hid + 2] = r[~go]
    for hid in rows:
        if state[hid] == 0:
            state[hid] = 2
    out[rank] = (state, feat, binv, nleft)
    dist.destroy_process_group()


@pytest.mark.parametrize("loss", [0, 1])
def test_two_rank_gloo_protocol_equals_single_process(orc, loss):
    from gen import gen
    w = gen.WORKLOADS["C1"] if loss == 0 else gen.WORKLOADS["C2"].scaled(n=3000, m=24, D=4)
    X = gen.features_host(w)
    Y = gen.targets_host(w, X).astype(np.float64)
    cuts, nbins, bins = orc.bin_matrix(X, w.B)
    ref = orc.train(bins, nbins, w.B, Y, loss=loss, T=1, D=w.D, lam=w.lam, gamma=w.gamma, lr=w.lr,
                    min_node=w.min_node)
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    mp.start_processes(_sharded_tree, args=(2, loss, port, out), nprocs=2, join=True, start_method="spawn")
    for rank in range(2):
        state, feat, binv, nleft = out[rank]
        np.testing.assert_array_equal(state, ref["state"][0])
        split = state == 1
        assert split.sum() >= 3
        np.testing.assert_array_equal(feat[split], ref["feat"][0][split])
        np.testing.assert_array_equal(binv[split], ref["bin"][0][split])
        np.testing.assert_array_equal(nleft[split], ref["n_left"][0][split])


def test_key_packing_orders_like_the_oracle_rule():
    from paper_conf_icpp_liupw25_b200 import parallel
    B = 256
    k1 = parallel.pack_key(10.0, 5, 3, B)
    k2 = parallel.pack_key(10.0, 5, 4, B)     # same gain: smaller bin wins
    k3 = parallel.pack_key(10.0, 4, 200, B)   # same gain: smaller feature wins
    k4 = parallel.pack_key(10.5, 900, 0, B)   # larger gain wins
    assert max(k1, k2) == k1 and max(k1, k3) == k3 and max(k3, k4) == k4
    assert parallel.pack_key(0.0, 1, 1, B) == 0 and parallel.pack_key(-1.0, 1, 1, B) == 0
    assert parallel.unpack_key(k3, B)[:2] == (4, 200)
    assert abs(parallel.unpack_key(k4, B)[2] - 10.5) < 10.5 * 2 ** -27
    assert parallel.shard_range(4096, 3, 8) == (1536, 2048)
