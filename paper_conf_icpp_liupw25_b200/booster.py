"""Driver of Algorithm 1 over the C ABI — host orchestration only.

Every arithmetic step runs in libgbdtmo.so kernels; this module allocates device buffers
with torch (plumbing), issues the ABI calls level by level, and — when a process group is
given — performs the two per-level exchanges of the feature-partitioned multi-GPU scheme
 with torch.distributed (NCCL): a MAX all-reduce of the packed split keys and
a SUM all-reduce of the owners' split records + row-direction bitmap.  Nothing in a tree
waits for the host, so a whole tree can be replayed as one CUDA graph.
"""
from __future__ import annotations

import dataclasses
import math
import os
from typing import Optional

import torch

from . import _abi
from . import parallel
from ._abi import Context, Problem, LOSS_MSE, LOSS_SOFTMAX


@dataclasses.dataclass
class Params:
    """Training parameters; defaults are the paper's: 100 trees, depth 7,
    learning rate 1, >= 20 instances per node, 256 bins; lambda = 1, gamma = 0 (readings R1, R2)."""
    loss: int = LOSS_MSE
    T: int = 100
    D: int = 7
    B: int = 256
    lam: float = 1.0
    gamma: float = 0.0
    lr: float = 1.0
    min_node: int = 20


# Measured variant table (tools/calibrate_hist.py -> hist_variant_table.json), per workload shape:
# gmem_max_rows = largest node (rows) built with the global-atomic histogram variant,
# small_max_rows = largest pair of siblings searched by sort-and-segment (small.cu) instead of
# histograms.  0 = off; missing table: shared-memory histograms everywhere.
_VARIANT_TABLE = None


def variant_threshold(V: int, m: int, key: str = "gmem_max_rows", n: Optional[int] = None) -> int:
    global _VARIANT_TABLE
    if _VARIANT_TABLE is None:
        import json
        import os
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "hist_variant_table.json")
        try:
            _VARIANT_TABLE = json.load(open(path))
        except (OSError, ValueError):
            _VARIANT_TABLE = {}
    entries = _VARIANT_TABLE.get("entries", [])
    if not entries:
        return 0
    # nearest measured shape: channel count first, then features and rows (log distance)
    def dist(e):
        dn = abs(math.log2(max(n, 1) / max(e.get("n", 1), 1))) if n else 0.0
        return (abs(math.log2(max(V, 1) / max(e["V"], 1))), abs(math.log2(max(m, 1) / max(e.get("m", 1), 1))) + dn)
    e = min(entries, key=dist)
    return int(e.get(key, 0))


class PeerExchangeError(RuntimeError):
    """A bounded peer-flag wait of the fused exchange expired (gbdtmo_peer_status error word != 0):
    the trees trained since are not valid (every later node becomes a leaf)."""


def _align(x, a):
    return (x + a - 1) // a * a


@dataclasses.dataclass
class Dataset:
    """Binned feature shard resident in HBM: bins uint8 [n][ld_bins] (row-major), cuts, nbins."""
    bins: torch.Tensor          # flat uint8 of gbdtmo_bins_bytes(n, ld_bins)
    nbins: torch.Tensor         # int32 [m]
    cuts: torch.Tensor          # float32 [m][B-1]
    n: int
    m: int
    ld_bins: int
    B: int
    f_begin: int = 0
    m_global: int = 0
    dflt: Optional[torch.Tensor] = None   # int32 [m] default (most frequent) bin per feature
    # CSC storage kept by bin_features_csc for gbdtmo_build_hist_csc: column
    # pointers int64 [m+1], row indices int32 [nnz], bins of the stored values uint8 [nnz], bin of an
    # implicit zero per feature int32 [m]
    csc_col_ptr: Optional[torch.Tensor] = None
    csc_row_idx: Optional[torch.Tensor] = None
    csc_nz_bins: Optional[torch.Tensor] = None
    csc_zbin: Optional[torch.Tensor] = None
    csc_nnz: int = 0


def bin_features(ctx: Context, X: torch.Tensor, B: int, f_begin: int = 0, m_global: Optional[int] = None,
                 bins_out: Optional[torch.Tensor] = None, ws: Optional[torch.Tensor] = None) -> Dataset:
    """gbdtmo_bin on a device float32 matrix [n][m] (row stride X.stride(0))."""
    assert X.is_cuda and X.dtype == torch.float32 and X.stride(1) == 1
    n, m = X.shape
    ld = _align(m, 16)
    nbytes = ctx.gbdtmo_bins_bytes(n, ld)
    bins = bins_out if bins_out is not None else torch.zeros(nbytes, dtype=torch.uint8, device=X.device)
    cuts = torch.empty((m, B - 1), dtype=torch.float32, device=X.device)
    nbins = torch.empty(m, dtype=torch.int32, device=X.device)
    wsb = ctx.gbdtmo_bin_workspace_bytes(n, m, B)
    if ws is None or ws.numel() < wsb:
        ws = torch.empty(wsb, dtype=torch.uint8, device=X.device)
    ctx.gbdtmo_set_stream(torch.cuda.current_stream(X.device).cuda_stream)
    ctx.gbdtmo_bin(X, n, m, X.stride(0), B, bins, ld, cuts, nbins, ws, wsb)
    # sparsity-aware default bins: only features whose top bin holds >= 1/16 of the rows
    dflt = torch.empty(m, dtype=torch.int32, device=X.device)
    ctx.gbdtmo_default_bins(bins, n, m, ld, B, max(1, n // 16), dflt)
    if not bool((dflt >= 0).any()):          # (one small D2H per dataset, not per tree)
        dflt = None
    return Dataset(bins, nbins, cuts, n, m, ld, B, f_begin, m_global if m_global is not None else m, dflt)


def bin_features_host(ctx: Context, Xh: torch.Tensor, B: int, device, f_begin: int = 0,
                      m_global: Optional[int] = None, strip: int = 512) -> Dataset:
    """gbdtmo_bin_host on a HOST float32 matrix [n][m] (pinned for asynchronous copies): the library
    uploads it in column strips on its copy stream while the previous strip is binned (binning is per
    column), so the device never holds all of X.  Same Dataset as bin_features on the whole matrix."""
    assert Xh.device.type == "cpu" and Xh.dtype == torch.float32 and Xh.is_contiguous()
    dev = torch.device(device)
    n, m = Xh.shape
    ld = _align(m, 16)
    bins = torch.zeros(ctx.gbdtmo_bins_bytes(n, ld), dtype=torch.uint8, device=dev)
    cuts = torch.empty((m, B - 1), dtype=torch.float32, device=dev)
    nbins = torch.empty(m, dtype=torch.int32, device=dev)
    wsb = ctx.gbdtmo_bin_host_workspace_bytes(n, m, B, strip)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    ctx.gbdtmo_set_stream(torch.cuda.current_stream(dev).cuda_stream)
    ctx.gbdtmo_bin_host(Xh.data_ptr(), n, m, m, B, bins, ld, cuts, nbins, ws, wsb, strip)
    dflt = torch.empty(m, dtype=torch.int32, device=dev)
    ctx.gbdtmo_default_bins(bins, n, m, ld, B, max(1, n // 16), dflt)
    if not bool((dflt >= 0).any()):          # (syncs the stream: Xh and ws are done with after this)
        dflt = None
    del ws
    return Dataset(bins, nbins, cuts, n, m, ld, B, f_begin, m_global if m_global is not None else m, dflt)


def bin_features_csc(ctx: Context, values: torch.Tensor, row_idx: torch.Tensor, col_ptr: torch.Tensor, n: int,
                     B: int, f_begin: int = 0, m_global: Optional[int] = None) -> Dataset:
    """gbdtmo_bin_csc on the paper's sparse storage: values float32 [nnz],
    row_idx int32 [nnz] (device), col_ptr int64 [m+1] (host or device).  Same Dataset as
    bin_features on the dense matrix."""
    cp_host = col_ptr.detach().to("cpu", torch.int64).contiguous()
    dev = values.device
    assert values.is_cuda and values.dtype == torch.float32 and row_idx.dtype == torch.int32
    cp_dev = cp_host.to(dev)
    m = cp_host.numel() - 1
    ld = _align(m, 16)
    bins = torch.zeros(ctx.gbdtmo_bins_bytes(n, ld), dtype=torch.uint8, device=dev)
    cuts = torch.empty((m, B - 1), dtype=torch.float32, device=dev)
    nbins = torch.empty(m, dtype=torch.int32, device=dev)
    wsb = ctx.gbdtmo_bin_workspace_bytes(n, m, B)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    ctx.gbdtmo_set_stream(torch.cuda.current_stream(dev).cuda_stream)
    ctx.gbdtmo_bin_csc(values if values.numel() else None, row_idx if row_idx.numel() else None, cp_dev, cp_host,
                       n, m, B, bins, ld, cuts, nbins, ws, wsb)
    dflt = torch.empty(m, dtype=torch.int32, device=dev)
    ctx.gbdtmo_default_bins(bins, n, m, ld, B, max(1, n // 16), dflt)
    if not bool((dflt >= 0).any()):
        dflt = None
    nnz = int(cp_host[-1])
    nz_bins = torch.empty(max(nnz, 1), dtype=torch.uint8, device=dev)
    zbin = torch.empty(m, dtype=torch.int32, device=dev)
    ctx.gbdtmo_csc_nz_bins(m, B, cp_dev, row_idx if nnz else None, bins, ld, cuts, nz_bins, zbin)
    return Dataset(bins, nbins, cuts, n, m, ld, B, f_begin, m_global if m_global is not None else m, dflt,
                   csc_col_ptr=cp_dev, csc_row_idx=row_idx, csc_nz_bins=nz_bins, csc_zbin=zbin, csc_nnz=nnz)


class Booster:
    """One GBDT-MO model being trained on one GPU (one feature shard when `group` is given)."""

    def __init__(self, ctx: Context, ds: Dataset, y: torch.Tensor, params: Params,
                 group=None, pred: Optional[torch.Tensor] = None, keep_model: bool = True,
                 sparse_default: bool = False, gmem_max_rows: Optional[int] = None,
                 small_max_rows: Optional[int] = None, hist_kernel: Optional[int] = None,
                 packed_bins: Optional[bool] = None, exchange: str = "collective", cache_root_counts: bool = True,
                 fs_channel_groups: int = 0, csc_hist: Optional[bool] = None, csc_levels: Optional[int] = None,
                 hist_waves: Optional[int] = None):
        """exchange (only with `group`): "collective" = torch.distributed all-reduces per level;
        "peer" = the fused peer-memory exchange (NEXT-4, gbdtmo_*_peer): the keys / records are
        read from the other ranks' windows inside split_record / partition, no host collective.
        fs_channel_groups: GBDTMO_OPT_FS_CHANNEL_GROUPS (0 automatic, 1 off, 2 / 4 / 8 forced).
        csc_hist: build the histograms of levels < csc_levels (all by default) from the dataset's CSC
        non-zeros (gbdtmo_build_hist_csc; datasets from bin_features_csc), the deeper ones from the bins;
        None = automatic: on for CSC datasets below 4% density (measured crossover ~5%: C3 at 1% of its
        entries 2.43 vs 4.36 ms per tree, at 20% 9.7 vs 4.6; profiles/r02c_csc_probe.jsonl)."""
        self.ctx, self.ds, self.params, self.group = ctx, ds, params, group
        assert exchange in ("collective", "peer")
        self.exchange = exchange if group is not None else "collective"
        # histogram variant selection: nodes with <= gmem_max_rows
        # rows use the global-atomic variant; None = the measured table for this channel count
        V = y.shape[1] * (2 if params.loss == LOSS_SOFTMAX else 1)
        self.gmem_max_rows = variant_threshold(V, ds.m, n=ds.n) if gmem_max_rows is None else int(gmem_max_rows)
        self.small_max_rows = variant_threshold(V, ds.m, "small_max_rows", n=ds.n) if small_max_rows is None \
            else int(small_max_rows)
        # shared-memory lane mapping: 0 row-pair tiles, 1 diagonal K = 4 tiles (measured per shape)
        self.hist_kernel = variant_threshold(V, ds.m, "hist_kernel", n=ds.n) if hist_kernel is None \
            else int(hist_kernel)
        # histogram work items per level in SM multiples (GBDTMO_OPT_HIST_WAVES; measured per shape)
        self.hist_waves = variant_threshold(V, ds.m, "hist_waves", n=ds.n) if hist_waves is None else int(hist_waves)
        # sparsity-aware default-bin skip; None = accumulate every bin.  Off by
        # default: measured slower on C2 (8.55 vs 7.84 ms/tree), where per-node overheads dominate.
        self.dflt = ds.dflt if sparse_default else None
        if csc_hist is None:
            csc_hist = ds.csc_zbin is not None and ds.csc_nnz < 0.04 * ds.n * ds.m
        self.csc_hist = bool(csc_hist)
        self.csc_levels = params.D if csc_levels is None else int(csc_levels)
        if self.csc_hist:
            assert ds.csc_zbin is not None, "csc_hist needs a dataset from bin_features_csc"
            cache_root_counts = False
            if self.csc_levels >= params.D:      # no level reads the bins for histograms
                self.gmem_max_rows = 0
                packed_bins = False
        self.fs_channel_groups = int(fs_channel_groups)
        dev = ds.bins.device
        self.device = dev
        n, d = y.shape
        assert n == ds.n and y.dtype == torch.float32 and y.is_contiguous()
        self.y = y
        self.d = d
        self.p = Problem(n=n, m=ds.m, f_begin=ds.f_begin, m_global=ds.m_global or ds.m, d=d, B=ds.B, D=params.D,
                         loss=params.loss, min_node=params.min_node, lambda_=params.lam, gamma=params.gamma,
                         lr=params.lr, ld_bins=ds.ld_bins)
        V = self.p.V
        D = params.D
        self.pred = pred if pred is not None else torch.zeros((n, d), dtype=torch.float64, device=dev)
        assert self.pred.dtype == torch.float64
        self.q = torch.empty((n, V), dtype=torch.int32, device=dev)
        self.gh = torch.empty((n, V), dtype=torch.float64, device=dev)   # fp64 g/h for exact leaf sums
        self.scales = torch.empty(V, dtype=torch.float32, device=dev)
        self.state = torch.empty(ctx.gbdtmo_state_bytes(self.p), dtype=torch.uint8, device=dev)
        self.hist, self.cnt = [None, None], [None, None]
        for lvl in (D - 1, D - 2):
            if lvl < 0:
                continue
            hb, cb = ctx.gbdtmo_hist_bytes(self.p, lvl)
            self.hist[lvl % 2] = torch.empty(hb // 8, dtype=torch.int64, device=dev)
            self.cnt[lvl % 2] = torch.empty(cb // 4, dtype=torch.int32, device=dev)
        if self.hist[1] is None:
            self.hist[1], self.cnt[1] = self.hist[0], self.cnt[0]
        # tile-packed bins for the row-pair histogram kernel (gbdtmo_pack_bins):
        # default on wherever the shape allows it and that kernel is selected
        nb = ctx.gbdtmo_packed_bins_bytes(self.p)
        use_packed = (nb > 0 and self.hist_kernel == 0) if packed_bins is None else bool(packed_bins)
        self.packed = None
        if use_packed:
            assert nb > 0, "this problem shape has no packed bin layout"
            self.packed = torch.empty(nb, dtype=torch.uint8, device=dev)
            ctx.gbdtmo_set_stream(torch.cuda.current_stream(dev).cuda_stream)
            ctx.gbdtmo_pack_bins(self.p, ds.bins, self.packed)
        self.keys = torch.zeros(1 << max(D - 1, 0), dtype=torch.int64, device=dev)
        self.xchg = torch.zeros(ctx.gbdtmo_xchg_count(self.p), dtype=torch.int64, device=dev)
        # root counts are the same for every tree (all rows): cached after the first tree's level 0
        self.cache_root_counts = cache_root_counts
        self.root_cnt = None
        self.peer_keys = None
        self._peer_host = None          # pinned int64 [2]: (epoch, error) copied after every tree
        self._peer_evt = None
        if self.exchange == "peer":
            self._peer_connect()
        NH = (1 << (D + 1)) - 1
        self.NH = NH
        self.leaf = torch.empty((NH, d), dtype=torch.float64, device=dev)
        self.keep_model = keep_model
        self.trees = []            # per tree: dict of device tensors (heap-indexed tree record)
        self._graph = None
        self.hist_events = []      # optional per-level (start, end) CUDA events around build_hist
        self.phase_marks = []      # optional per-tree phase marks (time_hist=True), see phase_ms()
        self._marks = []

    def _peer_connect(self):
        """Open this rank's window, exchange the IPC handles over the process group (plumbing),
        map the peers' windows; keys of level l are then written straight into the window."""
        import torch.distributed as dist
        rank, world = dist.get_rank(self.group), dist.get_world_size(self.group)
        torch.cuda.synchronize(self.device)
        if os.environ.get("GBDTMO_PEER_TIMEOUT_MS"):         # (tests: force expiry)
            self.ctx.gbdtmo_set_option(_abi.OPT_PEER_TIMEOUT_MS, int(os.environ["GBDTMO_PEER_TIMEOUT_MS"]))
        # every rank takes part in both gathers whatever happens locally, and all ranks agree on
        # the outcome, so a failure anywhere raises everywhere (no rank left in a collective)
        err = None
        try:
            h = self.ctx.gbdtmo_peer_open(self.p, rank, world)
        except _abi.GbdtmoError as ex:
            h, err = None, ex
        handles = [None] * world
        dist.all_gather_object(handles, h, group=self.group)
        if err is None and all(x is not None for x in handles):
            try:
                self.ctx.gbdtmo_peer_connect(b"".join(handles))
            except _abi.GbdtmoError as ex:
                err = ex
        elif err is None:
            err = RuntimeError("gbdtmo_peer_open failed on another rank")
        oks = [None] * world
        dist.all_gather_object(oks, err is None, group=self.group)
        if not all(oks):
            self.ctx.gbdtmo_peer_close()
            raise RuntimeError(f"peer exchange unavailable (rank {rank}: {err or 'ok'}; ranks ok: {oks})")
        self.peer_keys = [self.ctx.gbdtmo_peer_buffers(self.p, lvl)[0] for lvl in range(self.params.D)]

    def peer_status(self):
        """(exchanges completed, error word) of the peer window (synchronous); error 0 = healthy."""
        return self.ctx.gbdtmo_peer_status()

    def check_peer(self, block: bool = False):
        """Raise PeerExchangeError if the peer window's (sticky) error word is set.  Reads the
        copy enqueued after the last tree (gbdtmo_peer_status_async); block=False only looks if
        that copy has landed (no device synchronisation), block=True waits for it."""
        if self._peer_evt is None:
            return
        if not block and not self._peer_evt.query():
            return
        self._peer_evt.synchronize()
        epoch, err = int(self._peer_host[0]), int(self._peer_host[1])
        if err:
            raise PeerExchangeError(
                f"peer exchange wait expired (error word {err:#x}: epoch {err >> 8}, phase {err & 0xFF}; "
                f"{epoch} exchanges completed): trees trained since then are invalid")

    def _peer_after_tree(self):
        """Once per tree, asynchronously: check the previous tree's status copy if it has landed,
        then enqueue a copy of this tree's (epoch, error) words (no host synchronisation)."""
        if self.exchange != "peer":
            return
        self.check_peer(block=False)
        if self._peer_host is None:
            self._peer_host = torch.zeros(2, dtype=torch.int64).pin_memory()
        self.ctx.gbdtmo_set_stream(torch.cuda.current_stream(self.device).cuda_stream)
        self.ctx.gbdtmo_peer_status_async(self._peer_host)
        self._peer_evt = torch.cuda.Event()
        self._peer_evt.record(torch.cuda.current_stream(self.device))

    # ------------------------------------------------------------------ one tree
    def _level(self, lvl: int, time_hist: bool = False):
        ctx, p = self.ctx, self.p
        cur, par = lvl % 2, (lvl - 1) % 2
        ph = self.hist[par] if lvl > 0 else None
        pc = self.cnt[par] if lvl > 0 else None
        if time_hist:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
        if self.csc_hist and lvl < self.csc_levels:
            ds = self.ds
            ctx.gbdtmo_build_hist_csc(p, lvl, ds.csc_col_ptr, ds.csc_row_idx, ds.csc_nz_bins, ds.csc_nnz, ds.csc_zbin,
                                      self.q, self.state, self.hist[cur], self.cnt[cur])
        elif self.packed is not None:
            ctx.gbdtmo_build_hist_packed(p, lvl, self.ds.bins, self.packed, self.dflt, self.q, self.state,
                                         self.hist[cur], self.cnt[cur])
        else:
            ctx.gbdtmo_build_hist(p, lvl, self.ds.bins, self.dflt, self.q, self.state, self.hist[cur], self.cnt[cur])
        if time_hist:
            e1.record()
            self.hist_events.append((e0, e1))
        self._mark("find_split", time_hist)
        peer = self.exchange == "peer"
        keys = self.peer_keys[lvl] if peer else self.keys     # peer: this level's window keys
        ctx.gbdtmo_find_split(p, lvl, self.ds.nbins, self.dflt, self.scales, self.state, self.hist[cur], self.cnt[cur],
                              ph, pc, keys)
        if self.small_max_rows > 0:
            ctx.gbdtmo_search_small(p, lvl, self.ds.bins, self.q, self.ds.nbins, self.scales, self.state, keys)
        self._mark("split_record", time_hist)
        if peer:
            ctx.gbdtmo_split_record_peer(p, lvl, self.ds.bins, self.dflt, self.q, self.scales, self.state,
                                         self.hist[cur], self.cnt[cur], ph, pc, self.keys)
            self._mark("partition", time_hist)
            ctx.gbdtmo_partition_peer(p, lvl, self.state, self.xchg)
            return
        if self.group is not None:
            parallel.exchange_keys(self.keys[: 1 << lvl], self.group)
        ctx.gbdtmo_split_record(p, lvl, self.ds.bins, self.dflt, self.q, self.scales, self.state, self.hist[cur],
                                self.cnt[cur],
                                ph, pc, self.keys, self.xchg)
        if self.group is not None:
            parallel.exchange_records(self.xchg, self.group)
        self._mark("partition", time_hist)
        ctx.gbdtmo_partition(p, lvl, self.state, self.xchg)

    def _apply_options(self):
        """Context state for this booster's calls: stream and histogram-variant thresholds."""
        ctx = self.ctx
        ctx.gbdtmo_set_stream(torch.cuda.current_stream(self.device).cuda_stream)
        ctx.gbdtmo_set_option(_abi.OPT_GMEM_MAX_ROWS, self.gmem_max_rows)
        ctx.gbdtmo_set_option(_abi.OPT_SMALL_MAX_ROWS, self.small_max_rows)
        ctx.gbdtmo_set_option(_abi.OPT_HIST_KERNEL, self.hist_kernel)
        ctx.gbdtmo_set_option(_abi.OPT_FS_CHANNEL_GROUPS, self.fs_channel_groups)
        ctx.gbdtmo_set_option(_abi.OPT_HIST_WAVES, self.hist_waves)
        ctx.gbdtmo_set_root_counts(self.root_cnt)

    def _mark(self, name: str, on: bool):
        """(timing) an event recorded before the phase `name`; the phase lasts until the next mark."""
        if on:
            e = torch.cuda.Event(enable_timing=True)
            e.record()
            self._marks.append((name, e))

    def phase_ms(self, trees):
        """Per-phase device ms summed over the last `trees` timed trees (from the marks)."""
        tot = {}
        for marks in self.phase_marks[-trees:]:
            for (name, e0), (_, e1) in zip(marks[:-1], marks[1:]):
                tot[name] = tot.get(name, 0.0) + e0.elapsed_time(e1)
        return tot

    def _tree(self, time_hist: bool = False):
        ctx, p = self.ctx, self.p
        self._apply_options()
        self._marks = []
        self._mark("grad", time_hist)
        ctx.gbdtmo_grad(p, self.y, self.pred, self.q, self.scales, self.state, self.gh)
        for lvl in range(self.params.D):
            self._mark("build_hist", time_hist)
            self._level(lvl, time_hist)
            if lvl == 0 and self.cache_root_counts and self.root_cnt is None:
                # (plumbing: one device copy per dataset) the level-0 counts after find_split
                self.root_cnt = self.cnt[0][: self.p.m * self.p.B].clone()
        self._mark("leaf+update", time_hist)
        ctx.gbdtmo_leaf_values(p, self.scales, self.state, self.leaf, self.gh)   # fp64 row sums (R17)
        ctx.gbdtmo_update_pred(p, self.state, self.leaf, self.pred)
        self._mark("end", time_hist)
        if time_hist:
            self.phase_marks.append(self._marks)

    def step(self, time_hist: bool = False):
        """One boosting iteration (one tree) on the current stream; asynchronous.  With the peer
        exchange, raises PeerExchangeError as soon as a failed wait of an earlier tree is seen."""
        self._tree(time_hist)
        self._peer_after_tree()
        if self.keep_model:
            self.trees.append(self.export())

    def export(self):
        NH, dev = self.NH, self.device
        rec = dict(node_state=torch.empty(NH, dtype=torch.int32, device=dev),
                   feature=torch.empty(NH, dtype=torch.int32, device=dev),
                   bin=torch.empty(NH, dtype=torch.int32, device=dev),
                   gain=torch.empty(NH, dtype=torch.float64, device=dev),
                   n_rows=torch.empty(NH, dtype=torch.int64, device=dev),
                   n_left=torch.empty(NH, dtype=torch.int64, device=dev),
                   threshold=torch.empty(NH, dtype=torch.float32, device=dev))
        # the current stream (after a graph capture the context still names the capture stream)
        self.ctx.gbdtmo_set_stream(torch.cuda.current_stream(dev).cuda_stream)
        self.ctx.gbdtmo_tree_export(self.p, self.state, rec["node_state"], rec["feature"], rec["bin"], rec["gain"],
                                    rec["n_rows"], rec["n_left"], self.ds.cuts, rec["threshold"])
        if self.group is not None:   # thresholds live with the feature's owner: SUM merges them
            parallel.exchange_records(rec["threshold"], self.group)
        rec["leaf"] = self.leaf.clone()
        return rec

    def fit(self, T: Optional[int] = None, graph: Optional[bool] = None):
        """Train T trees.  graph=None: small single-process problems (n m <= 1e8, T >= 4), whose trees
        are launch-bound (~100 launches of a few microseconds), replay trees 2.. from one captured
        CUDA graph (identical results, tested); graph=True/False forces either."""
        T = T if T is not None else self.params.T
        if graph is None:
            graph = self.group is None and T >= 4 and self.ds.n * self.ds.m <= 100_000_000
        if graph and self.group is None and T >= 2:
            self.step()                                  # tree 1 eagerly: allocations, attributes
            self.capture(warmup=False)
            for _ in range(T - 1):
                self.step_graph()
        else:
            for _ in range(T):
                self.step()
        self.check_peer(block=True)
        return self

    # ----------------------------------------------------------------- graphs
    def capture(self, warmup: bool = True):
        """Capture one tree (grad .. update_pred) as a CUDA graph; replay with step_graph().
        warmup=False when a tree has already run eagerly on this Booster (attributes are set)."""
        s = torch.cuda.Stream(self.device)
        s.wait_stream(torch.cuda.current_stream(self.device))
        if warmup:
            saved = self.pred.clone()         # the warm-up tree is not part of the model
            with torch.cuda.stream(s):
                self._tree()                  # warm-up outside the graph (allocations, attributes)
                self.pred.copy_(saved)
            del saved
        torch.cuda.current_stream(self.device).wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            self._tree()
        self._graph = g
        return g

    def step_graph(self):
        self._graph.replay()
        self._peer_after_tree()
        if self.keep_model:
            self.trees.append(self.export())


def train(X, Y, params: Params, device: str = "cuda:0", ctx: Optional[Context] = None, group=None,
          f_begin: int = 0, m_global: Optional[int] = None, exchange: str = "collective"):
    """Public entry point: X float32 [n][m] and Y float32 [n][d] (host or device tensors or numpy
    arrays).  Copies the inputs to the GPU, bins the features, trains params.T trees, and
    returns the Booster (predictions in booster.pred, tree records in booster.trees)."""
    dev = torch.device(device)
    ctx = ctx or Context(dev.index or 0)
    Xt = torch.as_tensor(X)
    Yt = torch.as_tensor(Y)
    Yd = Yt.to(dev, non_blocking=True).contiguous().float()
    if Xt.device.type == "cpu" and Xt.dtype == torch.float32 and Xt.is_contiguous():
        # host matrix: strip-wise upload overlapped with binning (the device never holds all of X)
        ds = bin_features_host(ctx, Xt, params.B, dev, f_begin=f_begin, m_global=m_global)
    else:
        Xd = Xt.to(dev, non_blocking=True).contiguous().float()
        ds = bin_features(ctx, Xd, params.B, f_begin=f_begin, m_global=m_global)
        del Xd
    b = Booster(ctx, ds, Yd, params, group=group, exchange=exchange)
    b.fit()
    return b


def predict(ctx: Context, trees, X: torch.Tensor, D: int, d: int, pred: Optional[torch.Tensor] = None):
    """gbdtmo_predict: sum of the trees' leaf values for unseen rows X (device float32 [n][m_global]).
    `trees` is a list of exported tree records (Booster.trees)."""
    assert X.is_cuda and X.dtype == torch.float32 and X.stride(1) == 1
    n = X.shape[0]
    T = len(trees)
    dev = X.device
    pred = pred if pred is not None else torch.zeros((n, d), dtype=torch.float64, device=dev)
    if T == 0:
        return pred
    st = torch.stack([t["node_state"] for t in trees]).contiguous()
    ft = torch.stack([t["feature"] for t in trees]).contiguous()
    th = torch.stack([t["threshold"] for t in trees]).contiguous()
    lf = torch.stack([t["leaf"] for t in trees]).contiguous()
    ctx.gbdtmo_set_stream(torch.cuda.current_stream(dev).cuda_stream)
    ctx.gbdtmo_predict(X, n, X.shape[1], X.stride(0), T, D, d, st, ft, th, lf, pred)
    return pred
