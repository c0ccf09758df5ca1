"""Benchmark of the GBDT-MO hot path (one training tree = one step) on 1..8 B200s.

Default workload: BASELINE.json configs[4] (C5: n = 2,000,000, m = 4,096, d = 16 outputs,
256 bins, depth 8, MSE) -- the configuration the metric is quoted on at 1/2/4/8 GPUs.
Features are partitioned across ranks; every rank replicates y, yhat, g.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C5] [--impl ours|reference]

Prints ONE JSON line on rank 0.  `value` = logical histogram rows x outputs per second of the
whole job: sum over levels of the rows in the nodes searched at that level, times d, divided by
the device time per tree (max over ranks).  See DESIGN.md "Measurement".
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# BASELINE.json's metric; `value` is its throughput half (hist rows x outputs per second, whole
# job), `sec_per_tree` its time half, `roofline.hbm_view` its "% HBM roofline" part.
L2_BYTES = 126 * 1024 * 1024          # B200 L2 (B200_PROFILING.md)
METRIC = "sec/tree & hist rows\u00b7outputs/s at 1/2/4/8 B200; % HBM roofline"
UNIT = "rows*outputs/s"


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="C5")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--graph", action="store_true", help="replay each tree as a CUDA graph (1 GPU)")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N > 1 (gloo: lets N ranks share one GPU for testing)")
    ap.add_argument("--no-root-cache", action="store_true", help="(A/B) accumulate the root counts every tree")
    ap.add_argument("--predict", action="store_true",
                    help="NEXT-3 line: inference throughput (rows x trees / s) of gbdtmo_predict on unseen rows of "
                         "the workload, with a model of --predict-trees trees trained first (1 GPU)")
    ap.add_argument("--predict-trees", type=int, default=100)
    ap.add_argument("--exchange", default="auto", choices=["auto", "peer", "collective"],
                    help="N > 1 split exchange: peer = fused peer-memory exchange inside the kernels (NEXT-4), "
                         "collective = torch.distributed all-reduces; auto = peer, verified after the warm-up "
                         "(identical trees on every rank, no timeout) else collective")
    return ap.parse_args()


# --------------------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi samples during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1])); smax.append(float(f[2])); power.append(float(f[3]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(smax), "reasons": sorted(reasons),
                "samples": len(sm), "power_w_max": max(power)}


# ------------------------------------------------------------- same-run roofline denominators

def measure_atoms_peak(device):
    """Shared-memory atomic ceiling measured in this process right before the timed region
    (tools/microbench/peaks.cu): mode 0 = conflict-free red.shared.add.u32 (the pipe ceiling, the
    roofline peak), mode 1 = the histogram kernel's own row-pair lane map.  None if unavailable."""
    import ctypes as C
    path = os.path.join(ROOT, "tools", "microbench", "libgbdtmo_peaks.so")
    if not os.path.exists(path):
        return None
    L = C.CDLL(path)
    L.peaks_atoms.argtypes = [C.c_int, C.c_int, C.c_int] + [C.POINTER(C.c_double)] * 3
    out = {}
    for mode, name in ((0, "pipe"), (1, "hist_lane_map")):
        a, b, c = C.c_double(), C.c_double(), C.c_double()
        rc = L.peaks_atoms(device, mode, 80_000, C.byref(a), C.byref(b), C.byref(c))
        if rc != 0:
            return None
        out[name] = {"lane_ops_per_clk_sm": a.value, "lane_ops_per_s": b.value, "clk_mhz": c.value}
    return out


# ---------------------------------------------------------------------------- setup

def built_rows(tree_np, D):
    """Rows whose histograms were built (root + smaller child of every split with a searched child)."""
    st, nr, nl = tree_np["node_state"], tree_np["n_rows"], tree_np["n_left"]
    total = int(nr[0]) if st[0] in (1, 2) and tree_np["_searched"].get(0, False) else 0
    for h in range(len(st)):
        if st[h] == 1:
            lvl = int(np.floor(np.log2(h + 1)))
            if lvl + 1 >= D:
                continue
            l, r = 2 * h + 1, 2 * h + 2
            if tree_np["_searched"].get(l, False) or tree_np["_searched"].get(r, False):
                total += int(min(nl[h], nr[h] - nl[h]))
    return total


def built_rows_by_level(tree_np, D):
    """Rows built per level (level 0: the root; level l+1: smaller children of level-l splits)."""
    st, nr, nl = tree_np["node_state"], tree_np["n_rows"], tree_np["n_left"]
    out = [0] * D
    if st[0] in (1, 2) and tree_np["_searched"].get(0, False):
        out[0] = int(nr[0])
    for h in range(len(st)):
        if st[h] == 1:
            lvl = int(np.floor(np.log2(h + 1)))
            if lvl + 1 >= D:
                continue
            l, r = 2 * h + 1, 2 * h + 2
            if tree_np["_searched"].get(l, False) or tree_np["_searched"].get(r, False):
                out[lvl + 1] += int(min(nl[h], nr[h] - nl[h]))
    return out


def annotate_searched(tree_np, D, min_node):
    st, nr = tree_np["node_state"], tree_np["n_rows"]
    s = {}
    for h in range(len(st)):
        lvl = int(np.floor(np.log2(h + 1)))
        s[h] = st[h] in (1, 2) and lvl < D and nr[h] >= 2 * min_node
    tree_np["_searched"] = s
    return tree_np


def host_targets(w):
    from gen import gen
    return gen.targets_host(w)


# ------------------------------------------------------------------------ CPU oracle

_ORACLE_SAMPLES = {}


def cpu_oracle_sample(w, feats=128, trees=1):
    """The oracle as it stands (oracle_train, fp64, OpenMP) on a bounded sample of the workload:
    all n rows and d outputs, `feats` of the m features, `trees` trees of depth D.  The sample's
    columns are generated and binned once per (workload, feats) and reused (only training is timed)."""
    feats = min(feats, w.m)
    from oracle import oracle
    key = (w.name, feats)
    if key not in _ORACLE_SAMPLES:
        from gen import gen
        cols = np.linspace(0, w.m - 1, feats).astype(np.int64)
        X = np.empty((w.n, feats), np.float32)
        for j, c in enumerate(cols):
            X[:, j] = gen.features_host(w, 0, w.n, int(c), 1)[:, 0]
        cuts, nbins, bins = oracle.bin_matrix(X, w.B)
        del X
        _ORACLE_SAMPLES.clear()
        _ORACLE_SAMPLES[key] = (nbins, bins, host_targets(w).astype(np.float64))
    nbins, bins, Y = _ORACLE_SAMPLES[key]
    t0 = time.perf_counter()
    res = oracle.train(bins, nbins, w.B, Y, loss=w.loss, T=trees, D=w.D, lam=w.lam, gamma=w.gamma, lr=w.lr,
                       min_node=w.min_node)
    dt = time.perf_counter() - t0
    ro = 0
    for t in range(trees):
        tr = annotate_searched({"node_state": res["state"][t], "n_rows": res["nrows"][t],
                                "n_left": res["n_left"][t]}, w.D, w.min_node)
        ro += sum(int(tr["n_rows"][h]) for h, sv in tr["_searched"].items() if sv) * w.d
    # time scales with the feature count: rate for the full m = ro / (dt * m / feats)
    value = ro / (dt * w.m / feats)
    return {"value": value, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"oracle_train: {trees} tree(s), all {w.n} rows, d={w.d}, depth {w.D}, {feats} of {w.m} "
                      f"features (evenly spaced); time scaled x{w.m / feats:.0f} to all features",
            "seconds": dt, "sec_per_tree_full_m": dt / trees * w.m / feats}


# ------------------------------------------------------------------------------ main

def main():
    a = parse()
    rank, world, local = _env_int("RANK", 0), _env_int("WORLD_SIZE", 1), _env_int("LOCAL_RANK", 0)
    from gen import gen
    w = gen.sweep(int(a.workload[1:])) if a.workload.startswith("S") else gen.WORKLOADS[a.workload]

    if a.impl == "reference":
        # the oracle as it stands, on the host cores: W untimed + K timed bounded samples of this
        # workload (all rows and outputs, a feature subset sized so the run stays within minutes)
        if rank != 0:
            return 0
        first = cpu_oracle_sample(w)                       # (warm-up 1; also sizes the samples)
        budget_s = 120.0
        n_more = max(a.warmup - 1, 0) + a.steps
        feats = int(min(128, max(8, 128 * budget_s / max(n_more * first["seconds"], 1e-9))))
        for _ in range(max(a.warmup - 1, 0)):
            cpu_oracle_sample(w, feats=feats)
        timed = [cpu_oracle_sample(w, feats=feats) for _ in range(a.steps)]
        val = float(np.median([t["value"] for t in timed]))
        cb = dict(timed[len(timed) // 2], value=val)
        out = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": a.gpus,
               "steps": a.steps, "warmup": a.warmup, "ms_per_step": float(np.median([t["sec_per_tree_full_m"] for t in timed])) * 1e3,
               "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
               "data": "synthetic (seeded counter-based generator, gen/)",
               "config": {"workload": w.name, "n": w.n, "m": w.m, "d": w.d, "B": w.B, "D": w.D,
                          "loss": "mse" if w.loss == 0 else "softmax", "parallelism": "CPU oracle (fp64, OpenMP)"},
               "cpu_baseline": cb,
               "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(out))
        return 0

    import torch
    import torch.distributed as dist
    import paper_conf_icpp_liupw25_b200 as pkg

    if a.predict:
        if rank != 0:
            return 0
        return predict_main(a, w, local % torch.cuda.device_count())

    local = local % torch.cuda.device_count()       # (ranks may share a GPU with --backend gloo)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    group = None
    if world > 1:
        if a.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
        group = dist.group.WORLD
    from paper_conf_icpp_liupw25_b200.parallel import shard_range
    f0, f1 = shard_range(w.m, rank, world)
    m_loc = f1 - f0
    ctx = pkg.Context(local)
    params = pkg.Params(loss=w.loss, T=a.steps + a.warmup, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr,
                        min_node=w.min_node)

    # ---- inputs in HBM (untimed): X shard generated on the device, binned by gbdtmo_bin
    t_setup = time.perf_counter()
    # targets: computed once on rank 0's host and broadcast (every rank replicates y)
    if rank == 0:
        Y = torch.from_numpy(host_targets(w)).to(dev)
    else:
        Y = torch.empty((w.n, w.d), dtype=torch.float32, device=dev)
    if group is not None:
        dist.broadcast(Y, src=0, group=group)
    if w.classes_sweep:                 # features depend on the labels: generated on the host
        X = torch.from_numpy(gen.features_host(w, 0, w.n, f0, m_loc)).to(dev)
    else:
        X = torch.empty((w.n, m_loc), dtype=torch.float32, device=dev)
        gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, f0, m_loc, w.m, X.data_ptr(), m_loc,
                        torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    tb0 = torch.cuda.Event(enable_timing=True); tb1 = torch.cuda.Event(enable_timing=True)
    tb0.record()
    ds = pkg.bin_features(ctx, X, w.B, f_begin=f0, m_global=w.m)
    tb1.record()
    torch.cuda.synchronize()
    bin_ms_first = tb0.elapsed_time(tb1)          # includes first-touch allocation of bins + workspace
    tb0.record()                                   # warm: the steady-state cost of gbdtmo_bin
    ds2 = pkg.bin_features(ctx, X, w.B, f_begin=f0, m_global=w.m)
    tb1.record()
    torch.cuda.synchronize()
    bin_ms = tb0.elapsed_time(tb1)
    del ds2
    del X
    torch.cuda.empty_cache()
    exchange = a.exchange if a.exchange != "auto" else ("peer" if world > 1 else "collective")
    exchange_note = None
    try:
        booster = pkg.Booster(ctx, ds, Y, params, group=group, exchange=exchange,
                              cache_root_counts=not a.no_root_cache)
    except Exception as ex:            # e.g. CUDA IPC unavailable: the collective path
        if a.exchange == "peer":
            raise
        exchange, exchange_note = "collective", f"peer setup failed: {type(ex).__name__}: {ex}"[:200]
        booster = pkg.Booster(ctx, ds, Y, params, group=group, exchange=exchange)
    setup_s = time.perf_counter() - t_setup

    # ---- warm-up
    for _ in range(a.warmup):
        booster.step()
    if world > 1 and booster.exchange == "peer":
        ok = peer_consistent(booster, group, dev)
        if not ok and a.exchange == "auto":
            exchange, exchange_note = "collective", "peer exchange failed its post-warm-up check"
            pred0 = torch.zeros_like(booster.pred)
            del booster
            booster = pkg.Booster(ctx, ds, Y, params, group=group, exchange=exchange, pred=pred0)
            for _ in range(a.warmup):
                booster.step()
        elif not ok:
            raise RuntimeError("peer exchange failed its post-warm-up check")
    if a.graph and world == 1:
        booster.capture()
    torch.cuda.synchronize()
    if group is not None:
        dist.barrier()
    booster.hist_events.clear()
    atoms_peak = measure_atoms_peak(local)
    torch.cuda.synchronize()

    # ---- timed region: K trees, device time, max over ranks
    clk = ClockSampler(local)
    clk.start()
    time.sleep(0.3)
    # no Python GC pause inside the timed region (a gen-2 collection stalls the enqueueing thread
    # for tens of ms and the GPU idles: measured as a run-to-run tail on the small configs)
    gc.collect()
    gc.disable()
    l0 = ctx.gbdtmo_launch_count()
    torch.cuda.synchronize()
    if group is not None:
        dist.barrier()
    # L2 rule: a tree reads its bins, q and fp64 g/h from HBM; when those inputs fit twice in L2 the
    # trees are timed one by one with an L2 flush (a 256 MB write) between them, outside the events
    in_bytes = sum(int(x.numel()) * x.element_size() for x in
                   (ds.bins, booster.q, booster.gh, booster.pred, booster.y) + ((booster.packed,) if booster.packed is not None else ()))
    flush = in_bytes < 2 * L2_BYTES
    l2_note = (f"inputs larger than L2 ({in_bytes / 1e9:.2f} GB of bins, q, g/h per tree)" if not flush else
               f"L2 flushed between timed trees (256 MB write outside the timed events; inputs {in_bytes / 1e6:.0f} MB)")
    fbuf = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if flush else None
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    step_ev = []
    e0.record()
    for _ in range(a.steps):
        if flush:
            fbuf.fill_(1)
            s0 = torch.cuda.Event(enable_timing=True); s1 = torch.cuda.Event(enable_timing=True)
            s0.record()
        if a.graph and world == 1:
            booster.step_graph()
        else:
            booster.step(time_hist=True)
        if flush:
            s1.record()
            step_ev.append((s0, s1))
    e1.record()
    torch.cuda.synchronize()
    gc.enable()
    if group is not None:
        dist.barrier()
    l1 = ctx.gbdtmo_launch_count()
    clocks = clk.stop()
    booster.check_peer(block=True)        # a failed peer wait inside the timed region invalidates the run
    ms = sum(x.elapsed_time(y) for x, y in step_ev) if flush else e0.elapsed_time(e1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if group is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    ms_per_tree = ms / a.steps

    # ---- work accounting from the trees' records (after the timed region)
    trees = [annotate_searched({k: v.cpu().numpy() for k, v in tr.items()}, w.D, w.min_node)
             for tr in booster.trees[-a.steps:]]
    ro = sum(sum(int(tr["n_rows"][h]) for h, sv in tr["_searched"].items() if sv) * w.d for tr in trees)
    rows_built = sum(built_rows(tr, w.D) for tr in trees)
    value = ro / (ms * 1e-3)

    # ---- dominant kernel: build_hist (zero + k_hist_smem), CUDA events on the launching stream
    hist_ms = [e0_.elapsed_time(e1_) for (e0_, e1_) in booster.hist_events]
    hist_launches = len(hist_ms)
    hist_avg_ms = float(np.sum(hist_ms)) / max(hist_launches, 1)
    V = booster.p.V
    by_level = [[built_rows_by_level(tr, w.D)[l] for tr in trees] for l in range(w.D)]
    rows_lvl = [int(np.sum(v)) for v in by_level]                   # rows built per level, all timed trees
    root_cached = booster.root_cnt is not None
    # work per built (row, feature): V channel updates + 1 count (the root's count comes from the cache)
    updates = sum(r * m_loc * (V + (0 if (l == 0 and root_cached) else 1)) for l, r in enumerate(rows_lvl))
    lane_ops = sum(r * m_loc * (2 * V + (0 if (l == 0 and root_cached) else 1)) for l, r in enumerate(rows_lvl))
    upd_per_launch = updates / max(hist_launches, 1)
    achieved = upd_per_launch / (hist_avg_ms * 1e-3) if hist_launches else 0.0
    guide_peak_lane = 148 * 32 * 1.965e9                            # 32 ATOMS lanes/clk/SM at the max clock
    if atoms_peak:
        peak_lane = atoms_peak["pipe"]["lane_ops_per_s"]
        peak_src = (f"measured, same run: tools/microbench/peaks.cu red.shared.add.u32 on 32 distinct banks, "
                    f"{atoms_peak['pipe']['lane_ops_per_clk_sm']:.2f} lane-ops/clk/SM at "
                    f"{atoms_peak['pipe']['clk_mhz']:.0f} MHz = {atoms_peak['pipe']['lane_ops_per_s'] / 1e12:.2f} "
                    f"T lane-ops/s; 2 limb atomics per channel update + 1 count per (row, feature)")
    else:
        peak_lane, peak_src = guide_peak_lane, "guide (peaks library unavailable): 32 ATOMS lanes/clk/SM x 148 SMs x 1.965 GHz"
    peak = peak_lane * updates / lane_ops if lane_ops else 0.0      # updates/s at the atomic-pipe ceiling
    alg_bytes = rows_built * (m_loc + 4 * V + 4)          # bins + q + row id per built row
    hbm_gbs = alg_bytes / max(hist_launches, 1) / (hist_avg_ms * 1e-3) / 1e9 if hist_launches else 0.0
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except OSError:
        pass
    hbm_peak = float(peaks.get("hbm_gbs") or 6650.0)      # B200_PROFILING.md fallback when the file is absent
    hbm_peak_src = "MEASURED_PEAKS.json hbm_gbs" if peaks.get("hbm_gbs") else "of fallback (B200_PROFILING.md: 6.65 TB/s)"
    # DRAM traffic: bytes per built row per level from an ncu --set full capture of this bench's own
    # timed histogram launches (profiles/hist_traffic.json, tools/traffic_capture.sh), applied to the
    # rows this run built
    traffic, traffic_src = None, None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "hist_traffic.json")))
        bpr = prof.get("dram_bytes_per_built_row_by_level")
        if prof.get("workload") == w.name and world == 1 and bpr and len(bpr) == w.D:
            traffic = sum(b * r for b, r in zip(bpr, rows_lvl)) / max(hist_launches, 1)
            traffic_src = prof.get("source")
    except (OSError, ValueError):
        pass

    hist_total_ms = float(np.sum(hist_ms))
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": ms_per_tree, "sec_per_tree": ms_per_tree * 1e-3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int64",
        "dtype_detail": "31-bit fixed-point g/h, exact int64 histograms, fp64 gains and predictions",
        "data": f"synthetic (seeded counter-based generator, gen/); inputs resident in HBM ({in_bytes / 1e9:.2f} GB)",
        "config": {"workload": w.name, "n": w.n, "m": w.m, "d": w.d, "B": w.B, "D": w.D,
                   "loss": "mse" if w.loss == 0 else "softmax", "parallelism": f"feature-partition x{world}",
                   "exchange": (exchange if world > 1 else "none") + (f" ({exchange_note})" if exchange_note else ""),
                   "l2": l2_note, "graph": bool(a.graph and world == 1)},
        "hist_share": hist_total_ms / a.steps / ms_per_tree if ms_per_tree else None,
        "phase_ms_per_tree": ({k: round(v / a.steps, 3) for k, v in booster.phase_ms(a.steps).items()}
                              if not (a.graph and world == 1) else None),
        "rows_built_by_level": [int(np.mean([built_rows_by_level(tr, w.D)[l] for tr in trees])) for l in range(w.D)],
        "hist_ms_by_level": ([round(float(np.mean(hist_ms[l::w.D])), 3) for l in range(w.D)]
                             if len(hist_ms) == a.steps * w.D else None),
        "hist_rows_outputs_per_s_built": rows_built * w.d / (hist_total_ms * 1e-3) if hist_ms else None,
        "bin_ms": bin_ms, "bin_ms_first_call": bin_ms_first, "setup_s": setup_s,
        "roofline": {"bound": "alu", "kernel": "k_hist_smem (+k_zero_build) via gbdtmo_build_hist",
                     "achieved": achieved / 1e12, "peak": peak / 1e12, "unit": "Tupdate/s",
                     "frac": achieved / peak if peak else None, "traffic": traffic,
                     "peak_source": peak_src,
                     "frac_of_guide_peak": (achieved / (guide_peak_lane * updates / lane_ops)) if lane_ops else None,
                     "hbm_frac": hbm_gbs / hbm_peak,
                     "hbm_view": {"achieved_gbs": hbm_gbs, "peak_gbs": hbm_peak, "frac": hbm_gbs / hbm_peak,
                                  "peak_source": hbm_peak_src,
                                  "bytes": "algorithmic per built row: m bins + 4V q + 4 row id (north star's definition)"},
                     "traffic_source": traffic_src, "traffic_per_built_row": traffic * hist_launches / rows_built
                     if traffic else None,
                     "atoms_microbench": atoms_peak,
                     "launches": hist_launches, "avg_launch_ms": hist_avg_ms},
        "work": {"rows_built_per_tree": rows_built / a.steps, "logical_rows_per_tree": ro / w.d / a.steps,
                 "hist_ns_per_built_row": hist_total_ms * 1e6 / max(rows_built, 1),
                 "ms_per_tree_per_M_rows_built": ms_per_tree / (rows_built / a.steps / 1e6) if rows_built else None,
                 "note": "trees differ in rows built (which children are smaller); compare runs per built row"},
        "clocks": clocks,
        "gpu_launches": int(l1 - l0),
    }

    # ---- end to end through the public API with host buffers (H2D inside the timed region)
    del booster, ds
    torch.cuda.empty_cache()
    if not a.no_e2e:
        Yhost = Y.cpu().pin_memory()
        del Y
        out["e2e"] = e2e_run(w, a, rank, world, local, dev, group, f0, f1, Yhost, exchange)

    if group is not None:
        dist.barrier()
    if rank == 0:
        if not a.no_cpu_baseline and world == 1:
            try:
                out["cpu_baseline"] = cpu_oracle_sample(w)
            except Exception as ex:  # report, never fake
                out["cpu_baseline"] = {"error": repr(ex)}
        print(json.dumps(out))
    if group is not None:
        dist.destroy_process_group()
    return 0


def predict_main(a, w, local):
    """Inference line: train a model of --predict-trees trees on the
    workload, then time K passes of gbdtmo_predict over n UNSEEN rows (rows n..2n-1 of the same
    generator) resident in HBM.  value = rows x trees / s.  The kernel stages every row (m floats)
    once per pass, so it is bound by reading X from HBM: roofline bound "hbm", bytes = n m 4."""
    import torch
    import paper_conf_icpp_liupw25_b200 as pkg
    from gen import gen
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    ctx = pkg.Context(local)
    T = a.predict_trees

    def device_X(r0):
        if w.classes_sweep:
            return torch.from_numpy(gen.features_host(w, r0, w.n)).to(dev)
        X = torch.empty((w.n, w.m), dtype=torch.float32, device=dev)
        gen.matrix_cuda(w.seed, gen.STREAM_X, w.x_kind, r0, w.n, 0, w.m, w.m, X.data_ptr(), w.m,
                        torch.cuda.current_stream().cuda_stream)
        return X
    X = device_X(0)
    ds = pkg.bin_features(ctx, X, w.B)
    del X
    torch.cuda.empty_cache()
    Y = torch.from_numpy(host_targets(w)).to(dev)
    params = pkg.Params(loss=w.loss, T=T, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr, min_node=w.min_node)
    b = pkg.Booster(ctx, ds, Y, params)
    t0 = time.perf_counter()
    b.fit()
    torch.cuda.synchronize()
    train_s = time.perf_counter() - t0
    trees = b.trees
    del b, ds, Y
    torch.cuda.empty_cache()
    Xu = device_X(w.n)                                   # unseen rows
    pred = torch.zeros((w.n, w.d), dtype=torch.float64, device=dev)
    for _ in range(a.warmup):
        pkg.predict(ctx, trees, Xu, w.D, w.d, pred=pred)
    torch.cuda.synchronize()
    clk = ClockSampler(local)
    clk.start()
    time.sleep(0.3)
    l0 = ctx.gbdtmo_launch_count()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.steps):
        pkg.predict(ctx, trees, Xu, w.D, w.d, pred=pred)
    e1.record()
    torch.cuda.synchronize()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1) / a.steps
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except OSError:
        pass
    hbm_peak = float(peaks.get("hbm_gbs") or 6650.0)
    xbytes = w.n * w.m * 4
    gbs = xbytes / (ms * 1e-3) / 1e9
    out = {"metric": "inference rows*trees/s (gbdtmo_predict, unseen rows)", "value": w.n * T / (ms * 1e-3),
           "unit": "rows*trees/s", "n_gpus": 1, "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32 compare, f64 sums",
           "data": "synthetic (seeded counter-based generator, gen/); unseen rows n..2n-1, in HBM",
           "config": {"workload": w.name, "n": w.n, "m": w.m, "d": w.d, "D": w.D, "trees": T,
                      "l2": "inputs larger than L2" if xbytes > 126e6 else "X fits L2"},
           "train_s_for_model": train_s,
           "roofline": {"bound": "hbm", "kernel": "k_predict_tiles", "achieved": gbs, "peak": hbm_peak,
                        "unit": "GB/s", "frac": gbs / hbm_peak, "traffic": None,
                        "bytes": "n x m x 4 (every row staged once per pass)"},
           "clocks": clocks, "gpu_launches": int(ctx.gbdtmo_launch_count() - l0)}
    print(json.dumps(out))
    return 0


def peer_consistent(booster, group, dev):
    """After the warm-up trees: the peer window reports no expired wait on any rank, and every rank
    holds the same trees (node states, features, bins: replicated state, so any divergence of the
    exchange shows here)."""
    import torch
    import torch.distributed as dist
    torch.cuda.synchronize()
    _, err = booster.peer_status()
    sig = torch.zeros(1, dtype=torch.float64, device=dev)
    for tr in booster.trees:
        for k in ("node_state", "feature", "bin", "n_left"):
            v = tr[k].to(torch.float64)
            sig += (v * torch.arange(1, v.numel() + 1, dtype=torch.float64, device=dev)).sum()
    lo, hi = sig.clone(), sig.clone()
    dist.all_reduce(lo, op=dist.ReduceOp.MIN, group=group)
    dist.all_reduce(hi, op=dist.ReduceOp.MAX, group=group)
    bad = torch.tensor([1.0 if err else 0.0], dtype=torch.float64, device=dev)
    dist.all_reduce(bad, op=dist.ReduceOp.MAX, group=group)
    return bool(lo.item() == hi.item()) and bad.item() == 0.0


def e2e_run(w, a, rank, world, local, dev, group, f0, f1, Yh, exchange="collective"):
    """train(): pinned host X shard + y -> H2D -> gbdtmo_bin -> K trees -> D2H of yhat and the trees."""
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_liupw25_b200 as pkg
    from gen import gen
    m_loc = f1 - f0
    Xh = torch.empty((w.n, m_loc), dtype=torch.float32, pin_memory=True)
    Xh.numpy()[:] = gen.features_host(w, 0, w.n, f0, m_loc) if w.classes_sweep else \
        gen.matrix_host(w.seed, gen.STREAM_X, w.x_kind, 0, w.n, f0, m_loc, w.m, out=Xh.numpy())
    ctx = pkg.Context(local)
    params = pkg.Params(loss=w.loss, T=a.steps, D=w.D, B=w.B, lam=w.lam, gamma=w.gamma, lr=w.lr,
                        min_node=w.min_node)
    pred_h = torch.empty((w.n, w.d), dtype=torch.float64, pin_memory=True)   # the caller's output buffer
    torch.cuda.synchronize()
    if group is not None:
        dist.barrier()
    gc.collect()
    gc.disable()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    b = pkg.train(Xh, Yh, params, device=str(dev), ctx=ctx, group=group, f_begin=f0, m_global=w.m,
                  exchange=exchange)
    pred_h.copy_(b.pred, non_blocking=True)
    model_bytes = 0
    for tr in b.trees:
        for k, v in tr.items():
            model_bytes += v.numel() * v.element_size()
    model_h = [{k: v.to("cpu", non_blocking=True) for k, v in tr.items()} for tr in b.trees]
    e1.record()
    torch.cuda.synchronize()
    gc.enable()
    ms = e0.elapsed_time(e1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if group is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    ro = 0
    for tr in model_h:
        tn = annotate_searched({k: v.numpy() for k, v in tr.items()}, w.D, w.min_node)
        ro += sum(int(tn["n_rows"][h]) for h, sv in tn["_searched"].items() if sv) * w.d
    h2d = Xh.numel() * 4 + Yh.numel() * 4
    d2h = pred_h.numel() * 8 + model_bytes
    del b
    torch.cuda.empty_cache()
    return {"value": ro / (ms * 1e-3), "unit": UNIT, "h2d_bytes_per_step": h2d // a.steps,
            "d2h_bytes_per_step": d2h // a.steps, "ms_total": ms, "trees": a.steps,
            "what": "pkg.train(host X shard, host y): gbdtmo_bin_host (strip H2D overlapped with binning) + K trees + D2H of yhat and tree records"}


if __name__ == "__main__":
    sys.exit(main())
