"""Copy / summarise the outputs of tools/profile_all.sh from gpurun_out/ into profiles/.

  python tools/profile_collect.py r01
"""
import collections
import csv
import glob
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")


def last_json(path):
    try:
        lines = [ln for ln in open(path).read().splitlines() if ln.startswith("{")]
        return json.loads(lines[-1]) if lines else None
    except OSError:
        return None


def launch_summary(csv_path, txt_path):
    rows = list(csv.reader(open(csv_path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr, data = rows[hi], rows[hi + 1:]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in data:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("void ", "")
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        agg[name][0] += 1
        agg[name][1] += v
    setup = ("radix", "bin_", "k_sel_", "k_csc_", "gen_", "k_default_bins", "k_pack_bins", "at::", "k_atoms")
    tree = {k: v for k, v in agg.items() if not any(s in k for s in setup)}
    tot_tree = sum(v[1] for v in tree.values())
    with open(txt_path, "w") as f:
        f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none (cold, serialised; shares only)\n")
        f.write(f"# source: {os.path.basename(csv_path)}\n")
        f.write(f"{'kernel':60s} {'launches':>8s} {'total ms':>10s} {'share of tree kernels':>22s}\n")
        for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            share = f"{100 * t / tot_tree:6.1f}%" if k in tree else "  (setup)"
            f.write(f"{k[:60]:60s} {n:8d} {t / 1e6:10.3f} {share:>22s}\n")
        f.write(f"tree kernels total ms: {tot_tree / 1e6:.3f}\n")
    return tree


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    os.makedirs(PROF, exist_ok=True)
    lines = []
    for p in sorted(glob.glob(os.path.join(OUT, f"{tag}_bench_*.log"))):
        j = last_json(p)
        if j:
            lines.append(j)
    with open(os.path.join(PROF, f"{tag}_bench_lines.jsonl"), "w") as f:
        for j in lines:
            f.write(json.dumps(j) + "\n")
    lc = os.path.join(OUT, f"{tag}_launches_bench_c5.csv")
    if os.path.exists(lc):
        subprocess.run(["cp", lc, os.path.join(PROF, f"{tag}_launches_bench_c5.csv")])
        launch_summary(lc, os.path.join(PROF, f"{tag}_launches_bench_c5_summary.txt"))
    for name in ("hist", "fs"):
        txt = os.path.join(OUT, f"{tag}_ncu_{name}_c5.txt")
        if os.path.exists(txt):
            subprocess.run(["cp", txt, os.path.join(PROF, f"{tag}_ncu_{name}_c5.txt")])
        rawp = os.path.join(OUT, f"{tag}_prof_{name}_c5_raw.csv")
        if name == "hist" and os.path.exists(rawp):
            # dram bytes per launch (average over the captured launches) for bench.py's roofline.traffic
            rr = list(csv.reader(open(rawp)))
            h, units = rr[0], rr[1]
            tot, cnt = 0.0, 0
            for r in rr[2:]:
                try:
                    rd = float(r[h.index("dram__bytes_read.sum")].replace(",", ""))
                    wr = float(r[h.index("dram__bytes_write.sum")].replace(",", ""))
                except (ValueError, IndexError):
                    continue
                if rd != rd or wr != wr:      # NaN: a replay that failed to collect
                    continue
                unit = units[h.index("dram__bytes_read.sum")]
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
                tot += (rd + wr) * scale
                cnt += 1
            if cnt:
                json.dump({"workload": "C5-high-dim-feature-partitioned", "kernel": "k_hist_smem",
                           "dram_bytes_per_launch": tot / cnt, "launches": cnt,
                           "source": f"profiles/{tag}_ncu_hist_c5.txt (ncu --set full, one tree)"},
                          open(os.path.join(PROF, "hist_traffic.json"), "w"), indent=1)
    bp = os.path.join(OUT, f"{tag}_bin_probe_c5.log")
    if os.path.exists(bp):
        j = last_json(bp)
        if j:
            json.dump(j, open(os.path.join(PROF, f"{tag}_bin_probe_c5.json"), "w"), indent=1)
    bl = os.path.join(OUT, f"{tag}_launches_bin_c5.csv")
    if os.path.exists(bl):
        launch_summary(bl, os.path.join(PROF, f"{tag}_launches_bin_c5_summary.txt"))
    ab = os.path.join(OUT, f"{tag}_atom_bench.txt")
    if os.path.exists(ab):
        subprocess.run(["cp", ab, os.path.join(PROF, f"{tag}_microbench_atomics.txt")])
    print("collected", len(lines), "bench lines")


if __name__ == "__main__":
    main()
