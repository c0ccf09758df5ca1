"""profiles/hist_traffic.json from tools/traffic_capture.sh output: DRAM bytes (read + write) of
each histogram launch of the bench's first timed tree, divided by the rows that launch built
(the bench line's rows_built_by_level for that tree).  bench.py multiplies these per-level rates by
the rows its own timed trees built to report roofline.traffic per launch.

  python tools/traffic_collect.py r02 C5
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    tag, wl = sys.argv[1], sys.argv[2]
    out = os.path.join(ROOT, "gpurun_out")
    raw = list(csv.reader(open(os.path.join(out, f"{tag}_traffic_{wl}_raw.csv"))))
    h, units = raw[0], raw[1]
    def val(r, key):
        i = h.index(key)
        sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(units[i], 1)
        return float(r[i].replace(",", "")) * sc
    per_launch = [val(r, "dram__bytes_read.sum") + val(r, "dram__bytes_write.sum") for r in raw[2:]
                  if len(r) == len(h)]
    line = [ln for ln in open(os.path.join(out, f"{tag}_traffic_{wl}_bench.log")).read().splitlines()
            if ln.startswith("{")][-1]
    b = json.loads(line)
    rows = b["rows_built_by_level"]
    assert len(per_launch) == len(rows), (len(per_launch), len(rows))
    bpr = [t / r if r else 0.0 for t, r in zip(per_launch, rows)]
    res = {"workload": b["config"]["workload"], "kernel": "k_hist_smem",
           "dram_bytes_by_level": per_launch, "rows_built_by_level": rows,
           "dram_bytes_per_built_row_by_level": bpr,
           "algorithmic_bytes_per_built_row": b["config"]["m"] + 4 * b["config"]["d"] + 4,
           "source": f"profiles/{tag}_ncu_hist_{wl}_timed.txt: ncu --set full of bench.py's first timed tree "
                     f"(warm-up {b['warmup']} trees skipped), dram__bytes_read.sum + dram__bytes_write.sum"}
    json.dump(res, open(os.path.join(ROOT, "profiles", "hist_traffic.json"), "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
