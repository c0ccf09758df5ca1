"""Summarise an ncu report (details page + top SASS stall lines) into plain text for profiles/.

  python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--sass N] > profiles/rNN_<name>.txt
"""
import collections
import csv
import io
import subprocess
import sys

KEYS = [
    "Duration", "Elapsed Cycles", "SM Frequency", "DRAM Throughput", "Memory Throughput", "L1/TEX Cache Throughput",
    "L2 Cache Throughput", "Compute (SM) Throughput", "Executed Ipc Active", "Issue Slots Busy", "SM Busy",
    "L1/TEX Hit Rate", "L2 Hit Rate", "Mem Busy", "Max Bandwidth", "Eligible Warps Per Scheduler", "No Eligible",
    "Warp Cycles Per Issued Instruction", "Registers Per Thread", "Achieved Occupancy", "Dynamic Shared Memory Per Block",
    "Executed Instructions", "Block Size", "Grid Size",
]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed_op_shared_atom.sum",
       "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "lts__t_sectors_op_red.sum",
       "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
       "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum", "gpu__time_duration.sum"]


def run(args):
    return subprocess.run(["ncu"] + args, capture_output=True, text=True).stdout


def main():
    rep = sys.argv[1]
    nsass = int(sys.argv[sys.argv.index("--sass") + 1]) if "--sass" in sys.argv else 25
    det = list(csv.reader(io.StringIO(run(["-i", rep, "--page", "details", "--csv"]))))
    hdr = det[0]
    ki, ni, ui, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
    idi = hdr.index("ID")
    per = collections.OrderedDict()
    for r in det[1:]:
        if len(r) <= vi:
            continue
        key = (r[idi], r[ki].split("(")[0])
        per.setdefault(key, []).append(r)
    raw = list(csv.reader(io.StringIO(run(["-i", rep, "--page", "raw", "--csv"]))))
    rawd = {}
    if raw:
        rh = raw[0]
        for r in raw[2:]:
            rid = r[rh.index("ID")]
            rawd[rid] = {m: r[rh.index(m)] for m in RAW if m in rh}
    for (rid, name), rows in per.items():
        print(f"=== launch {rid}: {name}")
        seen = set()
        for r in rows:
            if r[ni] in KEYS and r[ni] not in seen:
                seen.add(r[ni])
                print(f"  {r[ni]:40s} {r[vi]:>18s} {r[ui]}")
        for m, v in rawd.get(rid, {}).items():
            print(f"  {m:40s} {v:>18s}")
        rt, rd = hdr.index("Rule Type"), hdr.index("Rule Description")
        for r in rows:
            if len(r) > rd and r[rt] in ("OPT", "WRN") and r[rd]:
                print("  rule:", r[rd][:220].replace("\n", " "))
    # SASS hot spots of every launch (stall samples)
    src = run(["-i", rep, "--page", "source", "--csv", "--print-source", "sass"])
    blocks = src.split('"Kernel Name"')
    for b in blocks[1:]:
        lines = list(csv.reader(io.StringIO('"Kernel Name"' + b)))
        title = lines[0][1][:90] if len(lines[0]) > 1 else "?"
        h = lines[1]
        si, ei = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
        data = [r for r in lines[2:] if len(r) > ei]
        tot = sum(float(r[si] or 0) for r in data) or 1.0
        print(f"--- SASS hot spots: {title}")
        for r in sorted(data, key=lambda r: -float(r[si] or 0))[:nsass]:
            print(f"  {float(r[si] or 0) / tot * 100:5.1f}%  {r[1][:100]}")


if __name__ == "__main__":
    main()
