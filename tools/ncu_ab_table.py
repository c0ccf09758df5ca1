"""Side-by-side table of selected ncu raw metrics for A/B captures (tools/ab_ncu.sh output).

  python tools/ncu_ab_table.py gpurun_out/ab_new1_raw.csv gpurun_out/ab_old_raw.csv ...
"""
import csv
import sys

KEYS = [
    "gpu__time_duration.sum", "smsp__inst_executed.sum", "smsp__inst_executed_op_shared_atom.sum",
    "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__lsuin_requests.avg.pct_of_peak_sustained_elapsed",
    "l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed",
    "sm__mio_pq_read_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
]


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, units, data = rows[0], rows[1], rows[2]
    return {k: (data[i], units[i]) for i, k in enumerate(hdr)}


def main():
    tabs = [load(p) for p in sys.argv[1:]]
    print("metric".ljust(72) + "".join(p.split("/")[-1][:18].rjust(20) for p in sys.argv[1:]))
    for k in KEYS:
        vals = [t.get(k, ("-", ""))[0] for t in tabs]
        unit = tabs[0].get(k, ("", ""))[1]
        print((k + f" [{unit}]")[:72].ljust(72) + "".join(v[:18].rjust(20) for v in vals))


if __name__ == "__main__":
    main()
