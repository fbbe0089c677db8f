"""Summarise ncu --set full reports (one kernel each) into a markdown table.

    python scripts/ncu_summary.py OUT.md TITLE label1=report1.ncu-rep label2=report2.ncu-rep#1 ...

(`#i` picks the i-th kernel of a report that holds several; default the first.)
"""
import csv
import io
import subprocess
import sys

METRICS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "l1tex__t_sector_hit_rate.pct",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_requests_pipe_lsu_mem_global_op_red.sum",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sector_hit_rate.pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__inst_executed.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__thread_inst_executed_per_inst_executed.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__shared_mem_per_block_dynamic",
    "sm__cycles_elapsed.avg",
    "sm__cycles_active.avg",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_red.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld_lookup_miss.sum",
    "smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
]


def raw(rep):
    idx = 0
    if "#" in rep:
        rep, idx = rep.rsplit("#", 1)
        idx = int(idx)
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2 + idx]
    return v[h.index("Kernel Name")], {k: (v[h.index(k)], u[h.index(k)]) for k in METRICS if k in h}


def main():
    out, title, specs = sys.argv[1], sys.argv[2], sys.argv[3:]
    cols = [(s.rsplit("=", 1)[0], *raw(s.rsplit("=", 1)[1])) for s in specs]
    lines = [f"# {title}", "", "| metric | " + " | ".join(f"{c[0]} (`{c[1][:32]}`)" for c in cols) + " |",
             "|---|" + "---|" * len(cols)]
    for m in METRICS:
        lines.append(f"| {m} | " + " | ".join(f"{c[2].get(m, ('-', ''))[0]} {c[2].get(m, ('', ''))[1]}".strip() for c in cols) + " |")
    open(out, "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
