"""Per-kernel summary of an ncu --set full report (raw page CSV on stdin)."""
import csv
import sys

rows = list(csv.reader(sys.stdin))
hdr = rows[0]
M = {"time_us": "gpu__time_duration.sum", "dram_rd_MB": "dram__bytes_read.sum", "dram_wr_MB": "dram__bytes_write.sum",
     "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
     "issue_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
     "alu_pct": "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
     "fma_pct": "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
     "lsu_pct": "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
     "warps_act_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
     "regs": "launch__registers_per_thread", "grid": "launch__grid_size", "inst_Mwarp": "smsp__inst_executed.sum",
     "st_long_sb": "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
     "st_wait": "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
     "st_barrier": "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
     "st_noinst": "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
     "st_short_sb": "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
     "st_mathpipe": "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
     "st_lg_thr": "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
     "st_mio": "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
     "st_branch": "smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio",
     "st_sleep": "smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio",
     "st_drain": "smsp__average_warps_issue_stalled_drain_per_issue_active.ratio"}
seen = set()
for r in rows[2:]:
    name = r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "")
    if name in seen:
        continue
    seen.add(name)
    out = []
    for k, m in M.items():
        if m in hdr:
            v = r[hdr.index(m)]
            try:
                f = float(v)
                if k == "inst_Mwarp":
                    f /= 1e6
                out.append(f"{k}={f:.3g}")
            except ValueError:
                out.append(f"{k}={v}")
    print(name + ": " + " ".join(out))
