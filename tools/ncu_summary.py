"""Text summary of an ncu --set full report: per kernel the key throughput /
occupancy / stall metrics, DRAM traffic, and the top source-line stall sites."""
import csv
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Hit Rate", "L2 Hit Rate",
        "Compute (SM) Throughput", "Issued Ipc Active", "Executed Instructions", "Registers Per Thread",
        "Theoretical Occupancy", "Achieved Occupancy", "Avg. Active Threads Per Warp",
        "Warp Cycles Per Issued Instruction", "Grid Size", "Block Size"]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "gpu__time_duration.sum",
       "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_selected_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_drain_per_issue_active.ratio",
       "smsp__average_warps_issue_stalled_membar_per_issue_active.ratio",
       "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
       "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active"]


def main(rep, top=15):
    det = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(det.splitlines()))
    h = rows[0]
    by = {}
    for r in rows[1:]:
        d = dict(zip(h, r))
        key = (d["ID"], d["Kernel Name"][:70])
        if d["Metric Name"] in KEYS:
            by.setdefault(key, []).append(f"  {d['Metric Name']:42s} {d['Metric Value']:>16s} {d['Metric Unit']}")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    rh, ru = rr[0], rr[1]
    for i, r in enumerate(rr[2:]):
        d = dict(zip(rh, r))
        key = (d.get("ID", str(i)), d.get("Kernel Name", "")[:70])
        for n in RAW:
            if n in d:
                by.setdefault(key, []).append(f"  {n:42s} {d[n]:>16s} {ru[rh.index(n)]}")
    for (i, name), lines in sorted(by.items()):
        print(f"== launch {i}: {name}")
        print("\n".join(lines))
    print("\n== warp-stall samples by source line (all profiled launches)")
    sys.stdout.flush()
    subprocess.run([sys.executable, __file__.replace("ncu_summary.py", "ncu_hot.py"), rep, str(top)])


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 15)
