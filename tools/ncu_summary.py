"""Per-kernel summary of an ncu report (run here, on the copied .ncu-rep).

usage: python tools/ncu_summary.py report.ncu-rep out.csv
Aggregates every captured launch of a kernel (mean per launch) over the
metrics the design decisions in DESIGN.md / profiles/README.md cite.
"""
import csv
import subprocess
import sys
from collections import defaultdict

METRICS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum",
    "launch__registers_per_thread",
    "launch__occupancy_limit_registers",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
]


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ik = hdr.index("Kernel Name")
    cols = [(m, hdr.index(m)) for m in METRICS if m in hdr]
    acc = defaultdict(lambda: [0, [0.0] * len(cols)])
    for r in data:
        name = r[ik].split("(")[0].replace("void ", "").split("::")[-1]
        a = acc[name]
        a[0] += 1
        for j, (_, i) in enumerate(cols):
            try:
                a[1][j] += float(r[i].replace(",", ""))
            except ValueError:
                pass
    with open(out, "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["kernel", "launches"] + [m for m, _ in cols])
        w.writerow(["", ""] + [units[i] for _, i in cols])
        for name, (n, s) in sorted(acc.items(), key=lambda kv: -kv[1][1][0]):
            w.writerow([name, n] + ["%.6g" % (v / n) for v in s])


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
