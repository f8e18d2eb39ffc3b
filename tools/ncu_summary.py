"""Per-kernel summary of an ncu report (run here, on the copied .ncu-rep).

usage: python tools/ncu_summary.py out.csv report.ncu-rep [report2.ncu-rep ...]
Aggregates every captured launch of a kernel (mean per launch) over the
metrics the design decisions in DESIGN.md / profiles/README.md cite.
Byte metrics are written in bytes, durations in ms (units row).
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


SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "msecond": 1.0, "ms": 1.0, "nsecond": 1e-6, "s": 1e3}


def load(rep, acc):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ik = hdr.index("Kernel Name")
    for r in data:
        name = r[ik].split("(")[0].replace("void ", "").split("::")[-1]
        a = acc[name]
        a[0] += 1
        for j, m in enumerate(METRICS):
            if m not in hdr:
                continue
            i = hdr.index(m)
            try:
                v = float(r[i].replace(",", ""))
            except ValueError:
                continue
            a[1][j] += v * SCALE.get(units[i], 1.0)


def main(out, reps):
    acc = defaultdict(lambda: [0, [0.0] * len(METRICS)])
    for rep in reps:
        load(rep, acc)
    unit = {"gpu__time_duration.sum": "ms", "dram__bytes_read.sum": "byte", "dram__bytes_write.sum": "byte"}
    with open(out, "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["kernel", "launches"] + METRICS)
        w.writerow(["", ""] + [unit.get(m, "") for m in METRICS])
        for name, (n, s) in sorted(acc.items(), key=lambda kv: -kv[1][1][0]):
            w.writerow([name, n] + ["%.6g" % (v / n) for v in s])


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2:])
