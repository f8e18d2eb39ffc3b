"""Writes the per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum)
of every kernel in an ncu summary (tools/ncu_summary.py output) into
profiles/ncu_traffic.json under the workload, stamped with the library source
hash (bench.src_sha) of the build that was profiled; bench.py reports a
kernel's `traffic` only from a capture of the same sources.

usage: python tools/ncu_traffic.py WORKLOAD SUMMARY.csv TAG
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(workload, summary, tag):
    from bench import src_sha
    rows = list(csv.reader(open(summary)))
    hdr = rows[0]
    ir, iw = hdr.index("dram__bytes_read.sum"), hdr.index("dram__bytes_write.sum")
    kernels = {r[0]: int(float(r[ir]) + float(r[iw])) for r in rows[2:]}
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(p))
    except (OSError, ValueError):
        d = {}
    sha = src_sha()
    if d.get("src_sha") != sha:
        d = {"src_sha": sha, "workloads": {}}
    d["capture"] = f"ncu --set full --clock-control none, one bench step ({tag})"
    d["workloads"][workload] = kernels
    json.dump(d, open(p, "w"), indent=1, sort_keys=True)
    print(json.dumps({workload: kernels}))


if __name__ == "__main__":
    main(*sys.argv[1:4])
