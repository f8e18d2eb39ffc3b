"""A/B summary of bench JSON lines (gpurun_out/<tag>_*.json): one line per file
with workload, ms per step, G records/s, the dominant kernel's launch ms and
roofline fraction, and the kernels above 0.05 ms per step.
usage: python tools/ab_summary.py gpurun_out/r2q_*.json > profiles/....txt"""
import json
import os
import sys

for path in sys.argv[1:]:
    try:
        d = json.loads(open(path).read().strip().splitlines()[-1])
    except (ValueError, IndexError):
        print(f"{os.path.basename(path)}: no JSON line")
        continue
    r = d.get("roofline") or {}
    ks = " ".join(f"{k}={v['ms_per_step']:.3f}" for k, v in (d.get("kernels") or {}).items() if v["ms_per_step"] > 0.05)
    dc = d.get("data_centric") or {}
    extra = f" data_centric={dc['ms_per_step']}ms" if dc else ""
    print(f"{os.path.basename(path)}: {d['config']['workload']} {d['ms_per_step']} ms {d['value'] / 1e9:.2f} G rec/s "
          f"{r.get('kernel')} {r.get('avg_launch_ms')} ms frac {r.get('frac')}{extra} | {ks}")
