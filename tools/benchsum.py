"""One-line summary of bench.py JSON lines on stdin: ms/step, G records/s,
dominant kernel ms and roofline fraction, top kernels (ms per step)."""
import json
import sys

for line in sys.stdin:
    line = line.strip()
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    r = d.get("roofline") or {}
    top = {k: v["ms_per_step"] for k, v in list((d.get("kernels") or {}).items())[:6]}
    print(d["config"]["workload"], d["ms_per_step"], round(d["value"] / 1e9, 2), r.get("kernel"), r.get("avg_launch_ms"),
          r.get("frac"), r.get("step_algorithmic_frac"), top)
