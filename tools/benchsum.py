import json,sys
for line in sys.stdin:
    line=line.strip()
    if not line.startswith('{'): continue
    d=json.loads(line)
    print(d["ms_per_step"], round(d["value"]/1e9,2), d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], {k:round(v["total_ms"]/v["launches"],3) for k,v in d["kernels"].items()})
