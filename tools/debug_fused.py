"""Debug helper: run the fused analysis on one random trace (for compute-sanitizer)."""
import sys
sys.path.insert(0, ".")
import numpy as np
import oracle as orc
import tracegen as tg
import paper_conf_cgo_shensll18_b200 as cadv

seed = int(sys.argv[1]) if len(sys.argv) > 1 else 0
t = tg.generate("rand", seed=seed, ctas=7, threads=160, instrs=40, lines=80, pstore=0.2, pbb=0.4)
ctx = cadv.create(0)
ctx.load_trace(cadv.to_device(t))
for flags in ("rd", "md", "bd", "rdmd", "rdbd", "mdbd", "all"):
    rd = (128, 0, 0, 66) if "rd" in flags or flags == "all" else None
    md = (32, 32) if "md" in flags or flags == "all" else None
    bd = 32 if "bd" in flags or flags == "all" else None
    try:
        out = ctx.analyze(rd=rd, md=md, bd=bd, nsites=t.nsites)
        ok = True
        if rd: ok &= bool((out["reuse"][0] == orc.reuse(t, 128, 0, 0, 66)[0]).all())
        if md: ok &= bool((out["mem_div"][0] == orc.mem_div(t, 32, 32)[0]).all())
        if bd: ok &= bool((out["branch_div"][1] == orc.branch_div(t, 32)[1]).all())
        print(flags, "ok" if ok else "MISMATCH", flush=True)
    except Exception as e:
        print(flags, "ERROR", e, flush=True)
        break
