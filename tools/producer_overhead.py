"""Instrumentation overhead of the device-side producer (include/cadv_record.cuh)
on this GPU: plain vs instrumented kernel time (CUDA events, mean of `reps`
launches after a warm-up), and the producer's record rate.  Writes one JSON
object (profiles/producer_overhead.json).  Context: the paper's LLVM-based
instrumentation costs 10-120x."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(out):
    from paper_conf_cgo_shensll18_b200 import producer as P
    res = {}
    for name, n, variant in (("sgemm_naive_256", 256, 0), ("sgemm_tiled_256", 256, 1), ("sgemm_naive_1024", 1024, 0),
                             ("sgemm_tiled_1024", 1024, 1)):
        recs = (n // 16) ** 2 * 256 * ((2 * n + 1) if variant == 0 else (2 * (n // 16) + 1))
        buf = P.TraceBuffer(recs, 2 * (n // 16) ** 2 * 8)
        plain = P.sgemm(n, variant, 0, None, reps=5)
        traced = P.sgemm(n, variant, 0, buf, reps=5)
        assert buf.n == recs
        res[name] = {"plain_ms": round(plain, 4), "instrumented_ms": round(traced, 4),
                     "slowdown": round(traced / plain, 2), "records": recs,
                     "records_per_s": round(recs / (traced / 1e3), 1)}
        del buf
    n, ctas, thr = 1 << 24, 148 * 8, 256
    recs = 3 * n + ctas * (thr // 32) * 32 * (2 + 2 * ((n + ctas * thr - 1) // (ctas * thr))) + 64 * 1024
    buf = P.TraceBuffer(recs, ctas * thr // 32)
    plain = P.vecadd(n, thr, ctas, None, reps=5)
    traced = P.vecadd(n, thr, ctas, buf, reps=5)
    res["vecadd_16M"] = {"plain_ms": round(plain, 4), "instrumented_ms": round(traced, 4),
                         "slowdown": round(traced / plain, 2), "records": buf.n,
                         "records_per_s": round(buf.n / (traced / 1e3), 1), "bb_records": True}
    import torch
    res["device"] = torch.cuda.get_device_name(0)
    res["paper_context"] = "CUDAAdvisor instrumentation: 10-120x (PAPER.md L396-398), K40c / P100"
    txt = json.dumps(res, indent=1)
    print(txt)
    if out:
        open(out, "w").write(txt + "\n")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else None)
