"""Small end-to-end workload for compute-sanitizer (tools/sanitize.sh): every
analysis entry point on C1 (vecAdd), a reduced C2 (SGEMM 64^3, both
kernels), a random trace with stores / BB records / > 512 sites, a small SRAD
(segment kernel, regroup scatter, data-centric rows), a
non-warp-contiguous trace and a kernel-scope call, each checked against the
oracle so a tool-induced change of results would show."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle as orc  # noqa: E402
import paper_conf_cgo_shensll18_b200 as cadv  # noqa: E402
import tracegen as tg  # noqa: E402


def main():
    traces = [("vecadd", tg.generate("vecadd"), True),
              ("sgemm64", tg.generate("sgemm", n=64, bb=1), True),
              ("rand", tg.generate("rand", seed=3, ctas=6, threads=128, instrs=20, lines=40, pstore=0.3, pbb=0.3,
                                   msites=600, bsites=40), True),
              ("srad64", tg.generate("srad", rows=64, cols=64, iters=1, bb=1), True),
              ("scramble", tg.generate("rand", seed=4, ctas=4, threads=96, instrs=15, lines=30, scramble=1,
                                       scramble_seed=4), False)]
    ctx = cadv.create(0)
    for name, t, contiguous in traces:
        ctx.load_trace(cadv.to_device(t), warp_contiguous=contiguous)
        o = ctx.analyze(rd=(128, 0, 0, 66), md=(32, 32), bd=32, nsites=t.nsites)
        assert (o["reuse"][0] == orc.reuse(t, 128, 0)[0]).all(), name
        assert (o["mem_div"][0] == orc.mem_div(t, 32, 32)[0]).all(), name
        assert (o["branch_div"][1] == orc.branch_div(t, 32)[1]).all(), name
        h, _ = ctx.reuse_histogram(32, 1, 1, 20)
        assert (h == orc.reuse(t, 32, 1, 1, 20)[0]).all(), name
        m, _ = ctx.mem_divergence(128, 8, t.nsites)
        assert (m == orc.mem_div(t, 128, 8)[0]).all(), name
        if name == "srad64":
            objs = tg.objects("srad", rows=64, cols=64, iters=1, bb=1)
            rh, mh = ctx.data_centric(objs, 128)
            rh_ref, mh_ref = orc.data_centric(t, objs, 128)
            assert (rh == rh_ref).all() and (mh == mh_ref).all(), name
        print("ok", name, t.n, flush=True)
    ctx.destroy()


if __name__ == "__main__":
    main()
