"""cadv_set_profiling modes (bench.py's timed loop uses mode 2): events around
every launch (1) or around the streaming pass k_scan<F> only (2); results do
not depend on the mode."""
import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu


def test_profiling_modes():
    import paper_conf_cgo_shensll18_b200 as cadv
    t = tg.generate("rand", seed=11, ctas=5, threads=128, instrs=30, lines=200, pstore=0.2, pbb=0.3)
    h_ref, s_ref = orc.reuse(t, 128, 0, 0, 66)
    with cadv.create(0) as ctx:
        ctx.load_trace(cadv.to_device(t))
        seen = {}
        for mode in (1, 2, 0):
            ctx.set_profiling(mode)
            out = ctx.analyze(rd=(128, cadv.SCOPE_CTA, cadv.BINS_LINEAR, 66), md=(128, 32), bd=32, nsites=t.nsites)
            h, st = out["reuse"]
            assert (h == h_ref).all() and st == s_ref, mode
            seen[mode] = ctx.last_kernel_times()
        ctx.set_profiling(0)
        names1 = [n for n, _ in seen[1]]
        names2 = [n for n, _ in seen[2]]
        assert len(names1) == ctx.last_launches() > len(names2)  # (every call of this trace launches the same kernels)
        assert names2 and all(n.startswith("k_scan<") for n in names2), names2
        assert [n for n in names1 if n.startswith("k_scan<")] == names2
        assert all(ms > 0 for _, ms in seen[2])
        assert seen[0] == []
        with pytest.raises(Exception):
            ctx.set_profiling(3)
