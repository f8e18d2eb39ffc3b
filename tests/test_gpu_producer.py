"""Device-side trace producer (include/cadv_record.cuh):
hand-instrumented sm_100a kernels write REAL traces on the GPU; the library
analyses them in place; results equal (a) the closed forms pinned for the
same programs' generated traces (config 1 vecAdd, config 2 SGEMM: they hold
for any warp-contiguous, lane-ascending record order) and (b) the CPU oracle
on a host copy of the very same trace."""
import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cadv():
    import paper_conf_cgo_shensll18_b200 as m
    return m


@pytest.fixture(scope="module")
def ctx(cadv):
    c = cadv.create(0)
    yield c
    c.destroy()


@pytest.fixture(scope="module")
def prod():
    from paper_conf_cgo_shensll18_b200 import producer
    return producer


def host_trace(buf, nsites):
    h = buf.to_host()
    return tg.from_arrays(*(h[k] for k, _ in tg.COLUMNS), nsites=nsites)


def test_vecadd_config1_real_trace(ctx, cadv, prod):
    buf = prod.TraceBuffer(4096, 2)
    prod.vecadd(683, 64, 1, buf)
    assert buf.n == 2049 + 1558
    ctx.load_trace(buf.columns())
    h, st = ctx.reuse_histogram(128, 0, 0, 66)
    assert h[0] == 1322 and h[-1] == 727 and h.sum() == 2049
    h32, _ = ctx.reuse_histogram(32, 0, 0, 66)
    assert h32[0] == 1194 and h32[-1] == 855
    hm, _ = ctx.mem_divergence(128, 32, 7)
    assert hm[0, 1] == 44 and hm[1, 1] == 22 and hm.sum() == 66
    ps, tot = ctx.branch_divergence(32, 7)
    assert list(tot) == [50, 2, 1558]
    assert list(ps[1]) == [24, 1, 747] and list(ps[2]) == [22, 1, 683]
    t = host_trace(buf, 7)
    for lb in (128, 32):
        assert (ctx.reuse_histogram(lb, 0, 0, 66)[0] == orc.reuse(t, lb, 0, 0, 66)[0]).all()
    assert (ctx.mem_divergence(32, 32, 7)[0] == orc.mem_div(t, 32)[0]).all()


def test_sgemm_config2_real_trace(ctx, cadv, prod):
    """Naive then tiled 256^3 SGEMM (CTA ids continue): the printed-shape MD
    closed forms of config 2."""
    n = 256
    nrec = 256 * 256 * ((2 * n + 1) + (2 * (n // 16) + 1))
    buf = prod.TraceBuffer(nrec, 2 * 256 * 8)
    prod.sgemm(n, 0, 0, buf, cta_base=0)
    prod.sgemm(n, 1, 0, buf, cta_base=256)
    assert buf.n == nrec == 35782656
    ctx.load_trace(buf.columns())
    pooled = ctx.mem_divergence(128, 32, 14)[0].sum(axis=0)
    assert pooled[1] == 524288 and pooled[2] == 526336 + 67584 and pooled.sum() == 524288 + 526336 + 67584
    pooled = ctx.mem_divergence(32, 32, 14)[0].sum(axis=0)
    assert pooled[2] == 1048576 and pooled[4] == 2048 + 67584


def test_sgemm_small_vs_oracle(ctx, cadv, prod):
    """64^3 naive + tiled with basic-block records: every analysis == oracle."""
    n = 64
    buf = prod.TraceBuffer(2_000_000, 2 * 16 * 8)
    prod.sgemm(n, 0, 1, buf, cta_base=0)
    prod.sgemm(n, 1, 1, buf, cta_base=16)
    t = host_trace(buf, 14)
    ctx.load_trace(buf.columns())
    for lb, sc in ((128, 0), (32, 1)):
        h, s = ctx.reuse_histogram(lb, sc, 0, 66)
        hr, sr = orc.reuse(t, lb, sc, 0, 66)
        assert (h == hr).all() and s == sr
    assert (ctx.mem_divergence(128, 32, 14)[0] == orc.mem_div(t, 128)[0]).all()
    ps, tot = ctx.branch_divergence(32, 14)
    psr, totr = orc.branch_div(t, 32)
    assert (tot == totr).all() and (ps == psr).all() and tot[1] == 0


def test_instrumentation_overhead_measured(prod):
    """The instrumented kernels run (and are slower than the plain ones)."""
    n = 256
    buf = prod.TraceBuffer(256 * 256 * (2 * n + 1), 2 * 256 * 8)
    plain = prod.sgemm(n, 0, 0, None, reps=3)
    traced = prod.sgemm(n, 0, 0, buf, reps=3)
    assert traced > plain > 0
