"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (one fused cadv_analyze on the whole trace resident in HBM).

* C3 (BFS, 1 M nodes) and C4 (SRAD 2048^2 x 6): every histogram and per-site
  counter element by element against the oracle (CTA scope; the oracle's
  LRU stack is per CTA, so it finishes in seconds to a minute).
* Kernel scope at full size, where the LRU oracle cannot finish: properties
  that hold at any size -- histogram mass = memory records; ∞ = stores +
  lines whose first access is a load (each renamed element's first use);
  streaming = renamed elements used exactly once -- computed from the
  definition with numpy; plus exact oracle parity on a 4 M-record prefix.
"""
import numpy as np
import pytest

import oracle as orc
import tracegen as tg
from props import kernel_scope_properties

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def cadv():
    import paper_conf_cgo_shensll18_b200 as m
    return m


@pytest.fixture(scope="module")
def ctx(cadv):
    c = cadv.create(0)
    yield c
    c.destroy()


def fused_vs_oracle(ctx, cadv, t, lb):
    ctx.load_trace(cadv.to_device(t))
    o = ctx.analyze(rd=(lb, 0, 0, 66), md=(lb, 32), bd=32, nsites=t.nsites)
    h_ref, s_ref = orc.reuse(t, lb, 0, 0, 66)
    assert (o["reuse"][0] == h_ref).all(), (o["reuse"][0], h_ref)
    assert o["reuse"][1] == s_ref
    mh, ms = orc.mem_div(t, lb, 32)
    assert (o["mem_div"][0] == mh).all() and (o["mem_div"][1] == ms).all()
    bs, bt = orc.branch_div(t, 32)
    assert (o["branch_div"][0] == bs).all() and (o["branch_div"][1] == bt).all()


def test_c3_bfs_full(ctx, cadv):
    t = tg.generate("bfs", nodes=1000000, seed=42)
    for lb in (128, 32):
        fused_vs_oracle(ctx, cadv, t, lb)


def test_c4_srad_full(ctx, cadv):
    t = tg.generate("srad", rows=2048, cols=2048, iters=6, bb=1)
    assert int(((t.meta & 3) < 2).sum()) == 478150656
    fused_vs_oracle(ctx, cadv, t, 128)


def test_kernel_scope_full_properties(ctx, cadv):
    t = tg.generate("srad", rows=2048, cols=2048, iters=6, bb=1)
    ctx.load_trace(cadv.to_device(t))
    h, st = ctx.reuse_histogram(128, 1, 1, 40)
    mass, inf, streaming = kernel_scope_properties(t, 128)
    assert int(h.sum()) == mass == st["accesses"]
    assert int(h[-1]) == inf == st["inf"]
    assert st["streaming"] == streaming
    # exact parity on a prefix the LRU oracle finishes
    p = tg.from_arrays(*(t.cols[k][:4_000_000] for k, _ in tg.COLUMNS), nsites=t.nsites)
    ctx.load_trace(cadv.to_device(p))
    h2, s2 = ctx.reuse_histogram(128, 1, 1, 40)
    h_ref, s_ref = orc.reuse(p, 128, 1, 1, 40)
    assert (h2 == h_ref).all() and s2 == s_ref
