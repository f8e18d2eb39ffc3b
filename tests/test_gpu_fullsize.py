"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (one fused cadv_analyze on the whole trace resident in HBM).

* C3 (BFS, 1 M nodes) and C4 (SRAD 2048^2 x 6): every histogram and per-site
  counter element by element against the oracle (CTA scope; the oracle's
  LRU stack is per CTA, so it finishes in seconds to a minute).
* C4-backprop (input 2^22, 1.02 G records with its BB trace): the same.
* Sub-warp analysis warp sizes (W = 8, 16) on C3 at full size (the
  warp-cooperative exact walk of every run).
* Kernel scope at full size, exact: the Fenwick-tree oracle variant
  (oracle.reuse_fenwick, pinned == LRU in test_oracle_pins.py) finishes
  where the LRU stack cannot; plus the size-free properties (mass, ∞,
  streaming) computed from the definition with numpy.
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


@pytest.mark.parametrize("name,kw", [("bfs", dict(nodes=1000000, seed=42)),
                                     ("srad", dict(rows=2048, cols=2048, iters=6, bb=1))])
def test_kernel_scope_full_exact(ctx, cadv, name, kw):
    """Kernel scope (the paper's "traditional definition") on C3 and
    C4 at full size, bit-exact against the Fenwick oracle; log2 and linear bins."""
    t = tg.generate(name, **kw)
    ctx.load_trace(cadv.to_device(t))
    for binning, nb in ((1, 40), (0, 66)):
        h, st = ctx.reuse_histogram(128, 1, binning, nb)
        h_ref, s_ref = orc.reuse_fenwick(t, 128, 1, binning, nb)
        assert (h == h_ref).all(), (name, binning, np.nonzero(h != h_ref))
        assert st == s_ref
    mass, inf, streaming = kernel_scope_properties(t, 128)
    assert int(h.sum()) == mass == st["accesses"] and int(h[-1]) == inf == st["inf"] and st["streaming"] == streaming


def test_c4_backprop_full(ctx, cadv):
    """C4's second shape: backprop, input 2^22, hidden 16, with BB records."""
    t = tg.generate("backprop", **{"in": 4194304})
    assert t.n > 1_000_000_000
    fused_vs_oracle(ctx, cadv, t, 128)


def test_c3_bfs_full_subwarp(ctx, cadv):
    """W = 16 and 8 (sub-warp groups: every run goes through the exact
    warp-cooperative walk) for memory and branch divergence at full size."""
    t = tg.generate("bfs", nodes=1000000, seed=42)
    ctx.load_trace(cadv.to_device(t))
    for W in (16, 8):
        o = ctx.analyze(rd=None, md=(128, W), bd=W, nsites=t.nsites)
        mh, ms = orc.mem_div(t, 128, W)
        assert (o["mem_div"][0] == mh).all() and (o["mem_div"][1] == ms).all(), W
        bs, bt = orc.branch_div(t, W)
        assert (o["branch_div"][0] == bs).all() and (o["branch_div"][1] == bt).all(), W
