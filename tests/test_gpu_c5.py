"""Config 5: the 4.0e9-record mixed memory trace -- SRAD
4096^2 x 3, backprop 2^23, SGEMM-naive 512^3, BFS 4 M nodes, tiled SGEMM
2048^3, then SRAD iterations, truncated at exactly 4.0e9 records
(tracegen "mixed", reading R20) -- analysed by ONE context in ONE
fused call (4.0e9 < 2^32 records per shard), bit-exact against the oracle.

The oracle runs launch-aligned chunk by chunk and the results are summed:
exact for CTA-scope reuse distance and for memory divergence, because no CTA
and no warp-level group spans two launches (CTA ids are unique per launch),
so every scope / group lies inside one chunk (the same decomposition
tests/test_dist_cpu.py checks against the whole-trace oracle).  The small
variant (div=256, 12 M records: every part, the SRAD fill and the
truncation) also checks kernel scope against the Fenwick oracle.
"""
import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cadv():
    import paper_conf_cgo_shensll18_b200 as m
    return m


def chunks(offs, target):
    """Launch-aligned [lo, hi) ranges of about `target` records."""
    out, lo = [], int(offs[0])
    for b in offs[1:]:
        if int(b) - lo >= target or int(b) == int(offs[-1]):
            out.append((lo, int(b)))
            lo = int(b)
    return out


def run_c5(cadv, params, target, kernel_scope):
    import torch
    torch.cuda.empty_cache()  # earlier modules' cached blocks: the library allocates with cudaMalloc
    offs = tg.launch_offsets("mixed", **params)
    n = int(offs[-1])
    dev = {k: torch.empty(n, dtype=torch.from_numpy(np.zeros(1, dt)).dtype, device="cuda") for k, dt in tg.COLUMNS}
    nsites = None
    h_ref, s_ref = np.zeros(66, np.uint64), dict(accesses=0, inf=0, streaming=0, overflow=0, finite_sum=0)
    m_ref, p_ref = None, None
    whole = [] if kernel_scope else None
    for t in tg.generate_ranges("mixed", chunks(offs, target), **params):
        for k, _ in tg.COLUMNS:
            dev[k][t.lo:t.lo + t.n].copy_(torch.from_numpy(t.cols[k]))
        nsites = t.nsites
        h, s = orc.reuse(t, 128, 0, 0, 66)
        h_ref += h
        for k in s_ref:
            s_ref[k] += s[k]
        mh, ps = orc.mem_div(t, 128, 32)
        m_ref = mh if m_ref is None else m_ref + mh
        p_ref = ps if p_ref is None else p_ref + ps
        if whole is not None:
            whole.append(t)
        del t
    ctx = cadv.create(0)
    try:
        ctx.load_trace(dev)
        o = ctx.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=None, nsites=nsites)
        assert (o["reuse"][0] == h_ref).all(), np.nonzero(o["reuse"][0] != h_ref)
        assert o["reuse"][1] == s_ref
        assert (o["mem_div"][0] == m_ref).all() and (o["mem_div"][1] == p_ref).all()
        if whole is not None:
            t = tg.concat(whole)
            hk, sk = ctx.reuse_histogram(128, 1, 1, 40)
            hr, sr = orc.reuse_fenwick(t, 128, 1, 1, 40)
            assert (hk == hr).all() and sk == sr
    finally:
        ctx.destroy()
        del dev
        torch.cuda.empty_cache()
    return n


def test_c5_mixed_small(cadv):
    n = run_c5(cadv, dict(div=256, records=12_000_000), 3_000_000, kernel_scope=True)
    assert n == 12_000_000


@pytest.mark.slow
def test_c5_mixed_full(cadv):
    n = run_c5(cadv, {}, 600_000_000, kernel_scope=False)
    assert n == 4_000_000_000
