"""GPU: the library on the paper's input domain (round-2 VERDICT items).

* Addresses: the paper records any i8* effective address.  The
  reuse path packs line numbers below 2^58 with flags above them, so a line
  >= 2^58 is CADV_ERR_UNSUPPORTED (a limit of this implementation, not a bad
  record) while the oracle still returns the histogram; memory divergence
  compares full addresses and accepts every address.
* Group rule (reading R19): records of one (cta, tid/32, winst)
  group share kind and site; the library rejects violations like the oracle.
* Non-warp-contiguous traces in ONE fused call (cadv_analyze,
  cadv_data_centric): reuse distance in trace order, divergence after the
  (cta, warp) regroup -- both equal the oracle.
"""
import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu
LD, ST, BB = 0, 1, 2


@pytest.fixture(scope="module")
def cadv():
    import paper_conf_cgo_shensll18_b200 as m
    return m


@pytest.fixture(scope="module")
def ctx(cadv):
    c = cadv.create(0)
    yield c
    c.destroy()


def shifted(t, shift):
    cols = {k: v.copy() for k, v in t.cols.items()}
    mem = (cols["meta"] & 3) != BB
    cols["addr"][mem] = cols["addr"][mem] + np.uint64(shift)
    return tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t.nsites)


@pytest.mark.parametrize("shift", [1 << 58, 0xC000000000000000])
def test_high_addresses(ctx, cadv, shift):
    t = shifted(tg.generate("rand", seed=5, ctas=3, threads=64, instrs=20, lines=30, pstore=0.3, pbb=0.3), shift)
    ctx.load_trace(cadv.to_device(t))
    # lines >= 2^58 (element model): the oracle answers, the library says UNSUPPORTED
    ref = orc.reuse(t, 1, 0)
    assert ref[0].sum() == ((t.meta & 3) != BB).sum()
    for call in (lambda: ctx.reuse_histogram(1, 0, 0, 66),
                 lambda: ctx.analyze(rd=(1, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)):
        with pytest.raises(cadv.CadvError) as e:
            call()
        assert e.value.status == cadv.CADV_ERR_UNSUPPORTED
    # lines < 2^58 (addr / 128 < 2^57): exact
    for sc in (0, 1):
        h, st = ctx.reuse_histogram(128, sc, 0, 66)
        hr, sr = orc.reuse(t, 128, sc, 0, 66)
        assert (h == hr).all() and st == sr
    # memory divergence: any address
    for lb in (1, 32, 128):
        h, ps = ctx.mem_divergence(lb, 32, t.nsites)
        hr, pr = orc.mem_div(t, lb, 32)
        assert (h == hr).all() and (ps == pr).all()
    out = ctx.analyze(rd=(128, 0, 0, 66), md=(1, 16), bd=32, nsites=t.nsites)
    assert (out["reuse"][0] == orc.reuse(t, 128, 0)[0]).all()
    assert (out["mem_div"][0] == orc.mem_div(t, 1, 16)[0]).all()
    assert (out["branch_div"][1] == orc.branch_div(t, 32)[1]).all()


def _mix(kind_of, site_of, n=40, warps=2, bb=False):
    """Groups of 20 lanes, warps 0..warps-1, winst 0..n/20-1 per warp; the
    callbacks give each record's kind and site (record index)."""
    recs = []
    for w in range(warps):
        for g in range(n // 20):
            for l in range(20):
                i = len(recs)
                recs.append((0x7F0000000000 + 128 * (g * 7 + l // 8), 32 * w + l, g, site_of(i),
                             (BB if bb else kind_of(i)) | (2 << 2)))
    a = np.array(recs, dtype=np.uint64)
    return tg.from_arrays(a[:, 0], np.zeros(len(a)), a[:, 1], a[:, 3], a[:, 2], a[:, 4], nsites=8)


@pytest.mark.parametrize("where", [0, 1, 19, 57])
def test_group_rule(ctx, cadv, where):
    good = _mix(lambda i: LD if (i // 20) % 2 else ST, lambda i: (i // 20) % 8)
    ctx.load_trace(cadv.to_device(good))
    h, ps = ctx.mem_divergence(128, 32, 8)
    hr, pr = orc.mem_div(good, 128, 32)
    assert (h == hr).all() and (ps == pr).all()
    bad_site = _mix(lambda i: LD, lambda i: 1 + (i == where and i % 20 != 0))
    bad_kind = _mix(lambda i: ST if (i == where and i % 20 != 0) else LD, lambda i: 1)
    bad_bb = _mix(None, lambda i: 3 + (i == where and i % 20 != 0), bb=True)
    for t, calls in ((bad_site, ("md",)), (bad_kind, ("md",)), (bad_bb, ("bd",))):
        if where % 20 == 0:      # the first record of a group defines it: nothing to violate
            continue
        ctx.load_trace(cadv.to_device(t))
        with pytest.raises(orc.OracleError):
            orc.mem_div(t, 128) if calls == ("md",) else orc.branch_div(t)
        for W in (32, 8):
            with pytest.raises(cadv.CadvError) as e:
                ctx.mem_divergence(128, W, 8) if calls == ("md",) else ctx.branch_divergence(W, 8)
            assert e.value.status == cadv.CADV_ERR_BAD_TRACE
        with pytest.raises(cadv.CadvError) as e:
            ctx.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=8)
        assert e.value.status == cadv.CADV_ERR_BAD_TRACE
        # reuse distance does not read the group columns: still exact
        h, st = ctx.reuse_histogram(128, 0, 0, 66)
        assert (h == orc.reuse(t, 128, 0)[0]).all()


@pytest.mark.parametrize("seed", range(4))
def test_fused_non_contiguous(ctx, cadv, seed):
    """One cadv_analyze call on a non-warp-contiguous trace: reuse distance
    over the trace order, divergence over the (cta, warp) groups."""
    t = tg.generate("rand", seed=seed, ctas=6, threads=128, instrs=15, lines=30, pstore=0.3, pbb=0.3,
                    scramble=1, scramble_seed=seed)
    ctx.load_trace(cadv.to_device(t), warp_contiguous=False)
    for (lb_rd, scope, lb_md, W, Wb) in ((128, 0, 32, 32, 32), (32, 1, 128, 16, 8)):
        out = ctx.analyze(rd=(lb_rd, scope, 0, 66), md=(lb_md, W), bd=Wb, nsites=t.nsites)
        h_ref, s_ref = orc.reuse(t, lb_rd, scope, 0, 66)
        assert (out["reuse"][0] == h_ref).all() and out["reuse"][1] == s_ref
        mh, ms = orc.mem_div(t, lb_md, W)
        assert (out["mem_div"][0] == mh).all() and (out["mem_div"][1] == ms).all()
        bs, bt = orc.branch_div(t, Wb)
        assert (out["branch_div"][1] == bt).all() and (out["branch_div"][0] == bs).all()
    base = np.array([int(t.addr[(t.meta & 3) != BB].min()) // 4096 * 4096], np.uint64)
    objs = (base, np.array([64 * 128 * 7], np.uint64))
    for scope in (0, 1):
        rh, mh = ctx.data_centric(objs, 128, scope, 0, 66, 32)
        rr, mr = orc.data_centric(t, objs, 128, scope, 0, 66, 32)
        assert (rh == rr).all() and (mh == mr).all()


@pytest.mark.parametrize("top", [(1 << 28) - 1, 1 << 28])
def test_bd_cta_id_boundary(ctx, cadv, top):
    """Branch divergence keeps T_c per CTA id: ids up to 2^28 - 1 are exact,
    an id of 2^28 is CADV_ERR_UNSUPPORTED (include/cadv.h) - for the separate
    and the fused call - while reuse and memory divergence take any id."""
    t0 = tg.generate("rand", seed=9, ctas=4, threads=96, instrs=20, lines=40, pstore=0.2, pbb=0.4)
    cols = {k: v.copy() for k, v in t0.cols.items()}
    cols["cta"] = (cols["cta"].astype(np.int64) + (top - int(cols["cta"].max()))).astype(np.uint32)
    t = tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t0.nsites)
    assert int(t.cta.max()) == top
    ctx.load_trace(cadv.to_device(t))
    h, st = ctx.reuse_histogram(128, 0, 0, 66)
    hr, sr = orc.reuse(t, 128, 0, 0, 66)
    assert (h == hr).all() and st == sr
    m, ps = ctx.mem_divergence(128, 32, t.nsites)
    assert (m == orc.mem_div(t, 128, 32)[0]).all()
    if top < (1 << 28):
        ps, tot = ctx.branch_divergence(32, t.nsites)
        psr, totr = orc.branch_div(t, 32)
        assert (tot == totr).all() and (ps == psr).all()
        out = ctx.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)
        assert (out["branch_div"][1] == totr).all()
    else:
        for call in (lambda: ctx.branch_divergence(32, t.nsites),
                     lambda: ctx.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)):
            with pytest.raises(cadv.CadvError) as e:
                call()
            assert e.value.status == cadv.CADV_ERR_UNSUPPORTED
