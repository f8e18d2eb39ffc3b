"""GPU parity of the data-centric attribution (cadv_data_centric, P:L123-133,
SURVEY.md NEXT-3): per-object reuse-distance and memory-divergence rows ==
the CPU oracle (oracle.data_centric), bit-exact, through the C ABI.

Object tables: the generators' own allocation tables (tracegen.objects) and
random line-disjoint tables over the trace's address range (gaps leave
unattributed lines; trims make objects end inside a line).
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


@pytest.fixture(scope="module")
def ctx(cadv):
    c = cadv.create(0)
    yield c
    c.destroy()


def random_table(t, L, k, seed):
    """Up to k ascending objects over the memory records' address range, no
    line shared by two objects (valid at line size L)."""
    rng = np.random.default_rng(seed)
    mem = (t.meta & 3) != 2
    if not mem.any():
        return np.zeros(0, np.uint64), np.zeros(0, np.uint64)
    lo_line, hi_line = int(t.addr[mem].min()) // L, int(t.addr[mem].max()) // L + 1
    cuts = sorted(set(int(x) for x in rng.integers(lo_line, hi_line + 1, 2 * k)))
    base, nbytes = [], []
    for a, b in zip(cuts[::2], cuts[1::2]):
        lo = a * L + int(rng.integers(0, max(1, L // 2)))
        hi = b * L - int(rng.integers(0, max(1, L // 2)))
        if hi > lo and (not base or (base[-1] + nbytes[-1] - 1) // L < lo // L):
            base.append(lo)
            nbytes.append(hi - lo)
    return np.array(base, np.uint64), np.array(nbytes, np.uint64)


def check(ctx, t, objs, L, scope=0, binning=0, nbins=66, W=32):
    rh, mh = ctx.data_centric(objs, L, scope, binning, nbins, W)
    rr, mr = orc.data_centric(t, objs, L, scope, binning, nbins, W)
    assert (rh == rr).all(), (L, scope, np.argwhere(rh != rr)[:8])
    assert (mh == mr).all(), (L, W, np.argwhere(mh != mr)[:8])


def test_vecadd_generator_objects(ctx, cadv):
    t = tg.generate("vecadd")
    ctx.load_trace(cadv.to_device(t))
    objs = tg.objects("vecadd")
    for L in (1, 4, 32, 128):
        for scope in (0, 1):
            check(ctx, t, objs, L, scope)
    # the closed form of tests/test_oracle_pins.py through the GPU path
    rh, mh = ctx.data_centric(objs, 128)
    assert list(rh[:, 0]) == [661, 661, 0, 0] and list(rh[:, 65]) == [22, 22, 683, 0]
    assert mh[0, 0, 1] == 22 and mh[1, 0, 1] == 22 and mh[2, 1, 1] == 22


RAND = [
    dict(ctas=3, threads=64, instrs=10, lines=16, pstore=0.3),
    dict(ctas=8, threads=96, instrs=20, lines=40, pbb=0.5),
    dict(ctas=2, threads=1024, instrs=30, lines=200),         # several tiles per CTA: cross-tile queries
    dict(ctas=1, threads=1024, instrs=80, lines=2000, pstore=0.1),
    dict(ctas=200, threads=64, instrs=6, lines=64, launches=3),
]


@pytest.mark.parametrize("case", range(len(RAND)))
@pytest.mark.parametrize("seed", [1, 2])
def test_random_tables(ctx, cadv, case, seed):
    t = tg.generate("rand", seed=seed, **RAND[case])
    ctx.load_trace(cadv.to_device(t))
    for j, (L, scope, binning, nb, W) in enumerate(((128, 0, 0, 66, 32), (32, 1, 0, 40, 32), (4, 0, 1, 12, 8),
                                                    (1, 1, 1, 20, 32))):
        check(ctx, t, random_table(t, L, 6, 100 * seed + j), L, scope, binning, nb, W)
    check(ctx, t, tg.objects("rand", seed=seed, **RAND[case]), 128)


def test_many_objects_global_tables(ctx, cadv):
    """> 63 objects: the scan's object tables and counters move to global
    memory; 200 rows x 66 bins exceed the tile kernel's shared histogram."""
    t = tg.generate("rand", seed=9, ctas=6, threads=256, instrs=40, lines=3000, pstore=0.2)
    ctx.load_trace(cadv.to_device(t))
    for L, k in ((128, 200), (32, 70), (128, 40)):
        objs = random_table(t, L, k, 7 + k)
        check(ctx, t, objs, L, 0)
        check(ctx, t, objs, L, 1, 1, 30)


def test_cross_tile_kernel_scope(ctx, cadv):
    """Kernel scope on a cyclic trace over 9000 lines (three tiles): the
    cross-tile phase (k_link, k_cross_final) attributes its queries too."""
    K, R = 9000, 3
    n = K * R
    addr = 0x7F0000000000 + 128 * (np.arange(n) % K)
    t = tg.from_arrays(addr, np.zeros(n), np.zeros(n), np.zeros(n), np.arange(n), np.full(n, 2 << 2), nsites=1)
    ctx.load_trace(cadv.to_device(t))
    objs = (np.array([0x7F0000000000 + 128 * 100, 0x7F0000000000 + 128 * 5000], np.uint64),
            np.array([128 * 3000, 128 * 2500], np.uint64))
    rh, mh = ctx.data_centric(objs, 128, 1, 0, K + 3)
    # closed form: each line is ∞ once and K-1 away R-1 times, in its own object's row
    assert rh[0, -1] == 3000 and rh[0, K - 1] == 3000 * (R - 1)
    assert rh[1, -1] == 2500 and rh[1, K - 1] == 2500 * (R - 1)
    assert rh[2, -1] == K - 5500 and rh[2].sum() == (K - 5500) * R
    check(ctx, t, objs, 128, 1, 0, K + 3)


@pytest.mark.parametrize("name,kw", [("srad", dict(rows=128, cols=128, iters=2)), ("bfs", dict(nodes=20000, seed=3)),
                                     ("sgemm", dict(n=64)), ("backprop", dict(**{"in": 4096}))])
def test_workload_objects(ctx, cadv, name, kw):
    t = tg.generate(name, **kw)
    ctx.load_trace(cadv.to_device(t))
    objs = tg.objects(name, **kw)
    assert len(objs[0]) >= 3
    for L in (128, 32):
        check(ctx, t, objs, L)


def test_rows_partition_and_errors(ctx, cadv):
    t = tg.generate("rand", seed=4, ctas=4, threads=128, instrs=20, lines=100, pstore=0.2)
    ctx.load_trace(cadv.to_device(t))
    objs = random_table(t, 128, 5, 3)
    rh, mh = ctx.data_centric(objs, 128)
    h, _ = ctx.reuse_histogram(128, 0, 0, 66)
    hm, _ = ctx.mem_divergence(128, 32)
    assert (rh.sum(axis=0) == h).all() and (mh.sum(axis=0) == hm).all()
    rh0, mh0 = ctx.data_centric((np.zeros(0, np.uint64), np.zeros(0, np.uint64)), 128)
    assert (rh0[0] == h).all() and (mh0[0] == hm).all()
    b = 0x7F0000000000
    for base, nb in (([b, b + 64], [64, 64]), ([b + 4096, b], [64, 64]), ([b], [0])):
        with pytest.raises(cadv.CadvError) as ei:
            ctx.data_centric((np.array(base, np.uint64), np.array(nb, np.uint64)), 128)
        assert ei.value.status == cadv.CADV_ERR_INVALID_ARG
    # RD only / MD only
    rh1, mh1 = ctx.data_centric(objs, 128, md=False)
    assert mh1 is None and (rh1 == rh).all()
    rh2, mh2 = ctx.data_centric(objs, 128, rd=False)
    assert rh2 is None and (mh2 == mh).all()


def test_long_chunks_objects(cadv):
    """One scan CTA (long warp chunks): duplicate-load runs cross steps."""
    import os
    old = os.environ.get("CADV_SCAN_CTAS")
    os.environ["CADV_SCAN_CTAS"] = "1"
    try:
        c = cadv.create(0)
    finally:
        if old is None:
            del os.environ["CADV_SCAN_CTAS"]
        else:
            os.environ["CADV_SCAN_CTAS"] = old
    try:
        for name, kw in (("srad", dict(rows=128, cols=128, iters=2)), ("rand", dict(seed=5, ctas=5, threads=33,
                                                                                      instrs=50, lines=3, pstore=0.5))):
            t = tg.generate(name, **kw)
            c.load_trace(cadv.to_device(t))
            for L in (128, 4):
                check(c, t, random_table(t, L, 4, 11), L, 0, 0, 66, 8)
                check(c, t, tg.objects(name, **kw), L, 1)
    finally:
        c.destroy()
