"""GPU parity: the CUDA path (through the C ABI) == the CPU oracle, bit-exact.

Every output is an integer, so comparisons are exact (`==`), element by
element: histograms, stats, per-site counters.  Inputs are seeded synthetic
traces from tracegen/ (DESIGN.md "Input recipe").
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


def load(ctx, cadv, t, contiguous=True, host=False):
    if host:
        ctx.load_trace(t.cols, warp_contiguous=contiguous)
    else:
        ctx.load_trace(cadv.to_device(t), warp_contiguous=contiguous)


def check_reuse(ctx, t, lb, scope, binning=0, nbins=66):
    h_gpu, s_gpu = ctx.reuse_histogram(lb, scope, binning, nbins)
    h_ref, s_ref = orc.reuse(t, lb, scope, binning, nbins)
    assert (h_gpu == h_ref).all(), (lb, scope, binning, np.nonzero(h_gpu != h_ref), h_gpu, h_ref)
    assert s_gpu == s_ref, (lb, scope, s_gpu, s_ref)


def check_md(ctx, t, lb, W=32):
    h_gpu, ps_gpu = ctx.mem_divergence(lb, W, t.nsites)
    h_ref, ps_ref = orc.mem_div(t, lb, W)
    assert (h_gpu == h_ref).all(), (lb, W, h_gpu, h_ref)
    assert (ps_gpu == ps_ref).all()


def check_bd(ctx, t, W=32):
    ps_gpu, tot_gpu = ctx.branch_divergence(W, t.nsites)
    ps_ref, tot_ref = orc.branch_div(t, W)
    assert (tot_gpu == tot_ref).all(), (W, tot_gpu, tot_ref)
    assert (ps_gpu == ps_ref).all()


def full_check(ctx, cadv, t, lbs=(128, 32), scopes=(0, 1), contiguous=True, W=(32,)):
    load(ctx, cadv, t, contiguous)
    for lb in lbs:
        for sc in scopes:
            check_reuse(ctx, t, lb, sc)
        check_md(ctx, t, lb)
    for w in W:
        check_bd(ctx, t, w)


# ----------------------------------------------------------------- config 1 + closed forms

def test_c1_vecadd_all(ctx, cadv):
    t = tg.generate("vecadd")
    load(ctx, cadv, t)
    for lb in (1, 4, 32, 128):
        for sc in (0, 1):
            for binning, nb in ((0, 66), (1, 12), (0, 3)):
                check_reuse(ctx, t, lb, sc, binning, nb)
        for W in (32, 16, 8, 4, 2, 1):
            check_md(ctx, t, lb, W)
    for W in (32, 16, 8, 1):
        check_bd(ctx, t, W)
    # closed forms through the GPU path too
    h, st = ctx.reuse_histogram(128, 0, 0, 66)
    assert h[0] == 1322 and h[-1] == 727
    ps, tot = ctx.branch_divergence(32, t.nsites)
    assert list(tot) == [50, 2, 1558]


def test_host_pointer_load(ctx, cadv):
    t = tg.generate("vecadd")
    load(ctx, cadv, t, host=True)
    check_reuse(ctx, t, 128, 0)
    check_md(ctx, t, 32)
    check_bd(ctx, t)


def test_paper_example_gpu(ctx, cadv):
    """ABCCDEFAAAB, RD(B) = 5; full histogram {0:3, 5:2, ∞:6}."""
    addr = [0x7F0000000000 + 4 * "ABCDEF".index(ch) for ch in "ABCCDEFAAAB"]
    n = len(addr)
    t = tg.from_arrays(addr, np.zeros(n), np.zeros(n), np.zeros(n), np.arange(n), [2 << 2] * n, nsites=1)
    load(ctx, cadv, t)
    h, st = ctx.reuse_histogram(4, 0, 0, 8)
    assert list(h) == [3, 0, 0, 0, 0, 2, 0, 6]


@pytest.mark.parametrize("K,R", [(3, 4), (100, 3), (5000, 2), (9000, 3)])
def test_cyclic_closed_form_gpu(ctx, cadv, K, R):
    """K lines read cyclically R times: K ∞ + K(R-1) at distance K-1 (spans tiles for K > 4096)."""
    n = K * R
    addr = 0x7F0000000000 + 128 * (np.arange(n) % K)
    t = tg.from_arrays(addr, np.zeros(n), np.zeros(n), np.zeros(n), np.arange(n), np.full(n, 2 << 2), nsites=1)
    load(ctx, cadv, t)
    h, st = ctx.reuse_histogram(128, 0, 0, K + 3)
    assert h[-1] == K and h[K - 1] == K * (R - 1) and h.sum() == n


# ----------------------------------------------------------------- random traces

RAND_CASES = [
    dict(ctas=1, threads=32, instrs=4, lines=4),
    dict(ctas=3, threads=64, instrs=10, lines=16, pstore=0.3),
    dict(ctas=8, threads=96, instrs=20, lines=40, pbb=0.5),
    dict(ctas=2, threads=1024, instrs=30, lines=200),        # large CTA segments -> several tiles
    dict(ctas=40, threads=128, instrs=12, lines=8, pfull=0.9),
    dict(ctas=5, threads=33, instrs=50, lines=3, pstore=0.5),
    dict(ctas=1, threads=1024, instrs=80, lines=2000, pstore=0.1),  # one giant CTA, many lines
    dict(ctas=200, threads=64, instrs=6, lines=64, launches=3),
]


@pytest.mark.parametrize("case", range(len(RAND_CASES)))
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_traces(ctx, cadv, case, seed):
    t = tg.generate("rand", seed=seed, **RAND_CASES[case])
    full_check(ctx, cadv, t, lbs=(1, 32, 128), W=(32, 8))


@pytest.mark.parametrize("seed", range(6))
def test_non_contiguous_traces(ctx, cadv, seed):
    """warp_contiguous = 0: records of the per-(cta, warp) streams randomly merged."""
    t = tg.generate("rand", seed=seed, ctas=6, threads=128, instrs=15, lines=30, scramble=1, scramble_seed=seed)
    full_check(ctx, cadv, t, lbs=(32, 128), contiguous=False, W=(32, 16))


@pytest.mark.parametrize("seed", range(4))
def test_lane_order_independence(ctx, cadv, seed):
    """Divergence depends on lane sets, not on the order lanes appear in a warp instruction."""
    t = tg.generate("rand", seed=seed, ctas=4, threads=64, instrs=20, lines=20)
    rng = np.random.default_rng(seed)
    # permute records inside each run of equal (cta, warp, winst, family)
    key = (t.cta.astype(np.int64) << 32) | ((t.tid.astype(np.int64) >> 5) << 24) | (t.winst.astype(np.int64) << 1) \
        | ((t.meta & 3) == 2)
    starts = np.r_[0, np.nonzero(np.diff(key))[0] + 1, t.n]
    order = np.arange(t.n)
    for a, b in zip(starts[:-1], starts[1:]):
        order[a:b] = a + rng.permutation(b - a)
    t2 = tg.from_arrays(*(t.cols[k][order] for k, _ in tg.COLUMNS), nsites=t.nsites)
    load(ctx, cadv, t2)
    check_md(ctx, t2, 32)
    check_bd(ctx, t2)
    h1, _ = orc.mem_div(t, 32)
    h2, _ = ctx.mem_divergence(32, 32, t.nsites)
    assert (h1 == h2).all()


# ----------------------------------------------------------------- adversarial / edge cases

def _mk(addr, cta, tid=None, meta=None, winst=None):
    n = len(addr)
    tid = np.zeros(n) if tid is None else tid
    meta = np.full(n, 2 << 2) if meta is None else meta
    winst = np.arange(n) if winst is None else winst
    return tg.from_arrays(addr, cta, tid, np.zeros(n), winst, meta, nsites=1)


def test_all_same_line(ctx, cadv):
    n = 20000
    t = _mk(np.full(n, 0x7F0000000000), np.zeros(n))
    full_check(ctx, cadv, t, lbs=(128,), W=(32,))


def test_all_distinct_lines(ctx, cadv):
    n = 20000
    t = _mk(0x7F0000000000 + 128 * np.arange(n), np.zeros(n))
    full_check(ctx, cadv, t, lbs=(128, 4096), W=(32,))


@pytest.mark.parametrize("k", [1, 2, 7])
def test_stores_every_k(ctx, cadv, k):
    rng = np.random.default_rng(k)
    n = 30000
    addr = 0x7F0000000000 + 4 * rng.integers(0, 300, n)
    meta = np.where(np.arange(n) % k == 0, (2 << 2) | 1, 2 << 2)
    t = _mk(addr, rng.integers(0, 3, n), meta=meta)
    full_check(ctx, cadv, t, lbs=(4, 32, 128), W=(32,))


def test_many_tiny_ctas(ctx, cadv):
    rng = np.random.default_rng(5)
    n = 100000
    cta = np.sort(rng.integers(0, 60000, n))
    addr = 0x7F0000000000 + 8 * rng.integers(0, 50, n)
    t = _mk(addr, cta)
    full_check(ctx, cadv, t, lbs=(8, 128), W=(32,))


def test_empty_and_bb_only(ctx, cadv):
    t = _mk(np.zeros(0, np.uint64), np.zeros(0))
    load(ctx, cadv, t)
    h, st = ctx.reuse_histogram(128, 0, 0, 10)
    assert h.sum() == 0 and st["accesses"] == 0
    hm, _ = ctx.mem_divergence(128, 32, 1)
    assert hm.sum() == 0
    _, tot = ctx.branch_divergence(32, 1)
    assert tot.sum() == 0
    t = tg.generate("nw", ctas=3)
    full_check(ctx, cadv, t, lbs=(128,), W=(32, 16))


def test_large_nbins_global_atomics(ctx, cadv):
    t = tg.generate("rand", seed=9, ctas=2, threads=512, instrs=40, lines=900)
    load(ctx, cadv, t)
    check_reuse(ctx, t, 32, 0, 0, 5000)
    check_reuse(ctx, t, 32, 1, 0, 5000)


def test_bad_trace_detected(ctx, cadv):
    t = tg.generate("vecadd")
    cols = {k: v.copy() for k, v in t.cols.items()}
    cols["meta"][100] = 3
    ctx.load_trace(cadv.to_device(tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t.nsites)))
    for call in (lambda: ctx.reuse_histogram(128, 0, 0, 10), lambda: ctx.mem_divergence(128, 32, 7),
                 lambda: ctx.branch_divergence(32, 7)):
        with pytest.raises(cadv.CadvError) as e:
            call()
        assert e.value.status == cadv.CADV_ERR_BAD_TRACE
    cols = {k: v.copy() for k, v in t.cols.items()}
    mem = np.nonzero((cols["meta"] & 3) < 2)[0]
    cols["addr"][mem[5]] += 1
    ctx.load_trace(cadv.to_device(tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t.nsites)))
    with pytest.raises(cadv.CadvError) as e:
        ctx.reuse_histogram(128, 0, 0, 10)
    assert e.value.status == cadv.CADV_ERR_BAD_TRACE


def test_long_run_detected(ctx, cadv):
    """A warp-level group of 40 records (same cta, warp, winst) violates the format."""
    n = 40
    t = _mk(0x7F0000000000 + 4 * np.arange(n), np.zeros(n), tid=np.arange(n) % 32, winst=np.zeros(n))
    ctx.load_trace(cadv.to_device(t))
    with pytest.raises(cadv.CadvError) as e:
        ctx.mem_divergence(128, 32, 1)
    assert e.value.status == cadv.CADV_ERR_BAD_TRACE


@pytest.mark.parametrize("bb", [False, True])
@pytest.mark.parametrize("lead,size,dup", [(0, 32, (3, 4)), (5, 20, (0, 19)), (13, 32, (30, 31)), (250, 12, (2, 9))])
def test_repeated_lane_detected(ctx, cadv, bb, lead, size, dup):
    """A warp-level group of <= 32 records with one lane twice (the run's lane
    masks are accumulated by addition in the scan: the carry must still fail
    the popcount check), at various offsets inside a 256-record step; the
    same trace without the repeat is valid and matches the oracle."""
    def build(repeat):
        recs = []  # (addr, tid, winst)
        for g in range(lead):      # filler groups of 1 record (warp 1), before the tested group
            recs.append((0x7F0000000000 + 128 * g, 32, g))
        lanes = list(range(size))
        if repeat:
            lanes[dup[1]] = lanes[dup[0]]
        for q, l in enumerate(lanes):
            recs.append((0x7F0000100000 + 4 * q, l, 0))
        for g in range(40):        # trailing groups
            recs.append((0x7F0000200000 + 128 * g, 32, lead + g))
        a = np.array(recs, dtype=np.uint64)
        meta = np.full(len(a), (2 if bb else 0) | (2 << 2))
        return tg.from_arrays(a[:, 0], np.zeros(len(a)), a[:, 1], np.zeros(len(a)), a[:, 2], meta, nsites=1)
    ok = build(False)
    ctx.load_trace(cadv.to_device(ok))
    if bb:
        psb, tot = ctx.branch_divergence(32, 1)
        psb_ref, tot_ref = orc.branch_div(ok, 32)
        assert (tot == tot_ref).all() and (psb == psb_ref).all()
    else:
        hm, psm = ctx.mem_divergence(128, 32, 1)
        hm_ref, psm_ref = orc.mem_div(ok, 128, 32)
        assert (hm == hm_ref).all() and (psm == psm_ref).all()
    ctx.load_trace(cadv.to_device(build(True)))
    with pytest.raises(cadv.CadvError) as e:
        ctx.branch_divergence(32, 1) if bb else ctx.mem_divergence(128, 32, 1)
    assert e.value.status == cadv.CADV_ERR_BAD_TRACE


def test_invalid_args(ctx, cadv):
    t = tg.generate("vecadd")
    load(ctx, cadv, t)
    for args in ((48, 0, 0, 10), (128, 2, 0, 10), (128, 0, 5, 10), (128, 0, 0, 2), (8192, 0, 0, 10)):
        with pytest.raises(cadv.CadvError) as e:
            ctx.reuse_histogram(*args)
        assert e.value.status == cadv.CADV_ERR_INVALID_ARG
    with pytest.raises(cadv.CadvError):
        ctx.mem_divergence(128, 64, 7)
    with pytest.raises(cadv.CadvError) as e:
        ctx.mem_divergence(128, 32, 3)  # sites up to 6 exist
    assert e.value.status == cadv.CADV_ERR_INVALID_ARG


# ----------------------------------------------------------------- fused pass (cadv_analyze)

@pytest.mark.parametrize("seed", range(4))
def test_fused_analyze_equals_oracle(ctx, cadv, seed):
    t = tg.generate("rand", seed=seed, ctas=7, threads=160, instrs=40, lines=80, pstore=0.2, pbb=0.4)
    load(ctx, cadv, t)
    for (lb_rd, scope, lb_md, W, Wb) in ((128, 0, 32, 32, 32), (32, 1, 128, 16, 8), (4, 0, 4, 8, 32)):
        out = ctx.analyze(rd=(lb_rd, scope, 0, 66), md=(lb_md, W), bd=Wb, nsites=t.nsites)
        h_ref, s_ref = orc.reuse(t, lb_rd, scope, 0, 66)
        assert (out["reuse"][0] == h_ref).all() and out["reuse"][1] == s_ref
        mh, ms = orc.mem_div(t, lb_md, W)
        assert (out["mem_div"][0] == mh).all() and (out["mem_div"][1] == ms).all()
        bs, bt = orc.branch_div(t, Wb)
        assert (out["branch_div"][1] == bt).all() and (out["branch_div"][0] == bs).all()


def test_fused_subsets(ctx, cadv):
    t = tg.generate("srad", rows=64, cols=64, iters=1)
    load(ctx, cadv, t)
    out = ctx.analyze(rd=None, md=(128, 32), bd=None, nsites=t.nsites)
    assert set(out) == {"mem_div"}
    assert (out["mem_div"][0] == orc.mem_div(t, 128, 32)[0]).all()
    out = ctx.analyze(rd=(128, 0, 1, 20), md=None, bd=32, nsites=t.nsites, per_site=False)
    assert (out["reuse"][0] == orc.reuse(t, 128, 0, 1, 20)[0]).all()
    assert (out["branch_div"][1] == orc.branch_div(t, 32)[1]).all()


# ----------------------------------------------------------------- shaped workloads (reduced sizes)

def test_sgemm_small(ctx, cadv):
    full_check(ctx, cadv, tg.generate("sgemm", n=64, bb=1), lbs=(32, 128))


def test_srad_small(ctx, cadv):
    full_check(ctx, cadv, tg.generate("srad", rows=128, cols=128, iters=2), lbs=(32, 128))


def test_bfs_small(ctx, cadv):
    full_check(ctx, cadv, tg.generate("bfs", nodes=20000, seed=3), lbs=(32, 128))


def test_backprop_small(ctx, cadv):
    full_check(ctx, cadv, tg.generate("backprop", **{"in": 4096}), lbs=(32, 128))


def test_polybench_md_printed_gpu(ctx, cadv):
    """The paper's printed BICG/Syrk memory-divergence shares, via the GPU path."""
    t = tg.generate("bicg", nx=1024, ny=1024)
    load(ctx, cadv, t)
    h, _ = ctx.mem_divergence(128, 32, t.nsites)
    pooled = h.sum(axis=0).astype(float)
    assert round(100 * pooled[1] / pooled.sum()) == 75 and round(100 * pooled[32] / pooled.sum()) == 25
    check_md(ctx, t, 32)
    t = tg.generate("syrk", ni=8, nj=32, m=1024)
    load(ctx, cadv, t)
    h, _ = ctx.mem_divergence(128, 32, t.nsites)
    pooled = h.sum(axis=0).astype(float)
    assert round(100 * pooled[1] / pooled.sum(), 2) == 50.02


# ----------------------------------------------------------------- full-size configs

@pytest.mark.slow
def test_c2_sgemm_full(ctx, cadv):
    """Config 2 at full size (35,782,656 records), both line sizes, bit-exact."""
    t = tg.generate("sgemm", n=256)
    assert t.n == 35782656
    full_check(ctx, cadv, t, lbs=(32, 128), scopes=(0,))


# ----------------------------------------------------------------- store chains / long warp chunks

def _chain_trace(seed, n_chains=400, max_len=300):
    """Store chains of random length (1 .. max_len, also >16 and across lanes,
    steps and chunks), each followed by 0-3 loads of the same line (duplicates,
    RD 0) and a few unrelated loads, over a handful of CTAs."""
    rng = np.random.default_rng(seed)
    addr, cta, meta = [], [], []
    for _ in range(n_chains):
        line = int(rng.integers(0, 64))
        c = int(rng.integers(0, 3))
        L = int(rng.choice([1, 2, 15, 16, 17, 31, 32, 33, 255, 256, 257, int(rng.integers(1, max_len))]))
        base = 0x7F0000000000 + 128 * line
        addr += [base + 4 * int(o) for o in rng.integers(0, 32, L)]
        cta += [c] * L
        meta += [(2 << 2) | 1] * L
        nd = int(rng.integers(0, 4))
        addr += [base] * nd
        cta += [c] * nd
        meta += [2 << 2] * nd
        no = int(rng.integers(0, 4))
        addr += [0x7F0000000000 + 128 * int(x) for x in rng.integers(0, 64, no)]
        cta += [c] * no
        meta += [2 << 2] * no
    n = len(addr)
    return _mk(np.array(addr, np.uint64), np.array(cta), meta=np.array(meta))


@pytest.mark.parametrize("seed", [11, 12, 13])
def test_store_chains(ctx, cadv, seed):
    t = _chain_trace(seed)
    full_check(ctx, cadv, t, lbs=(4, 128), W=(32,))


@pytest.fixture(scope="module")
def ctx_long(cadv):
    """A context whose streaming pass uses 1 CTA: warp chunks of many 256-record steps."""
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
    yield c
    c.destroy()


LONG_CASES = [
    ("chains", dict(seed=21)),
    ("rand", dict(seed=4, ctas=8, threads=96, instrs=20, lines=40, pbb=0.5)),
    ("rand", dict(seed=5, ctas=5, threads=33, instrs=50, lines=3, pstore=0.5)),
    ("rand", dict(seed=6, ctas=2, threads=1024, instrs=30, lines=200, pstore=0.3)),
    ("srad", dict(rows=128, cols=128, iters=2)),
    ("bfs", dict(nodes=20000, seed=3)),
    ("nw", dict(ctas=3)),
]


@pytest.mark.parametrize("case", range(len(LONG_CASES)))
def test_long_chunks(ctx_long, cadv, case):
    name, kw = LONG_CASES[case]
    t = _chain_trace(kw["seed"]) if name == "chains" else tg.generate(name, **kw)
    full_check(ctx_long, cadv, t, lbs=(4, 128), W=(32, 8))
    out = ctx_long.analyze(rd=(128, 1, 0, 66), md=(32, 32), bd=32, nsites=t.nsites)
    assert (out["reuse"][0] == orc.reuse(t, 128, 1, 0, 66)[0]).all()
    assert (out["mem_div"][0] == orc.mem_div(t, 32, 32)[0]).all()
    assert (out["branch_div"][1] == orc.branch_div(t, 32)[1]).all()


def test_long_chunks_non_contiguous(ctx_long, cadv):
    t = tg.generate("rand", seed=7, ctas=6, threads=128, instrs=15, lines=30, scramble=1, scramble_seed=7)
    full_check(ctx_long, cadv, t, lbs=(32,), contiguous=False, W=(32, 16))


@pytest.mark.parametrize("spread", [40, 57])
def test_tile_key_widths(ctx, cadv, spread):
    """Tiles whose line range needs 64-bit packed sort keys (2^20 <= range <
    2^52 lines) or separate line / position arrays (>= 2^52, 1-byte lines):
    addresses spread over 2^spread bytes, with repeats so reuses exist."""
    rng = np.random.default_rng(spread)
    n = 30000
    base = rng.integers(0, 1 << spread, 500, dtype=np.uint64) & ~np.uint64(15)
    addr = base[rng.integers(0, 500, n)]
    meta = np.where(rng.random(n) < 0.2, (2 << 2) | 1, 2 << 2)
    t = _mk(addr, rng.integers(0, 3, n), meta=meta)
    full_check(ctx, cadv, t, lbs=(1, 128), W=(32,))


def test_eq1_from_gpu_outputs(ctx, cadv):
    """NEXT-4: Eq. (1) from the library's outputs equals the
    same metric from the oracle's (R.D. from the exact finite-distance sum)."""
    from paper_conf_cgo_shensll18_b200 import metrics as M
    t = tg.generate("srad", rows=128, cols=128, iters=2)
    load(ctx, cadv, t)
    o = ctx.analyze(rd=(128, 0, 0, 20), md=(128, 32), bd=None, nsites=t.nsites)
    h_ref, s_ref = orc.reuse(t, 128, 0, 0, 20)
    assert o["reuse"][1] == s_ref and s_ref["overflow"] > 0   # the mean needs the exact sum, not the bins
    rd, md = M.mean_reuse_distance(o["reuse"][1]), M.md_degree(o["mem_div"][0])
    assert rd == M.mean_reuse_distance(s_ref) and md == M.md_degree(orc.mem_div(t, 128)[0])
    assert M.opt_num_warps(16384, rd, 128, md, 4) == M.opt_num_warps(16384, M.mean_reuse_distance(s_ref), 128,
                                                                       orc.md_degree(orc.mem_div(t, 128)[0]), 4)


@pytest.mark.parametrize("ctas", [40, 1500])
def test_regroup_tables_and_overflow(ctx, ctx_long, cadv, ctas):
    """CTA regroup through per-region CTA tables (regroup.cu): with 1 scan CTA
    (16 regions) 1500 CTAs overflow a region's table (> RG_MAX = 768
    distinct CTAs) and the squeeze + radix-sort path takes over; 40 CTAs fit.
    Both contexts, both line sizes, CTA scope, against the oracle."""
    t = tg.generate("rand", seed=31, ctas=ctas, threads=64, instrs=12, lines=50, pstore=0.2, pbb=0.2)
    for c in (ctx, ctx_long):
        load(c, cadv, t)
        check_reuse(c, t, 128, 0)
        check_reuse(c, t, 32, 0, 1, 20)


def test_cta_id_all_ones(ctx, cadv):
    """CTA id 0xffffffff (the regroup tables' empty marker) in a reuse trace:
    such a trace takes the radix-sort regroup and still matches the oracle."""
    rng = np.random.default_rng(5)
    n = 5000
    cta = rng.choice(np.array([0, 7, 0xFFFFFFFF, 12345], dtype=np.uint64), n)
    addr = 0x7F0000000000 + 128 * rng.integers(0, 300, n).astype(np.uint64)
    t = _mk(addr, cta, tid=rng.integers(0, 64, n), meta=np.full(n, 2 << 2))
    load(ctx, cadv, t)
    check_reuse(ctx, t, 128, 0)
    check_reuse(ctx, t, 128, 1)


@pytest.mark.parametrize("case", [("srad", dict(rows=128, cols=128, iters=2)), ("bfs", dict(nodes=20000, seed=3)),
                                  ("rand", dict(seed=12, ctas=30, threads=64, instrs=10, lines=40, pstore=0.3))])
def test_segment_kernel_equals_tiles(ctx, cadv, case):
    """CTA segments of <= 256 kept records go to the segment kernel (k_rd_seg);
    CADV_RD_TILES forces the tile kernels on the same trace: both equal the
    oracle (histogram, stats incl. streaming and the finite sum), both bin modes."""
    import os
    name, kw = case
    t = tg.generate(name, **kw)
    load(ctx, cadv, t)
    for lb, binning, nb in ((128, 0, 66), (32, 1, 20)):
        ref = orc.reuse(t, lb, 0, binning, nb)
        seg = ctx.reuse_histogram(lb, 0, binning, nb)
        os.environ["CADV_RD_TILES"] = "1"
        try:
            til = ctx.reuse_histogram(lb, 0, binning, nb)
        finally:
            del os.environ["CADV_RD_TILES"]
        for h, st in (seg, til):
            assert (h == ref[0]).all() and st == ref[1], (name, lb)


@pytest.mark.parametrize("reuse_frac", [0.0, 0.25])
def test_segment_kernel_full_hash_tables(ctx, cadv, reuse_frac):
    """Every CTA segment holds exactly 256 kept records (the segment kernel's
    limit) over up to 256 distinct random lines spread across a 2^40-line
    range: each warp's hash table runs at its highest load, with long probe
    chains and wrap-around; the result equals the oracle and the tile path."""
    import os
    rng = np.random.default_rng(31)
    nct, per = 300, 256
    addr, cta = [], []
    for c in range(nct):
        nd = per - int(per * reuse_frac)
        lines = rng.choice(1 << 40, nd, replace=False).astype(np.uint64)
        seq = np.concatenate([lines, rng.choice(lines, per - nd)])
        rng.shuffle(seq)
        for k in range(1, per):  # no two consecutive equal lines (no duplicate-load compression)
            if seq[k] == seq[k - 1]:
                seq[k], seq[0] = seq[0], seq[k]
        addr.append(0x10000000000 + 128 * seq)
        cta.append(np.full(per, c, dtype=np.uint64))
    addr, cta = np.concatenate(addr), np.concatenate(cta)
    meta = np.where(rng.random(len(addr)) < 0.1, (2 << 2) | 1, 2 << 2)
    t = _mk(addr, cta, tid=rng.integers(0, 256, len(addr)), meta=meta)
    load(ctx, cadv, t)
    ref = orc.reuse(t, 128, 0, 0, 66)
    seg = ctx.reuse_histogram(128, 0, 0, 66)
    os.environ["CADV_RD_TILES"] = "1"
    try:
        til = ctx.reuse_histogram(128, 0, 0, 66)
    finally:
        del os.environ["CADV_RD_TILES"]
    for h, st in (seg, til):
        assert (h == ref[0]).all() and st == ref[1]


@pytest.mark.parametrize("longest", [4096, 4097])
def test_segment_lists_mixed_lengths(ctx, cadv, longest):
    """CTA segments of every length class in one trace: <= 256 kept records
    (segment kernel), 257 .. 4096 (one tile each from the segment list, no
    cross-tile queries; line ranges for all three tile key widths) and, with
    longest = 4097, one segment that sends the call to the bounds-tiled path
    with its cross-tile phase.  Both scopes, both bin modes, against the
    oracle and the forced tile path."""
    import os
    rng = np.random.default_rng(longest)
    lens = [1, 2, 255, 256, 257, 300, 1000, 2048, 4095, longest] + list(rng.integers(1, 700, 60))
    addr, cta = [], []
    for c, n in enumerate(lens):
        span = [1 << 12, 1 << 30, 1 << 55][c % 3]  # MODE 0 / 1 / 2 tiles (line range < 2^20, < 2^52, wider)
        nd = max(1, int(n * rng.uniform(0.2, 0.9)))
        lines = np.sort(rng.choice(span, nd, replace=False).astype(np.uint64))
        seq = rng.choice(lines, int(n))
        for k in range(1, int(n)):  # no two consecutive equal lines: every record is kept
            if seq[k] == seq[k - 1]:
                seq[k] = lines[(np.searchsorted(lines, seq[k]) + 1) % nd] if nd > 1 else seq[k]
        addr.append(128 * seq)
        cta.append(np.full(int(n), c, dtype=np.uint64))
    order = rng.permutation(len(lens))  # CTAs interleaved in blocks, as resident CTAs would be
    addr = np.concatenate([addr[i] for i in order])
    cta = np.concatenate([cta[i] for i in order])
    meta = np.where(rng.random(len(addr)) < 0.15, (2 << 2) | 1, 2 << 2)
    t = _mk(addr, cta, tid=rng.integers(0, 256, len(addr)), meta=meta)
    load(ctx, cadv, t)
    for lb, scope, binning, nb in ((128, 0, 0, 66), (128, 0, 1, 20), (128, 1, 0, 66)):
        ref = orc.reuse(t, lb, scope, binning, nb)
        got = ctx.reuse_histogram(lb, scope, binning, nb)
        os.environ["CADV_RD_TILES"] = "1"
        try:
            til = ctx.reuse_histogram(lb, scope, binning, nb)
        finally:
            del os.environ["CADV_RD_TILES"]
        for h, st in (got, til):
            assert (h == ref[0]).all() and st == ref[1], (lb, scope, binning)


@pytest.mark.parametrize("seed", [1, 2])
def test_many_sites_global_counters(ctx, cadv, seed):
    """More than 512 sites (NSITE_SMEM): the per-site counters of memory and
    branch divergence take the global-atomic path; fused and separate calls,
    W = 32 and 8, against the oracle."""
    t = tg.generate("rand", seed=seed, ctas=20, threads=256, instrs=40, lines=100, msites=3000, bsites=1000,
                    pbb=0.4, pstore=0.2)
    assert t.nsites == 4000
    full_check(ctx, cadv, t, lbs=(32, 128), scopes=(0,), W=(32, 8))
    out = ctx.analyze(rd=(128, 0, 0, 66), md=(128, 16), bd=16, nsites=t.nsites)
    mh, ms = orc.mem_div(t, 128, 16)
    assert (out["mem_div"][0] == mh).all() and (out["mem_div"][1] == ms).all()
    bs, bt = orc.branch_div(t, 16)
    assert (out["branch_div"][0] == bs).all() and (out["branch_div"][1] == bt).all()
