"""Multi-rank parity on one GPU: G loopback ranks (threads of this process,
each with its own context and stream) analyse consecutive position-range
shards of one trace; every rank must return the oracle's whole-trace result,
bit-exact.  The loopback group drives the same collective
call sequence the NCCL path runs (include/cadv.h cadv_create_loopback).
"""
import threading

import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cadv():
    import paper_conf_cgo_shensll18_b200 as m
    return m


def run_ranks(cadv, t, cuts, fn, contiguous=True):
    """fn(ctx) on every rank r with shard [cuts[r], cuts[r+1]); returns per-rank results."""
    import torch
    G = len(cuts) - 1
    grp = cadv.LoopbackGroup(G)
    out, err = [None] * G, [None] * G

    def work(r):
        try:
            stream = torch.cuda.Stream()
            lo, hi = cuts[r], cuts[r + 1]
            cols = {k: torch.from_numpy(np.ascontiguousarray(t.cols[k][lo:hi])).cuda() for k in cadv.COLUMNS}
            torch.cuda.synchronize()
            ctx = grp.context(r, stream=stream.cuda_stream)
            try:
                ctx.load_trace(cols, global_offset=lo, warp_contiguous=contiguous)
                out[r] = fn(ctx)
            finally:
                ctx.destroy()
        except Exception as e:  # noqa: BLE001 - re-raised in the main thread
            err[r] = e

    th = [threading.Thread(target=work, args=(r,)) for r in range(G)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=300)
    assert not any(x.is_alive() for x in th), "a rank hung in a collective"
    grp.destroy()
    return out, err


def random_cuts(n, G, seed, empty=False):
    rng = np.random.default_rng(seed)
    inner = sorted(int(x) for x in rng.integers(0, n + 1, G - 1))
    if empty and G > 2:
        inner[1] = inner[0]  # one empty shard
    return [0] + inner + [n]


def snapped_cuts(t, G, seed):
    return tg.snap_cuts(t.cols, random_cuts(t.n, G, seed))


def check_all_equal(out, ref):
    for r, o in enumerate(out):
        assert o is not None, f"rank {r} returned nothing"
        for a, b in zip(o, ref):
            assert np.array_equal(np.asarray(a), np.asarray(b)), (r, a, b)


TRACES = {
    "rand_stores": lambda: tg.generate("rand", seed=3, ctas=9, threads=96, instrs=25, lines=40, pstore=0.3, pbb=0.3),
    "rand_bigcta": lambda: tg.generate("rand", seed=4, ctas=2, threads=1024, instrs=30, lines=300, pstore=0.2),
    "srad": lambda: tg.generate("srad", rows=128, cols=128, iters=2),
    "bfs": lambda: tg.generate("bfs", nodes=20000, seed=3),
}


@pytest.mark.parametrize("name", sorted(TRACES))
@pytest.mark.parametrize("G", [2, 3, 4])
@pytest.mark.parametrize("scope", [0, 1])
def test_reuse_position_shards(cadv, name, G, scope):
    """Reuse distance on arbitrary (unsnapped) position splits, CTA and kernel scope."""
    t = TRACES[name]()
    cuts = random_cuts(t.n, G, seed=G * 7 + scope, empty=(G == 4))
    h_ref, s_ref = orc.reuse(t, 128, scope, 0, 66)
    out, err = run_ranks(cadv, t, cuts, lambda c: c.reuse_histogram(128, scope, 0, 66))
    assert not any(err), err
    for h, s in out:
        assert (h == h_ref).all(), (np.nonzero(h != h_ref), h, h_ref)
        assert s == s_ref


@pytest.mark.parametrize("name", sorted(TRACES))
@pytest.mark.parametrize("G", [2, 4])
def test_fused_snapped_shards(cadv, name, G):
    """All three analyses in one call on group-snapped shards."""
    t = TRACES[name]()
    cuts = snapped_cuts(t, G, seed=G)
    ref_rd = orc.reuse(t, 32, 0, 1, 20)
    ref_md = orc.mem_div(t, 128, 32)
    ref_bd = orc.branch_div(t, 32)

    def fn(c):
        o = c.analyze(rd=(32, 0, 1, 20), md=(128, 32), bd=32, nsites=t.nsites)
        return o["reuse"][0], o["reuse"][1]["streaming"], o["mem_div"][0], o["mem_div"][1], \
            o["branch_div"][0], o["branch_div"][1]

    out, err = run_ranks(cadv, t, cuts, fn)
    assert not any(err), err
    check_all_equal(out, (ref_rd[0], ref_rd[1]["streaming"], ref_md[0], ref_md[1], ref_bd[0], ref_bd[1]))


def test_divergence_subwarp_shards(cadv):
    t = TRACES["rand_stores"]()
    cuts = snapped_cuts(t, 3, seed=1)
    out, err = run_ranks(cadv, t, cuts, lambda c: (c.mem_divergence(32, 8, t.nsites)[0],
                                                  c.branch_divergence(16, t.nsites)[1]))
    assert not any(err), err
    check_all_equal(out, (orc.mem_div(t, 32, 8)[0], orc.branch_div(t, 16)[1]))


def test_split_group_rejected(cadv):
    """A shard boundary inside a warp-level group: divergence is refused on
    every rank (BAD_TRACE), reuse distance is still exact."""
    t = TRACES["srad"]()
    gs = tg.group_starts(t.cols["cta"], t.cols["tid"], t.cols["winst"], t.cols["meta"])
    mid = int(np.flatnonzero(~gs[t.n // 2:])[0]) + t.n // 2  # inside a group
    cuts = [0, mid, t.n]

    def fn(c):
        with pytest.raises(cadv.CadvError) as e:
            c.mem_divergence(128, 32, t.nsites)
        assert e.value.status == cadv.CADV_ERR_BAD_TRACE
        return c.reuse_histogram(128, 0, 0, 66)

    out, err = run_ranks(cadv, t, cuts, fn)
    assert not any(err), err
    h_ref, _ = orc.reuse(t, 128, 0, 0, 66)
    for h, _ in out:
        assert (h == h_ref).all()


def test_bad_record_on_one_rank(cadv):
    """A bad record on rank 1 fails the call on every rank (no rank hangs)."""
    t = TRACES["rand_stores"]()
    cols = {k: v.copy() for k, v in t.cols.items()}
    cuts = snapped_cuts(t, 3, seed=5)
    cols["meta"][cuts[1] + 3] = 3
    t2 = tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t.nsites)

    def fn(c):
        with pytest.raises(cadv.CadvError) as e:
            c.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)
        return e.value.status

    out, err = run_ranks(cadv, t2, cuts, fn)
    assert not any(err), err
    assert all(s == cadv.CADV_ERR_BAD_TRACE for s in out), out


def test_nccl_single_rank_context(cadv):
    """The NCCL backend itself (dlopen, ncclCommInitRank, all-reduce,
    all-gather, grouped send/recv to self) on a one-rank communicator, which
    runs the whole multi-rank code path on this one GPU."""
    import torch
    t = TRACES["rand_stores"]()
    ctx = cadv.create(0, torch.cuda.current_stream().cuda_stream, nccl_id=cadv.nccl_unique_id(), rank=0, nranks=1)
    try:
        ctx.load_trace(cadv.to_device(t))
        o = ctx.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)
        h_ref, s_ref = orc.reuse(t, 128, 0, 0, 66)
        assert (o["reuse"][0] == h_ref).all() and o["reuse"][1] == s_ref
        assert (o["mem_div"][0] == orc.mem_div(t, 128, 32)[0]).all()
        assert (o["branch_div"][1] == orc.branch_div(t, 32)[1]).all()
        h, _ = ctx.reuse_histogram(32, 1, 1, 20)
        assert (h == orc.reuse(t, 32, 1, 1, 20)[0]).all()
    finally:
        ctx.destroy()


@pytest.mark.parametrize("scope", [0, 1])
def test_exchange_collective_baseline(cadv, monkeypatch, scope):
    """CADV_EXCHANGE=nccl: the kept-record exchange through the communicator's
    all-to-all (NCCL send / recv) instead of the peer-memory store kernel;
    same result."""
    monkeypatch.setenv("CADV_EXCHANGE", "nccl")
    t = TRACES["rand_bigcta"]()
    cuts = random_cuts(t.n, 3, seed=99)
    h_ref, s_ref = orc.reuse(t, 32, scope, 0, 66)
    out, err = run_ranks(cadv, t, cuts, lambda c: c.reuse_histogram(32, scope, 0, 66))
    assert not any(err), err
    for h, s in out:
        assert (h == h_ref).all() and s == s_ref


@pytest.mark.parametrize("name", ["srad", "rand_stores"])
@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("scope", [0, 1])
def test_data_centric_shards(cadv, name, G, scope):
    """Data-centric attribution (cadv_data_centric) on snapped shards: every
    rank returns the oracle's global per-object rows."""
    t = TRACES[name]()
    cuts = snapped_cuts(t, G, seed=3 * G + scope)
    if name == "srad":
        objs = tg.objects("srad", rows=128, cols=128, iters=2)
    else:
        base = int(t.addr[(t.meta & 3) != 2].min())
        objs = (np.array([base, base + 2048], np.uint64), np.array([1024, 1 << 20], np.uint64))
    ref = orc.data_centric(t, objs, 128, scope, 0, 66, 32)
    out, err = run_ranks(cadv, t, cuts, lambda c: c.data_centric(objs, 128, scope, 0, 66, 32))
    assert not any(err), err
    check_all_equal(out, ref)


@pytest.mark.parametrize("G", [2, 3, 4])
def test_kernel_scope_spread_cyclic(cadv, G):
    """Kernel scope over ranks keeps every kept record on its rank: K lines
    read cyclically R times (27,000 records, several tiles per rank) split at
    random positions; the cross-tile entries travel to rank 0.  Closed form:
    K at ∞ and K (R - 1) at distance K - 1, on every rank."""
    K, R = 9000, 3
    n = K * R
    addr = 0x7F0000000000 + 128 * (np.arange(n) % K)
    t = tg.from_arrays(addr, np.zeros(n), np.zeros(n), np.zeros(n), np.arange(n), np.full(n, 2 << 2), nsites=1)
    cuts = random_cuts(n, G, seed=40 + G, empty=(G == 4))
    out, err = run_ranks(cadv, t, cuts, lambda c: c.reuse_histogram(128, 1, 0, K + 3))
    assert not any(err), err
    for h, s in out:
        assert h[-1] == K and h[K - 1] == K * (R - 1) and h.sum() == n
        assert s["streaming"] == 0 and s["finite_sum"] == K * (R - 1) * (K - 1)


@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("seed", [0, 1])
def test_non_contiguous_shards(cadv, G, seed):
    """warp_contiguous = 0 on several ranks, unsnapped cuts (a warp-level
    group may lie on two ranks): every (cta, warp32) stream moves to one rank
    (exchange_by_warp), reuse distance keeps the trace order -- one fused call
    per rank equals the whole-trace oracle."""
    t = tg.generate("rand", seed=seed, ctas=8, threads=128, instrs=15, lines=30, pstore=0.3, pbb=0.3, scramble=1,
                    scramble_seed=seed)
    cuts = random_cuts(t.n, G, seed=seed + 11, empty=(G == 3))
    ref = (orc.reuse(t, 128, 0, 0, 66)[0], orc.mem_div(t, 128, 32)[0], orc.mem_div(t, 128, 32)[1],
           orc.branch_div(t, 32)[0], orc.branch_div(t, 32)[1], orc.mem_div(t, 32, 16)[0], orc.branch_div(t, 8)[1])

    def fn(c):
        o = c.analyze(rd=(128, 0, 0, 66), md=(128, 32), bd=32, nsites=t.nsites)
        m16, _ = c.mem_divergence(32, 16, t.nsites)
        _, b8 = c.branch_divergence(8, t.nsites)
        return o["reuse"][0], o["mem_div"][0], o["mem_div"][1], o["branch_div"][0], o["branch_div"][1], m16, b8

    out, err = run_ranks(cadv, t, cuts, fn, contiguous=False)
    assert not any(err), err
    check_all_equal(out, ref)


@pytest.mark.parametrize("G", [2, 3])
def test_cta_scope_segment_paths_per_rank(cadv, G):
    """CTA scope over ranks: after the CTA-range exchange each rank resolves its
    own CTA segments - segment kernel (<= 256 kept records), packed
    segment-list tiles (<= 4096) - unless one of its segments is longer, which
    sends that rank alone to the bounds-tiled path.  Short and medium CTAs
    first, long (5000-record) CTAs last, so the ranks take different paths."""
    rng = np.random.default_rng(G)
    lens = list(rng.integers(1, 257, 40)) + list(rng.integers(257, 4097, 8)) + [5000, 4096, 5000]
    addr, cta = [], []
    for c, n in enumerate(lens):
        lines = np.sort(rng.choice(1 << 20, max(2, int(n) // 3), replace=False)).astype(np.uint64)
        seq = rng.choice(lines, int(n))
        for k in range(1, int(n)):  # no two consecutive equal lines: every record is kept
            if seq[k] == seq[k - 1]:
                seq[k] = lines[(np.searchsorted(lines, seq[k]) + 1) % len(lines)]
        addr.append(0x7F0000000000 + 128 * seq)
        cta.append(np.full(int(n), c, dtype=np.uint64))
    addr, cta = np.concatenate(addr), np.concatenate(cta)
    n = len(addr)
    meta = np.where(rng.random(n) < 0.1, (2 << 2) | 1, 2 << 2)
    t = tg.from_arrays(addr, cta, rng.integers(0, 256, n), np.zeros(n), np.arange(n), meta, nsites=1)
    cuts = random_cuts(t.n, G, seed=11 * G)
    for binning, nb in ((0, 66), (1, 20)):
        h_ref, s_ref = orc.reuse(t, 128, 0, binning, nb)
        out, err = run_ranks(cadv, t, cuts, lambda c: c.reuse_histogram(128, 0, binning, nb))
        assert not any(err), err
        for h, s in out:
            assert (h == h_ref).all() and s == s_ref
