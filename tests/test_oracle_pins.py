"""Pins the CPU oracle to things other than itself (CPU only, no GPU).

Each pin cites the PAPER.md passage or the closed form it checks (DESIGN.md
"Oracle pins").  Chosen so that a plausible oracle mistake fails at least one:
  - dropped write rule / wrong epoch           -> write-rule cases, brute force
  - distinct *accesses* instead of elements    -> paper example, cyclic closed form
  - off-by-one window (inclusive bounds)       -> paper example (5, not 6)
  - addresses instead of lines (MD)            -> BICG/Syrk printed %, SGEMM closed form
  - 32 instead of launched lanes (BD)          -> vecAdd and NW closed forms
  - wrong binning index                        -> explicit bin-boundary cases
"""
import json
import math
import os

import numpy as np
import pytest

import oracle as orc
import tracegen as tg

LD, ST, BB = 0, 1, 2


def meta(kind, nbytes=4):
    return kind | (int(np.log2(nbytes)) << 2) if kind != BB else BB


def literal(seq, elem=4, cta=None):
    """Trace of single-thread 4-byte accesses; seq items 'X' load or 'X!' store."""
    names = {}
    addr, m = [], []
    for tok in seq:
        st = tok.endswith("!")
        key = tok.rstrip("!")
        names.setdefault(key, len(names))
        addr.append(0x7F0000000000 + names[key] * elem)
        m.append(meta(ST if st else LD, elem))
    n = len(addr)
    c = np.zeros(n, np.uint32) if cta is None else np.asarray(cta, np.uint32)
    return tg.from_arrays(addr, c, np.zeros(n), np.zeros(n), np.arange(n), m, nsites=1)


# ----------------------------------------------------------------- reuse distance

def test_paper_worked_example(golden_dir):
    """'ABCCDEFAAAB ... The reuse distance of B is 5.'"""
    g = json.load(open(os.path.join(golden_dir, "paper_rd_example.json")))
    t = literal(list(g["sequence"]))
    pos, want = g["printed"]["position"], g["printed"]["reuse_distance"]
    rd = orc.reuse_rd(t, line_bytes=4)
    assert g["sequence"][pos] == g["printed"]["element"]
    assert rd[pos] == want
    _, _, rdb = orc.reuse_brute(t, line_bytes=4)
    assert rdb[pos] == want
    # the rest of the sequence follows from the same definition: A@7 also sees
    # {B,C,D,E,F} -> 5; the C/A repeats are 0; first touches are ∞.
    assert list(rd) == [-1, -1, -1, 0, -1, -1, -1, 5, 0, 0, 5]
    h, st = orc.reuse(t, line_bytes=4, nbins=8)
    assert h[0] == 3 and h[5] == 2 and h[7] == 6 and h.sum() == 11
    # Eq. (1)'s average reuse distance over the finite distances: 10 / 5
    assert st["finite_sum"] == 10 and st["finite_sum"] / (st["accesses"] - st["inf"]) == 2.0


@pytest.mark.parametrize("K,R", [(1, 5), (3, 4), (7, 3), (40, 2), (130, 3)])
def test_cyclic_closed_form(K, R):
    """Textbook LRU case: K distinct lines read cyclically R times ->
    K first touches (∞) and K(R-1) reuses at distance K-1."""
    t = literal([f"x{k}" for _ in range(R) for k in range(K)])
    h, st = orc.reuse(t, line_bytes=4, nbins=K + 3)
    assert h[-1] == K
    assert h[K - 1] == K * (R - 1)
    assert h.sum() == K * R
    assert st["streaming"] == (K if R == 1 else 0)
    assert st["finite_sum"] == K * (R - 1) * (K - 1)


def test_write_rule_restarts_counting():
    """once A is written it is counted as another address A';
    L252: ∞ = never reused or not reused before the next write."""
    rd = orc.reuse_rd(literal(["A", "A!", "A"]), line_bytes=4)
    assert list(rd) == [-1, -1, 0]          # the store is A' (first access), the load reuses A'
    rd = orc.reuse_rd(literal(["B", "A", "A!", "A", "B"]), line_bytes=4)
    # B@4 sees A (old) and A' (new) between its uses: two distinct elements
    assert list(rd) == [-1, -1, -1, 0, 2]
    rd = orc.reuse_rd(literal(["A", "B", "A!", "A", "B"]), line_bytes=4)
    # here the old A precedes B@1, so only A' lies between the two uses of B
    assert list(rd) == [-1, -1, -1, 0, 1]
    rd = orc.reuse_rd(literal(["A", "A", "A!", "A!", "B", "A"]), line_bytes=4)
    assert list(rd) == [-1, 0, -1, -1, -1, 1]


def test_line_model_vs_element_model():
    """element-based and line-based models; two 4-byte elements
    of one 128 B line are one line but two elements."""
    t = literal(["a", "b", "a"])  # a and b are 4 bytes apart
    assert list(orc.reuse_rd(t, line_bytes=4)) == [-1, -1, 1]
    assert list(orc.reuse_rd(t, line_bytes=128)) == [-1, 0, 0]


def test_binning_boundaries():
    """LINEAR: bins 0..B-3 exact, B-2 overflow, B-1 ∞.  LOG2: bin k = [2^(k-1), 2^k-1]."""
    for d in range(0, 20):
        seq = ["A"] + [f"x{k}" for k in range(d)] + ["A"]
        t = literal(seq)
        h, st = orc.reuse(t, line_bytes=4, nbins=8)
        assert h[min(d, 6)] == 1 and h[7] == d + 1
        assert st["overflow"] == (1 if d >= 6 else 0)
        h, _ = orc.reuse(t, line_bytes=4, binning=orc.BINS_LOG2, nbins=6)
        k = 0 if d == 0 else int(d).bit_length()
        assert h[k if k <= 3 else 4] == 1


def _rand_literal(rng, n, ncta, nelem, pstore):
    seq = [f"e{rng.integers(nelem)}" + ("!" if rng.random() < pstore else "") for _ in range(n)]
    return literal(seq, cta=rng.integers(ncta, size=n))


@pytest.mark.parametrize("seed", range(40))
def test_lru_equals_brute_force_random(seed):
    """LRU-stack oracle == literal O(n^2) definition on random tiny traces,
    with stores, in both scopes and both binnings."""
    rng = np.random.default_rng(seed)
    t = _rand_literal(rng, int(rng.integers(1, 120)), int(rng.integers(1, 4)), int(rng.integers(1, 12)),
                      float(rng.choice([0.0, 0.1, 0.3])))
    for scope in (orc.SCOPE_CTA, orc.SCOPE_KERNEL):
        for binning, nbins in ((orc.BINS_LINEAR, 9), (orc.BINS_LOG2, 5)):
            for lb in (4, 8):
                h1, s1 = orc.reuse(t, lb, scope, binning, nbins)
                h2, s2, rd2 = orc.reuse_brute(t, lb, scope, binning, nbins)
                assert (h1 == h2).all() and s1 == s2
                assert (orc.reuse_rd(t, lb, scope) == rd2).all()


@pytest.mark.parametrize("seed", range(12))
def test_lru_equals_brute_force_generated(seed):
    """Same equivalence on generator traces with warps, masks, mixed widths and BB records."""
    t = tg.generate("rand", ctas=2, threads=40, instrs=3, lines=4, seed=seed, pstore=0.25)
    for lb in (1, 32, 128):
        for scope in (orc.SCOPE_CTA, orc.SCOPE_KERNEL):
            h1, s1 = orc.reuse(t, lb, scope)
            h2, s2, _ = orc.reuse_brute(t, lb, scope)
            assert (h1 == h2).all() and s1 == s2


def test_reuse_invariants_generated():
    """(i) histogram mass = #memory records (north_star); (ii) ∞ = #stores +
    #first accesses of (scope, line) epochs; store-free: ∞ = #distinct
    (scope, line) ("cold misses equal the distinct-line count"); (vi) streaming <= ∞."""
    t = tg.generate("rand", ctas=5, threads=96, instrs=20, lines=50, seed=3, pstore=0.0)
    mem = (t.meta & 3) != BB
    for lb in (4, 32, 128):
        h, st = orc.reuse(t, lb)
        assert h.sum() == mem.sum() == st["accesses"]
        distinct = len(set(zip(t.cta[mem].tolist(), (t.addr[mem] // lb).tolist())))
        assert st["inf"] == distinct
        assert st["streaming"] <= st["inf"]
    t = tg.generate("rand", ctas=5, threads=96, instrs=20, lines=50, seed=4, pstore=0.3)
    h, st = orc.reuse(t, 32)
    assert h.sum() == ((t.meta & 3) != BB).sum()
    assert st["inf"] >= ((t.meta & 3) == ST).sum()


def test_cta_scope_invariant_to_interleaving():
    """CTA scope depends only on each CTA's own order (P:L237 regroup by CTA)."""
    t = tg.generate("rand", ctas=6, threads=64, instrs=12, lines=20, seed=9)
    rng = np.random.default_rng(0)
    # random merge of the per-CTA streams
    keys = rng.random(t.n)
    order = np.empty(t.n, np.int64)
    for c in np.unique(t.cta):
        idx = np.nonzero(t.cta == c)[0]
        keys[idx] = np.sort(keys[idx])
    order = np.argsort(keys, kind="stable")
    t2 = tg.from_arrays(*(t.cols[k][order] for k, _ in tg.COLUMNS), nsites=t.nsites)
    for lb in (32, 128):
        assert (orc.reuse(t, lb)[0] == orc.reuse(t2, lb)[0]).all()


def test_coarser_lines_shift_cdf_left_store_free():
    """Without stores, a coarser line never increases a reuse distance, so the
    CDF at 2L dominates the one at L (element model <= line model)."""
    t = tg.generate("rand", ctas=3, threads=64, instrs=30, lines=40, seed=5, pstore=0.0)
    prev = None
    for lb in (1, 4, 16, 64, 256):
        h, _ = orc.reuse(t, lb, nbins=200)
        cdf = np.cumsum(h[:-1])
        if prev is not None:
            assert (cdf >= prev).all()
        prev = cdf


def test_vecadd_reuse_closed_form():
    """Config 1 (vecAdd, 683 fp32, 64 threads): every 128 B line of a/b is
    touched by one warp-instruction whose lanes are adjacent -> 1 ∞ + RD 0 for
    the rest; each store is a fresh element.  128 B: ∞ = 683 + 2*22, 32 B:
    ∞ = 683 + 2*86 (ceil(683/32) = 22, ceil(683/8) = 86)."""
    t = tg.generate("vecadd")
    h, st = orc.reuse(t, 128)
    assert h[0] == 1366 - 44 and h[-1] == 683 + 44 and h.sum() == 2049
    h, st = orc.reuse(t, 32)
    assert h[0] == 1366 - 172 and h[-1] == 683 + 172


# ----------------------------------------------------------------- memory divergence

def _pct(hist):
    pooled = hist.sum(axis=0).astype(np.float64)
    return 100.0 * pooled / pooled.sum()


def test_polybench_md_printed(golden_dir):
    """printed BICG / Syrk / Syr2k memory-divergence shares."""
    g = json.load(open(os.path.join(golden_dir, "paper_md_polybench.json")))
    traces = {"bicg": tg.generate("bicg", nx=1024, ny=1024),
              "syrk": tg.generate("syrk", ni=8, nj=32, m=1024),
              "syr2k": tg.generate("syr2k", ni=8, nj=32, m=1024)}
    for row in g["rows"]:
        hist, _ = orc.mem_div(traces[row["app"]], line_bytes=row["line_bytes"])
        pct = _pct(hist)
        for k, v in row["printed"].items():
            assert round(pct[int(k)], row["decimals"]) == pytest.approx(v), (row, pct[int(k)])


def test_coalescing_bound_printed():
    """a bool/float warp access touches one 128 B line and up to
    four 32 B lines when fully coalesced."""
    for nbytes, want32 in ((4, 4), (1, 1)):
        base = 0x7F0000001000
        addr = [base + l * nbytes for l in range(32)]
        t = tg.from_arrays(addr, np.zeros(32), np.arange(32), np.zeros(32), np.zeros(32),
                           [meta(LD, nbytes)] * 32, nsites=1)
        h128, _ = orc.mem_div(t, 128)
        h32, _ = orc.mem_div(t, 32)
        assert h128[0, 1] == 1 and h32[0, want32] == 1


def test_sgemm_md_closed_form():
    """Config 2, SGEMM 256^3, warp = 2 rows x 16 cols: naive ld A -> 2 lines,
    ld B -> 1 (128 B) / 2 (32 B), st C -> 2 / 4; tiled A, B, C -> 2 / 4."""
    t = tg.generate("sgemm", n=256)
    h, ps = orc.mem_div(t, 128)
    pooled = h.sum(axis=0)
    assert pooled[1] == 524288 and pooled[2] == 526336 + 67584 and pooled.sum() == 524288 + 526336 + 67584
    h, _ = orc.mem_div(t, 32)
    pooled = h.sum(axis=0)
    assert pooled[2] == 1048576 and pooled[4] == 2048 + 67584 and pooled.sum() == 1048576 + 2048 + 67584


def test_vecadd_md_closed_form():
    t = tg.generate("vecadd")
    h, ps = orc.mem_div(t, 128)
    assert h[0, 1] == 44 and h[1, 1] == 22 and h.sum() == 66
    h, ps = orc.mem_div(t, 32)
    assert h.sum(axis=0)[4] == 63 and h.sum(axis=0)[2] == 3
    assert ps[:, 0].sum() == 66


def test_md_invariants_generated():
    t = tg.generate("rand", ctas=4, threads=128, instrs=40, lines=30, seed=11)
    mem = (t.meta & 3) != BB
    ngroups = len(set(zip(t.cta[mem].tolist(), (t.tid[mem] // 32).tolist(), t.winst[mem].tolist())))
    prev = None
    for lb in (1, 8, 32, 128, 4096):
        h, ps = orc.mem_div(t, lb)
        assert h.sum() == ngroups == ps[:, 0].sum()
        assert h[:, 0].sum() == 0
        k = np.arange(33)
        assert (h * k).sum() == ps[:, 1].sum()
        mean = (h * k).sum() / h.sum()
        if prev is not None:
            assert mean <= prev      # coarser lines never touch more lines
        prev = mean
    for W in (1, 2, 4, 8, 16, 32):
        h, _ = orc.mem_div(t, 32, warp_size=W)
        assert h.shape == (2, W + 1) and h[:, 0].sum() == 0
        if W == 1:
            assert h[:, 1].sum() == mem.sum()


def test_md_degree_weighted_average():
    """degree = average of the weighted sum of the distribution."""
    h = np.zeros((2, 33), np.uint64)
    h[0, 1] = 3
    h[1, 32] = 1
    assert orc.md_degree(h) == pytest.approx((3 * 1 + 32) / 4)


# ----------------------------------------------------------------- branch divergence

def test_table3_percent_arithmetic(golden_dir):
    """PAPER.md Table 3: % divergence = 100 * divergent / total (all rows)."""
    g = json.load(open(os.path.join(golden_dir, "paper_table3.json")))
    for app, div, tot, pct in g["rows"]:
        assert round(100.0 * div / tot, 2) == pytest.approx(pct), app


def test_vecadd_bd_closed_form():
    """vecAdd BB trace: entry, header, body, exit; warp 1's last header and body
    have 11 of 32 lanes -> 2 divergent of 50 warp-level block executions."""
    t = tg.generate("vecadd")
    ps, tot = orc.branch_div(t)
    assert list(tot) == [50, 2, 1558]
    assert list(ps[1]) == [24, 1, 747] and list(ps[2]) == [22, 1, 683]
    assert list(ps[0]) == [2, 0, 64] and list(ps[3]) == [2, 0, 64]


def test_nw_bd_closed_form():
    """NW-shaped 16-thread CTA (1 warp, 16 launched lanes; Table 2 'nw: 1
    warp/CTA'): divergent = 'if (tx == 0)' + 15 + 15 'if (tx <= m)' blocks
    = 31 of 165 executions per CTA.  With 32 as the reference lane count every
    execution would be divergent (165/165)."""
    for ctas in (1, 3):
        t = tg.generate("nw", ctas=ctas)
        ps, tot = orc.branch_div(t)
        assert tot[0] == 165 * ctas and tot[1] == 31 * ctas
        assert tot[2] == ((t.meta & 3) == BB).sum()


def test_uniform_kernel_has_no_divergence():
    """Uniform control flow -> 0 divergent blocks (Table 3 bicg/syrk rows)."""
    t = tg.generate("sgemm", n=32, bb=1)
    ps, tot = orc.branch_div(t)
    assert tot[1] == 0 and tot[0] > 0


def test_bd_invariants_generated():
    t = tg.generate("rand", ctas=5, threads=100, instrs=30, seed=13, pbb=0.6)
    bbm = (t.meta & 3) == BB
    for W in (4, 8, 32):
        ps, tot = orc.branch_div(t, warp_size=W)
        assert tot[1] <= tot[0]
        assert tot[2] == bbm.sum()
        assert (ps.sum(axis=0) == tot).all()


# ----------------------------------------------------------------- validation

def test_bad_trace_rejected():
    t = literal(["A", "B"])
    t.cols["meta"][1] = 3          # kind 3 does not exist
    with pytest.raises(orc.OracleError) as e:
        orc.reuse(t, 4)
    assert e.value.code == 2
    t = literal(["A", "B"])
    t.cols["addr"][0] += 2         # misaligned 4-byte access
    with pytest.raises(orc.OracleError):
        orc.mem_div(t, 32)
    with pytest.raises(orc.OracleError) as e:
        orc.reuse(literal(["A"]), line_bytes=48)
    assert e.value.code == 1


def test_kernel_scope_properties_match_oracle():
    """The size-free properties used by the full-size GPU tests (mass, ∞ =
    first use of every renamed element, streaming = elements used once)
    equal the LRU oracle's on random traces with stores, both line models."""
    from props import kernel_scope_properties
    for seed in range(4):
        t = tg.generate("rand", seed=seed, ctas=4, threads=64, instrs=20, lines=30, pstore=0.3)
        for lb in (1, 4, 128):
            for scope in (1,):
                h, s = orc.reuse(t, lb, scope, 0, 40)
                assert kernel_scope_properties(t, lb) == (int(h.sum()), int(h[-1]), s["streaming"])


def test_eq1_bypass_warps_arithmetic():
    """PAPER.md L363 Eq. (1): floor(L1 / (R.D. * line * M.D. * CTAs/SM)),
    with R.D. and M.D. from the analyses' outputs (here the oracle's)."""
    from paper_conf_cgo_shensll18_b200 import metrics as M
    assert M.opt_num_warps(16 * 1024, 2.0, 128, 2.0, 1) == 32
    assert M.opt_num_warps(48 * 1024, 3.0, 128, 4.0, 2) == 16
    assert M.opt_num_warps(24 * 1024, 0.0, 128, 2.0, 1) == -1
    t = literal(list("ABCCDEFAAAB"))
    _, st = orc.reuse(t, line_bytes=4, nbins=8)
    assert M.mean_reuse_distance(st) == 2.0
    h = np.zeros((2, 33), np.uint64)
    h[0, 1] = 3
    h[1, 32] = 1
    assert M.md_degree(h) == pytest.approx(orc.md_degree(h)) == pytest.approx(35 / 4)
    s = M.instance_stats([1.0, 2.0, 3.0, 6.0])
    assert s["mean"] == 3.0 and s["min"] == 1.0 and s["max"] == 6.0 and s["stddev"] == pytest.approx(math.sqrt(3.5))


# ----------------------------------------------------------------- data-centric attribution (NEXT-3)
# each access is associated with the data object whose range
# holds its effective address; reading R18 fixes line granularity.

def _brute_rd_py(t, L, scope):
    """Literal P:L248 in pure Python loops (tiny traces): distinct renamed
    elements strictly between an access and the previous use of its element."""
    n = t.n
    key = [None] * n
    for i in range(n):
        if (int(t.meta[i]) & 3) == BB:
            continue
        s = int(t.cta[i]) if scope == orc.SCOPE_CTA else 0
        line = int(t.addr[i]) // L
        stores = sum(1 for j in range(i + 1) if (int(t.meta[j]) & 3) == ST and key_line(t, j, L, scope) == (s, line))
        key[i] = (s, line, stores)
    rd = [None] * n
    for i in range(n):
        if key[i] is None:
            continue
        rd[i] = -1
        if (int(t.meta[i]) & 3) == LD:
            for j in range(i - 1, -1, -1):
                if key[j] == key[i]:
                    rd[i] = len({key[m] for m in range(j + 1, i) if key[m] is not None and key[m][0] == key[i][0]})
                    break
    return rd


def key_line(t, j, L, scope):
    return (int(t.cta[j]) if scope == orc.SCOPE_CTA else 0, int(t.addr[j]) // L)


def _row_py(line, L, objs):
    lo, hi = line * L, line * L + L
    for k, (b, nb) in enumerate(zip(*objs)):
        if lo < int(b) + int(nb) and int(b) < hi:
            return k
    return len(objs[0])


def _bin_py(d, nbins):
    return nbins - 1 if d < 0 else min(d, nbins - 2)


@pytest.mark.parametrize("L", [128, 32])
def test_data_centric_vecadd_closed_form(L):
    """vecAdd (C1): c[i] = a[i] + b[i], N = 683 fp32, arrays 4 KiB aligned.
    Per object: a and b are read once per element, so each of their
    ceil(4N / L) lines is first touched once (∞) and every other load is a
    reuse at distance 0; every store to c opens a new element (∞).
    MD: every warp instruction touches one object; 22 per array, all
    coalesced (1 line at 128 B; at 32 B 4 lines, the 11-lane tail 2 lines)."""
    N = 683
    t = tg.generate("vecadd")
    objs = tg.objects("vecadd")
    assert len(objs[0]) == 3 and all(int(b) % 4096 == 0 for b in objs[0])
    rh, mh = orc.data_centric(t, objs, L, nbins=66)
    lines = -(-4 * N // L)
    for k in (0, 1):
        assert rh[k, 0] == N - lines and rh[k, 65] == lines and rh[k].sum() == N
    assert rh[2, 65] == N and rh[2].sum() == N
    assert rh[3].sum() == 0
    for k, kind in ((0, LD), (1, LD), (2, ST)):
        row = mh[k, kind]
        if L == 128:
            assert row[1] == 22 and row.sum() == 22
        else:
            assert row[4] == 21 and row[2] == 1 and row.sum() == 22
        assert mh[k, 1 - kind].sum() == 0


@pytest.mark.parametrize("seed", range(10))
def test_data_centric_equals_python_brute_force(seed):
    """Per-object RD and MD vs a pure-Python literal computation on tiny
    random traces, with random object tables (gaps, unattributed lines)."""
    rng = np.random.default_rng(1000 + seed)
    L = int(rng.choice([1, 4, 16, 32, 128]))
    scope = int(rng.integers(0, 2))
    n = int(rng.integers(20, 120))
    ncta = int(rng.integers(1, 4))
    nelem = int(rng.integers(2, 40))
    base0 = 0x7F0000000000
    addr = base0 + 4 * rng.integers(0, nelem, n)
    kinds = np.where(rng.random(n) < 0.25, ST, LD)
    cta = rng.integers(0, ncta, n)
    tid = rng.integers(0, 64, n)
    # winst per (cta, warp): every record its own warp instruction, except a few shared
    t = tg.from_arrays(addr, cta, tid, np.zeros(n), np.arange(n), [meta(k) for k in kinds], nsites=1)
    # object table: random line-disjoint ranges over [base0, base0 + 4 nelem),
    # each trimmed inside its first / last line (so partial lines occur)
    nlines = 4 * nelem // L + 2
    cuts = sorted(set(int(x) for x in rng.integers(0, nlines, 6)))
    objs_b, objs_n = [], []
    for a, b in zip(cuts[::2], cuts[1::2]):
        lo = base0 + a * L + int(rng.integers(0, max(1, L // 2)))
        hi = base0 + b * L - int(rng.integers(0, max(1, L // 2)))
        if hi > lo and (not objs_b or (objs_b[-1] + objs_n[-1] - 1) // L < lo // L):
            objs_b.append(lo)
            objs_n.append(hi - lo)
    assert seed % 5 or objs_b  # most seeds have objects (checked on a subset)
    objs = (np.array(objs_b, np.uint64), np.array(objs_n, np.uint64))
    nb = 10
    rh, mh = orc.data_centric(t, objs, L, scope=scope, nbins=nb, warp_size=32)
    rd = _brute_rd_py(t, L, scope)
    want = np.zeros((len(objs_b) + 1, nb), np.uint64)
    for i in range(n):
        want[_row_py(int(addr[i]) // L, L, objs), _bin_py(rd[i], nb)] += 1
    assert (rh == want).all()
    # MD: every record is its own group (distinct winst) -> degree 1 in its object's row
    wm = np.zeros((len(objs_b) + 1, 2, 33), np.uint64)
    for i in range(n):
        wm[_row_py(int(addr[i]) // L, L, objs), kinds[i], 1] += 1
    assert (mh == wm).all()


def test_data_centric_rows_partition_the_analyses():
    """Rows partition the whole-trace histograms (every access / group lands
    in exactly one row), on a generated trace with stores, both scopes."""
    t = tg.generate("rand", seed=3, ctas=5, threads=128, instrs=30, lines=200, pstore=0.2, pbb=0.2)
    base = int(t.addr[(t.meta & 3) != BB].min()) // 4096 * 4096
    objs = (np.array([base, base + 8192, base + 40960], np.uint64), np.array([4096, 8192, 1 << 20], np.uint64))
    for L, scope in ((128, 0), (32, 1), (4, 0)):
        rh, mh = orc.data_centric(t, objs, L, scope=scope, nbins=40)
        h, _ = orc.reuse(t, L, scope, 0, 40)
        assert (rh.sum(axis=0) == h).all()
        hm, _ = orc.mem_div(t, L, 32)
        assert (mh.sum(axis=0) == hm).all()
    # no objects: everything is unattributed
    rh, mh = orc.data_centric(t, (np.zeros(0, np.uint64), np.zeros(0, np.uint64)), 128, nbins=40)
    assert rh.shape == (1, 40) and (rh[0] == orc.reuse(t, 128, 0, 0, 40)[0]).all()


def test_data_centric_rejects_bad_tables():
    t = tg.generate("vecadd")
    b = 0x7F0000000000
    bad = [
        ([b, b + 64], [64, 64]),       # both objects share line b at 128 B
        ([b + 4096, b], [64, 64]),     # not ascending
        ([b], [0]),                    # empty object
    ]
    for base, nb in bad:
        with pytest.raises(orc.OracleError):
            orc.data_centric(t, (np.array(base, np.uint64), np.array(nb, np.uint64)), 128)
    # the same pair is fine at 64 B lines (no line intersects both)
    orc.data_centric(t, (np.array([b, b + 64], np.uint64), np.array([64, 64], np.uint64)), 64)


# ----------------------------------------------------------------- round 2 pins

def test_vecadd_md_per_site_closed_form():
    """Config 1 per site (P:L264 per instruction): each of ld a / ld b / st c
    is 22 warp-level instructions (683 = 10*64 + 43: warp 0 runs 11 full
    iterations, warp 1 runs 11, the last with 11 lanes); a full group covers
    128 contiguous bytes = 1 line at 128 B, 4 at 32 B; the 11-lane group
    covers bytes 2688..2731 = 1 line at 128 B, 2 at 32 B ->
    {22, 22} at 128 B and {22, 21*4 + 2 = 86} at 32 B."""
    t = tg.generate("vecadd")
    _, ps = orc.mem_div(t, 128)
    mem_sites = sorted(set(t.site[(t.meta & 3) != BB].tolist()))
    assert len(mem_sites) == 3
    for s in mem_sites:
        assert list(ps[s]) == [22, 22]
    _, ps = orc.mem_div(t, 32)
    for s in mem_sites:
        assert list(ps[s]) == [22, 86]
    assert ps.sum(axis=0).tolist() == [66, 258]


def test_sgemm_md_per_site_closed_form():
    """Config 2 per site: naive ld A[row*N+k] (2 rows, one k -> 2 lines at any
    L), ld B[k*N+col] (16 consecutive floats = 64 B, 64-B aligned -> 1 line at
    128 B, 2 at 32 B), st C (2 rows x 64 B -> 2 / 4); 256 CTAs x 8 warps x 256
    iterations = 524,288 groups per loop site, 2,048 per store; tiled: 16 tile
    steps -> 32,768 groups per tile load, each 2 rows x 64 B -> 2 / 4 lines."""
    t = tg.generate("sgemm", n=256)
    _, p128 = orc.mem_div(t, 128)
    _, p32 = orc.mem_div(t, 32)
    rows128 = [tuple(r) for r in p128.tolist() if r[0]]
    rows32 = [tuple(r) for r in p32.tolist() if r[0]]
    assert rows128 == [(524288, 1048576), (524288, 524288), (2048, 4096), (32768, 65536), (32768, 65536), (2048, 4096)]
    assert rows32 == [(524288, 1048576), (524288, 1048576), (2048, 8192), (32768, 131072), (32768, 131072), (2048, 8192)]


def test_address_domain_is_the_full_u64():
    """P:L242 records an i8* effective address: no upper limit.  Shifting every
    address by a multiple of the line size (here into [2^62, 2^64)) relabels
    lines one-to-one, so every analysis must give the same result."""
    t = tg.generate("rand", seed=5, ctas=3, threads=64, instrs=20, lines=30, pstore=0.3)
    for shift in (np.uint64(1 << 58), np.uint64(0xC000000000000000)):
        cols = {k: v.copy() for k, v in t.cols.items()}
        mem = (cols["meta"] & 3) != BB
        cols["addr"][mem] = cols["addr"][mem] + shift
        t2 = tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=t.nsites)
        for lb in (1, 128):
            for sc in (0, 1):
                a, b = orc.reuse(t, lb, sc), orc.reuse(t2, lb, sc)
                assert (a[0] == b[0]).all() and a[1] == b[1]
                f = orc.reuse_fenwick(t2, lb, sc)
                assert (a[0] == f[0]).all() and a[1] == f[1]
            assert all((x == y).all() for x, y in zip(orc.mem_div(t, lb), orc.mem_div(t2, lb)))


def _group_trace(sites, kinds, tids=None):
    n = len(sites)
    tids = np.arange(n) if tids is None else np.asarray(tids)
    addr = 0x7F0000000000 + 4 * np.arange(n)
    return tg.from_arrays(addr, np.zeros(n), tids, np.asarray(sites), np.zeros(n),
                          [meta(k) for k in kinds], nsites=max(sites) + 1)


def test_group_invariant_enforced():
    """A dynamic warp-level instruction comes from one static instruction
    (P:L235 Record() per instrumented load/store, P:L345 passBasicBlock() per
    block): the records of one (cta, tid/32, winst) group share kind and
    site; a group that mixes them is a malformed trace (BAD_TRACE), also when
    the analysis warp size splits the warp (the group is the warp32's)."""
    ok = _group_trace([3] * 8, [LD] * 8)
    orc.mem_div(ok, 128)
    for bad in (_group_trace([3] * 7 + [4], [LD] * 8), _group_trace([3] * 8, [LD] * 7 + [ST])):
        for W in (32, 4):
            with pytest.raises(orc.OracleError) as e:
                orc.mem_div(bad, 128, W)
            assert e.value.code == 2
        orc.reuse(bad, 128)           # reuse distance does not read the group columns
    bb = _group_trace([1] * 5 + [2] * 3, [BB] * 8)
    with pytest.raises(orc.OracleError) as e:
        orc.branch_div(bb)
    assert e.value.code == 2
    # the two half-warps of one winst are still one warp32 instruction
    with pytest.raises(orc.OracleError):
        orc.branch_div(_group_trace([1] * 16 + [2] * 16, [BB] * 32), warp_size=16)
    # different warps (tid / 32) are different groups: no constraint between them
    orc.branch_div(_group_trace([1] * 4 + [2] * 4, [BB] * 8, tids=[0, 1, 2, 3, 32, 33, 34, 35]))


@pytest.mark.parametrize("seed", range(6))
def test_fenwick_equals_brute_force(seed):
    """The Fenwick variant against the literal O(n^2) definition on
    random traces with stores, both scopes, both binnings."""
    t = tg.generate("rand", seed=100 + seed, ctas=3, threads=40, instrs=12, lines=12, pstore=0.3)
    for lb in (1, 32, 128):
        for sc in (0, 1):
            for b, nb in ((0, 40), (1, 8)):
                hb, sb, _ = orc.reuse_brute(t, lb, sc, b, nb)
                hf, sf = orc.reuse_fenwick(t, lb, sc, b, nb)
                assert (hb == hf).all() and sb == sf, (seed, lb, sc, b)


def test_fenwick_pins():
    """The paper example (RD(B) = 5) and the cyclic closed form."""
    t = literal(list("ABCCDEFAAAB"))
    h, st = orc.reuse_fenwick(t, line_bytes=4, nbins=8)
    assert list(h) == [3, 0, 0, 0, 0, 2, 0, 6] and st["finite_sum"] == 10
    K, R = 130, 3
    h, st = orc.reuse_fenwick(literal([f"x{k}" for _ in range(R) for k in range(K)]), line_bytes=4, nbins=K + 3)
    assert h[-1] == K and h[K - 1] == K * (R - 1) and st["finite_sum"] == K * (R - 1) * (K - 1)


@pytest.mark.parametrize("name,kw", [("vecadd", {}), ("sgemm", dict(n=64, bb=1)), ("bfs", dict(nodes=8000, seed=42)),
                                     ("srad", dict(rows=128, cols=128, iters=2)), ("backprop", {"in": 2048})])
def test_fenwick_equals_lru_on_configs(name, kw):
    """the Fenwick variant is cross-checked == LRU on C1-C4
    (C1 at full size, C2-C4 shapes at reduced size), both scopes."""
    t = tg.generate(name, **kw)
    for lb in (32, 128):
        for sc in (0, 1):
            a, f = orc.reuse(t, lb, sc), orc.reuse_fenwick(t, lb, sc)
            assert (a[0] == f[0]).all() and a[1] == f[1], (name, lb, sc)
