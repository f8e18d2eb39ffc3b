"""Seeded synthetic trace generator (shared input module).

Holds no analysis arithmetic: it only emits the records an instrumented
kernel would produce (PAPER.md L235-237 Record(), L322/L345 passBasicBlock()).
Both the oracle side and the CUDA side of the tests and of bench.py read the
arrays it produces.  See tracegen.cpp for the record layout and the virtual
scheduler, DESIGN.md "Input recipe" for the workloads.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libtracegen.so")
_lib = None

COLUMNS = (("addr", np.uint64), ("cta", np.uint32), ("tid", np.uint16),
           ("site", np.uint32), ("winst", np.uint32), ("meta", np.uint8))

KIND_LOAD, KIND_STORE, KIND_BB = 0, 1, 2


def _load():
    global _lib
    if _lib is not None:
        return _lib
    src = os.path.join(_HERE, "tracegen.cpp")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["/usr/bin/g++" if os.path.exists("/usr/bin/g++") else "g++", "-O2", "-std=c++17", "-fopenmp", "-shared", "-fPIC",
                               "-o", _SO, src])
    lib = ctypes.CDLL(_SO)
    P, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
    lib.tg_plan.restype = P
    lib.tg_plan.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.c_char_p, ctypes.c_int]
    for fn, rt in (("tg_num_records", u64), ("tg_num_sites", u32), ("tg_num_ctas", u32),
                   ("tg_num_launches", u32), ("tg_info", ctypes.c_char_p)):
        getattr(lib, fn).restype = rt
        getattr(lib, fn).argtypes = [P]
    lib.tg_fill_range.restype = ctypes.c_int
    lib.tg_fill_range.argtypes = [P, u64, u64] + [P] * 6
    lib.tg_launch_offsets.restype = None
    lib.tg_launch_offsets.argtypes = [P, P]
    lib.tg_free.restype = None
    lib.tg_free.argtypes = [P]
    lib.tg_objects.restype = u32
    lib.tg_objects.argtypes = [P, P, P]
    _lib = lib
    return lib


@dataclass
class Trace:
    """One synthetic trace (or one position-range shard of it), SoA columns."""
    workload: str
    params: dict
    n: int                      # records in this object
    n_total: int                # records in the whole trace
    nsites: int
    nctas: int
    nlaunches: int
    info: str
    lo: int = 0                 # first global position held here
    cols: dict = field(default_factory=dict)

    def __getattr__(self, k):
        cols = self.__dict__.get("cols", {})
        if k in cols:
            return cols[k]
        raise AttributeError(k)

    def nbytes(self) -> int:
        return sum(a.nbytes for a in self.cols.values())


def _param_str(params: dict) -> str:
    return ",".join(f"{k}={v}" for k, v in params.items())


def plan(workload: str, **params):
    """Returns (handle, n_total, nsites, nctas, nlaunches, info) without generating."""
    lib = _load()
    err = ctypes.create_string_buffer(256)
    h = lib.tg_plan(workload.encode(), _param_str(params).encode(), err, 256)
    if not h:
        raise ValueError(err.value.decode())
    return (h, int(lib.tg_num_records(h)), int(lib.tg_num_sites(h)), int(lib.tg_num_ctas(h)),
            int(lib.tg_num_launches(h)), lib.tg_info(h).decode())


def launch_offsets(workload: str, **params) -> np.ndarray:
    """Start position of every kernel launch in the trace, plus the total."""
    lib = _load()
    h, n_total, nsites, nctas, nl, info = plan(workload, **params)
    try:
        out = np.zeros(nl + 1, np.uint64)
        lib.tg_launch_offsets(h, out.ctypes.data)
        return out
    finally:
        lib.tg_free(h)


def objects(workload: str, **params):
    """The workload's data objects (its allocated arrays): (base, bytes) as
    two uint64 arrays, ascending base (the allocation map of P:L131; input
    description, not analysis arithmetic)."""
    lib = _load()
    h, *_ = plan(workload, **params)
    try:
        k = int(lib.tg_objects(h, None, None))
        base, nbytes = np.zeros(k, np.uint64), np.zeros(k, np.uint64)
        if k:
            lib.tg_objects(h, base.ctypes.data, nbytes.ctypes.data)
        return base, nbytes
    finally:
        lib.tg_free(h)


def shard_bounds(workload: str, rank: int, world: int, **params):
    """[lo, hi) of this rank's shard: launch-aligned position ranges of about
    equal size (no CTA spans two shards: CTAs never span launches)."""
    off = launch_offsets(workload, **params).astype(np.int64)
    n = int(off[-1])
    cut = [0]
    for r in range(1, world):
        target = r * n // world
        k = int(np.argmin(np.abs(off - target)))
        cut.append(max(cut[-1], int(off[k])))
    cut.append(n)
    return cut[rank], cut[rank + 1]


def group_starts(cta, tid, winst, meta) -> np.ndarray:
    """Boolean mask of records that start a warp-level group run: the first
    record, or one whose (cta, tid // 32, winst, BB-or-memory) differs from
    its predecessor's.  Sharding plumbing (where a position split may fall
    without cutting a group), not analysis arithmetic."""
    n = len(cta)
    m = np.ones(n, dtype=bool)
    if n > 1:
        fam = (np.asarray(meta) & 3) == 2
        w = np.asarray(tid).astype(np.uint32) >> 5
        m[1:] = ((cta[1:] != cta[:-1]) | (w[1:] != w[:-1]) | (winst[1:] != winst[:-1]) | (fam[1:] != fam[:-1]))
    return m


def snap_cuts(cols, cuts):
    """Moves every interior cut point forward to the next group start."""
    gs = group_starts(cols["cta"], cols["tid"], cols["winst"], cols["meta"])
    idx = np.flatnonzero(gs)
    out = []
    for c in cuts:
        k = np.searchsorted(idx, c)
        out.append(int(idx[k]) if k < len(idx) else len(gs))
    return out


def position_bounds(workload: str, world: int, snap: bool = True, **params):
    """world + 1 cut points of equal position-range shards of the whole trace
    (SURVEY.md 8(e)); with snap, each interior cut moves to the next group
    start (found in a 64-record window generated around it), so divergence
    groups are never split.  Deterministic: every rank computes the same."""
    h, n, *_ = plan(workload, **params)
    _load().tg_free(h)
    cuts = [0]
    for r in range(1, world):
        c = r * n // world
        if snap and 0 < c < n:
            lo, hi = max(0, c - 64), min(n, c + 64)
            w = generate(workload, lo, hi, **params)
            gs = group_starts(w.cols["cta"], w.cols["tid"], w.cols["winst"], w.cols["meta"])
            gs[0] = lo == 0
            k = np.flatnonzero(gs[c - lo:])
            c = c + int(k[0]) if len(k) else hi
        cuts.append(max(cuts[-1], c))
    cuts.append(n)
    return cuts


def generate(workload: str, lo: int | None = None, hi: int | None = None, alloc=None, **params) -> Trace:
    """Generates records [lo, hi) (default: all) of a workload.

    alloc(n, dtype) -> numpy array may be given to place the columns in
    caller-owned memory (e.g. pinned host memory for bench.py's e2e leg).
    """
    lib = _load()
    h, n_total, nsites, nctas, nl, info = plan(workload, **params)
    try:
        lo = 0 if lo is None else int(lo)
        hi = n_total if hi is None else int(hi)
        n = hi - lo
        alloc = alloc or (lambda m, dt: np.empty(m, dtype=dt))
        cols = {name: alloc(n, dt) for name, dt in COLUMNS}
        for name, dt in COLUMNS:
            a = cols[name]
            assert a.dtype == dt and a.flags.c_contiguous and a.shape == (n,)
        if n > 0:
            rc = lib.tg_fill_range(h, lo, hi, *[cols[name].ctypes.data for name, _ in COLUMNS])
            if rc != 0:
                raise ValueError(f"tg_fill_range failed ({rc})")
        return Trace(workload, dict(params), n, n_total, nsites, nctas, nl, info, lo, cols)
    finally:
        lib.tg_free(h)


def generate_ranges(workload: str, ranges, alloc=None, **params):
    """Yields the Trace of every [lo, hi) in `ranges`, planning the workload
    once (C5's plan counts 4e9 records; full-size tests generate it in
    launch-aligned chunks)."""
    lib = _load()
    h, n_total, nsites, nctas, nl, info = plan(workload, **params)
    try:
        alloc = alloc or (lambda m, dt: np.empty(m, dtype=dt))
        for lo, hi in ranges:
            lo, hi = int(lo), int(hi)
            cols = {name: alloc(hi - lo, dt) for name, dt in COLUMNS}
            if hi > lo:
                rc = lib.tg_fill_range(h, lo, hi, *[cols[name].ctypes.data for name, _ in COLUMNS])
                if rc != 0:
                    raise ValueError(f"tg_fill_range failed ({rc})")
            yield Trace(workload, dict(params), hi - lo, n_total, nsites, nctas, nl, info, lo, cols)
    finally:
        lib.tg_free(h)


def from_arrays(addr, cta, tid, site, winst, meta, nsites=None, workload="custom") -> Trace:
    """Wraps hand-built columns (tests, golden fixtures) as a Trace."""
    cols = {}
    for (name, dt), a in zip(COLUMNS, (addr, cta, tid, site, winst, meta)):
        cols[name] = np.ascontiguousarray(np.asarray(a, dtype=dt))
    n = len(cols["addr"])
    assert all(len(a) == n for a in cols.values())
    ns = int(nsites) if nsites is not None else (int(cols["site"].max()) + 1 if n else 1)
    nc = int(cols["cta"].max()) + 1 if n else 0
    return Trace(workload, {}, n, n, ns, nc, 1, "", 0, cols)


def concat(traces) -> Trace:
    cols = {name: np.concatenate([t.cols[name] for t in traces]) for name, _ in COLUMNS}
    return from_arrays(*[cols[name] for name, _ in COLUMNS],
                       nsites=max(t.nsites for t in traces), workload="+".join(t.workload for t in traces))


# Named configurations of BASELINE.json; params per workload.
CONFIGS = {
    "c1_vecadd": ("vecadd", {}),
    "c2_sgemm": ("sgemm", {"n": 256}),
    "c3_bfs": ("bfs", {"nodes": 1000000, "seed": 42}),
    "c4_srad": ("srad", {"rows": 2048, "cols": 2048, "iters": 6}),
    "c4_backprop": ("backprop", {"in": 4194304}),
    "c5_mixed": ("mixed", {}),
}
