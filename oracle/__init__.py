"""CPU oracle for the CUDAAdvisor trace analyses — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (its cpu_baseline leg and
--impl reference) may import this package.  The product path
(paper_conf_cgo_shensll18_b200) never imports it and shares no code with it.

Functions follow PAPER.md (see oracle.cpp header for the passages):
  reuse(trace, ...)        LRU-stack reuse-distance histogram
  reuse_rd(trace, ...)     per-record reuse distances
  reuse_brute(trace, ...)  O(n^2) literal definition
  reuse_fenwick(trace, ...) Fenwick-tree distinct counts (same outputs; large traces)
  mem_div(trace, ...)      unique lines per warp instruction
  branch_div(trace, ...)   divergent warp-level block executions
  data_centric(trace, objects, ...)  per-data-object RD / MD histograms
Every function is pinned in tests/test_oracle_pins.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

SCOPE_CTA, SCOPE_KERNEL = 0, 1
BINS_LINEAR, BINS_LOG2 = 0, 1


class OracleError(RuntimeError):
    def __init__(self, code):
        super().__init__({1: "invalid argument", 2: "bad trace"}.get(code, f"error {code}"))
        self.code = code


def _load():
    global _lib
    if _lib is not None:
        return _lib
    src = os.path.join(_HERE, "oracle.cpp")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["/usr/bin/g++" if os.path.exists("/usr/bin/g++") else "g++", "-O2", "-std=c++17", "-fopenmp", "-shared", "-fPIC", "-o", _SO, src])
    lib = ctypes.CDLL(_SO)
    P, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    lib.oracle_reuse.argtypes = [P, P, P, P, u64, u32, i32, i32, u32, P, P]
    lib.oracle_reuse_rd.argtypes = [P, P, P, P, u64, u32, i32, P]
    lib.oracle_reuse_brute.argtypes = [P, P, P, P, u64, u32, i32, i32, u32, P, P, P]
    lib.oracle_reuse_fenwick.argtypes = [P, P, P, P, u64, u32, i32, i32, u32, P, P]
    lib.oracle_mem_div.argtypes = [P, P, P, P, P, P, u64, u32, u32, u32, P, P]
    lib.oracle_branch_div.argtypes = [P, P, P, P, P, u64, u32, u32, P, P]
    lib.oracle_data_centric.argtypes = [P, P, P, P, P, P, u64, P, P, u32, u32, i32, i32, u32, u32, P, P]
    for f in ("oracle_reuse", "oracle_reuse_rd", "oracle_reuse_brute", "oracle_mem_div",
              "oracle_branch_div", "oracle_data_centric", "oracle_num_threads", "oracle_reuse_fenwick"):
        getattr(lib, f).restype = ctypes.c_int
    lib.oracle_set_num_threads.restype = None
    lib.oracle_set_num_threads.argtypes = [ctypes.c_int]
    _lib = lib
    return lib


def _p(a):
    return a.ctypes.data if a is not None else None


def _check(rc):
    if rc != 0:
        raise OracleError(rc)


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def set_num_threads(k: int) -> None:
    """OpenMP threads of the following oracle calls (0 = all cores)."""
    _load().oracle_set_num_threads(int(k))


def reuse(t, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66):
    """Returns (hist[nbins] u64, stats dict)."""
    lib = _load()
    hist = np.zeros(nbins, np.uint64)
    st = np.zeros(5, np.uint64)
    _check(lib.oracle_reuse(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.meta), t.n, line_bytes, scope, binning,
                            nbins, _p(hist), _p(st)))
    return hist, dict(zip(("accesses", "inf", "streaming", "overflow", "finite_sum"), map(int, st)))


def reuse_fenwick(t, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66):
    """Same outputs as reuse(), Fenwick-tree (Bennett-Kruskal) distinct counts:
    O(n log n) per scope, for kernel scope at full size."""
    lib = _load()
    hist = np.zeros(nbins, np.uint64)
    st = np.zeros(5, np.uint64)
    _check(lib.oracle_reuse_fenwick(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.meta), t.n, line_bytes, scope, binning,
                                    nbins, _p(hist), _p(st)))
    return hist, dict(zip(("accesses", "inf", "streaming", "overflow", "finite_sum"), map(int, st)))


def reuse_rd(t, line_bytes=128, scope=SCOPE_CTA):
    """Per-record reuse distance: >=0 finite, -1 = ∞, -2 = not a memory record."""
    lib = _load()
    rd = np.zeros(t.n, np.int64)
    _check(lib.oracle_reuse_rd(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.meta), t.n, line_bytes, scope, _p(rd)))
    return rd


def reuse_brute(t, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66):
    """O(n^2) literal definition; returns (hist, stats, rd per record)."""
    lib = _load()
    hist = np.zeros(nbins, np.uint64)
    st = np.zeros(5, np.uint64)
    rd = np.zeros(t.n, np.int64)
    _check(lib.oracle_reuse_brute(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.meta), t.n, line_bytes, scope, binning,
                                  nbins, _p(hist), _p(st), _p(rd)))
    return hist, dict(zip(("accesses", "inf", "streaming", "overflow", "finite_sum"), map(int, st))), rd


def mem_div(t, line_bytes=128, warp_size=32, nsites=None, per_site=True):
    """Returns (hist[2][W+1] u64, per_site[nsites][2] u64 or None)."""
    lib = _load()
    nsites = t.nsites if nsites is None else nsites
    hist = np.zeros((2, warp_size + 1), np.uint64)
    ps = np.zeros((nsites, 2), np.uint64) if per_site else None
    _check(lib.oracle_mem_div(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.winst), _p(t.site), _p(t.meta), t.n,
                              line_bytes, warp_size, nsites, _p(hist), _p(ps)))
    return hist, ps


def branch_div(t, warp_size=32, nsites=None, per_site=True):
    """Returns (per_site[nsites][3] u64 or None, totals[3] u64 = exec, divergent, threads)."""
    lib = _load()
    nsites = t.nsites if nsites is None else nsites
    ps = np.zeros((nsites, 3), np.uint64) if per_site else None
    tot = np.zeros(3, np.uint64)
    _check(lib.oracle_branch_div(_p(t.cta), _p(t.tid), _p(t.winst), _p(t.site), _p(t.meta), t.n, warp_size,
                                 nsites, _p(ps), _p(tot)))
    return ps, tot


def data_centric(t, objects, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66, warp_size=32,
                 rd=True, md=True):
    """objects = (base u64[k], bytes u64[k]).  Returns (rd_hist[k+1][nbins] or
    None, md_hist[k+1][2][W+1] or None); row k = unattributed lines."""
    lib = _load()
    base = np.ascontiguousarray(objects[0], dtype=np.uint64)
    nb = np.ascontiguousarray(objects[1], dtype=np.uint64)
    k = len(base)
    rh = np.zeros((k + 1, nbins), np.uint64) if rd else None
    mh = np.zeros((k + 1, 2, warp_size + 1), np.uint64) if md else None
    _check(lib.oracle_data_centric(_p(t.addr), _p(t.cta), _p(t.tid), _p(t.winst), _p(t.site), _p(t.meta), t.n, _p(base), _p(nb),
                                   k, line_bytes, scope, binning, nbins, warp_size, _p(rh), _p(mh)))
    return rh, mh


def md_degree(hist):
    """Memory divergence degree: sum_k k*h_k / sum_k h_k over pooled loads+stores."""
    h = np.asarray(hist, dtype=np.float64).sum(axis=0)
    k = np.arange(len(h))
    return float((k * h).sum() / h.sum()) if h.sum() else 0.0
