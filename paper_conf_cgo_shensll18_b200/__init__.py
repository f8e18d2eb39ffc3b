"""paper_conf_cgo_shensll18_b200 — B200-native CUDAAdvisor trace analysis.

Thin ctypes binding over libcadv.so (include/cadv.h).  Argument marshalling
only: every step of every analysis runs in the library's sm_100a kernels.
There is no CPU fallback — without the built library or without an sm_100
device every call raises CadvError.

Names mirror the C ABI:
    ctx = create(device=0, stream=None)          # cadv_create
    ctx.load_trace(cols, warp_contiguous=True)   # cadv_load_trace
    ctx.reuse_histogram(line_bytes, scope, binning, nbins)   # cadv_reuse_histogram
    ctx.mem_divergence(line_bytes, warp_size, nsites)        # cadv_mem_divergence
    ctx.branch_divergence(warp_size, nsites)                 # cadv_branch_divergence
    ctx.destroy()                                            # cadv_destroy
Trace columns may be torch CUDA tensors (borrowed, zero copy) or host numpy
arrays / CPU tensors (copied by cadv_load_trace).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CADV_LIB") or os.path.join(_HERE, "libcadv.so")  # CADV_LIB: A/B builds

CADV_OK, CADV_ERR_INVALID_ARG, CADV_ERR_BAD_TRACE, CADV_ERR_NO_TRACE = 0, 1, 2, 3
CADV_ERR_OOM, CADV_ERR_CUDA, CADV_ERR_NCCL, CADV_ERR_UNSUPPORTED = 4, 5, 6, 7
SCOPE_CTA, SCOPE_KERNEL = 0, 1
BINS_LINEAR, BINS_LOG2 = 0, 1
STATUS_NAMES = {0: "OK", 1: "INVALID_ARG", 2: "BAD_TRACE", 3: "NO_TRACE", 4: "OOM", 5: "CUDA", 6: "NCCL",
                7: "UNSUPPORTED"}
COLUMNS = ("addr", "cta", "tid", "site", "winst", "meta")
_DTYPES = {"addr": np.uint64, "cta": np.uint32, "tid": np.uint16, "site": np.uint32, "winst": np.uint32,
           "meta": np.uint8}


class CadvError(RuntimeError):
    def __init__(self, status, msg=""):
        super().__init__(f"cadv error {STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class TraceDesc(ctypes.Structure):
    _fields_ = [("addr", ctypes.c_void_p), ("cta", ctypes.c_void_p), ("tid", ctypes.c_void_p),
                ("site", ctypes.c_void_p), ("winst", ctypes.c_void_p), ("meta", ctypes.c_void_p),
                ("n", ctypes.c_uint64), ("on_device", ctypes.c_int), ("warp_contiguous", ctypes.c_int)]


class Analysis(ctypes.Structure):
    _fields_ = [("rd_line_bytes", ctypes.c_uint32), ("rd_scope", ctypes.c_int), ("rd_binning", ctypes.c_int),
                ("rd_nbins", ctypes.c_uint32), ("md_line_bytes", ctypes.c_uint32), ("md_warp_size", ctypes.c_uint32),
                ("bd_warp_size", ctypes.c_uint32), ("nsites", ctypes.c_uint32)]


class ReuseStats(ctypes.Structure):
    _fields_ = [("accesses", ctypes.c_uint64), ("inf", ctypes.c_uint64), ("streaming", ctypes.c_uint64),
                ("overflow", ctypes.c_uint64), ("finite_sum", ctypes.c_uint64)]


_lib = None


def lib():
    """Loads libcadv.so (built by `make` / __graft_entry__.build()); raises if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise CadvError(CADV_ERR_CUDA, f"{LIB_PATH} is not built (run `make` or __graft_entry__.build())")
    L = ctypes.CDLL(LIB_PATH)
    P, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    L.cadv_create.argtypes = [ctypes.POINTER(P), i32, P, P, i32, i32]
    L.cadv_load_trace.argtypes = [P, ctypes.POINTER(TraceDesc), u64]
    L.cadv_reuse_histogram.argtypes = [P, u32, i32, i32, P, u32, ctypes.POINTER(ReuseStats)]
    L.cadv_mem_divergence.argtypes = [P, u32, u32, P, P, u32]
    L.cadv_branch_divergence.argtypes = [P, u32, P, u32, P]
    L.cadv_analyze.argtypes = [P, ctypes.POINTER(Analysis), P, ctypes.POINTER(ReuseStats), P, P, P, P]
    L.cadv_data_centric.argtypes = [P, P, u32, u32, i32, i32, u32, u32, P, P]
    L.cadv_destroy.argtypes = [P]
    for f in ("cadv_create", "cadv_load_trace", "cadv_reuse_histogram", "cadv_mem_divergence",
              "cadv_branch_divergence", "cadv_analyze", "cadv_data_centric", "cadv_destroy"):
        getattr(L, f).restype = i32
    L.cadv_last_error.argtypes = [P]
    L.cadv_last_error.restype = ctypes.c_char_p
    L.cadv_last_elapsed_ms.argtypes = [P]
    L.cadv_last_elapsed_ms.restype = ctypes.c_float
    L.cadv_last_launches.argtypes = [P]
    L.cadv_last_launches.restype = u32
    L.cadv_set_profiling.argtypes = [P, i32]
    L.cadv_set_profiling.restype = i32
    L.cadv_last_kernel_times.argtypes = [P, P, P, u32]
    L.cadv_last_kernel_times.restype = u32
    L.cadv_last_count.argtypes = [P, i32]
    L.cadv_last_count.restype = u64
    L.cadv_version.restype = ctypes.c_char_p
    L.cadv_nccl_unique_id.argtypes = [P]
    L.cadv_nccl_unique_id.restype = i32
    L.cadv_loopback_group_create.argtypes = [i32]
    L.cadv_loopback_group_create.restype = P
    L.cadv_loopback_group_destroy.argtypes = [P]
    L.cadv_loopback_group_destroy.restype = i32
    L.cadv_create_loopback.argtypes = [ctypes.POINTER(P), i32, P, P, i32]
    L.cadv_create_loopback.restype = i32
    L.cadv_create_peer.argtypes = [ctypes.POINTER(P), i32, P, ctypes.c_char_p, i32, i32]
    L.cadv_create_peer.restype = i32
    L.cadv_bootstrap_selftest.argtypes = [ctypes.c_char_p, i32, i32, P, P, u64]
    L.cadv_bootstrap_selftest.restype = i32
    _lib = L
    return L


def _ptr_and_kind(a, name):
    """(pointer, on_device, keepalive) for a torch tensor or numpy array column."""
    dt = _DTYPES[name]
    try:
        import torch
        if isinstance(a, torch.Tensor):
            tmap = {np.uint64: torch.uint64, np.uint32: torch.uint32, np.uint16: torch.uint16, np.uint8: torch.uint8}
            if a.dtype != tmap[dt] or not a.is_contiguous() or a.dim() != 1:
                raise CadvError(CADV_ERR_INVALID_ARG, f"column {name}: need contiguous 1-D {tmap[dt]}")
            return a.data_ptr(), bool(a.is_cuda), a
    except ImportError:
        pass
    arr = np.ascontiguousarray(a)
    if arr.dtype != dt or arr.ndim != 1:
        raise CadvError(CADV_ERR_INVALID_ARG, f"column {name}: need 1-D {np.dtype(dt)}")
    return arr.ctypes.data, False, arr


class Context:
    """One analysis context (one per GPU / rank): cadv_create ... cadv_destroy."""

    def __init__(self, device: int = 0, stream=None, nccl_id: bytes | None = None, rank: int = 0, nranks: int = 1,
                 loopback=None, peer_addr: str | None = None):
        L = lib()
        h = ctypes.c_void_p()
        if peer_addr is not None:
            s = L.cadv_create_peer(ctypes.byref(h), int(device), ctypes.c_void_p(stream or 0), peer_addr.encode(),
                                   int(rank), int(nranks))
        elif loopback is not None:
            s = L.cadv_create_loopback(ctypes.byref(h), int(device), ctypes.c_void_p(stream or 0), loopback.handle,
                                       int(rank))
            nranks = loopback.nranks
        else:
            idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
            s = L.cadv_create(ctypes.byref(h), int(device), ctypes.c_void_p(stream or 0), idbuf, int(rank),
                              int(nranks))
        if s != CADV_OK:
            raise CadvError(s, "cadv_create failed (needs an sm_100 GPU and the CUDA driver; NCCL for nranks > 1)")
        self._h = h
        self._keep = None
        self.device = device
        self.rank, self.nranks = rank, nranks

    # -- helpers
    def _check(self, s):
        if s != CADV_OK:
            raise CadvError(s, lib().cadv_last_error(self._h).decode())

    @property
    def handle(self):
        return self._h

    def last_elapsed_ms(self) -> float:
        return float(lib().cadv_last_elapsed_ms(self._h))

    def last_launches(self) -> int:
        return int(lib().cadv_last_launches(self._h))

    def set_profiling(self, enable):
        """cadv_set_profiling: CUDA events around every kernel launch (True / 1)
        or around the streaming-pass (k_scan<F>) launches only (2)."""
        self._check(lib().cadv_set_profiling(self._h, int(enable)))

    def last_kernel_times(self):
        """cadv_last_kernel_times: [(kernel name, device ms)] of the last call."""
        L = lib()
        k = L.cadv_last_kernel_times(self._h, None, None, 0)
        names = (ctypes.c_char_p * max(k, 1))()
        ms = (ctypes.c_float * max(k, 1))()
        k = L.cadv_last_kernel_times(self._h, ctypes.cast(names, ctypes.c_void_p), ctypes.cast(ms, ctypes.c_void_p), k)
        return [(names[i].decode(), float(ms[i])) for i in range(k)]

    def last_count(self, which: int) -> int:
        """cadv_last_count: 0 kept records, 1 cross-tile entries, 2 cross-tile queries, 3 tiles."""
        return int(lib().cadv_last_count(self._h, which))

    # -- cadv_load_trace
    def load_trace(self, cols, n=None, warp_contiguous=True, global_offset=0):
        """cols: mapping (or object with attributes) addr/cta/tid/site/winst/meta."""
        get = (lambda k: cols[k]) if isinstance(cols, dict) else (lambda k: getattr(cols, k))
        ptrs, devs, keep = {}, set(), []
        for k in COLUMNS:
            p, d, ka = _ptr_and_kind(get(k), k)
            ptrs[k] = p
            devs.add(d)
            keep.append(ka)
        if len(devs) != 1:
            raise CadvError(CADV_ERR_INVALID_ARG, "all columns must be on the device or all on the host")
        n = len(keep[0]) if n is None else int(n)
        d = TraceDesc(ptrs["addr"], ptrs["cta"], ptrs["tid"], ptrs["site"], ptrs["winst"], ptrs["meta"], n,
                      1 if devs.pop() else 0, 1 if warp_contiguous else 0)
        self._check(lib().cadv_load_trace(self._h, ctypes.byref(d), int(global_offset)))
        self._keep = keep  # borrowed device columns stay alive while loaded

    # -- cadv_reuse_histogram
    def reuse_histogram(self, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66):
        hist = np.zeros(nbins, np.uint64)
        st = ReuseStats()
        self._check(lib().cadv_reuse_histogram(self._h, line_bytes, scope, binning, hist.ctypes.data, nbins,
                                               ctypes.byref(st)))
        return hist, {"accesses": st.accesses, "inf": st.inf, "streaming": st.streaming, "overflow": st.overflow,
                      "finite_sum": st.finite_sum}

    # -- cadv_mem_divergence
    def mem_divergence(self, line_bytes=128, warp_size=32, nsites=0):
        hist = np.zeros((2, warp_size + 1), np.uint64)
        ps = np.zeros((nsites, 2), np.uint64) if nsites else None
        self._check(lib().cadv_mem_divergence(self._h, line_bytes, warp_size, hist.ctypes.data,
                                              ps.ctypes.data if ps is not None else None, nsites))
        return hist, ps

    # -- cadv_branch_divergence
    def branch_divergence(self, warp_size=32, nsites=0):
        ps = np.zeros((nsites, 3), np.uint64) if nsites else None
        tot = np.zeros(3, np.uint64)
        self._check(lib().cadv_branch_divergence(self._h, warp_size, ps.ctypes.data if ps is not None else None,
                                                 nsites, tot.ctypes.data))
        return ps, tot

    # -- cadv_analyze (one fused pass)
    def analyze(self, rd=(128, SCOPE_CTA, BINS_LINEAR, 66), md=(128, 32), bd=32, nsites=0, per_site=True):
        """Any of rd / md / bd may be None.  Returns dict with the outputs of
        reuse_histogram / mem_divergence / branch_divergence."""
        a = Analysis(rd[0] if rd else 1, rd[1] if rd else 0, rd[2] if rd else 0, rd[3] if rd else 3,
                     md[0] if md else 1, md[1] if md else 32, bd if bd else 32, nsites)
        out = {}
        rh = np.zeros(rd[3], np.uint64) if rd else None
        st = ReuseStats()
        mh = np.zeros((2, md[1] + 1), np.uint64) if md else None
        ms = np.zeros((nsites, 2), np.uint64) if (md and per_site and nsites) else None
        bt = np.zeros(3, np.uint64) if bd else None
        bs = np.zeros((nsites, 3), np.uint64) if (bd and per_site and nsites) else None
        p = lambda x: x.ctypes.data if x is not None else None
        self._check(lib().cadv_analyze(self._h, ctypes.byref(a), p(rh), ctypes.byref(st) if rd else None, p(mh),
                                       p(ms), p(bt), p(bs)))
        if rd:
            out["reuse"] = (rh, {"accesses": st.accesses, "inf": st.inf, "streaming": st.streaming,
                                 "overflow": st.overflow, "finite_sum": st.finite_sum})
        if md:
            out["mem_div"] = (mh, ms)
        if bd:
            out["branch_div"] = (bs, bt)
        return out

    # -- cadv_data_centric
    def data_centric(self, objects, line_bytes=128, scope=SCOPE_CTA, binning=BINS_LINEAR, nbins=66, warp_size=32,
                     rd=True, md=True):
        """objects = (base, bytes) arrays (ascending).  Returns (rd_hist[k+1][nbins]
        or None, md_hist[k+1][2][W+1] or None); row k = unattributed lines."""
        base = np.asarray(objects[0], dtype=np.uint64)
        nb = np.asarray(objects[1], dtype=np.uint64)
        k = len(base)
        tab = np.ascontiguousarray(np.stack([base, nb], axis=1)) if k else np.zeros((0, 2), np.uint64)
        rh = np.zeros((k + 1, nbins), np.uint64) if rd else None
        mh = np.zeros((k + 1, 2, warp_size + 1), np.uint64) if md else None
        p = lambda x: x.ctypes.data if x is not None else None
        self._check(lib().cadv_data_centric(self._h, tab.ctypes.data if k else None, k, line_bytes, scope, binning,
                                            nbins, warp_size, p(rh), p(mh)))
        return rh, mh

    # -- cadv_destroy
    def destroy(self):
        if getattr(self, "_h", None):
            lib().cadv_destroy(self._h)
            self._h = None
            self._keep = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.destroy()


def create(device: int = 0, stream=None, nccl_id: bytes | None = None, rank: int = 0, nranks: int = 1,
           peer_addr: str | None = None) -> Context:
    """cadv_create.  nranks > 1: one process per GPU, all ranks pass the same
    nccl_id (from nccl_unique_id() on rank 0) -- or the same peer_addr
    ("127.0.0.1:port" of rank 0) for cadv_create_peer, the library's own
    collectives over CUDA IPC peer memory."""
    return Context(device, stream, nccl_id, rank, nranks, peer_addr=peer_addr)


def bootstrap_selftest(addr: str, rank: int, nranks: int, payload: bytes) -> bytes:
    """cadv_bootstrap_selftest: host-only allgather over the peer backend's TCP
    bootstrap (no GPU); returns the nranks payloads concatenated in rank order."""
    out = ctypes.create_string_buffer(len(payload) * nranks)
    rc = lib().cadv_bootstrap_selftest(addr.encode(), int(rank), int(nranks), ctypes.c_char_p(payload), out,
                                       len(payload))
    if rc != 0:
        raise CadvError(CADV_ERR_NCCL, f"bootstrap self-test failed ({rc})")
    return out.raw


def nccl_unique_id() -> bytes:
    """cadv_nccl_unique_id: 128 bytes to broadcast to every rank."""
    buf = ctypes.create_string_buffer(128)
    s = lib().cadv_nccl_unique_id(buf)
    if s != CADV_OK:
        raise CadvError(s, "cadv_nccl_unique_id failed")
    return buf.raw


class LoopbackGroup:
    """cadv_loopback_group_create: N in-process ranks on one GPU (tests)."""

    def __init__(self, nranks: int):
        self.nranks = nranks
        self.handle = lib().cadv_loopback_group_create(int(nranks))
        if not self.handle:
            raise CadvError(CADV_ERR_INVALID_ARG, "bad loopback group size")

    def context(self, rank: int, device: int = 0, stream=None) -> Context:
        return Context(device, stream, rank=rank, loopback=self)

    def destroy(self):
        if self.handle:
            lib().cadv_loopback_group_destroy(self.handle)
            self.handle = None


def version() -> str:
    return lib().cadv_version().decode()


def to_device(trace, device="cuda"):
    """Copies a tracegen.Trace's columns to torch CUDA tensors (plumbing only)."""
    import torch
    return {k: torch.from_numpy(np.ascontiguousarray(trace.cols[k])).to(device) for k in COLUMNS}
