"""Device-side trace producer (include/cadv_record.cuh) and its demo kernels.

ctypes binding of libcadv_demo.so: hand-instrumented sm_100a kernels (config
1 vecAdd, config 2 naive / tiled SGEMM) write REAL traces into device
buffers allocated here with torch (plumbing only); the buffers are SoA
columns ready for `Context.load_trace`.  SURVEY.md NEXT-2.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libcadv_demo.so")


class DevTrace(ctypes.Structure):
    """cadv_dev_trace (include/cadv_record.cuh)."""
    _fields_ = [("addr", ctypes.c_void_p), ("cta", ctypes.c_void_p), ("tid", ctypes.c_void_p),
                ("site", ctypes.c_void_p), ("winst", ctypes.c_void_p), ("meta", ctypes.c_void_p),
                ("count", ctypes.c_void_p), ("capacity", ctypes.c_ulonglong), ("winst_ctr", ctypes.c_void_p),
                ("cta_base", ctypes.c_uint32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is not built (run `make`)")
        L = ctypes.CDLL(LIB_PATH)
        L.cadv_demo_vecadd.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(DevTrace),
                                       ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
        L.cadv_demo_sgemm.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(DevTrace),
                                      ctypes.c_uint32, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
        L.cadv_demo_vecadd.restype = L.cadv_demo_sgemm.restype = ctypes.c_int
        _lib = L
    return _lib


class TraceBuffer:
    """Device SoA trace columns + record counter + per-warp winst counters."""

    def __init__(self, capacity: int, max_warps: int, device="cuda"):
        import torch
        self.capacity = int(capacity)
        self.cols = {"addr": torch.zeros(capacity, dtype=torch.uint64, device=device),
                     "cta": torch.zeros(capacity, dtype=torch.uint32, device=device),
                     "tid": torch.zeros(capacity, dtype=torch.uint16, device=device),
                     "site": torch.zeros(capacity, dtype=torch.uint32, device=device),
                     "winst": torch.zeros(capacity, dtype=torch.uint32, device=device),
                     "meta": torch.zeros(capacity, dtype=torch.uint8, device=device)}
        self.count = torch.zeros(1, dtype=torch.int64, device=device)
        self.winst_ctr = torch.zeros(2 * max_warps, dtype=torch.int32, device=device)

    def desc(self, cta_base=0) -> DevTrace:
        c = self.cols
        return DevTrace(c["addr"].data_ptr(), c["cta"].data_ptr(), c["tid"].data_ptr(), c["site"].data_ptr(),
                        c["winst"].data_ptr(), c["meta"].data_ptr(), self.count.data_ptr(), self.capacity,
                        self.winst_ctr.data_ptr(), cta_base)

    @property
    def n(self) -> int:
        n = int(self.count.item())
        if n > self.capacity:
            raise RuntimeError(f"trace buffer overflow: {n} records > capacity {self.capacity}")
        return n

    def columns(self):
        n = self.n
        return {k: v[:n] for k, v in self.cols.items()}

    def to_host(self):
        """numpy columns (for the CPU oracle in tests)."""
        return {k: v.cpu().numpy() for k, v in self.columns().items()}


def _check(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} failed: cudaError {rc}")


def vecadd(n=683, threads=64, ctas=1, buf: TraceBuffer | None = None, reps=1) -> float:
    """vecAdd (config 1 = defaults); traced into `buf` if given.  Returns ms per launch."""
    ms = ctypes.c_float()
    d = buf.desc() if buf is not None else None
    _check(lib().cadv_demo_vecadd(n, ctas, threads, ctypes.byref(d) if d is not None else None, reps,
                                  ctypes.byref(ms)), "cadv_demo_vecadd")
    return ms.value


def sgemm(n=256, variant=0, bb=0, buf: TraceBuffer | None = None, cta_base=0, reps=1) -> float:
    """Config-2 SGEMM (variant 0 naive, 1 tiled), appended to `buf` if given."""
    ms = ctypes.c_float()
    d = buf.desc(cta_base) if buf is not None else None
    _check(lib().cadv_demo_sgemm(n, variant, bb, ctypes.byref(d) if d is not None else None, cta_base, reps,
                                 ctypes.byref(ms)), "cadv_demo_sgemm")
    return ms.value


SGEMM_RECORDS_PER_CTA = {0: lambda n, bb: 256 * (2 * n + 1) + (8 * (2 * n + 3) * 32 if bb else 0),
                         1: lambda n, bb: 256 * (2 * (n // 16) + 1) + (8 * (2 * (n // 16) + 3) * 32 if bb else 0)}
