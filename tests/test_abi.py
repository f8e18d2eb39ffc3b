"""C-ABI library checks that need no GPU: the library loads, exports every
entry point include/cadv.h declares, and fails loudly without a device."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_cgo_shensll18_b200")


def _declared():
    src = open(os.path.join(ROOT, "include", "cadv.h")).read()
    return sorted(set(re.findall(r"CADV_API\s+[^;(]*?\b(cadv_\w+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for want in ("cadv_create", "cadv_load_trace", "cadv_reuse_histogram", "cadv_mem_divergence",
                 "cadv_branch_divergence", "cadv_destroy", "cadv_last_error", "cadv_last_elapsed_ms"):
        assert want in names


def test_library_exports_every_declared_symbol():
    import paper_conf_cgo_shensll18_b200 as cadv
    L = cadv.lib()
    for name in _declared():
        assert hasattr(L, name), name
    assert cadv.version().startswith("cadv")


def test_create_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_cgo_shensll18_b200 as cadv
    with pytest.raises(cadv.CadvError) as e:
        cadv.create(0)
    assert e.value.status == cadv.CADV_ERR_CUDA
    h = ctypes.c_void_p()
    assert cadv.lib().cadv_create(ctypes.byref(h), 0, None, None, 0, 1) == cadv.CADV_ERR_CUDA


def test_null_arguments_rejected():
    import paper_conf_cgo_shensll18_b200 as cadv
    L = cadv.lib()
    assert L.cadv_create(None, 0, None, None, 0, 1) == cadv.CADV_ERR_INVALID_ARG
    assert L.cadv_load_trace(None, None, 0) == cadv.CADV_ERR_INVALID_ARG
    assert L.cadv_reuse_histogram(None, 128, 0, 0, None, 10, None) == cadv.CADV_ERR_INVALID_ARG
    assert L.cadv_data_centric(None, None, 0, 128, 0, 0, 66, 32, None, None) == cadv.CADV_ERR_INVALID_ARG
    assert L.cadv_destroy(None) == cadv.CADV_ERR_INVALID_ARG


def test_product_path_is_independent_of_the_oracle():
    """The product package and its CUDA sources never reference oracle/."""
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, re.M), f
                assert "oracle.cpp" not in txt and "liboracle" not in txt, f


def test_sm100a_only_build():
    mk = open(os.path.join(ROOT, "Makefile")).read()
    assert "arch=compute_100a,code=sm_100a" in mk


def _boot_worker(addr, rank, nranks, q):
    import paper_conf_cgo_shensll18_b200 as cadv
    try:
        q.put((rank, cadv.bootstrap_selftest(addr, rank, nranks, bytes([rank + 1]) * 5)))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)))


@pytest.mark.parametrize("nranks", [2, 3])
def test_peer_bootstrap_multiprocess(nranks):
    """The peer backend's host bootstrap (TCP star through rank 0, the part of
    cadv_create_peer that needs no GPU): nranks processes allgather a blob."""
    import multiprocessing as mp
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_boot_worker, args=(f"127.0.0.1:{port}", r, nranks, q)) for r in range(nranks)]
    for p in ps:
        p.start()
    got = dict(q.get(timeout=60) for _ in range(nranks))
    for p in ps:
        p.join(timeout=30)
    want = b"".join(bytes([r + 1]) * 5 for r in range(nranks))
    assert all(got[r] == want for r in range(nranks)), got
