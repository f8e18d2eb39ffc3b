"""Multi-rank path with ONE PROCESS PER RANK on one GPU.

Each rank is a separate process holding a cadv context created with
cadv_create_peer: the library's own collectives (device kernels reading the
other processes' staged buffers through CUDA IPC mappings, TCP bootstrap on
127.0.0.1).  This drives the cross-process code the in-process loopback
ranks cannot: cudaIpcGetMemHandle / cudaIpcOpenMemHandle of the exchange
buffers, k_push storing straight into another process's receive buffer, the
T_c max-reduce, the histogram sum, the kernel-scope entry gather and the
agreed error path.  Shards are consecutive position ranges (snapped to group
starts for divergence); every rank must return the whole-trace oracle result.
"""
import multiprocessing as mp
import os
import socket

import numpy as np
import pytest

import oracle as orc
import tracegen as tg

pytestmark = pytest.mark.gpu

CASES = {
    "rand": ("rand", dict(seed=3, ctas=40, threads=128, instrs=20, lines=60, pstore=0.25, pbb=0.3, launches=2)),
    "srad": ("srad", dict(rows=256, cols=256, iters=2)),
    "bfs": ("bfs", dict(nodes=30000, seed=7)),
}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(addr, rank, nranks, name, kw, snap, env, q, contiguous=True):
    try:
        os.environ.update(env)
        import torch
        import paper_conf_cgo_shensll18_b200 as cadv
        torch.cuda.set_device(0)
        if contiguous:
            cuts = tg.position_bounds(name, nranks, snap=snap, **kw)
        else:  # (scrambled traces are generated whole: unsnapped equal cuts)
            n = tg.generate(name, **kw).n
            cuts = [r * n // nranks for r in range(nranks)] + [n]
        t = tg.generate(name, **kw) if not contiguous else None
        t = tg.from_arrays(*(t.cols[k][cuts[rank]:cuts[rank + 1]] for k, _ in tg.COLUMNS), nsites=t.nsites) \
            if t is not None else tg.generate(name, cuts[rank], cuts[rank + 1], **kw)
        ctx = cadv.create(0, peer_addr=addr, rank=rank, nranks=nranks)
        ctx.load_trace(cadv.to_device(t), global_offset=cuts[rank], warp_contiguous=contiguous)
        out = {}
        for lb, sc in ((128, 0), (32, 0), (128, 1)):
            h, st = ctx.reuse_histogram(lb, sc, 0, 66)
            out[("rd", lb, sc)] = (h, st)
        if snap or not contiguous:
            o = ctx.analyze(rd=(128, 0, 1, 20), md=(128, 32), bd=32, nsites=t.nsites)
            out["fused"] = (o["reuse"][0], o["mem_div"][0], o["mem_div"][1], o["branch_div"][0], o["branch_div"][1])
            out["md16"] = ctx.mem_divergence(32, 16, t.nsites)
            out["bd8"] = ctx.branch_divergence(8, t.nsites)
        ctx.destroy()
        q.put((rank, out))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, "ERR " + repr(e) + traceback.format_exc()))


def _run(name, kw, nranks, snap, env=None, contiguous=True):
    addr = f"127.0.0.1:{_free_port()}"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(addr, r, nranks, name, kw, snap, env or {}, q, contiguous))
          for r in range(nranks)]
    for p in ps:
        p.start()
    res = {}
    for _ in range(nranks):
        r, v = q.get(timeout=300)
        res[r] = v
    for p in ps:
        p.join(timeout=60)
    for r, v in res.items():
        assert not isinstance(v, str), v
    return res


@pytest.mark.parametrize("case", sorted(CASES))
@pytest.mark.parametrize("nranks", [2, 3])
def test_peer_processes_equal_oracle(case, nranks):
    name, kw = CASES[case]
    t = tg.generate(name, **kw)
    res = _run(name, kw, nranks, snap=True)
    ref_rd = {k: orc.reuse(t, k[1], k[2], 0, 66) for k in res[0] if isinstance(k, tuple)}
    rh20 = orc.reuse(t, 128, 0, 1, 20)[0]
    mh, ms = orc.mem_div(t, 128, 32)
    bs, bt = orc.branch_div(t, 32)
    m16 = orc.mem_div(t, 32, 16)
    b8 = orc.branch_div(t, 8)
    for r in range(nranks):
        for k, (h, st) in ref_rd.items():
            assert (res[r][k][0] == h).all() and res[r][k][1] == st, (r, k)
        f = res[r]["fused"]
        assert (f[0] == rh20).all() and (f[1] == mh).all() and (f[2] == ms).all()
        assert (f[3] == bs).all() and (f[4] == bt).all()
        assert (res[r]["md16"][0] == m16[0]).all() and (res[r]["md16"][1] == m16[1]).all()
        assert (res[r]["bd8"][0] == b8[0]).all() and (res[r]["bd8"][1] == b8[1]).all()


def test_peer_processes_unsnapped_reuse_and_alltoallv():
    """Unsnapped position cuts (reuse distance accepts any split) and the
    alltoallv exchange path (CADV_EXCHANGE=nccl selects the grouped
    send / receive form, served here by the peer backend's alltoallv)."""
    name, kw = CASES["rand"]
    t = tg.generate(name, **kw)
    for env in ({}, {"CADV_EXCHANGE": "nccl"}):
        res = _run(name, kw, 2, snap=False, env=env)
        for k in res[0]:
            h, st = orc.reuse(t, k[1], k[2], 0, 66)
            for r in range(2):
                assert (res[r][k][0] == h).all() and res[r][k][1] == st, (env, r, k)


def test_peer_processes_non_contiguous():
    """warp_contiguous = 0 shards in two processes: the per-warp stream
    exchange (exchange_by_warp) runs over the peer collectives."""
    kw = dict(seed=2, ctas=8, threads=128, instrs=15, lines=30, pstore=0.3, pbb=0.3, scramble=1, scramble_seed=2)
    t = tg.generate("rand", **kw)
    res = _run("rand", kw, 2, snap=False, contiguous=False)
    rh20 = orc.reuse(t, 128, 0, 1, 20)[0]
    mh, ms = orc.mem_div(t, 128, 32)
    bs, bt = orc.branch_div(t, 32)
    for r in range(2):
        f = res[r]["fused"]
        assert (f[0] == rh20).all() and (f[1] == mh).all() and (f[2] == ms).all()
        assert (f[3] == bs).all() and (f[4] == bt).all()
        assert (res[r]["md16"][0] == orc.mem_div(t, 32, 16)[0]).all()
        assert (res[r]["bd8"][1] == orc.branch_div(t, 8)[1]).all()
