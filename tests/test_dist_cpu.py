"""Multi-process (world_size 2, gloo, CPU) checks of the data-parallel
decomposition the multi-GPU path relies on:

  * launch-aligned position shards (tracegen.shard_bounds) cover the trace
    exactly and never split a CTA (CTAs never span kernel instances);
  * per-shard CTA-scope reuse histograms and per-shard MD / BD counters,
    summed with an all-reduce, equal the analysis of the whole trace
    (the analyzer runs per kernel instance; L237: reuse is
    per CTA) -- checked with the oracle on each rank;
  * bench.py's weak-scaling combination: two independent traces (different
    seeds) analysed on two ranks sum to the analysis of their concatenation
    with disjoint CTA ids;
  * bench.py's position-range sharding (the N>1 default): every rank derives
    the same cut points of the N-times-larger global trace, the shards tile
    it exactly, every cut falls on a warp-level group start, and the shard
    contents equal the corresponding slices of the global trace.  (The
    library's cross-rank exchange itself is covered on one GPU by
    tests/test_gpu_multirank.py with in-process loopback ranks.)
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _analyse(t, lb):
    import oracle as orc
    h, st = orc.reuse(t, lb, orc.SCOPE_CTA, orc.BINS_LINEAR, 40)
    hm, psm = orc.mem_div(t, lb, 32)
    psb, tot = orc.branch_div(t, 32)
    return np.concatenate([h.astype(np.int64), np.array([st["streaming"]]), hm.ravel().astype(np.int64),
                           psm.ravel().astype(np.int64), psb.ravel().astype(np.int64), tot.astype(np.int64)])


def _worker(rank, world, port, mode, q):
    import sys
    sys.path.insert(0, ROOT)
    import tracegen as tg
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        if mode == "shard":
            params = dict(rows=64, cols=64, iters=2)
            lo, hi = tg.shard_bounds("srad", rank, world, **params)
            t = tg.generate("srad", lo=lo, hi=hi, **params)
            t.nsites = tg.plan("srad", **params)[2]
            # a CTA must not appear on both ranks
            ctas = torch.zeros(4096, dtype=torch.int64)
            ctas[np.unique(t.cta).astype(np.int64)] = 1
            dist.all_reduce(ctas)
            assert int(ctas.max()) <= 1
        elif mode == "position":
            import bench
            bench.WORKLOADS["t_srad"] = ("srad", dict(rows=64, cols=64, iters=1, bb=1))
            bench.SCALE["t_srad"] = "iters"
            name, params = bench.workload_params("t_srad", world, "position")
            assert params["iters"] == world
            t, off, total, mode2 = bench.make_trace("t_srad", rank, world, "position", pinned=False)
            assert mode2 == "position"
            cuts = torch.tensor(tg.position_bounds(name, world, snap=True, **params), dtype=torch.int64)
            allc = [torch.zeros_like(cuts) for _ in range(world)]
            dist.all_gather(allc, cuts)
            assert all((c == cuts).all() for c in allc)
            assert off == int(cuts[rank]) and off + t.n == int(cuts[rank + 1]) and total == int(cuts[-1])
            whole = tg.generate(name, **params)
            assert total == whole.n
            for k, _ in tg.COLUMNS:
                assert (t.cols[k] == whole.cols[k][off:off + t.n]).all()
            gs = tg.group_starts(whole.cta, whole.tid, whole.winst, whole.meta)
            assert gs[off] or off == 0
            v = torch.tensor([t.n], dtype=torch.int64)
            dist.all_reduce(v)
            if rank == 0:
                q.put(np.array([int(v[0]), total]))
            return
        else:
            t = tg.generate("rand", seed=10 + rank, ctas=5, threads=96, instrs=25, lines=40, launches=2)
        v = torch.from_numpy(_analyse(t, 32))
        dist.all_reduce(v)
        if rank == 0:
            q.put(v.numpy())
    finally:
        dist.destroy_process_group()


def _run(mode):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, mode, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def test_shard_bounds_cover_and_align():
    import tracegen as tg
    params = dict(rows=64, cols=64, iters=3)
    off = tg.launch_offsets("srad", **params)
    for world in (1, 2, 3, 4, 8):
        b = [tg.shard_bounds("srad", r, world, **params) for r in range(world)]
        assert b[0][0] == 0 and b[-1][1] == int(off[-1])
        for (lo, hi), (lo2, _) in zip(b, b[1:]):
            assert hi == lo2 and lo <= hi
        for lo, hi in b:
            assert lo in set(off.tolist()) and hi in set(off.tolist())


def test_sharded_analysis_sums_to_whole_trace():
    import tracegen as tg
    got = _run("shard")
    params = dict(rows=64, cols=64, iters=2)
    want = _analyse(tg.generate("srad", **params), 32)
    assert (got == want).all()


def test_weak_scaling_combination():
    import tracegen as tg
    got = _run("weak")
    a = tg.generate("rand", seed=10, ctas=5, threads=96, instrs=25, lines=40, launches=2)
    b = tg.generate("rand", seed=11, ctas=5, threads=96, instrs=25, lines=40, launches=2)
    cols = {k: np.concatenate([a.cols[k], b.cols[k] + (a.cta.max() + 1 if k == "cta" else 0)])
            for k, _ in tg.COLUMNS}
    cat = tg.from_arrays(*(cols[k] for k, _ in tg.COLUMNS), nsites=max(a.nsites, b.nsites))
    want = _analyse(cat, 32)
    assert (got == want).all()


def test_bench_position_sharding():
    got = _run("position")
    assert got[0] == got[1]
