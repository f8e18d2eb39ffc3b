#!/usr/bin/env python
"""bench.py — throughput of the CUDAAdvisor trace-analysis hot path on B200.

One step = the whole hot path over
one synthetic trace resident in HBM:
    cadv_load_trace (R0 ingest) + cadv_reuse_histogram (128 B lines, CTA
    scope) + cadv_mem_divergence (128 B, warp 32) + cadv_branch_divergence.
Metric (BASELINE.json): trace records analysed per second (reuse +
divergence), whole job, plus the dominant kernel's HBM roofline fraction.

Workload (N=1): config 4, Rodinia-shaped SRAD 2048x2048, 6 iterations, with
its basic-block trace (tracegen "srad"); 478,150,656 memory records.
N>1 (torchrun, one rank per GPU), --sharding position (default): weak
scaling over ONE global trace N times the N=1 workload (SRAD: 6N
iterations), cut into N equal position ranges snapped to warp-level group
boundaries; each rank holds one shard and the library's
NCCL context does the exchange (kept records redistributed by CTA range,
T_c max-reduce, histogram all-reduce), so every rank gets the global
result.  --sharding independent: every rank its own trace (seed 42 + rank),
histograms summed with torch.distributed.

--impl reference: the CPU oracle (oracle/) as it stands, on this host's
cores, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    "c4_srad": ("srad", dict(rows=2048, cols=2048, iters=6, bb=1)),
    "c2_sgemm": ("sgemm", dict(n=256, bb=1)),
    "c3_bfs": ("bfs", dict(nodes=1000000, seed=42)),
    "c4_backprop": ("backprop", {"in": 4194304}),
    # C5 per GPU: 5e8 records of the mixed trace; at N = 8 the global trace is C5 (4.0e9)
    "c5_mixed": ("mixed", {"records": 500000000}),
}
# how a workload grows with N for position-range weak scaling (param, factor per GPU)
SCALE = {"c4_srad": "iters", "c4_backprop": "in", "c5_mixed": "records"}
METRIC = "trace records analysed/sec (reuse+divergence)"
UNIT = "records/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="cadv", choices=["cadv", "reference"])
    ap.add_argument("--workload", default="c4_srad", choices=sorted(WORKLOADS))
    ap.add_argument("--line-bytes", type=int, default=128)
    ap.add_argument("--rd-scope", default="cta", choices=["cta", "kernel"],
                    help="reuse-distance scope (kernel = whole trace, SURVEY.md NEXT-1)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="target CPU time of the oracle sample")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile-run", action="store_true", help="short run for ncu (no clocks / baselines)")
    ap.add_argument("--sharding", default="position", choices=["position", "independent"],
                    help="N>1: shards of one global trace (library NCCL exchange) or one trace per rank")
    ap.add_argument("--no-data-centric", action="store_true", help="skip the data-centric attribution leg")
    ap.add_argument("--separate", action="store_true",
                    help="one library call per analysis (three passes) instead of the fused cadv_analyze")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="N>1 position sharding: weak = N times the N=1 workload, strong = the N=1 workload split N ways")
    ap.add_argument("--no-per-analysis", action="store_true", help="skip the per-analysis (separate) rates")
    return ap.parse_args()


# ----------------------------------------------------------------- helpers

def log(*a):
    print(*a, file=sys.stderr, flush=True)


class Clocks:
    """SM clocks and throttle reasons sampled DURING the timed region
    (B200_PROFILING.md clocks line): NVML in a background thread every 2 ms
    (works for timed regions of a few ms); nvidia-smi if NVML is missing."""

    def __init__(self, device):
        self.device = device
        self.samples = []
        self.err = None
        self._stop = None
        self._th = None

    def start(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            # torch's device index -> NVML handle (CUDA_VISIBLE_DEVICES may remap)
            h = nv.nvmlDeviceGetHandleByIndex(self._nvml_index(nv))
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        except Exception as e:  # noqa: BLE001
            self.err = f"NVML unavailable: {e}"
            return
        self.samples = []
        self._stop = threading.Event()
        first = threading.Event()

        def run():
            while True:
                try:
                    self.samples.append((nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM),
                                         nv.nvmlDeviceGetCurrentClocksEventReasons(h)))
                except Exception:  # noqa: BLE001
                    pass
                first.set()
                if self._stop.wait(0.002):
                    break

        self._th = threading.Thread(target=run, daemon=True)
        self._th.start()
        first.wait(2.0)

    def _nvml_index(self, nv):
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        if vis:
            ids = [x.strip() for x in vis.split(",") if x.strip()]
            if self.device < len(ids) and ids[self.device].isdigit():
                return int(ids[self.device])
        return self.device

    def stop(self):
        if self._th is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [self.err or "no sampler"], "samples": 0}
        self._stop.set()
        self._th.join(timeout=5)
        import pynvml as nv
        names = {"hw_slowdown": nv.nvmlClocksEventReasonHwSlowdown,
                 "hw_thermal_slowdown": nv.nvmlClocksEventReasonHwThermalSlowdown,
                 "sw_thermal_slowdown": nv.nvmlClocksEventReasonSwThermalSlowdown,
                 "sw_power_cap": nv.nvmlClocksEventReasonSwPowerCap}
        sm = [float(c) for c, _ in self.samples]
        reasons = sorted({nm for _, r in self.samples for nm, bit in names.items() if r & bit})
        under = [x for x in sm if x > 300] or sm
        return {"sm_mhz": statistics.median(under) if under else None, "sm_max_mhz": float(self.max_mhz),
                "reasons": reasons, "samples": len(sm), "source": "NVML, 2 ms"}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def workload_params(workload, world, sharding, scaling="weak"):
    """(generator, params) of the global trace analysed by `world` GPUs."""
    name, params = WORKLOADS[workload]
    params = dict(params)
    if world > 1 and sharding == "position" and workload in SCALE and scaling == "weak":
        params[SCALE[workload]] = params[SCALE[workload]] * world
    return name, params


def make_trace(workload, rank, world, sharding, pinned, scaling="weak"):
    """This rank's trace: its position-range shard of the global trace, or
    (independent / unscalable workloads) a whole trace of its own.  Returns
    (trace, global_offset, global_records, mode)."""
    import tracegen as tg
    name, params = workload_params(workload, world, sharding, scaling)
    mode = "position" if (world > 1 and sharding == "position" and (workload in SCALE or scaling == "strong")) else (
        "independent" if world > 1 else "single")
    if mode == "independent" and rank:
        params["seed"] = params.get("seed", 42) + rank
    alloc = None
    if pinned:
        import torch
        tmap = {np.uint64: torch.uint64, np.uint32: torch.uint32, np.uint16: torch.uint16, np.uint8: torch.uint8}

        def alloc(n, dt):
            return torch.empty(n, dtype=tmap[dt], pin_memory=True).numpy()
    t0 = time.time()
    if mode == "position":
        cuts = tg.position_bounds(name, world, snap=True, **params)
        t = tg.generate(name, cuts[rank], cuts[rank + 1], alloc=alloc, **params)
        off, total = cuts[rank], cuts[-1]
    else:
        t = tg.generate(name, alloc=alloc, **params)
        off, total = 0, t.n * world
    log(f"[bench] rank {rank}: generated {workload} ({name} {params}) [{off:,}, {off + t.n:,}) of {total:,} "
        f"records in {time.time() - t0:.1f}s")
    return t, off, total, mode


# Algorithmic bytes per launch of each kernel, SURVEY.md 8(d) "Algorithmic
# bytes per record" (what the method must move): MD 23 B per memory record
# (addr 8, cta 4, tid 2, winst 4, site 4, meta 1), BD 15 B per BB record
# (cta, tid, winst, site, meta), reuse 13 B per memory record read (addr,
# cta, meta) + the previous-occurrence array P (4 B written + 4 B read).
# The fused pass k_scan<7> streams the trace once: 23 B x mem + 15 B x BB.
# Its other bytes (the BB records' addr column, the kept records it writes
# for the reuse tail) are implementation passes, reported separately.
def algorithmic_bytes(kname, st):
    mem, bb, kept = st["n_mem"], st["n_bb"], st["kept"]
    table = {
        "k_scan<7>": 23 * mem + 15 * bb,
        "k_scan<1>": 13 * mem,
        "k_scan<2>": 23 * mem,
        "k_scan<4>": 15 * bb,
        "k_scan<11>": 23 * mem,                     # data-centric (reuse + MD per object)
        "k_rd_seg": 8 * kept,                       # P of the kept records (4 B in + 4 B out, in registers)
        "k_rd_tile<0>": 8 * kept,
    }
    return table.get(kname)


def implementation_bytes(kname, st):
    """Bytes the kernel moves beyond algorithmic_bytes (not counted in frac)."""
    if kname in ("k_scan<7>", "k_scan<1>", "k_scan<11>"):
        return {"bb_addr_column": 8 * st["n_bb"] if kname == "k_scan<7>" else 0, "kept_record_writes": 12 * st["kept"]}
    return {}


def src_sha():
    """Identity of the library build: hash of its sources and Makefile."""
    import glob
    import hashlib
    h = hashlib.sha256()
    files = sorted(glob.glob(os.path.join(ROOT, "paper_conf_cgo_shensll18_b200", "csrc", "*"))) + \
        [os.path.join(ROOT, "include", "cadv.h"), os.path.join(ROOT, "Makefile")]
    for f in files:
        with open(f, "rb") as fh:
            h.update(os.path.basename(f).encode())
            h.update(fh.read())
    return h.hexdigest()[:16]


def ncu_traffic(kname, workload):
    """DRAM bytes (read + write) per launch of `kname` from profiles/ncu_traffic.json,
    written by tools/ncu_capture.sh from one `ncu --set full` capture of this
    bench's workload -- used only when it was taken on the SAME library
    sources (src_sha) and workload; else (None, reason)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(p))
    except (OSError, ValueError):
        return None, "no profiles/ncu_traffic.json"
    if d.get("src_sha") != src_sha():
        return None, f"profiles/ncu_traffic.json is from sources {d.get('src_sha')}, not {src_sha()}"
    k = d.get("workloads", {}).get(workload, {}).get(kname)
    if k is None:
        return None, f"no {kname} capture for {workload}"
    return int(k), f"profiles/ncu_traffic.json ({d.get('capture', 'ncu --set full')}, sources {d['src_sha']})"


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


# ----------------------------------------------------------------- CPU oracle (baseline / reference arm)

def oracle_sample(t, target_s, line_bytes):
    """Times the oracle (reuse + MD + BD, as it stands) on a growing prefix of
    the trace until one sample takes >= target_s/3; returns the last sample's
    (records, seconds, cores, description)."""
    import oracle as orc
    import tracegen as tg
    n = min(t.n, 200_000)
    while True:
        sub = tg.from_arrays(*(t.cols[k][:n] for k, _ in tg.COLUMNS), nsites=t.nsites)
        t0 = time.time()
        orc.reuse(sub, line_bytes, 0, 0, 66)
        orc.mem_div(sub, line_bytes, 32)
        orc.branch_div(sub, 32)
        dt = time.time() - t0
        if dt >= target_s / 3 or n >= t.n:
            return n, dt, orc.num_threads(), f"first {n:,} records of the trace (reuse + MD + BD)"
        n = min(t.n, int(n * max(2.0, min(8.0, (target_s / 3) / max(dt, 1e-3)))))


def oracle_one_thread(t, nrec, line_bytes):
    """The same oracle calls on the first nrec records with ONE thread."""
    import oracle as orc
    import tracegen as tg
    sub = tg.from_arrays(*(t.cols[k][:nrec] for k, _ in tg.COLUMNS), nsites=t.nsites)
    orc.set_num_threads(1)
    try:
        t0 = time.time()
        orc.reuse(sub, line_bytes, 0, 0, 66)
        orc.mem_div(sub, line_bytes, 32)
        orc.branch_div(sub, 32)
        return time.time() - t0
    finally:
        orc.set_num_threads(0)


# ----------------------------------------------------------------- main

def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    import torch
    import torch.distributed as dist

    import paper_conf_cgo_shensll18_b200 as cadv
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    t, goff, gtotal, mode = make_trace(args.workload, rank, world, args.sharding, pinned=True, scaling=args.scaling)
    n = t.n
    n_mem = int(((t.meta & 3) < 2).sum())
    n_bb = n - n_mem
    nsites = t.nsites
    dev = {k: torch.from_numpy(t.cols[k]).to(f"cuda:{local}", non_blocking=True) for k in cadv.COLUMNS}
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    if mode == "position":
        # one NCCL communicator inside the library; rank 0's id broadcast over torch.distributed
        obj = [cadv.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ctx = cadv.create(local, stream.cuda_stream, nccl_id=obj[0], rank=rank, nranks=world)
    else:
        ctx = cadv.create(local, stream.cuda_stream)
    lb = args.line_bytes
    NB = 66
    SC = cadv.SCOPE_CTA if args.rd_scope == "cta" else cadv.SCOPE_KERNEL

    def step(cols, allreduce=True):
        launches = 0
        ktimes = []
        ctx.load_trace(cols, global_offset=goff)
        launches += ctx.last_launches(); ktimes += ctx.last_kernel_times()
        if args.separate:
            h, st = ctx.reuse_histogram(lb, SC, cadv.BINS_LINEAR, NB)
            launches += ctx.last_launches(); ktimes += ctx.last_kernel_times()
            kept = ctx.last_count(0)
            hm, _ = ctx.mem_divergence(lb, 32, nsites)
            launches += ctx.last_launches(); ktimes += ctx.last_kernel_times()
            _, tot = ctx.branch_divergence(32, nsites)
            launches += ctx.last_launches(); ktimes += ctx.last_kernel_times()
        else:
            out = ctx.analyze(rd=(lb, SC, cadv.BINS_LINEAR, NB), md=(lb, 32), bd=32, nsites=nsites)
            launches += ctx.last_launches(); ktimes += ctx.last_kernel_times()
            kept = ctx.last_count(0)
            h, st = out["reuse"]
            hm, _ = out["mem_div"]
            _, tot = out["branch_div"]
        if mode == "independent" and allreduce:
            r = torch.from_numpy(np.concatenate([h, hm.ravel(), tot]).astype(np.int64)).cuda()
            dist.all_reduce(r)
            launches += 1
        return launches, ktimes, dict(n=n, n_mem=n_mem, n_bb=n_bb, kept=kept, md_groups=int(hm.sum()),
                                      bd_groups=int(tot[0]))

    # ---- warm-up (allocates the library workspace)
    for _ in range(max(args.warmup, 0)):
        step(dev)
    # ---- timed region (CUDA events around the streaming pass only: the
    # dominant kernel's live duration without two event records per launch)
    ctx.set_profiling(2)
    clocks = Clocks(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if not args.profile_run:
        clocks.start()
    else:
        # ncu --profile-from-start off: capture the timed steps only (not the
        # warm-up, whose first call also sizes the workspace)
        torch.cuda.profiler.start()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    launches, kt, stats = 0, [], None
    for _ in range(args.steps):
        L, k, stats = step(dev)
        launches += L
        kt += k
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ck = clocks.stop() if not args.profile_run else {}
    if args.profile_run:
        torch.cuda.profiler.stop()
    ctx.set_profiling(False)
    ms = e0.elapsed_time(e1)
    ms_max = ms
    total_records = n
    if world > 1:
        v = torch.tensor([ms, float(n)], dtype=torch.float64, device="cuda")
        mx = v.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        sm = v.clone()
        dist.all_reduce(sm, op=dist.ReduceOp.SUM)
        ms_max = float(mx[0])
        total_records = int(sm[1])
    ms_step = ms_max / max(args.steps, 1)
    value = total_records * args.steps / (ms_max / 1e3)
    total_mem = n_mem
    if world > 1:
        v = torch.tensor([float(n_mem)], dtype=torch.float64, device="cuda")
        dist.all_reduce(v)
        total_mem = int(v[0])

    # ---- dominant kernel roofline (live CUDA-event durations of the timed region)
    agg = {}
    for name, t_ms in kt:
        a = agg.setdefault(name, [0.0, 0])
        a[0] += t_ms
        a[1] += 1
    dom = max(agg.items(), key=lambda kv: kv[1][0])[0] if agg else None
    peak, peak_src = peaks()
    roof = None
    if dom:
        tot_ms, cnt = agg[dom]
        per = algorithmic_bytes(dom, stats)
        avg_ms = tot_ms / cnt
        if per is not None:
            gbs = per / (avg_ms / 1e3) / 1e9
            traffic, tsrc = ncu_traffic(dom, args.workload)
            # the whole step by SURVEY 8(d) bytes: 31 B per memory record (23 B read
            # once + the P array 4 B written and read) + 15 B per BB record
            step_bytes = 31 * n_mem + 15 * n_bb
            roof = {"bound": "hbm", "kernel": dom, "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                    "frac": round(gbs / peak, 4), "traffic": traffic, "peak_source": peak_src,
                    "traffic_source": tsrc, "avg_launch_ms": round(avg_ms, 4),
                    "algorithmic_bytes_per_launch": per,
                    "algorithmic_bytes_rule": "SURVEY 8(d): 23 B x memory records + 15 B x BB records (k_scan<7>)",
                    "implementation_bytes_per_launch": implementation_bytes(dom, stats),
                    "share_of_step": round(tot_ms / (ms * 1.0), 4),
                    "step_algorithmic_frac": round(step_bytes / (ms_step / 1e3) / 1e9 / peak, 4),
                    "step_algorithmic_bytes": step_bytes}
    # ---- per-kernel breakdown of the step: a separate, untimed pass with
    # events around every launch
    kernels = {}
    if not args.profile_run:
        ctx.set_profiling(1)
        nb = max(1, min(args.steps, 3))
        kall = {}
        for _ in range(nb):
            _, k, _ = step(dev)
            for name, t_ms in k:
                a = kall.setdefault(name, [0.0, 0])
                a[0] += t_ms
                a[1] += 1
        torch.cuda.synchronize()
        ctx.set_profiling(False)
        kernels = {k: {"launches_per_step": v[1] / nb, "ms_per_step": round(v[0] / nb, 4)}
                   for k, v in sorted(kall.items(), key=lambda kv: -kv[1][0])}

    # ---- per-analysis rates (reuse, MD and BD records/s
    # separately, and "reuse+divergence" = memory records / (t_reuse + t_md)),
    # each analysis alone through its own C-ABI call, CUDA events, untimed
    # for the headline value
    per_an = None
    if world == 1 and not args.profile_run and not args.no_per_analysis:
        calls = {"reuse": lambda: ctx.reuse_histogram(lb, SC, cadv.BINS_LINEAR, NB),
                 "mem_div": lambda: ctx.mem_divergence(lb, 32, nsites),
                 "branch_div": lambda: ctx.branch_divergence(32, nsites)}
        per_an = {}
        ksteps = max(3, min(args.steps, 10))
        for nm, fn in calls.items():
            fn()
            torch.cuda.synchronize()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            for _ in range(ksteps):
                fn()
            a1.record(stream)
            torch.cuda.synchronize()
            ams = a0.elapsed_time(a1) / ksteps
            recs = n_bb if nm == "branch_div" else n_mem
            per_an[nm] = {"ms_per_call": round(ams, 4), "records": recs,
                          "records_per_s": round(recs / (ams / 1e3), 1),
                          "record_kind": "BB records" if nm == "branch_div" else "memory records"}
        per_an["reuse_plus_divergence"] = {
            "records_per_s": round(n_mem / ((per_an["reuse"]["ms_per_call"] + per_an["mem_div"]["ms_per_call"]) / 1e3), 1),
            "definition": "memory records / (t_reuse + t_mem_div), SURVEY 8(d)"}
        per_an["fused_mem_records_per_s"] = round(n_mem * args.steps / (ms / 1e3), 1)

    # ---- data-centric attribution: the same trace, per-object
    # RD + MD rows over the workload's allocation table (one fused pass)
    dcen = None
    if world == 1 and not args.profile_run and not args.no_data_centric:
        import tracegen as tg
        gname, gparams = WORKLOADS[args.workload]
        objs = tg.objects(gname, **gparams)
        if len(objs[0]):
            def dstep():
                ctx.data_centric(objs, lb, SC, cadv.BINS_LINEAR, NB, 32)
                return ctx.last_launches(), ctx.last_kernel_times(), ctx.last_count(0)
            for _ in range(2):
                dstep()
            ctx.set_profiling(2)
            torch.cuda.synchronize()
            g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            g0.record(stream)
            dk, dl, dkept = [], 0, 0
            for _ in range(args.steps):
                L_, k_, dkept = dstep()
                dl += L_
                dk += k_
            g1.record(stream)
            torch.cuda.synchronize()
            ctx.set_profiling(False)
            dms = g0.elapsed_time(g1) / max(args.steps, 1)
            dagg = {}
            for name_, t_ms in dk:
                a = dagg.setdefault(name_, [0.0, 0])
                a[0] += t_ms
                a[1] += 1
            ddom = max(dagg.items(), key=lambda kv: kv[1][0])[0]
            per = algorithmic_bytes(ddom, dict(n=n, n_mem=n_mem, n_bb=n_bb, kept=dkept, md_groups=0, bd_groups=0))
            davg = dagg[ddom][0] / dagg[ddom][1]
            dcen = {"value": round(n / (dms / 1e3), 1), "unit": UNIT, "ms_per_step": round(dms, 3),
                    "objects": int(len(objs[0])), "call": "cadv_data_centric(rd + md rows per object)",
                    "gpu_launches": dl,
                    "roofline": ({"bound": "hbm", "kernel": ddom, "achieved": round(per / (davg / 1e3) / 1e9, 1),
                                  "peak": peak, "unit": "GB/s", "frac": round(per / (davg / 1e3) / 1e9 / peak, 4),
                                  "avg_launch_ms": round(davg, 4), "algorithmic_bytes_per_launch": per}
                                 if per else None)}

    # ---- e2e: the same step through the C ABI with HOST buffers (H2D inside the timed region)
    e2e = None
    if args.e2e_steps > 0 and not args.profile_run:
        # the step's inputs in pinned host memory (copied to the device inside the timed region)
        host = {k: torch.from_numpy(t.cols[k]).pin_memory() for k in cadv.COLUMNS}
        step(host, allreduce=False)  # warm the host-copy workspace
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(args.e2e_steps):
            step(host)
        f1.record(stream)
        torch.cuda.synchronize()
        ems = f0.elapsed_time(f1)
        if world > 1:
            v = torch.tensor([ems], dtype=torch.float64, device="cuda")
            dist.all_reduce(v, op=dist.ReduceOp.MAX)
            ems = float(v[0])
        h2d = int(sum(t.cols[k].nbytes for k in cadv.COLUMNS))
        d2h = 8 * (NB + 4) + 8 * 2 * 33 + 8 * 2 * nsites + 8 * 3 + 8 * 3 * nsites
        e2e = {"value": round(total_records * args.e2e_steps / (ems / 1e3), 1), "unit": UNIT,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h}

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.profile_run:
        rec, dt, cores, desc = oracle_sample(t, args.cpu_seconds, lb)
        n1 = max(1, rec // max(1, cores))
        dt1 = oracle_one_thread(t, n1, lb)
        cpu = {"value": round(rec / dt, 1), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc,
               "seconds": round(dt, 2), "cpu_model": cpu_model(),
               "one_thread": {"value": round(n1 / dt1, 1), "unit": UNIT, "records": n1, "seconds": round(dt1, 2)}}

    if rank == 0:
        name, params = WORKLOADS[args.workload]
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_step, 3), "higher_is_better": True,
            "scaling": args.scaling if world > 1 else "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic",
            "mem_records_per_s": round(total_mem * args.steps / (ms_max / 1e3), 1),
            "config": {"workload": args.workload, "generator": name, "params": params,
                       "records_per_gpu": n, "mem_records_per_gpu": int(((t.meta & 3) < 2).sum()),
                       "line_bytes": lb, "warp_size": 32, "rd_scope": args.rd_scope, "rd_bins": "linear 66",
                       "analyses": ("load_trace + reuse + mem_div + branch_div (three calls)" if args.separate else
                                    "load_trace + cadv_analyze(reuse, mem_div, branch_div: one fused pass)"),
                       "l2": "inputs larger than L2 (trace >> 126 MB), no flush needed",
                       "global_records": gtotal, "sharding": mode, "src_sha": src_sha(),
                       "parallelism": (f"position-range shards of one trace over {world} GPUs (library NCCL: "
                                       "kept records exchanged by CTA range, T_c max, histograms all-reduced)"
                                       if mode == "position" else
                                       f"dp{world} (independent trace per GPU, histograms all-reduced)"
                                       if world > 1 else "single GPU")},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": ck, "kernels": kernels, "per_analysis": per_an, "data_centric": dcen,
        }
        print(json.dumps(line), flush=True)
    ctx.destroy()
    if world > 1:
        dist.destroy_process_group()


def run_reference(args, rank, world):
    """The oracle as it stands, on this host's cores, one bounded sample per step."""
    if rank != 0:
        return
    import oracle as orc
    import tracegen as tg
    name, params = WORKLOADS[args.workload]
    lb = args.line_bytes
    # a bounded sample: the first launch's worth of records, capped
    t = make_trace(args.workload, 0, 1, args.sharding, pinned=False)[0]
    nsamp, dt_probe, cores, desc = oracle_sample(t, max(args.cpu_seconds / 2, 2.0), lb)
    sub = tg.from_arrays(*(t.cols[k][:nsamp] for k, _ in tg.COLUMNS), nsites=t.nsites)

    def step():
        orc.reuse(sub, lb, 0, 0, 66)
        orc.mem_div(sub, lb, 32)
        orc.branch_div(sub, 32)

    for _ in range(args.warmup):
        step()
    t0 = time.time()
    for _ in range(args.steps):
        step()
    dt = time.time() - t0
    value = nsamp * args.steps / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * dt / max(args.steps, 1), 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": args.workload, "generator": name, "params": params, "line_bytes": lb,
                   "sample_records": nsamp},
        "cpu_baseline": {"value": round(value, 1), "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": desc, "cpu_model": cpu_model()},
        "e2e": {"value": round(value, 1), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
