"""One data-centric call (cadv_data_centric) on a bench workload, bracketed by
cudaProfilerStart/Stop for `ncu --profile-from-start off` (the bench's
--profile-run covers the fused analysis only).
usage: python tools/dc_profile.py [workload]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_shensll18_b200 as cadv  # noqa: E402
import tracegen as tg  # noqa: E402


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "c4_srad"
    name, params = bench.WORKLOADS[wl]
    t = tg.generate(name, **params)
    objs = tg.objects(name, **params)
    with cadv.create(0) as ctx:
        ctx.load_trace(cadv.to_device(t))
        for _ in range(2):
            ctx.data_centric(objs, 128, 0, cadv.BINS_LINEAR, 66, 32)
        torch.cuda.synchronize()
        torch.cuda.profiler.start()
        ctx.data_centric(objs, 128, 0, cadv.BINS_LINEAR, 66, 32)
        torch.cuda.synchronize()
        torch.cuda.profiler.stop()
    print("data-centric call profiled:", wl, t.n, "records", len(objs[0]), "objects")


if __name__ == "__main__":
    main()
