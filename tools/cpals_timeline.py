#!/usr/bin/env python
"""Where a CP-ALS sweep's device time goes (sf_cpals on a planned tensor): GPU kernels of a
few sweeps recorded with torch.profiler (CUPTI), summed per kernel name, plus the host wall
time per sweep.

  python tools/cpals_timeline.py nell1 [--iters 3]
"""
import argparse
import collections
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="nell1")
    ap.add_argument("--iters", type=int, default=3)
    args = ap.parse_args()
    import torch
    from torch.profiler import ProfilerActivity, profile

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[args.config]
    R = cfg.rank
    inds, vals = synth.config_tensor_device(cfg)
    facs = synth.config_factors_device(cfg)
    with sf.Tensor(cfg.dims, inds, vals) as T:
        del inds, vals
        A = [f.clone() for f in facs]
        T.cp_als(A, iters=1)  # plans + warm-up
        torch.cuda.synchronize()
        A = [f.clone() for f in facs]
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            t0 = time.perf_counter()
            T.cp_als(A, iters=args.iters)
            torch.cuda.synchronize()
            wall = (time.perf_counter() - t0) * 1e3
        by = collections.Counter()
        for e in prof.events():
            if e.device_type == torch.autograd.DeviceType.CUDA:
                by[e.name[:80]] += e.time_range.end - e.time_range.start
        total = sum(by.values())
        print(json.dumps({"config": cfg.name, "iters": args.iters, "wall_ms_per_sweep": wall / args.iters,
                          "gpu_ms_per_sweep": total / 1e3 / args.iters,
                          "per_kernel_ms_per_sweep": {k: round(v / 1e3 / args.iters, 3) for k, v in by.most_common(15)}}))


if __name__ == "__main__":
    main()
