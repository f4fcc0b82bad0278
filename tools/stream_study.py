#!/usr/bin/env python
"""segments x streams study of the paper's pipeline (§IV-C
L201-229, Fig. 11 "fix the number of segments to 4 ... fix the number of CUDA
streams to 4"), on B200 with synthetic tensors shaped like the paper's workloads.

For a host-resident (pinned) COO tensor and one mode (and, under "all_modes_one_upload", every
mode from one upload with sf_mttkrp_streamed_modes):
  T_h2d      the COO upload alone (cudaMemcpy of the N+1 arrays)
  T_(1,1)    sf_mttkrp_streamed with 1 segment on 1 stream (no overlap)
  T_compute  = T_(1,1) - T_h2d
  T_(S,K)    sf_mttkrp_streamed with S segments over K streams
  overlap    = (T_h2d + T_compute - T_(S,K)) / min(T_h2d, T_compute)
and, for comparison, the resident path (create + plan + fragment MTTKRP) end to end.
"""
from __future__ import annotations

import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["vast", "nell2"]
    out = {}
    for name in names:
        cfg = synth.CONFIGS[name]
        d_inds, d_vals = synth.config_tensor_device(cfg)
        h_inds = [a.cpu().pin_memory() for a in d_inds]
        h_vals = d_vals.cpu().pin_memory()
        del d_inds, d_vals
        facs = synth.config_factors_device(cfg)
        n = 0
        R = cfg.rank
        y = torch.empty((cfg.dims[n], R), device="cuda")
        dev_bufs = [torch.empty_like(a, device="cuda") for a in h_inds] + [torch.empty_like(h_vals, device="cuda")]

        def wall(fn, reps=5):
            fn()
            torch.cuda.synchronize()
            ts = []
            for _ in range(reps):
                t0 = time.perf_counter()
                fn()
                torch.cuda.synchronize()
                ts.append(time.perf_counter() - t0)
            return float(np.median(ts)) * 1e3

        def h2d():
            for dbuf, h in zip(dev_bufs, h_inds + [h_vals]):
                dbuf.copy_(h, non_blocking=True)

        t_h2d = wall(h2d)
        h_y = torch.empty((cfg.dims[n], R), dtype=torch.float32).pin_memory()

        def d2h():
            h_y.copy_(y, non_blocking=True)
        t_d2h = wall(d2h)
        grid = {}
        for S in (1, 2, 4, 8, 16, 32):
            for K in (1, 2, 4, 8):
                if K > S:
                    continue
                grid[f"{S}x{K}"] = wall(lambda: sf.mttkrp_streamed(cfg.dims, h_inds, h_vals, facs, n, y, S, K))
        t11 = grid["1x1"]
        t_comp = max(t11 - t_h2d, 1e-6)
        ov = {k: (t_h2d + t_comp - v) / min(t_h2d, t_comp) for k, v in grid.items()}

        # every mode from one upload (sf_mttkrp_streamed_modes): the N MTTKRPs of a step
        ys = [torch.empty((d, R), device="cuda") for d in cfg.dims]
        reps_all = 2 if cfg.nnz > 5e8 else 5
        grid_all = {}
        for S in (1, 4, 8, 16, 32):
            for K in (1, 2, 4):
                if K > S:
                    continue
                grid_all[f"{S}x{K}"] = wall(lambda: sf.mttkrp_streamed_modes(cfg.dims, h_inds, h_vals, facs, ys, S, K),
                                            reps=reps_all)
        t11a = grid_all["1x1"]
        t_comp_all = max(t11a - t_h2d, 1e-6)
        ov_all = {k: (t_h2d + t_comp_all - v) / min(t_h2d, t_comp_all) for k, v in grid_all.items()}
        best_all = min(grid_all, key=grid_all.get)
        all_modes = {"t_streamed_ms": grid_all, "t_compute_ms": t_comp_all, "overlap_ratio": ov_all,
                     "best": best_all, "best_over_h2d": grid_all[best_all] / t_h2d,
                     "speedup_best_vs_1x1": t11a / grid_all[best_all]}
        del ys

        def resident():
            with sf.Tensor(cfg.dims, h_inds, h_vals, segments=8, streams=4) as T:
                T.plan(n, R)
                T.mttkrp(n, facs, y)
                torch.cuda.synchronize()
        t_res = wall(resident, reps=3)
        best = min(grid, key=grid.get)
        # device footprint of the streamed path (O(streams x segment), not O(tensor): tensors larger
        # than HBM stream through it) at 32 segments / 4 streams vs the tensor's bytes
        sf.device_bytes(reset_peak=True)
        sf.mttkrp_streamed(cfg.dims, h_inds, h_vals, facs, n, y, 32, 4)
        torch.cuda.synchronize()
        peak_streamed = sf.device_bytes()[1]
        out[name] = {"nnz": cfg.nnz, "bytes_h2d": int(sum(a.numel() * 4 for a in h_inds) + h_vals.numel() * 4),
                     "t_h2d_ms": t_h2d, "h2d_GBps": (sum(a.numel() * 4 for a in h_inds) + h_vals.numel() * 4) / t_h2d / 1e6,
                     "t_compute_ms": t_comp, "t_streamed_ms": grid, "overlap_ratio": ov,
                     "best": best, "speedup_best_vs_1x1": t11 / grid[best],
                     "t_resident_path_ms": t_res, "mode": n, "t_d2h_ms": t_d2h,
                     "breakdown_ms": {"h2d": t_h2d, "kernel": t_comp, "d2h": t_d2h,
                                      "serial_sum": t_h2d + t_comp + t_d2h,
                                      "streamed_best_plus_d2h": grid[best] + t_d2h},
                     "streamed_peak_device_bytes_32seg": int(peak_streamed),
                     "all_modes_one_upload": all_modes}
        print(json.dumps({name: out[name]}), flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    path = os.path.join(ROOT, "gpurun_out", "stream_study.json")
    json.dump(out, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
