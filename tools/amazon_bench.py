#!/usr/bin/env python
"""Largest config (BASELINE.json configs[4], amazon-reviews-shaped, nnz = 1.74 B, R = 16) on ONE
B200: bench.py keeps every mode's plan resident, which does not fit 180 GB for this tensor, so
here each mode is planned by the selector, timed (CUDA events, warm-up first, 10 launches) and
released before the next.  Prints one JSON line: per-mode ms, plan ms, launch, and the
all-modes GFLOP/s (N*nnz*R per mode) -- the 1-GPU point of the N = 1/8 scaling target."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "amazon"]
    R, N = cfg.rank, cfg.nmodes
    facs = synth.config_factors_device(cfg)
    inds, vals = synth.config_tensor_device(cfg)
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    s = torch.cuda.current_stream()
    per_mode = {}
    for n in range(N):
        T.plan(n, R)
        info = T.plan_info(n, R)
        out = torch.empty((cfg.dims[n], R), dtype=torch.float32, device="cuda")
        for _ in range(3):
            T.mttkrp(n, facs, out)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(10):
            T.mttkrp(n, facs, out)
        e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        per_mode[n] = {"ms": ms, "gflops": N * cfg.nnz * R / (ms * 1e-3) / 1e9, "plan_ms": info["plan_ms"],
                       "launch": info["launch"], "num_tiles": info["num_tiles"]}
        del out
        T.plan_release(n, R)
        torch.cuda.empty_cache()
    step = sum(v["ms"] for v in per_mode.values())
    print(json.dumps({"config": cfg.name, "nnz": cfg.nnz, "rank": R, "dims": list(cfg.dims),
                      "value": N * N * cfg.nnz * R / (step * 1e-3) / 1e9, "unit": "GFLOP/s",
                      "ms_per_step": step, "per_mode": per_mode,
                      "note": "one plan resident at a time (plan, time, release per mode)"}))
    T.close()


if __name__ == "__main__":
    main()
