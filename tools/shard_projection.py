#!/usr/bin/env python
"""Projected multi-GPU scaling from shards timed one at a time on ONE B200 (gpurun gives one
GPU).  For P in --ranks, every rank's shard of every mode (sf_set_shard(P, p),
the exact plans a P-GPU run builds) is planned by the selector and its sf_mttkrp timed
(CUDA events, 3 warm-up + --reps launches); a P-GPU step would take the max over ranks of the
per-rank step (ranks run concurrently on their own GPUs, each with its own HBM and L2) plus the
boundary exchange (one allgather of R*4 bytes per rank and mode: microseconds on NVLink, not
included).  Prints one JSON line per P: per-rank step ms, the max, and speedup vs P = 1.

  python tools/shard_projection.py amazon --ranks 1,2,4,8
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--ranks", default="1,2,4,8")
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[args.config]
    R, N = cfg.rank, cfg.nmodes
    facs = synth.config_factors_device(cfg)
    inds, vals = synth.config_tensor_device(cfg)
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    s = torch.cuda.Stream()
    base = None
    for P in [int(x) for x in args.ranks.split(",")]:
        per_rank = []
        for p in range(P):
            T.set_shard(P, p)
            step = 0.0
            modes = {}
            for n in range(N):
                T.plan(n, R)
                info = T.plan_info(n, R)
                out = torch.empty((max(1, info["out_rows"]), R), device="cuda")
                for _ in range(3):
                    T.mttkrp(n, facs, out, stream=s)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for _ in range(args.reps):
                    T.mttkrp(n, facs, out, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / args.reps
                modes[n] = {"ms": round(ms, 4), "nnz_local": info["nnz_local"], "hot_kb": info["launch"]["hot_kb"],
                            "l2tiles": bool(info["launch"]["flags"] & sf.LAUNCH_L2_TILES)}
                step += ms
                T.plan_release(n, R)
                del out
                torch.cuda.empty_cache()
            per_rank.append({"rank": p, "step_ms": round(step, 4), "modes": modes})
        mx = max(r["step_ms"] for r in per_rank)
        if base is None and P == 1:
            base = mx
        flops = N * N * cfg.nnz * R
        print(json.dumps({"config": cfg.name, "P": P, "max_rank_step_ms": mx,
                          "projected_gflops": flops / (mx * 1e-3) / 1e9,
                          "speedup_vs_1": (base / mx) if base else None,
                          "balance": min(r["step_ms"] for r in per_rank) / mx, "per_rank": per_rank}), flush=True)
    T.close()


if __name__ == "__main__":
    main()
