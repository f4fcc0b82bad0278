#!/usr/bin/env python
"""Hot-row cache budget sweep (launch.hot_kb; DESIGN.md §5 "hot-row cache").

For every mode of a config: take the selector's launch, then re-plan it with hot_kb in
{0, 16, 32, 64, 128, 256} MiB (and, for L2-tiled picks, the same without the L2 tiles) and time
10 sf_mttkrp launches each (CUDA events, 3 warm-up).  One JSON line per (mode, variant).

  python tools/hot_sweep.py nell1,deli4d [--budgets 0,32,64,128]
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
    ap.add_argument("configs")
    ap.add_argument("--budgets", default="0,16,32,64,128,256")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--modes", default=None)
    ap.add_argument("--no-tiles-variant", action="store_true", help="only the selector's tiling choice")
    args = ap.parse_args()
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    budgets = [int(x) for x in args.budgets.split(",")]
    for name in args.configs.split(","):
        cfg = synth.CONFIGS[name]
        R, N = cfg.rank, cfg.nmodes
        facs = synth.config_factors_device(cfg)
        inds, vals = synth.config_tensor_device(cfg)
        T = sf.Tensor(cfg.dims, inds, vals)
        del inds, vals
        torch.cuda.empty_cache()
        s = torch.cuda.Stream()
        modes = range(N) if args.modes is None else [int(x) for x in args.modes.split(",")]
        for n in modes:
            T.plan(n, R)
            base = T.plan_info(n, R)["launch"]
            out = torch.empty((cfg.dims[n], R), dtype=torch.float32, device="cuda")
            variants = []
            tv = [True, False] if (base["flags"] & sf.LAUNCH_L2_TILES) and not args.no_tiles_variant else [None]
            for tiles in tv:
                for hb in budgets:
                    variants.append((tiles, hb))
            for tiles, hb in variants:
                staged = {m: base["block_rows"][m] for m in range(N) if base["staged_mask"] >> m & 1}
                flags = base["flags"]
                if tiles is False:
                    staged, flags = {}, flags & ~sf.LAUNCH_L2_TILES
                L = sf.Launch.make(kernel=sf.KERNEL_FRAG, block_threads=base["block_threads"],
                                   ctas_per_sm=base["ctas_per_sm"], chunk_nnz=base["chunk_nnz"], staged=staged,
                                   flags=flags, hot_kb=hb * 1024)
                T.set_launch(n, R, L)
                info = T.plan_info(n, R)
                for _ in range(3):
                    T.mttkrp(n, facs, out, stream=s)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for _ in range(args.reps):
                    T.mttkrp(n, facs, out, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / args.reps
                print(json.dumps({"config": name, "mode": n, "l2tiles": bool(flags & sf.LAUNCH_L2_TILES),
                                  "hot_mb": hb, "ms": round(ms, 4),
                                  "plan_ms": round(info["plan_ms"], 2), "selector": base}), flush=True)
            T.plan_release(n, R)
            del out
            torch.cuda.empty_cache()
        T.close()
        del facs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
