#!/usr/bin/env python
"""L2-tiled schedule study (SF_LAUNCH_L2_TILES; DESIGN.md §5 "L2 tiles").

For every mode of the given configs: time the selector's launch, then the unstaged
frag3 launch with one gathered mode tiled into L2-sized row blocks (every CTA sweeps the
tiles in the same order), for each gathered factor larger than --min-mb and a few block
sizes.  One JSON line per (config, mode, launch) to stdout.

usage: python tools/l2tile_study.py nell1,amazon,deli4d
"""
from __future__ import annotations

import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def random_configs(count, seed):
    """Held-out check of the selection rule: random tensors (never a BASELINE/Table III shape)
    large enough that gathered factors exceed L2."""
    import numpy as np
    rng = np.random.default_rng(seed)
    out = []
    for k in range(count):
        N = int(rng.choice([3, 3, 4]))
        R = int(rng.choice([16, 32]))
        nnz = int(10 ** rng.uniform(7.5, 8.2))
        dims = [int(10 ** rng.uniform(4.0, 7.3)) for _ in range(N)]
        zipf = [float(rng.choice([0.0, 0.5, 0.8, 1.0, 1.2])) for _ in range(N)]
        out.append(synth.Config(f"rand{k}", tuple(dims), nnz, R, tuple(zipf), 40000000 + k, 40001000 + k,
                                "random held-out tensor (tools/l2tile_study.py)"))
    return out


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["nell1"]
    if names[0].startswith("random"):  # random:COUNT:SEED
        _, cnt, sd = (names[0].split(":") + ["8", "1"])[:3]
        cfgs = random_configs(int(cnt), int(sd))
    else:
        cfgs = [synth.CONFIGS[nm] for nm in names]
    min_mb = float(os.environ.get("MIN_MB", "24"))
    block_mb = [float(x) for x in os.environ.get("BLOCK_MB", "16,32,64").split(",")]
    for cfg in cfgs:
        name = cfg.name
        d_inds, d_vals = synth.config_tensor_device(cfg)
        facs = synth.config_factors_device(cfg)
        R = cfg.rank
        T = sf.Tensor(cfg.dims, d_inds, d_vals)
        del d_inds, d_vals
        torch.cuda.empty_cache()
        s = torch.cuda.current_stream()

        def timed(n, out, reps=5):
            for _ in range(2):
                T.mttkrp(n, facs, out)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(reps):
                T.mttkrp(n, facs, out)
            e1.record(s)
            torch.cuda.synchronize()
            return e0.elapsed_time(e1) / reps

        for n in range(cfg.nmodes):
            out = torch.empty((cfg.dims[n], R), dtype=torch.float32, device="cuda")
            # the selector without the L2-tile rule is the reference ("auto"); with it: "rule"
            os.environ["SF_DEBUG"] = "no_l2tiles"
            T.plan(n, R)
            auto = timed(n, out)
            ref = out.clone()
            info = T.plan_info(n, R)
            print(json.dumps({"config": name, "dims": list(cfg.dims), "nnz": cfg.nnz, "rank": R, "mode": n,
                              "launch": "auto", "ms": auto, "picked": info["launch"]}), flush=True)
            T.plan_release(n, R)
            os.environ.pop("SF_DEBUG", None)
            T.plan(n, R)
            ms = timed(n, out)
            print(json.dumps({"config": name, "mode": n, "launch": "rule", "ms": ms, "speedup_vs_auto": auto / ms,
                              "picked": T.plan_info(n, R)["launch"]}), flush=True)
            T.plan_release(n, R)
            for m in range(cfg.nmodes):
                fac_mb = cfg.dims[m] * R * 4 / 2**20
                if m == n or fac_mb < min_mb:
                    continue
                for bmb in block_mb:
                    rows = int(bmb * 2**20 / (R * 4))
                    if rows >= cfg.dims[m]:
                        continue
                    for flags in (sf.LAUNCH_L2_TILES,):
                        L = sf.Launch.make(kernel=sf.KERNEL_FRAG, chunk_nnz=128, staged={m: rows}, flags=flags)
                        try:
                            T.set_launch(n, R, L)
                        except sf.SfError as e:
                            print(json.dumps({"config": name, "mode": n, "tiled": m, "err": str(e)}), flush=True)
                            continue
                        ms = timed(n, out)
                        rel = float(((out - ref).abs().max() / ref.abs().max().clamp_min(1e-30)).item())
                        print(json.dumps({"config": name, "mode": n, "launch": "l2tiles", "tiled": m,
                                          "fac_mb": round(fac_mb, 1), "block_mb": bmb, "rows": rows,
                                          "tiles": T.plan_info(n, R)["num_tiles"], "ms": ms,
                                          "speedup_vs_auto": auto / ms, "max_rel_diff_vs_auto": rel}),
                              flush=True)
                        T.plan_release(n, R)
            # two tiled modes (every gathered factor above MIN_MB), 32 MB blocks each
            big = [m for m in range(cfg.nmodes) if m != n and cfg.dims[m] * R * 4 / 2**20 >= min_mb]
            if len(big) >= 2:
                rows = int(32 * 2**20 / (R * 4))
                staged = {m: min(rows, cfg.dims[m]) for m in big[:2]}
                L = sf.Launch.make(kernel=sf.KERNEL_FRAG, chunk_nnz=128, staged=staged, flags=sf.LAUNCH_L2_TILES)
                T.set_launch(n, R, L)
                ms = timed(n, out)
                print(json.dumps({"config": name, "mode": n, "launch": "l2tiles2", "tiled": big[:2], "block_mb": 32,
                                  "tiles": T.plan_info(n, R)["num_tiles"], "ms": ms, "speedup_vs_auto": auto / ms}),
                      flush=True)
                T.plan_release(n, R)
            del out, ref
            torch.cuda.empty_cache()
        T.close()
        del facs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
