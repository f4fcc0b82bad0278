#!/usr/bin/env python
"""Held-out check of the hot-row selection rules: random hyper-sparse tensors
that are NOT BASELINE.json / Table III shapes (random N, R, dims, nnz, Zipf exponents; seeds
disjoint from every other study).  For every mode: the selector's pick, the pick with the
hot-row rules disabled (SF_DEBUG=no_hot: round 1's tree + L2-tile rule), the hot-row class with
and without L2 tiles of each gathered factor (2^19-row blocks, 16 / 32 MB hot), and the
unstaged plan without hot rows.  One JSON line per mode with every time and pick / best.

  python tools/hot_heldout.py --count 12 --seed 77
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def random_tensor(rng, k):
    N = int(rng.choice([3, 3, 4]))
    R = int(rng.choice([16, 32]))
    nnz = int(10 ** rng.uniform(7.3, 8.1))
    dims = [int(10 ** rng.uniform(5.5, 7.4)) for _ in range(N)]
    if N == 4:
        dims[int(rng.integers(0, 4))] = int(10 ** rng.uniform(2.5, 4))  # one short mode, like deli/flickr
    zipf = [float(rng.choice([0.5, 0.7, 0.8, 1.0, 1.2])) for _ in range(N)]
    return dict(name=f"heldout{k}", dims=dims, nnz=nnz, rank=R, zipf=zipf, seed=91000000 + 101 * k)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--count", type=int, default=12)
    ap.add_argument("--seed", type=int, default=77)
    ap.add_argument("--configs", default="", help="also run these named configs (synth.CONFIGS)")
    args = ap.parse_args()
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    rng = np.random.default_rng(args.seed)
    s = torch.cuda.Stream()

    def time_it(T, n, R, facs, out):
        for _ in range(2):
            T.mttkrp(n, facs, out, stream=s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(5):
            T.mttkrp(n, facs, out, stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / 5

    tensors = [random_tensor(rng, k) for k in range(args.count)]
    for name in [x for x in args.configs.split(",") if x]:
        cfg = synth.CONFIGS[name]
        tensors.append(dict(name=name, dims=list(cfg.dims), nnz=cfg.nnz, rank=cfg.rank, zipf=list(cfg.zipf),
                            seed=cfg.seed, config=name))
    for c in tensors:
        R, N = c["rank"], len(c["dims"])
        if "config" in c:
            inds, vals = synth.config_tensor_device(synth.CONFIGS[c["config"]])
            facs = synth.config_factors_device(synth.CONFIGS[c["config"]])
        else:
            inds, vals = synth.gen_coo_device(c["dims"], c["nnz"], c["seed"], c["zipf"])
            facs = synth.gen_factors_device(c["dims"], R, c["seed"] + 7)
        # exact row counts per mode -> hot coverage (share of nonzeros in the hottest 16 MB of rows)
        counts = [torch.bincount(a.long(), minlength=d) for a, d in zip(inds, c["dims"])]
        hot_rows = (16 << 20) // (4 * R)
        cover = [float(torch.topk(cn, min(hot_rows, cn.numel())).values.sum()) / c["nnz"] for cn in counts]
        with sf.Tensor(c["dims"], inds, vals) as T:
            del inds, vals
            for n in range(N):
                out = torch.empty((c["dims"][n], R), device="cuda")
                cn = counts[n].double()
                rho = {}
                for m in range(N):
                    if m != n and c["dims"][m] > (1 << 19):
                        Tt = -(-c["dims"][m] // (1 << 19))
                        rho[m] = float(Tt * (1 - torch.exp(-1.44 * cn / Tt)).sum() / c["nnz"])
                times = {}
                auto = sf.Launch()
                auto.kernel = 0
                T.set_launch(n, R, auto)
                pick = T.plan_info(n, R)["launch"]
                times["pick"] = time_it(T, n, R, facs, out)
                os.environ["SF_DEBUG"] = "no_hot"
                T.set_launch(n, R, auto)
                os.environ.pop("SF_DEBUG", None)
                nohot = T.plan_info(n, R)["launch"]
                times["no_hot_rules"] = time_it(T, n, R, facs, out)
                chunk = 64 if R >= 32 else 128
                variants = {"unstaged": sf.Launch.make(kernel=sf.KERNEL_FRAG, block_threads=1024, chunk_nnz=chunk),
                            "hot32": sf.Launch.make(kernel=sf.KERNEL_FRAG, block_threads=1024, chunk_nnz=chunk,
                                                    hot_kb=32 << 10)}
                for m in range(N):
                    if m == n or c["dims"][m] <= (1 << 19):
                        continue
                    for hot in (16, 32):
                        variants[f"tile{m}+hot{hot}"] = sf.Launch.make(
                            kernel=sf.KERNEL_FRAG, block_threads=1024, chunk_nnz=128, staged={m: 1 << 19},
                            flags=sf.LAUNCH_L2_TILES, hot_kb=hot << 10)
                for name, L in variants.items():
                    try:
                        T.set_launch(n, R, L)
                        times[name] = time_it(T, n, R, facs, out)
                    except sf.SfError:
                        times[name] = None
                T.plan_release(n, R)
                del out
                torch.cuda.empty_cache()
                ok = {k2: v for k2, v in times.items() if v}
                best = min(ok.values())
                print(json.dumps({"tensor": c, "mode": n, "pick": pick, "no_hot_pick": nohot, "cover": cover,
                                  "rho": rho, "y_mb": c["dims"][n] * R * 4 / 2**20,
                                  "times_ms": {k2: (round(v, 4) if v else None) for k2, v in times.items()},
                                  "pick_over_best": best / times["pick"],
                                  "no_hot_over_best": best / times["no_hot_rules"]}), flush=True)
        del facs, counts
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
