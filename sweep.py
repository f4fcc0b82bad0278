#!/usr/bin/env python
"""Exhaustive launch sweep (validates the adaptive selector, §8(a) A4; PAPER.md
§III-A Fig. 4 L157-167 and §IV-B).

For each mode of a config: time sf_mttkrp under every launch in a grid
(kernel x staged-mode subset x block rows x chunk length x threads), then report the
selector's pick, its rank and its throughput relative to the sweep best.
Writes one JSON object per line to stdout (and --out).
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def time_launch(T, n, R, facs, out, L, sf, torch, reps=5):
    try:
        T.set_launch(n, R, L)
    except sf.SfError as e:
        return None, str(e)
    s = torch.cuda.current_stream()
    for _ in range(2):
        T.mttkrp(n, facs, out)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(reps):
        T.mttkrp(n, facs, out)
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps, None


def grid(dims, n, R, quick):
    others = [m for m in range(len(dims)) if m != n]
    row_opts = [128, 256, 384, 512, 775] if not quick else [256, 512]
    chunks = [64, 128, 256, 512] if not quick else [128]
    threads = [256, 512, 1024] if not quick else [512]
    staged_sets = [()]
    for k in range(1, len(others) + 1):
        staged_sets += list(itertools.combinations(others, k))
    for st in staged_sets:
        opts = {m: sorted(set(row_opts + ([dims[m]] if dims[m] <= 2048 else []))) for m in st}
        rows_choices = [()] if not st else itertools.product(*[opts[m] for m in st])
        for rows in rows_choices:
            for C, th, fl in itertools.product(chunks, threads, (0,) if not st else (8,)):
                yield {"kernel": 2, "block_threads": th, "chunk_nnz": C, "flags": fl & ~8,
                       "staged": {m: min(r, dims[m]) for m, r in zip(st, rows)}}
    # L2-tiled plans (SF_LAUNCH_L2_TILES = 64): one gathered factor >= 16 MB in 16/32/64 MB blocks
    for m in others:
        fac = dims[m] * R * 4
        if fac < 16 * 2**20:
            continue
        for mb in ((64,) if quick else (16, 32, 64)):
            rows = int(mb * 2**20 / (R * 4))
            if rows >= dims[m]:
                continue
            for C, th in itertools.product(chunks, threads):
                yield {"kernel": 2, "block_threads": th, "chunk_nnz": C, "flags": 64, "staged": {m: rows}}
    yield {"kernel": 1}


def grid_sparse(dims, n, R):
    """Exhaustive grid for hyper-sparse modes (gathered factors >> L2, SURVEY C-6): unstaged
    (owner stores / memset + atomics), L2 tiles of every gathered factor >= 16 MB in
    16/32/64/128 MB blocks (one mode, and two modes), each with hot-row caches of
    0/8/16/32/64/128 MB, x chunk length x threads; shared-memory block staging for contrast."""
    others = [m for m in range(len(dims)) if m != n]
    hots = [0, 8, 16, 32, 64, 128]
    for fl in (0, 4):
        for C, th, hb in itertools.product([64, 128, 256], [512, 1024], hots):
            yield {"kernel": 2, "block_threads": th, "chunk_nnz": C, "flags": fl, "staged": {}, "hot_kb": hb * 1024}
    big = [m for m in others if dims[m] * R * 4 >= 16 * 2**20]
    for m in big:
        for mb in (16, 32, 64, 128):
            rows = int(mb * 2**20 / (R * 4))
            if rows >= dims[m]:
                continue
            for C, th, hb in itertools.product([128, 256], [512, 1024], hots):
                yield {"kernel": 2, "block_threads": th, "chunk_nnz": C, "flags": 64, "staged": {m: rows},
                       "hot_kb": hb * 1024}
    for a, b in itertools.combinations(big, 2):
        for mb in (32, 64):
            ra, rb = (min(int(mb * 2**20 / (R * 4)), dims[x]) for x in (a, b))
            for hb in (0, 16, 32):
                yield {"kernel": 2, "block_threads": 512, "chunk_nnz": 128, "flags": 64, "staged": {a: ra, b: rb},
                       "hot_kb": hb * 1024}
    for m in others:
        for rows in (256, 512):
            yield {"kernel": 2, "block_threads": 512, "chunk_nnz": 128, "flags": 0, "staged": {m: min(rows, dims[m])}}
    yield {"kernel": 1}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="nell2")
    ap.add_argument("--modes", default=None)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--sparse", action="store_true", help="the hyper-sparse grid (grid_sparse)")
    ap.add_argument("--out", default=None)
    ap.add_argument("--only-staged", default=None, help="restrict to this staged set, e.g. '1:256'")
    args = ap.parse_args()
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[args.config]
    inds, vals = synth.config_tensor_device(cfg)
    facs = synth.config_factors_device(cfg)
    R = cfg.rank
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    modes = [int(x) for x in args.modes.split(",")] if args.modes else range(cfg.nmodes)
    outf = open(args.out, "w") if args.out else None
    flops = cfg.nmodes * cfg.nnz * R
    for n in modes:
        out = torch.empty((cfg.dims[n], R), device="cuda")
        T.plan(n, R)
        pick = T.plan_info(n, R)["launch"]
        t_pick, _ = time_launch(T, n, R, facs, out, sf.Launch.make(
            kernel=2 if pick["kernel"] == "frag" else 1, block_threads=pick["block_threads"],
            ctas_per_sm=pick["ctas_per_sm"], chunk_nnz=pick["chunk_nnz"],
            staged={m: r for m, r in enumerate(pick["block_rows"]) if pick["staged_mask"] >> m & 1},
            flags=pick.get("flags", 0), hot_kb=pick.get("hot_kb", 0)),
            sf, torch)
        results = []
        t0 = time.time()
        for g in (grid_sparse(cfg.dims, n, R) if args.sparse else grid(cfg.dims, n, R, args.quick)):
            if args.only_staged is not None:
                want = {} if args.only_staged == "none" else {int(a): int(b) for a, b in
                                                              (x.split(":") for x in args.only_staged.split(","))}
                if g.get("kernel") != 2 or g.get("staged") != want:
                    continue
            L = sf.Launch.make(**g)
            ms, err = time_launch(T, n, R, facs, out, L, sf, torch)
            rec = {"mode": n, "launch": g, "ms": ms, "err": err,
                   "gflops": flops / cfg.nmodes / ms / 1e6 if ms else None}
            results.append(rec)
            line = json.dumps(rec)
            print(line, flush=True)
            if outf:
                outf.write(line + "\n")
                outf.flush()
        ok = sorted([r for r in results if r["ms"]], key=lambda r: r["ms"])
        best = ok[0]
        rank_of_pick = sum(1 for r in ok if r["ms"] < t_pick) + 1
        summ = {"summary": True, "config": cfg.name, "mode": n, "pick": pick, "pick_ms": t_pick,
                "best": best["launch"], "best_ms": best["ms"], "pick_over_best": best["ms"] / t_pick,
                "pick_rank": rank_of_pick, "n_launches": len(ok), "sweep_s": time.time() - t0}
        print(json.dumps(summ), flush=True)
        if outf:
            outf.write(json.dumps(summ) + "\n")
            outf.flush()
        T.plan_release(n, R)  # one plan resident at a time (amazon: 1.74 B nonzeros)
        del out
        torch.cuda.empty_cache()
    T.close()


if __name__ == "__main__":
    main()
