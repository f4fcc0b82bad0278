#!/usr/bin/env python
"""Offline calibration of the L2-tile cost model (sf_select.cpp `l2_tile_choice`).

Model (per mode n, unstaged frag3 plan, factor rows of RB = 4R bytes):
  * an ideal frequency-ordered L2 of C bytes holds the hottest gathered rows (all gathered
    modes compete; the per-row frequency histogram of each mode in log2 bins);
  * misses cost RB bytes of DRAM each;
  * tiling gathered mode m into blocks of B bytes makes every mode-m gather a hit (its
    rows cost F_m once), leaves C - B for the other modes' hot rows, and revisits Y once
    per (tile, touched row): 2 RB bytes each unless Y fits in L2 next to the block.
Inputs: gpurun_out/c13_rowfreq.jsonl (tools/row_freq_dump.py) and the measured study
lines (tools/l2tile_study.py).  Prints predicted vs measured speedups.
"""
import json
import math
import sys


def hot_hits(hists, cap_rows):
    """Nonzeros served by the cap_rows hottest rows over the given (rows, nnz) histograms."""
    bins = []
    for rows, nnz in hists:
        for b in range(len(rows)):
            if rows[b]:
                bins.append((nnz[b] / rows[b], rows[b], nnz[b]))
    bins.sort(reverse=True)
    hits, left = 0.0, cap_rows
    for f, r, z in bins:
        if left <= 0:
            break
        take = min(r, left)
        hits += take * f
        left -= take
    return hits


def touched(hist, T):
    rows, nnz = hist
    return sum(r * (1.0 - math.exp(-(z / r) / T)) for r, z in zip(rows, nnz) if r)


def model(cfg, n, C, tiled=None, block_bytes=0):
    R = cfg["rank"]
    RB = 4 * R
    nnz = cfg["nnz"]
    dims = cfg["dims"]
    G = [m for m in range(len(dims)) if m != n]
    hist = {m: (cfg["modes"][m]["rows"], cfg["modes"][m]["nnz"]) for m in range(len(dims))}
    stream = 16 * nnz
    if tiled is None:
        hits = hot_hits([hist[m] for m in G], C / RB)
        return stream + (len(G) * nnz - hits) * RB + dims[n] * RB
    others = [m for m in G if m != tiled]
    T = math.ceil(dims[tiled] * RB / block_bytes)
    cap = max(0.0, C - block_bytes)
    hits = hot_hits([hist[m] for m in others], cap / RB)
    miss = (len(others) * nnz - hits) * RB + dims[tiled] * RB
    ybytes = dims[n] * RB
    yrev = 0.0 if ybytes + block_bytes <= C else 2 * RB * T * touched(hist[n], T)
    return stream + miss + yrev + ybytes


def main():
    freq = {}
    for line in open(sys.argv[1]):
        d = json.loads(line)
        freq[d["config"]] = d
    meas = {}
    for path in sys.argv[2:]:
        for line in open(path):
            d = json.loads(line)
            if "ms" not in d:
                continue
            key = (d["config"], d["mode"])
            meas.setdefault(key, []).append(d)
    for C_mb in (48, 64, 80, 96):
        C = C_mb * 2**20
        agree, loss = 0, []
        for (name, n), rows in sorted(meas.items()):
            if name not in freq:
                continue
            cfg = freq[name]
            auto = [r for r in rows if r["launch"] == "auto"][0]["ms"]
            base = model(cfg, n, C)
            opts = [("auto", None, auto, 1.0)]
            for r in rows:
                if r["launch"] != "l2tiles":
                    continue
                pred = base / model(cfg, n, C, r["tiled"], r["block_mb"] * 2**20)
                opts.append(((r["tiled"], r["block_mb"]), pred, r["ms"], auto / r["ms"]))
            best_meas = min(opts, key=lambda o: o[2])
            cand = [o for o in opts[1:] if o[1] >= 1.10]
            pick = max(cand, key=lambda o: o[1]) if cand else opts[0]
            loss.append(pick[2] / best_meas[2])
            agree += pick is best_meas
            if C_mb == 64:
                print(f"{name:9s} m{n} best={best_meas[0]} {best_meas[3]:.2f}x  pick={pick[0]} "
                      f"meas {auto / pick[2]:.2f}x  preds=" +
                      " ".join(f"{o[0]}:{o[1]:.2f}/{o[3]:.2f}" for o in opts[1:]))
        print(f"C={C_mb} MB: pick==best {agree}/{len(loss)}, mean time vs best {sum(loss) / len(loss):.3f}, "
              f"worst {max(loss):.3f}")


if __name__ == "__main__":
    main()
