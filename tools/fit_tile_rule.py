#!/usr/bin/env python
"""Fit / evaluate the hot+L2-tile rule on tools/hot_heldout.py output (offline, no GPU).

Rule: when the hot-row class applies, tile the gathered factor m (2^19-row L2
tiles, 16 MB hot rows on the others) that minimises the hot coverage cover_m among candidates
with T_m = ceil(I_m / 2^19) in [2, tmax], Y revisit ratio rho_m <= rmax and cover_m < cmax;
else hot rows alone.  For each (cmax, rmax, tmax) on a grid: mean and min of best / chosen time
over the modes where the hot class applies.

  python tools/fit_tile_rule.py train.jsonl [eval.jsonl]
"""
import itertools
import json
import sys


def load(path):
    return [json.loads(l) for l in open(path)]


def chosen_time(d, cmax, rmax, tmax):
    t = d["times_ms"]
    N = len(d["tensor"]["dims"])
    n = d["mode"]
    best_m, best_c = None, 2.0
    for m in range(N):
        if m == n or str(m) not in {str(k) for k in d["rho"]}:
            continue
        T = -(-d["tensor"]["dims"][m] // (1 << 19))
        rho = d["rho"].get(str(m), d["rho"].get(m))
        c = d["cover"][m]
        if T < 2 or T > tmax or rho > rmax or c >= cmax or t.get(f"tile{m}+hot16") is None:
            continue
        if c < best_c:
            best_m, best_c = m, c
    return t[f"tile{best_m}+hot16"] if best_m is not None else t["hot32"]


def evaluate(rows, cmax, rmax, tmax):
    ratios = []
    for d in rows:
        R, dims, n = d["tensor"]["rank"], d["tensor"]["dims"], d["mode"]
        gathered = sum(dims[m] * R * 4 for m in range(len(dims)) if m != n and dims[m] * R * 4 >= 16 << 20)
        if gathered < 160 << 20:
            continue  # the hot class does not apply (factors near L2 size)
        if d["times_ms"].get("hot32") is None:
            continue
        best = min(v for v in d["times_ms"].values() if v)
        ratios.append(best / chosen_time(d, cmax, rmax, tmax))
    return (min(ratios), sum(ratios) / len(ratios), len(ratios)) if ratios else (None, None, 0)


def main():
    train = load(sys.argv[1])
    evals = load(sys.argv[2]) if len(sys.argv) > 2 else []
    res = []
    for cmax, rmax, tmax in itertools.product([0.0, 0.4, 0.5, 0.6, 0.65, 0.7, 0.75, 0.8, 0.85, 1.01],
                                              [0.1, 0.25, 0.5], [8, 16, 32, 64]):
        mn, mean, k = evaluate(train, cmax, rmax, tmax)
        res.append((mean, mn, cmax, rmax, tmax, k))
    res.sort(reverse=True)
    print("train: mean, min, cmax, rmax, tmax, modes")
    for r in res[:12]:
        print("  %.4f %.3f %.2f %.2f %d %d" % r)
    if evals:
        for r in res[:5]:
            mn, mean, k = evaluate(evals, r[2], r[3], r[4])
            print("eval with cmax %.2f rmax %.2f tmax %d: mean %.4f min %.3f over %d modes" % (r[2], r[3], r[4], mean, mn, k))
        mn, mean, k = evaluate(evals, 0.0, 0.25, 16)
        print("eval hot-only (no tiles): mean %.4f min %.3f" % (mean, mn))


if __name__ == "__main__":
    main()
