#!/usr/bin/env python
"""Lower bound on a launch's DRAM traffic under an ideal static row cache.

For every mode n of a config: DRAM bytes >= records + Y + (gathers of factor rows outside the
cache) x 4R, where the cache holds the C bytes of the most frequently gathered rows over all
gathered factors (the optimal static cache for independent draws: the synthetic generator draws
every index independently from its bucketed Zipf table, `synth.zipf_table`, so no reordering of
the nonzeros can give a row more reuse than its frequency).  Factors of <= 1 MB are assumed
staged in shared memory (no DRAM gathers).  Prints, per mode, the cold gathers per nonzero and
the bound at cache sizes C, next to the ncu-measured traffic (`profiles/ncu_traffic.json`), and
the roofline fraction the bound allows at the DRAM throughput the measured launch achieved.

  python tools/cache_bound.py [nell1 deli4d amazon ...]
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def row_probs(I, s):
    """(per-row gather probability, rows) per bucket of the generator's Zipf table."""
    e, _ = synth.zipf_table(int(I), float(s))
    if len(e) == 0:
        return np.array([1.0 / I]), np.array([float(I)])
    e = e.astype(np.float64)
    a, b = e[:-1] + 1.0, e[1:] + 1.0
    w = np.log(b / a) if abs(s - 1.0) < 1e-12 else (b ** (1 - s) - a ** (1 - s)) / (1 - s)
    w /= w.sum()
    width = e[1:] - e[:-1]
    return w / width, width


def cold_per_nnz(cfg, n, cache_bytes):
    R = cfg.rank
    ps, cs = [], []
    for m in range(cfg.nmodes):
        if m == n or cfg.dims[m] * R * 4 <= (1 << 20):
            continue
        p, c = row_probs(cfg.dims[m], cfg.zipf[m])
        ps.append(p)
        cs.append(c)
    if not ps:
        return 0.0, 0
    p, c = np.concatenate(ps), np.concatenate(cs)
    o = np.argsort(-p)
    p, c = p[o], c[o]
    K = cache_bytes / (4.0 * R)
    cum = np.cumsum(c)
    k = int(np.searchsorted(cum, K))
    cov = float((p[:k] * c[:k]).sum())
    if k < len(p):
        cov += float(p[k] * (K - (cum[k - 1] if k else 0.0)))
    return len(ps) - cov, len(ps)


def main():
    names = sys.argv[1:] or ["nell1", "deli4d", "amazon", "nell2"]
    traffic = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))["configs"]
    for name in names:
        cfg = synth.CONFIGS[name]
        N, R, nnz = cfg.nmodes, cfg.rank, cfg.nnz
        rec = 16 if N <= 4 else 32
        alg = 4 * (N + 1) * nnz + 4 * R * sum(cfg.dims)
        meas = traffic.get(name, {}).get("per_mode")
        for n in range(N):
            y = cfg.dims[n] * R * 4
            row = {"config": name, "mode": n, "algorithmic_GB": round(alg / 1e9, 3)}
            for C in (16, 32, 64, 126):
                cold, _ = cold_per_nnz(cfg, n, C * 2 ** 20)
                b = rec * nnz + y + cold * nnz * 4 * R
                row[f"bound_{C}MB_GB"] = round(b / 1e9, 2)
                row[f"cold_per_nnz_{C}MB"] = round(cold, 3)
            if meas:
                row["ncu_GB"] = round(meas[n] / 1e9, 2)
                # how far the measured bytes are above each bound: at the same DRAM rate the
                # roofline fraction could rise by at most this factor
                for C in (32, 126):
                    row[f"ncu_over_{C}MB"] = round(row["ncu_GB"] / row[f"bound_{C}MB_GB"], 3)
            print(json.dumps(row))


if __name__ == "__main__":
    main()
