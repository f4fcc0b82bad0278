#!/usr/bin/env python
"""Compare launch pickers on l2tile_study outputs: for each (tensor, mode), the picked launch's
time over the best of every launch timed for it.  usage:
selector_compare.py OLD.jsonl NEW.jsonl   (OLD 'rule' lines = old tree + hand rule when present,
else its 'auto'; NEW 'auto' = the retrained tree)"""
import collections
import json
import math
import sys


def load(path):
    by = collections.OrderedDict()
    for line in open(path):
        r = json.loads(line)
        if "ms" not in r or r["launch"] == "l2tiles2":
            continue
        d = by.setdefault((r["config"], r["mode"]), {})
        key = r["launch"] if r["launch"] in ("auto", "rule") else (r["tiled"], r["block_mb"])
        d[key] = r["ms"]
    return by


def main():
    old, new = load(sys.argv[1]), load(sys.argv[2])
    rows = []
    for k in new:
        if k not in old:
            continue
        o, n = old[k], new[k]
        best = min(list(o.values()) + list(n.values()))
        base = o["auto"]  # the old tree alone
        t_old = o.get("rule", o["auto"])
        t_new = n["auto"]
        rows.append((k, base / best, base / t_old, base / t_new, t_old / best, t_new / best))
    g = lambda xs: math.exp(sum(map(math.log, xs)) / len(xs))
    print(f"{len(rows)} modes: speedup over the old tree alone, geomean: best {g([r[1] for r in rows]):.3f}, "
          f"old tree + rule {g([r[2] for r in rows]):.3f}, new tree {g([r[3] for r in rows]):.3f}; "
          f"time / best mean: old+rule {sum(r[4] for r in rows) / len(rows):.3f} (worst {max(r[4] for r in rows):.2f}), "
          f"new {sum(r[5] for r in rows) / len(rows):.3f} (worst {max(r[5] for r in rows):.2f})")
    if len(sys.argv) > 3:
        for r in rows:
            print(r[0], " ".join(f"{x:.2f}" for x in r[1:]))


if __name__ == "__main__":
    main()
