#!/usr/bin/env python
"""Markdown table of sweep summaries (sweep.py output): per (config, mode) the selector's pick
time, the sweep best, pick / best, the pick's rank and the number of launches swept.

  python tools/sweep_table.py profiles/r02/sweeps/final/*.jsonl
"""
import json
import sys


def main():
    rows = []
    for path in sys.argv[1:]:
        for line in open(path):
            d = json.loads(line)
            if d.get("summary"):
                rows.append(d)
    print("| config | mode | pick (ms) | sweep best (ms) | pick / best | rank | launches | pick class |")
    print("|---|---|---|---|---|---|---|---|")
    worst = 1.0
    for d in rows:
        p = d["pick"]
        cls = ("hot %d MB" % (p.get("hot_kb", 0) // 1024) if p.get("hot_kb") else "no hot") + \
              (" + L2 tiles" if p.get("flags", 0) & 64 else "") + \
              (" + smem blocks" if p.get("staged_mask") and not p.get("flags", 0) & 64 else "")
        r = d["pick_over_best"]
        worst = min(worst, r)
        print(f"| {d['config']} | {d['mode']} | {d['pick_ms']:.3f} | {d['best_ms']:.3f} | {r:.3f} | {d['pick_rank']} | "
              f"{d['n_launches']} | {cls} |")
    print(f"\nminimum pick / best: {worst:.3f} over {len(rows)} modes")


if __name__ == "__main__":
    main()
