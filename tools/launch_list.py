"""Aggregate an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel."""
import collections
import csv
import json
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}


def aggregate(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr = rows[hi]
    ki, mi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= mi:
            continue
        v = float(r[mi].replace(",", "")) * SCALE.get(r[ui], 1.0)
        a = agg.setdefault(r[ki][:90], [0, 0.0])
        a[0] += 1
        a[1] += v
    tot = sum(v[1] for v in agg.values())
    return {k: {"launches": v[0], "total_ms": round(v[1], 4), "share": round(v[1] / tot, 4)} for k, v in agg.items()}


if __name__ == "__main__":
    print(json.dumps(aggregate(sys.argv[1]), indent=1))
