"""Summarise an ncu launch list (gpu__time_duration per launch) into per-kernel
counts, total time and share, for the timed steps of a bench run."""
import csv
import json
import sys
from collections import defaultdict


def summarise(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    agg = defaultdict(lambda: {"launches": 0, "ns": 0.0, "grid": set(), "block": set()})
    for r in rows[start + 1:]:
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"].split("(")[0].replace("void ", "")
        a = agg[name]
        a["launches"] += 1
        a["ns"] += float(d["Metric Value"].replace(",", ""))
        a["grid"].add(d.get("Grid Size"))
        a["block"].add(d.get("Block Size"))
    total = sum(a["ns"] for a in agg.values())
    out = {}
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["ns"]):
        out[k] = {"launches": a["launches"], "total_ms": a["ns"] / 1e6, "share": a["ns"] / total,
                  "grids": sorted(g for g in a["grid"] if g), "blocks": sorted(b for b in a["block"] if b)}
    return out


if __name__ == "__main__":
    print(json.dumps(summarise(sys.argv[1]), indent=1))
