#!/usr/bin/env python3
"""Per-kernel launch counts, summed device time and share of an ncu launch list
(`ncu --metrics gpu__time_duration.sum --csv --log-file X.csv <cmd>`):

    python scripts/launch_shares.py profiles/r02/launches_road24m.csv road24m > profiles/r02/launch_shares_road24m.json
"""
import collections
import csv
import json
import re
import sys


def main(path, workload):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    idx = {h: i for i, h in enumerate(rows[0])}
    agg = collections.defaultdict(lambda: [0, 0.0])
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    for r in rows[1:]:
        if r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", r[idx["Kernel Name"]]).replace("void ", "").replace("b200dfs::", "")
        agg[name][0] += 1
        agg[name][1] += float(r[idx["Metric Value"]].replace(",", "")) * scale.get(r[idx["Metric Unit"]], 1.0)
    tot = sum(v[1] for v in agg.values())
    out = {k: {"launches": v[0], "ms_total": round(v[1], 3), "share": round(v[1] / tot, 4)}
           for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])}
    json.dump({"workload": workload, "source": "ncu --metrics gpu__time_duration.sum --clock-control none "
               "(cold-cache, serialised: shares, not absolutes)", "kernels": out}, sys.stdout, indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
