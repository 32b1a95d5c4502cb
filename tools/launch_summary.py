"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into per-kernel shares.

usage: python tools/launch_summary.py LAUNCHES.csv OUT.txt "command that produced it"
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
agg = {}
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        v *= {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}[d["Metric Unit"]]
        a = agg.setdefault(d["Kernel Name"], [0, 0.0])
        a[0] += 1
        a[1] += v
tot = sum(a[1] for a in agg.values())
with open(sys.argv[2], "w") as f:
    f.write(sys.argv[3] + "\n(cold-cache, serialised launches under ncu: compare shares, not absolutes)\n")
    for k, (n, us) in sorted(agg.items(), key=lambda x: -x[1][1]):
        f.write(f"{k:36s} launches={n:5d} total_us={us:12.1f} mean_us={us / n:10.2f} share={us / tot:6.3f}\n")
print(open(sys.argv[2]).read())
