"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: per kernel
name, count and total / mean duration, and each kernel's share of the total.
The last factorisation in the list (after the warm-up) is the timed step."""
import collections
import csv
import sys

rows = []
with open(sys.argv[1]) as f:
    lines = [l for l in f if l.startswith('"')]
for r in csv.DictReader(lines):
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    v = float(r["Metric Value"].replace(",", ""))
    unit = r.get("Metric Unit", "ns")
    scale = {"ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "nsecond": 1e-3}.get(unit, 1.0)
    name = r["Kernel Name"].split("(")[0].split("<")[0].replace("stfk::", "")
    rows.append((name, v * scale))
agg = collections.OrderedDict()
for name, us in rows:
    c, t = agg.get(name, (0, 0.0))
    agg[name] = (c + 1, t + us)
tot = sum(t for _, t in agg.values())
print("%-28s %8s %14s %12s %7s" % ("kernel", "launches", "total_us", "mean_us", "share"))
for name, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print("%-28s %8d %14.1f %12.2f %6.1f%%" % (name, c, t, t / c, 100 * t / tot))
print("total launches %d, total serialised kernel time %.1f ms" % (len(rows), tot / 1e3))
