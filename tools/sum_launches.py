"""Aggregate an ncu --metrics gpu__time_duration.sum CSV by kernel name."""
import csv
import sys
from collections import defaultdict

tot = defaultdict(float)
cnt = defaultdict(int)
with open(sys.argv[1]) as f:
    lines = [l for l in f if l.startswith('"')]
for r in csv.DictReader(lines):
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"][:90]
    v = float(r["Metric Value"].replace(",", ""))
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "nsecond": 1e-6}.get(r["Metric Unit"], 1e-6)
    tot[name] += v * scale
    cnt[name] += 1
total = sum(tot.values())
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{v:10.3f} ms {100*v/total:6.2f}% {cnt[k]:6d}x  {k}")
print(f"{total:10.3f} ms total")
