"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list: per kernel name, launches and mean time."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
tot = defaultdict(list)
for r in rows[1:]:
    try:
        tot[r[ki]].append(float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0))
    except ValueError:
        pass
print("==", sys.argv[2] if len(sys.argv) > 2 else sys.argv[1])
for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k[:70]:70s} n={len(v):3d} mean={sum(v)/len(v):9.4f} ms")
