"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list: per kernel name, launches and mean time."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
tot = defaultdict(list)
for r in rows[1:]:
    try:
        tot[r[ki]].append(float(r[vi].replace(",", "")))
    except ValueError:
        pass
print("==", sys.argv[2] if len(sys.argv) > 2 else sys.argv[1])
for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
    unit = 1e-6 if max(v) > 1e4 else 1e-3  # ns or us
    print(f"{k[:70]:70s} n={len(v):3d} mean={sum(v)/len(v)*unit:9.4f} ms")
