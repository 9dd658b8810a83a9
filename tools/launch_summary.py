"""Mean device time per kernel from an ncu --metrics gpu__time_duration.sum csv."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
agg = defaultdict(list)
for r in rows[1:]:
    name = r[ki].split("(")[0].replace("void ", "").replace("pc::", "")
    agg[name].append(float(r[vi].replace(",", "")))
tot = sum(sum(v) for v in agg.values())
for name, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{name:40s} n={len(v):4d} mean={sum(v)/len(v)/1e3:8.2f} us  total={sum(v)/1e3:9.1f} us  {100*sum(v)/tot:5.1f}%")
