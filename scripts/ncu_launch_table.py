"""Mean device time per kernel from an ncu launch-list CSV (--metrics gpu__time_duration.sum --csv):
python scripts/ncu_launch_table.py launches.csv"""
import csv
import sys
from collections import defaultdict

agg = defaultdict(list)
hdr = None
for r in csv.reader(open(sys.argv[1])):
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            unit = d.get("Metric Unit", "")
            v = float(d["Metric Value"].replace(",", ""))
            v = v / 1e3 if unit in ("ns", "nsecond") else (v * 1e3 if unit in ("ms", "msecond") else v)
            agg[d["Kernel Name"].split("(")[0][:60]].append(v)
for n, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{n:60s} n={len(v):4d} mean {sum(v) / len(v):9.2f} us  min {min(v):9.2f}  max {max(v):9.2f}")
