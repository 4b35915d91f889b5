"""Per-kernel launch count / mean / max duration (us) of an ncu --metrics gpu__time_duration.sum
--csv launch list.  usage: python scripts/launch_agg.py LAUNCHES.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, agg = None, collections.defaultdict(list)
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3,
                     "msecond": 1e3}.get(d.get("Metric Unit", "ns"), 1e-3)
            agg[d["Kernel Name"][:80]].append(float(d["Metric Value"].replace(",", "")) * scale)
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{len(v):4d} {sum(v) / len(v):12.1f} {max(v):12.1f}  {k}")
