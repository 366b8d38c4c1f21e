"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list per kernel.
  python tools/launch_summary.py launches.csv [max_rows]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, agg = None, collections.OrderedDict()
scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr is None or len(r) < len(hdr):
        continue
    d = dict(zip(hdr, r))
    if d.get("Metric Name") != "gpu__time_duration.sum":
        continue
    v = float(d["Metric Value"].replace(",", "")) * scale.get(d["Metric Unit"], 1.0)
    a = agg.setdefault(d["Kernel Name"][:60], [0, 0.0])
    a[0] += 1
    a[1] += v
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':62s}{'launches':>9s}{'total_us':>11s}{'mean_us':>9s}{'share':>8s}")
for k, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1])[: int(sys.argv[2]) if len(sys.argv) > 2 else 40]:
    print(f"{k:62s}{c:9d}{v:11.1f}{v / c:9.2f}{v / tot * 100:7.1f}%")
print(f"total {tot:.1f} us")
