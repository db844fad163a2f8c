"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV):
per-kernel launch count, total time and share of the listed launches."""
import csv, io, sys
from collections import defaultdict
txt = open(sys.argv[1]).read()
i = txt.find('"ID"')
rows = list(csv.DictReader(io.StringIO(txt[i:])))
agg = defaultdict(lambda: [0, 0.0])
scale = {"ns": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1.0}
for r in rows:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    n = r["Kernel Name"][:90]
    agg[n][0] += 1
    agg[n][1] += float(r["Metric Value"].replace(",", "")) * scale.get(r["Metric Unit"], 1.0)
tot = sum(v[1] for v in agg.values())
print(f"{'launches':>8} {'total_us':>12} {'share':>7}  kernel")
for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{c:8d} {t / 1e3:12.1f} {100 * t / tot:6.2f}%  {n}")
