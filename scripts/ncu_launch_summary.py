"""Summarise an ncu launch-list CSV (--metrics gpu__time_duration.sum) into kernel shares."""
import collections
import csv
import sys

src, cmd = sys.argv[1], (sys.argv[2] if len(sys.argv) > 2 else "")
lines = open(src).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
agg = collections.defaultdict(lambda: [0, 0.0])
for r in csv.DictReader(lines[start:]):
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "nsecond": 1e-6}[r["Metric Unit"]]
    a = agg[r["Kernel Name"]]
    a[0] += 1
    a[1] += float(r["Metric Value"].replace(",", "")) * scale
tot = sum(v[1] for v in agg.values())
print(f"# ncu launch list of `{cmd}`")
print("# (gpu__time_duration.sum, --clock-control none; cold-cache, serialised: compare SHARES)")
print(f"{'launches':>8s}  {'total_ms':>9s}  {'share':>6s}  kernel")
for k, (c, ms) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{c:8d}  {ms:9.3f}  {100 * ms / tot:5.1f}%  {k}")
