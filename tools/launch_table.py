"""Per-kernel totals of an ncu launch-list CSV (our kernels + NCCL), divided by the number of MSFs.

  python tools/launch_table.py launches.csv [msfs]
"""
import collections
import csv
import io
import sys

text = open(sys.argv[1]).read()
runs = int(sys.argv[2]) if len(sys.argv) > 2 else 1
rows = list(csv.DictReader(io.StringIO(text[text.index('"ID"'):])))
agg = collections.OrderedDict()
for r in rows:
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    k = r["Kernel Name"]
    if "eclmst" not in k and "nccl" not in k.lower():
        continue
    name = k.split("(")[0][-44:]
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += float(r["Metric Value"]) / 1e3
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':46s} {'launches/MSF':>12s} {'us/MSF':>10s} {'share':>6s}")
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:46s} {c / runs:12.1f} {t / runs:10.1f} {t / tot:6.1%}")
