"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) by kernel: launches and
share of the serialised device time.  Usage: python tools/launch_summary.py launches.csv"""
import csv
import re
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
agg = defaultdict(lambda: [0, 0.0])
for r in rows[hdr + 1:]:
    if len(r) <= vi:
        continue
    name = re.sub(r"\(.*", "", r[ki]).replace("void ", "").strip()
    a = agg[name]
    a[0] += 1
    a[1] += float(r[vi].replace(",", ""))
tot = sum(a[1] for a in agg.values())
print("| kernel | launches | total ms | share |")
print("|---|---|---|---|")
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print("| `%s` | %d | %.3f | %.1f %% |" % (k, c, t / 1e6, 100.0 * t / tot))
