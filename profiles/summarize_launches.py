"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel totals and shares.
usage: python profiles/summarize_launches.py launches.csv [title]"""
import csv
import sys
from collections import defaultdict

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, ui, vi = hdr.index("Kernel Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[1:]:
    name = r[ki].split("(")[0].replace("void ", "")
    tot[name] += float(r[vi].replace(",", "")) * SCALE[r[ui]]
    cnt[name] += 1
s = sum(tot.values())
print(sys.argv[2] if len(sys.argv) > 2 else sys.argv[1])
print("per-launch device times (ncu, cold cache, serialised): compare shares, not absolutes")
for k in sorted(tot, key=lambda k: -tot[k]):
    print(f"{k:36s} launches={cnt[k]:4d} total_ms={tot[k]:10.3f} share={tot[k] / s * 100:5.1f}%")
