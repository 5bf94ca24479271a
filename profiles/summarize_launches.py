"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum[,dram__bytes_read.sum,
dram__bytes_write.sum] --csv`): per-kernel totals, time shares and DRAM bytes per launch.
usage: python profiles/summarize_launches.py launches.csv [title] [--traffic-json out.json workload]

--traffic-json writes {workload: {kernel: dram_bytes_per_launch}} (read by bench.py to fill the
roofline "traffic" field of the dominant kernel: the DRAM bytes ncu counted for that kernel)."""
import csv
import json
import os
import sys
from collections import defaultdict

TSCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
BSCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "KB": 1e3, "MB": 1e6, "GB": 1e9}

args = sys.argv[1:]
tj = None
detects = None
if "--detects" in args:  # igd_detect calls the launch list covers (warmup + steps of the bench run)
    i = args.index("--detects")
    detects = int(args[i + 1])
    args = args[:i] + args[i + 2:]
if "--traffic-json" in args:
    i = args.index("--traffic-json")
    tj = (args[i + 1], args[i + 2])
    args = args[:i] + args[i + 3:]
rows = [r for r in csv.reader(open(args[0])) if len(r) > 10]
hdr = rows[0]
ki, ii, mi = hdr.index("Kernel Name"), hdr.index("ID"), hdr.index("Metric Name")
ui, vi = hdr.index("Metric Unit"), hdr.index("Metric Value")
per = defaultdict(dict)  # launch id -> metrics
names = {}
for r in rows[1:]:
    lid = int(r[ii])
    names[lid] = r[ki].split("(")[0].replace("void ", "")
    v = float(r[vi].replace(",", ""))
    m = r[mi]
    if m == "gpu__time_duration.sum":
        per[lid]["ms"] = v * TSCALE[r[ui]]
    elif m.startswith("dram__bytes"):
        per[lid]["dram"] = per[lid].get("dram", 0.0) + v * BSCALE.get(r[ui], 1.0)
tot, cnt, dram = defaultdict(float), defaultdict(int), defaultdict(float)
for lid, m in per.items():
    k = names[lid]
    tot[k] += m.get("ms", 0.0)
    cnt[k] += 1
    dram[k] += m.get("dram", 0.0)
s = sum(tot.values())
print(args[1] if len(args) > 1 else args[0])
print("per-launch device times (ncu, cold cache, serialised): compare shares, not absolutes")
for k in sorted(tot, key=lambda k: -tot[k]):
    line = f"{k:36s} launches={cnt[k]:4d} total_ms={tot[k]:10.3f} share={tot[k] / s * 100:5.1f}%"
    if dram[k]:
        line += f"  dram/launch={dram[k] / cnt[k] / 1e9:8.3f} GB  dram GB/s={dram[k] / (tot[k] / 1e3) / 1e9:7.1f}"
    print(line)
if tj:
    out, workload = tj
    d = json.load(open(out)) if os.path.exists(out) else {}
    d[workload] = {k: dram[k] / cnt[k] for k in dram if dram[k]}
    if detects:
        d[workload]["__dram_per_detect__"] = sum(dram.values()) / detects
    json.dump(d, open(out, "w"), indent=1, sort_keys=True)
