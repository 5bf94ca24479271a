"""Per-opcode instruction / stall-sample mix and the hottest SASS lines of one kernel in an
ncu report.  usage: python profiles/sass_hot.py report.ncu-rep kernel-regex [launch-skip] [top]"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep, kre = sys.argv[1], sys.argv[2]
skip = int(sys.argv[3]) if len(sys.argv) > 3 else 0
top = int(sys.argv[4]) if len(sys.argv) > 4 else 20
raw = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kre}",
                               "--launch-skip", str(skip), "--launch-count", "1", "--print-source", "sass"],
                              text=True, stderr=subprocess.DEVNULL)
rows = list(csv.reader(io.StringIO(raw)))
hdr = rows[1]
data = [r for r in rows[2:] if len(r) > 10]
ie, ss = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")


def I(x):
    try:
        return int(x)
    except ValueError:
        return 0


tot = sum(I(r[ie]) for r in data) or 1
stot = sum(I(r[ss]) for r in data) or 1
print(f"{rows[0][1]}: {tot} warp instructions, {stot} stall samples, {len(data)} SASS lines")
c, s = Counter(), Counter()
for r in data:
    t = r[1].split()
    if not t:
        continue
    op = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
    c[op] += I(r[ie])
    s[op] += I(r[ss])
print("opcode mix: " + "  ".join(f"{op} {v / tot * 100:.1f}%/{s[op] / stot * 100:.1f}%" for op, v in c.most_common(16)))
print(f"top {top} SASS lines by stall samples (index, %samples, %inst, line):")
for i in sorted(sorted(range(len(data)), key=lambda i: -I(data[i][ss]))[:top]):
    print(f"  {i:5d} {I(data[i][ss]) / stot * 100:5.1f}% {I(data[i][ie]) / tot * 100:5.2f}%  {data[i][1].strip()[:90]}")
