"""Per-CUDA-source-line warp instructions and stall samples of one kernel in an ncu report
(--page source --print-source cuda,sass; needs -lineinfo).  usage:
   python profiles/src_hot.py report.ncu-rep kernel-regex [top]"""
import csv
import io
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
raw = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kre}",
                               "--launch-skip", str(int(sys.argv[4]) if len(sys.argv) > 4 else 0), "--launch-count", "1", "--print-source", "cuda,sass"], text=True,
                              stderr=subprocess.DEVNULL)
rows = list(csv.reader(io.StringIO(raw)))
out = []
fname = "?"
hdr = None
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8 or not r[0].isdigit():
        continue
    ie = hdr.index("Instructions Executed")
    ss = hdr.index("Warp Stall Sampling (All Samples)")
    try:
        out.append((int(r[ie]), int(r[ss]), fname, int(r[0]), r[1][:110]))
    except ValueError:
        pass
tot = sum(o[0] for o in out) or 1
stot = sum(o[1] for o in out) or 1
print(f"{kre}: {tot} warp instructions, {stot} stall samples")
for ins, st, f, ln, src in sorted(out, reverse=True)[:top]:
    print(f"{100 * ins / tot:5.1f}% inst {100 * st / stot:5.1f}% stall  {f}:{ln}  {src}")
