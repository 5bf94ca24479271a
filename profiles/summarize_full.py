"""Key metrics per kernel from an `ncu --set full` report (text, for the repo).
usage: python profiles/summarize_full.py report.ncu-rep [title]"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram % of peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm % of peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
]
rep = sys.argv[1]
raw = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
rows = list(csv.reader(io.StringIO(raw)))
hdr, units = rows[0], rows[1]
print(sys.argv[2] if len(sys.argv) > 2 else rep)
for r in rows[2:]:
    print(f"== {r[hdr.index('Kernel Name')]}")
    for m, label in METRICS:
        if m in hdr:
            i = hdr.index(m)
            print(f"   {label:24s} {r[i]:>18s} {units[i]}")
det = subprocess.check_output(["ncu", "-i", rep, "--page", "details", "--csv"], text=True)
for r in csv.reader(io.StringIO(det)):
    if len(r) > 16 and r[15] in ("OPT",) and r[13] in ("CPIStall", "IssueSlotUtilization", "SharedMemoryConflicts",
                                                       "UncoalescedGlobalAccess", "UncoalescedSharedAccess",
                                                       "TheoreticalOccupancy"):
        print(f"-- {r[4].split('(')[0]}: {r[13]}: {r[16][:400]}")
