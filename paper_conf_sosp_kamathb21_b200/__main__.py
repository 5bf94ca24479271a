"""Command-line race check of a trace file:

    python -m paper_conf_sosp_kamathb21_b200 TRACE --blocks B --block-dim D [--coalesce]
        [--paper-counters] [--out reports.csv] [--device N]

TRACE is a raw little-endian array of 16-byte ``igd_event`` records (include/igd.h: u64 addr,
u32 tk = tid | kind << 24 | scope << 28, u32 active mask) in execution order.  Reports are written
as CSV (``addr,cur,prev,type,cur_kind,prev_kind``; type 1..5 = R1..R5 of Table 2), ascending by
``cur``, to ``--out`` or stdout.  The check runs on the GPU through libigd (no CPU fallback).
"""
from __future__ import annotations

import argparse
import sys

import numpy as np

RULES = {1: "R1 scoped atomic", 2: "R2 intra-warp (ITS)", 3: "R3 intra-block", 4: "R4 inter-block",
         5: "R5 missing lock"}


def parse_args(argv=None):
    ap = argparse.ArgumentParser(prog="python -m paper_conf_sosp_kamathb21_b200", description=__doc__.split("\n")[0])
    ap.add_argument("trace", help="raw file of 16-byte igd_event records")
    ap.add_argument("--blocks", type=int, required=True, help="grid size of the traced kernel (blocks)")
    ap.add_argument("--block-dim", type=int, required=True, help="threads per block")
    ap.add_argument("--coalesce", action="store_true", help="warp-coalesced check (IGD_DETECT_COALESCE)")
    ap.add_argument("--paper-counters", action="store_true",
                    help="Fig. 4-width synchronization IDs (IGD_DETECT_PAPER_COUNTERS)")
    ap.add_argument("--out", default="-", help="CSV output path ('-' = stdout)")
    ap.add_argument("--device", type=int, default=0)
    return ap.parse_args(argv)


def read_trace(path: str) -> np.ndarray:
    from .igd import EVENT_DTYPE

    raw = np.fromfile(path, dtype=np.uint8)
    if raw.size % EVENT_DTYPE.itemsize:
        raise SystemExit(f"{path}: {raw.size} bytes is not a whole number of 16-byte events")
    return raw.view(EVENT_DTYPE)


def write_csv(reports: np.ndarray, out) -> None:
    out.write("addr,cur,prev,type,cur_kind,prev_kind\n")
    for r in reports:
        out.write(f"{int(r['addr']):#x},{int(r['cur'])},{int(r['prev'])},{int(r['type'])},"
                  f"{int(r['cur_kind'])},{int(r['prev_kind'])}\n")


def main(argv=None) -> int:
    a = parse_args(argv)
    ev = read_trace(a.trace)
    from . import igd

    with igd.Detector(a.device) as d:
        d.load(ev, a.blocks, a.block_dim)
        n = d.detect(coalesce=a.coalesce, paper_counters=a.paper_counters)
        rep = d.reports()
    out = sys.stdout if a.out == "-" else open(a.out, "w")
    try:
        write_csv(rep, out)
    finally:
        if out is not sys.stdout:
            out.close()
    counts = np.bincount(rep["type"].astype(np.int64), minlength=6) if n else np.zeros(6, np.int64)
    summary = ", ".join(f"{RULES[t]}: {int(counts[t])}" for t in range(1, 6) if counts[t])
    print(f"{len(ev)} events, {n} races" + (f" ({summary})" if summary else ""), file=sys.stderr)
    return 0


if __name__ == "__main__":
    sys.exit(main())
