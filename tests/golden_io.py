"""Parser for the hand-written golden traces under tests/golden/*.trace.

Format (one directive per line, '#' starts a comment):
  geometry <n_blocks> <block_dim>
  word <NAME> <word number>
  <KIND> t<tid> [<WORD>] [BLOCK|DEVICE|SYSTEM] [m=0x<mask>]     accesses, FENCE, SYNCWARP
  SYNCTHREADS b<block> | CG_BLOCK_SYNC b<block>
  GRID_SYNC | CG_GRID_SYNC
  expect <WORD> <cur> <prev> R<k>                               one expected report
Event indices are the 0-based line order of event lines.
"""
from __future__ import annotations

import glob
import os

import numpy as np

import tracegen as tg

GOLDEN_DIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
_SCOPES = {"BLOCK": tg.BLOCK, "DEVICE": tg.DEVICE, "SYSTEM": tg.SYSTEM}


def parse(path):
    geom = None
    words = {}
    b = None
    expects = []
    with open(path) as f:
        for raw in f:
            line = raw.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            head = tok[0]
            if head == "geometry":
                geom = (int(tok[1]), int(tok[2]))
                b = tg.TraceBuilder(*geom)
                continue
            if head == "word":
                words[tok[1]] = int(tok[2], 0)
                continue
            if head == "expect":
                expects.append((words[tok[1]] << 2, int(tok[2]), int(tok[3]), int(tok[4][1:])))
                continue
            kind = tg.KIND_NAMES.index(head)
            tid, word, scope, mask = 0, 0, tg.NONE, None
            for t in tok[1:]:
                if t.startswith("t") and t[1:].isdigit():
                    tid = int(t[1:])
                elif t.startswith("b") and t[1:].isdigit():
                    tid = int(t[1:]) * geom[1]
                elif t in _SCOPES:
                    scope = _SCOPES[t]
                elif t.startswith("m="):
                    mask = int(t[2:], 0)
                elif t in words:
                    word = words[t]
                else:
                    raise ValueError(f"{path}: bad token {t!r}")
            if kind in (tg.SYNCTHREADS, tg.CG_BLOCK_SYNC, tg.GRID_SYNC, tg.CG_GRID_SYNC) and mask is None:
                mask = 0xFFFFFFFF
            b.ev(kind, tid, word, scope, mask)
    expects.sort(key=lambda r: r[1])
    return b.events(), geom[0], geom[1], expects


def all_golden():
    return sorted(glob.glob(os.path.join(GOLDEN_DIR, "*.trace")))


def report_tuples(reports):
    """(addr, cur, prev, type) tuples of a REPORT_DTYPE array, in array order."""
    return [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"])) for r in reports]


def full_tuples(reports):
    return [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"]), int(r["cur_kind"]),
             int(r["prev_kind"])) for r in reports]


def as_numpy_tuple_set(reports):
    return set(report_tuples(reports))


__all__ = ["parse", "all_golden", "report_tuples", "full_tuples", "np"]
