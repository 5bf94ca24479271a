"""Seeded synthetic trace generators -- shared INPUT module (no race-check arithmetic).

This package only *produces* traces in the 16-byte ``igd_event`` format of
include/igd.h; it never evaluates the race rules.  Both the oracle
(tests) and the CUDA path (tests, bench) consume what it produces.  The generator
families C1..C5 live in the C library ``tracegen/igdgen.c`` and are
wrapped by :mod:`tracegen.families`; this module holds the format, a hand-written trace
builder used by the golden fixtures and a small random-trace fuzzer.

Each family also returns an *injection ledger*: the races it deliberately planted
(which events, which rule was intended).  The ledger records generator intent, written
down when the injection is emitted; tests use it as an independent pin of the oracle.
"""
from __future__ import annotations

import numpy as np

EVENT_DTYPE = np.dtype([("addr", "<u8"), ("tk", "<u4"), ("mask", "<u4")])
assert EVENT_DTYPE.itemsize == 16

REPORT_DTYPE = np.dtype([("addr", "<u8"), ("cur", "<u8"), ("prev", "<u8"), ("type", "u1"),
                         ("cur_kind", "u1"), ("prev_kind", "u1"), ("pad", "u1", (5,))])
assert REPORT_DTYPE.itemsize == 32

# kind codes
LD, ST, ATOM, CAS, EXCH, FENCE, SYNCWARP, SYNCTHREADS, GRID_SYNC = range(9)
CG_TILE_SYNC, CG_BLOCK_SYNC, CG_GRID_SYNC = 9, 10, 11
KERNEL_BOUNDARY = 12  # multi-kernel traces
KIND_NAMES = ["LD", "ST", "ATOM", "CAS", "EXCH", "FENCE", "SYNCWARP", "SYNCTHREADS", "GRID_SYNC",
              "CG_TILE_SYNC", "CG_BLOCK_SYNC", "CG_GRID_SYNC", "KERNEL_BOUNDARY"]
# scope codes
NONE, BLOCK, DEVICE, SYSTEM = 0, 1, 2, 3
SCOPE_NAMES = ["NONE", "BLOCK", "DEVICE", "SYSTEM"]


def pack_tk(tid, kind, scope):
    return (np.asarray(tid, np.uint32) | (np.asarray(kind, np.uint32) << 24)
            | (np.asarray(scope, np.uint32) << 28)).astype(np.uint32)


def unpack(events):
    """Split an EVENT_DTYPE array into (addr, tid, kind, scope, mask) numpy arrays."""
    tk = events["tk"]
    return (events["addr"], tk & 0xFFFFFF, (tk >> 24) & 0xF, (tk >> 28) & 0x3, events["mask"])


class Geometry:
    """Grid geometry of the traced kernel."""

    def __init__(self, n_blocks: int, block_dim: int):
        self.n_blocks = int(n_blocks)
        self.block_dim = int(block_dim)
        self.wpb = (self.block_dim + 31) // 32

    @property
    def threads(self):
        return self.n_blocks * self.block_dim

    def lane(self, t):
        return (t % self.block_dim) % 32

    def warp(self, t):
        return (t // self.block_dim) * self.wpb + (t % self.block_dim) // 32

    def block(self, t):
        return t // self.block_dim


class TraceBuilder:
    """Append events one by one (hand-written traces: golden fixtures, unit tests).

    ``mask`` defaults to the single lane of ``tid``.  Word-level helpers take a *word*
    number and store the byte address ``word << 2``.
    """

    def __init__(self, n_blocks: int, block_dim: int):
        self.geom = Geometry(n_blocks, block_dim)
        self.rows = []

    def _lanebit(self, tid):
        return 1 << self.geom.lane(tid)

    def ev(self, kind, tid, word=0, scope=NONE, mask=None, addr=None):
        if mask is None:
            mask = self._lanebit(tid)
        if addr is None:
            addr = int(word) << 2
        self.rows.append((int(addr), int(tid), int(kind), int(scope), int(mask) & 0xFFFFFFFF))
        return len(self.rows) - 1

    def ld(self, tid, word, mask=None):
        return self.ev(LD, tid, word, NONE, mask)

    def st(self, tid, word, mask=None):
        return self.ev(ST, tid, word, NONE, mask)

    def atom(self, tid, word, scope=DEVICE, mask=None):
        return self.ev(ATOM, tid, word, scope, mask)

    def cas(self, tid, word, scope=DEVICE, mask=None):
        return self.ev(CAS, tid, word, scope, mask)

    def exch(self, tid, word, scope=DEVICE, mask=None):
        return self.ev(EXCH, tid, word, scope, mask)

    def fence(self, tid, scope=DEVICE, mask=None):
        return self.ev(FENCE, tid, 0, scope, mask)

    def syncwarp(self, tid, mask=0xFFFFFFFF):
        return self.ev(SYNCWARP, tid, 0, NONE, mask)

    def syncthreads(self, block):
        return self.ev(SYNCTHREADS, block * self.geom.block_dim, 0, NONE, 0xFFFFFFFF)

    def grid_sync(self):
        return self.ev(GRID_SYNC, 0, 0, NONE, 0xFFFFFFFF)

    def kernel_boundary(self, n_blocks: int = None, block_dim: int = None):
        """End the kernel.  With a grid, the next kernel runs on (n_blocks, block_dim): the
        boundary's addr carries (n_blocks << 32) | block_dim (per-kernel geometry)."""
        if n_blocks is None:
            return self.ev(KERNEL_BOUNDARY, 0, 0, NONE, 0xFFFFFFFF)
        i = self.ev(KERNEL_BOUNDARY, 0, 0, NONE, 0xFFFFFFFF, addr=geometry_code(n_blocks, block_dim))
        self.geom = Geometry(n_blocks, block_dim)
        return i

    def events(self):
        out = np.zeros(len(self.rows), EVENT_DTYPE)
        if self.rows:
            a = np.array(self.rows, dtype=np.uint64)
            out["addr"] = a[:, 0]
            out["tk"] = pack_tk(a[:, 1].astype(np.uint32), a[:, 2].astype(np.uint32),
                                a[:, 3].astype(np.uint32))
            out["mask"] = a[:, 4].astype(np.uint32)
        return out


def random_trace(seed: int, n: int, n_blocks: int = None, block_dim: int = None, n_words: int = 16,
                 weights=None, max_uses_per_word: int = 0, lock_words: int = 2, p_lock_data: float = 0.0):
    """Arbitrary event sequence for fuzzing.

    Geometry is 1-3 blocks x {32,64,96} threads unless given.  Kinds are drawn with
    weights, scopes at random, masks random but containing the lane.  With
    ``max_uses_per_word`` > 0 every data word is accessed at most that many times
    (the pairwise evaluator needs 2).  ``p_lock_data`` sends that fraction of LD/ST/ATOM to
    the lock words.  Returns (events, n_blocks, block_dim).
    """
    rng = np.random.default_rng(seed)
    if n_blocks is None:
        n_blocks = int(rng.integers(1, 4))
    if block_dim is None:
        block_dim = int(rng.choice([32, 64, 96]))
    g = Geometry(n_blocks, block_dim)
    if weights is None:
        weights = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    kinds = np.arange(len(weights))  # 13 weights: kernel boundaries too
    w = np.asarray(weights, float)
    w = w / w.sum()
    b = TraceBuilder(n_blocks, block_dim)
    uses = {}
    next_fresh = 1000
    for _ in range(n):
        k = int(rng.choice(kinds, p=w))
        t = int(rng.integers(0, g.threads))
        lane = g.lane(t)
        mask = (int(rng.integers(0, 1 << 32)) | (1 << lane)) & 0xFFFFFFFF
        if rng.random() < 0.5:
            mask = 1 << lane
        if k in (LD, ST, ATOM):
            if max_uses_per_word:
                # pick a word that still has budget, else a fresh one
                cands = [x for x, u in uses.items() if u < max_uses_per_word]
                if cands and rng.random() < 0.6:
                    word = int(rng.choice(cands))
                else:
                    word = next_fresh
                    next_fresh += 1
                uses[word] = uses.get(word, 0) + 1
            elif p_lock_data and rng.random() < p_lock_data:
                word = 500 + int(rng.integers(0, lock_words))   # plain access to a lock word
            else:
                word = int(rng.integers(0, n_words))
            scope = NONE if k in (LD, ST) else int(rng.integers(1, 4))
            b.ev(k, t, word, scope, mask)
        elif k in (CAS, EXCH):
            # lock words live in their own range; their own accesses are atomics
            word = 500 + int(rng.integers(0, lock_words))
            b.ev(k, t, word, int(rng.integers(1, 4)), mask)
        elif k == FENCE:
            b.ev(FENCE, t, 0, int(rng.integers(1, 4)), mask)
        elif k in (SYNCWARP, CG_TILE_SYNC):
            b.ev(k, t, 0, NONE, mask)
        elif k in (SYNCTHREADS, CG_BLOCK_SYNC):
            b.ev(k, t, 0, NONE, 0xFFFFFFFF)
        else:
            b.ev(k, 0, 0, NONE, 0xFFFFFFFF)
    return b.events(), n_blocks, block_dim


def geometry_code(n_blocks: int, block_dim: int) -> int:
    """A KERNEL_BOUNDARY's addr announcing the next kernel's grid: (n_blocks << 32) | block_dim."""
    return (int(n_blocks) << 32) | int(block_dim)


def boundary_event(n_blocks: int = None, block_dim: int = None) -> np.ndarray:
    """One KERNEL_BOUNDARY event (tid 0, scope NONE); addr 0 keeps the geometry, else it carries
    the next kernel's grid."""
    e = np.zeros(1, EVENT_DTYPE)
    e["tk"] = pack_tk(0, KERNEL_BOUNDARY, NONE)
    e["mask"] = 0xFFFFFFFF
    if n_blocks is not None:
        e["addr"] = geometry_code(n_blocks, block_dim)
    return e


def concat_kernels(traces, geoms=None) -> np.ndarray:
    """Join per-kernel traces into one multi-kernel trace, a KERNEL_BOUNDARY between consecutive
    kernels.  ``geoms``: per-kernel (n_blocks, block_dim); when given, each boundary announces the
    next kernel's grid (the trace descriptor carries the first).  Returns the trace; kernel k's
    events start at sum(len(t) + 1 for t in traces[:k])."""
    parts = []
    for k, t in enumerate(traces):
        if k:
            parts.append(boundary_event(*geoms[k]) if geoms is not None else boundary_event())
        parts.append(np.asarray(t, EVENT_DTYPE))
    return np.concatenate(parts) if parts else np.zeros(0, EVENT_DTYPE)


def warp_instr_trace(seed: int, n_instr: int, n_blocks: int = 2, block_dim: int = 64, n_words: int = 24,
                     p_shared: float = 0.5, weights=None):
    """Warp-instruction-shaped fuzz trace: each step picks a warp, an active mask and a kind and
    emits one event per active lane in ascending lane order (the trace convention of
    include/igd.h).  With probability ``p_shared`` an access instruction's lanes all touch one
    word (the shape §6.5's coalescing targets), else each lane picks its own word.
    Returns (events, n_blocks, block_dim)."""
    rng = np.random.default_rng(seed)
    g = Geometry(n_blocks, block_dim)
    b = TraceBuilder(n_blocks, block_dim)
    if weights is None:
        weights = [30, 14, 16, 3, 2, 8, 4, 3, 1]   # LD ST ATOM CAS EXCH FENCE SYNCWARP SYNCTHREADS GRID
    w = np.asarray(weights, float)
    w = w / w.sum()
    for _ in range(n_instr):
        k = int(rng.choice(len(weights), p=w))
        blk = int(rng.integers(0, n_blocks))
        wi = int(rng.integers(0, (block_dim + 31) // 32))
        lanes_here = min(32, block_dim - wi * 32)
        full = (1 << lanes_here) - 1
        r = rng.random()
        mask = full if r < 0.4 else (int(rng.integers(1, 1 << lanes_here)) if r < 0.9 else 1 << int(rng.integers(0, lanes_here)))
        lanes = [l for l in range(lanes_here) if (mask >> l) & 1]
        tid0 = blk * block_dim + wi * 32
        if k in (LD, ST, ATOM, CAS, EXCH):
            scope = NONE if k in (LD, ST) else int(rng.integers(1, 4))
            if k in (CAS, EXCH):
                shared_word = 500 + int(rng.integers(0, 3))
            else:
                shared_word = int(rng.integers(0, n_words))
            shared = rng.random() < p_shared or k in (CAS, EXCH)
            for l in lanes:
                word = shared_word if shared else int(rng.integers(0, n_words))
                b.ev(k, tid0 + l, word, scope, mask)
        elif k == FENCE:
            s = int(rng.integers(1, 4))
            for l in lanes:
                b.ev(FENCE, tid0 + l, 0, s, mask)
        elif k == SYNCWARP:
            b.ev(SYNCWARP, tid0 + lanes[0], 0, NONE, mask)
        elif k == SYNCTHREADS:
            b.ev(SYNCTHREADS, blk * block_dim, 0, NONE, 0xFFFFFFFF)
        else:
            b.ev(GRID_SYNC, 0, 0, NONE, 0xFFFFFFFF)
    _ = g
    return b.events(), n_blocks, block_dim
