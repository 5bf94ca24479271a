"""Independent evaluators that pin the oracle.

None of these shares code with oracle/igd_oracle.c or with the CUDA path.  Each restates
PAPER.md Table 2 from a different angle:

* ``bf_scratch``     -- from-scratch per-access evaluation: for every access rescan the
                        word's whole history and count synchronization events strictly
                        between md and the access (no incremental shadow state).  O(n^2).
* ``pairwise``       -- for traces whose data words have <= 2 accesses: a scoped
                        happens-before predicate per conflicting pair (C.7 2).
* ``closed_form_syncfree`` -- vectorised numpy formulation for LD/ST/ATOM-only traces
                        (no sync events, no locks), usable at 10^6-10^8 events (C.7 4).
"""
from __future__ import annotations

import numpy as np

import tracegen as tg

LD, ST, ATOM, CAS, EXCH, FENCE = 0, 1, 2, 3, 4, 5
SYNCWARP, SYNCTHREADS, GRID = 6, 7, 8
CG_TILE, CG_BLOCK, CG_GRID = 9, 10, 11
KERNEL_BOUNDARY = 12
ACCESS = (LD, ST, ATOM, CAS, EXCH)
ATOMICS = (ATOM, CAS, EXCH)


def _decode(events):
    addr, tid, kind, scope, mask = tg.unpack(events)
    kind = kind.astype(np.int64).copy()
    kind[kind == CG_TILE] = SYNCWARP       # A15: CG syncs are their constituents
    kind[kind == CG_BLOCK] = SYNCTHREADS
    kind[kind == CG_GRID] = GRID
    scope = scope.astype(np.int64).copy()
    scope[scope == 3] = 2                  # A12: SYSTEM == DEVICE
    return ([int(x) for x in addr], [int(x) for x in tid], [int(x) for x in kind],
            [int(x) for x in scope], [int(x) for x in mask], [int(x) for x in tg.unpack(events)[2]])


class _Geo:
    def __init__(self, nb, bd):
        self.D = bd
        self.Wb = (bd + 31) // 32

    def block(self, t):
        return t // self.D

    def warp(self, t):
        return (t // self.D) * self.Wb + (t % self.D) // 32

    def lane(self, t):
        return (t % self.D) % 32


def _h18(word):
    # reading A8, restated: low 32 bits of word * 0x9E3779B1, top 18 bits
    return ((word & 0xFFFFFFFF) * 0x9E3779B1 & 0xFFFFFFFF) >> 14


def _bloom(h):
    return (1 << (h % 16)) | (1 << ((h // 16) % 16))


def lock_replay(events, nb, bd):
    """Held-lock Bloom of each event's own thread just before the event (independent
    restatement of §6.3, readings A9-A11, A15).  Returns a list L[i]."""
    geo = _Geo(nb, bd)
    addr, tid, kind, scope, mask, _ = _decode(events)
    warp_tab = {}     # warp -> list of [hash, scope, active]
    thr_tab = {}      # tid  -> list of [hash, scope, active]
    per_thread = set()
    L = [0] * len(kind)

    def table(t):
        w = geo.warp(t)
        if w in per_thread:
            return thr_tab.setdefault(t, [])
        return warp_tab.setdefault(w, [])

    for i in range(len(kind)):
        k, t = kind[i], tid[i]
        if k in ACCESS:
            L[i] = 0
            for h, s, act in table(t):
                if act:
                    L[i] |= _bloom(h)
        if k == FENCE:
            for e in table(t):
                if e[1] <= scope[i]:
                    e[2] = True
        elif k == GRID:
            for tab in list(warp_tab.values()) + list(thr_tab.values()):
                for e in tab:
                    e[2] = True          # every scope <= DEVICE
        elif k == CAS:
            if bin(mask[i]).count("1") > 1:
                per_thread.add(geo.warp(t))
            tab = table(t)
            h = _h18(addr[i] >> 2)
            if not any(e[0] == h and e[1] == scope[i] for e in tab) and len(tab) < 3:
                tab.append([h, scope[i], False])
        elif k == EXCH:
            tab = table(t)
            h = _h18(addr[i] >> 2)
            tab[:] = [e for e in tab if not (e[0] == h and e[1] == scope[i])]
    return L


def _sync_between(kind, tid, scope, geo, lo, hi, what, ent):
    """Is there a sync event of class ``what`` for entity ``ent`` strictly inside (lo, hi)?"""
    for x in range(lo + 1, hi):
        k = kind[x]
        if what == "any_fence" and ((k == FENCE and tid[x] == ent) or k == GRID):
            return True
        if what == "dev_fence" and ((k == FENCE and tid[x] == ent and scope[x] >= 2) or k == GRID):
            return True
        if what == "warp_bar" and k == SYNCWARP and geo.warp(tid[x]) == ent:
            return True
        if what == "block_bar" and ((k == SYNCTHREADS and geo.block(tid[x]) == ent) or k == GRID):
            return True
    return False


def _sync_count(kind, tid, scope, geo, lo, hi, what, ent):
    """Number of events strictly inside (lo, hi) that advance the paper's ID ``what`` of
    entity ``ent`` (Fig. 4 fields; grid syncs are a device fence by every thread and a barrier
    for every block, A15)."""
    n = 0
    for x in range(lo + 1, hi):
        k = kind[x]
        if what == "WarpBarID":
            n += k == SYNCWARP and geo.warp(tid[x]) == ent
        elif what == "BlkBarID":
            n += (k == SYNCTHREADS and geo.block(tid[x]) == ent) or k == GRID
        elif what == "DevFenceID":
            n += (k == FENCE and tid[x] == ent and scope[x] >= 2) or k == GRID
        elif what == "BlkFenceID":
            n += k == FENCE and tid[x] == ent and scope[x] == 1
    return n


WIDTH = {"WarpBarID": 6, "BlkBarID": 8, "DevFenceID": 6, "BlkFenceID": 6}  # Fig. 4


def bf_scratch(events, nb, bd, paper_counters=False):
    """From-scratch evaluator (C.7 1).  Returns a list of (addr, cur, prev, type, cur_kind,
    prev_kind) sorted by cur.  ``paper_counters``: an ID counts as changed only when the number
    of its events since md is not a multiple of 2^width (reading A33)."""
    geo = _Geo(nb, bd)
    addr, tid, kind, scope, mask, rawkind = _decode(events)
    L = lock_replay(events, nb, bd)
    out = []
    hist = {}  # word -> list of access indices (so far)
    for i in range(len(kind)):
        k = kind[i]
        if k not in ACCESS:
            continue
        a = addr[i] >> 2
        H = hist.setdefault(a, [])
        if H:
            c = tid[i]
            LA = H[-1]
            writes = [j for j in H if kind[j] != LD]
            LW = writes[-1] if writes else None
            seq = H + [i]
            devS = any(geo.block(tid[x]) != geo.block(tid[y]) for x, y in zip(seq, seq[1:]))
            blkS = any(geo.block(tid[x]) == geo.block(tid[y]) and geo.warp(tid[x]) != geo.warp(tid[y])
                       for x, y in zip(seq, seq[1:]))
            ats = [j for j in H if kind[j] in ATOMICS]
            atomic = bool(ats)
            ascope = scope[ats[-1]] if ats else 0
            locks = L[LA]
            if not (k == LD and LW is None):
                md = LW if k == LD else LA
                p = tid[md]
                same_w = geo.warp(p) == geo.warp(c)
                same_b = geo.block(p) == geo.block(c)
                P3 = p == c
                if paper_counters:
                    def moved(what, ent):
                        return _sync_count(kind, tid, scope, geo, md, i, what, ent) % (1 << WIDTH[what]) != 0
                    P4 = same_w and (moved("WarpBarID", geo.warp(c)) or (mask[i] >> geo.lane(p)) & 1 == 1)
                    P5 = same_b and moved("BlkBarID", geo.block(c))
                else:
                    P4 = same_w and (_sync_between(kind, tid, scope, geo, md, i, "warp_bar", geo.warp(c))
                                     or (mask[i] >> geo.lane(p)) & 1 == 1)
                    P5 = same_b and _sync_between(kind, tid, scope, geo, md, i, "block_bar", geo.block(c))
                P6 = atomic and k in ATOMICS and (same_b or ascope == 2)
                if not (P3 or P4 or P5 or P6):
                    if paper_counters:
                        noDev = not moved("DevFenceID", p)
                        noAny = noDev and not moved("BlkFenceID", p)
                    else:
                        noAny = not _sync_between(kind, tid, scope, geo, md, i, "any_fence", p)
                        noDev = not _sync_between(kind, tid, scope, geo, md, i, "dev_fence", p)
                    typ = 0
                    if atomic and ascope == 1 and geo.block(tid[LW]) != geo.block(c):
                        typ = 1
                    elif same_w and noAny and not devS and not blkS:
                        typ = 2
                    elif same_b and noAny and not devS:
                        typ = 3
                    elif not same_b and noDev:
                        typ = 4
                    elif (locks | L[i]) != 0 and (locks & L[i]) == 0:
                        typ = 5
                    if typ:
                        out.append((a << 2, i, md, typ, rawkind[i], rawkind[md]))
        H.append(i)
    return out


def pairwise(events, nb, bd):
    """Pairwise evaluator (C.7 2) for words with at most two accesses.  Returns (reports,
    words_with_two_accesses); reports are (addr, cur, prev, type) for those words only."""
    geo = _Geo(nb, bd)
    addr, tid, kind, scope, mask, _ = _decode(events)
    L = lock_replay(events, nb, bd)
    by_word = {}
    for i, k in enumerate(kind):
        if k in ACCESS:
            by_word.setdefault(addr[i] >> 2, []).append(i)
    out = []
    eligible = set()
    for a, idxs in by_word.items():
        if len(idxs) > 2:
            continue
        eligible.add(a)
        if len(idxs) < 2:
            continue
        j, i = idxs
        if kind[j] == LD and kind[i] == LD:
            continue
        tj, ti = tid[j], tid[i]
        same_w = geo.warp(tj) == geo.warp(ti)
        same_b = geo.block(tj) == geo.block(ti)

        def between(pred):
            return any(pred(x) for x in range(j + 1, i))

        safe = (tj == ti
                or (same_w and (between(lambda x: kind[x] == SYNCWARP and geo.warp(tid[x]) == geo.warp(ti))
                                or (mask[i] >> geo.lane(tj)) & 1 == 1))
                or (same_b and between(lambda x: (kind[x] == SYNCTHREADS and geo.block(tid[x]) == geo.block(ti))
                                       or kind[x] == GRID))
                or (kind[j] in ATOMICS and kind[i] in ATOMICS and (same_b or scope[j] == 2)))
        if safe:
            continue
        fenced = between(lambda x: (kind[x] == FENCE and tid[x] == tj) or kind[x] == GRID)
        dfenced = between(lambda x: (kind[x] == FENCE and tid[x] == tj and scope[x] == 2) or kind[x] == GRID)
        typ = 0
        if kind[j] in ATOMICS and scope[j] == 1 and not same_b:
            typ = 1
        elif same_w and not fenced:
            typ = 2
        elif same_b and not fenced:
            typ = 3
        elif not same_b and not dfenced:
            typ = 4
        elif (L[j] | L[i]) != 0 and (L[j] & L[i]) == 0:
            typ = 5
        if typ:
            out.append((a << 2, i, j, typ))
    out.sort(key=lambda r: r[1])
    return out, eligible


def closed_form_syncfree(events, nb, bd):
    """Vectorised evaluation for traces whose kinds are all LD/ST/ATOM (C.7 4).
    Returns arrays (addr, cur, prev, type) sorted by cur."""
    addr, tid, kind, scope, mask = tg.unpack(events)
    kind = kind.astype(np.int64)
    assert np.all((kind == LD) | (kind == ST) | (kind == ATOM)), "sync-free traces only"
    n = len(kind)
    if n == 0:
        e = np.zeros(0, np.int64)
        return e.astype(np.uint64), e, e, e
    scope = np.where(scope == 3, 2, scope).astype(np.int64)
    tid = tid.astype(np.int64)
    word = (addr >> np.uint64(2)).astype(np.uint64)
    idx = np.arange(n, dtype=np.int64)
    order = np.lexsort((idx, word))
    w, ix, t, k, s, m = word[order], idx[order], tid[order], kind[order], scope[order], mask[order].astype(np.int64)
    D, Wb = bd, (bd + 31) // 32
    blk = t // D
    wrp = blk * Wb + (t % D) // 32
    lane = (t % D) % 32
    pos = np.arange(n, dtype=np.int64)
    head = np.ones(n, bool)
    head[1:] = w[1:] != w[:-1]
    seg_start = np.maximum.accumulate(np.where(head, pos, 0))
    # last write / last atomic strictly before each position, within the segment
    wpos = np.maximum.accumulate(np.where(k != LD, pos, -1))
    apos = np.maximum.accumulate(np.where(k == ATOM, pos, -1))
    lw = np.full(n, -1, np.int64)
    la_at = np.full(n, -1, np.int64)
    lw[1:] = wpos[:-1]
    la_at[1:] = apos[:-1]
    lw = np.where(lw >= seg_start, lw, -1)
    la_at = np.where(la_at >= seg_start, la_at, -1)
    # sharing flags: inclusive segmented OR of adjacent-pair predicates
    prev_blk = np.roll(blk, 1)
    prev_wrp = np.roll(wrp, 1)
    devp = (~head) & (prev_blk != blk)
    blkp = (~head) & (prev_blk == blk) & (prev_wrp != wrp)

    def seg_or(x):
        c = np.cumsum(x.astype(np.int64))
        base = np.where(head, c - x.astype(np.int64), 0)
        base = np.maximum.accumulate(np.where(head, base, -1))
        return (c - base) > 0

    devS = seg_or(devp)
    blkS = seg_or(blkp)
    atomic = la_at >= 0
    ascope = np.where(atomic, s[np.maximum(la_at, 0)], 0)
    md = np.where(k == LD, lw, pos - 1)
    valid = ~head
    p2 = (k == LD) & (lw < 0)
    cand = valid & ~p2
    mdc = np.maximum(md, 0)
    p = t[mdc]
    same_w = wrp[mdc] == wrp
    same_b = blk[mdc] == blk
    P3 = p == t
    P4 = same_w & (((m >> lane[mdc]) & 1) == 1)
    P6 = atomic & (k == ATOM) & (same_b | (ascope == 2))
    chk = cand & ~(P3 | P4 | P6)
    lwc = np.maximum(lw, 0)
    R1 = atomic & (ascope == 1) & (blk[lwc] != blk)
    R2 = same_w & ~devS & ~blkS
    R3 = same_b & ~devS
    R4 = ~same_b
    typ = np.where(R1, 1, np.where(R2, 2, np.where(R3, 3, np.where(R4, 4, 0))))
    sel = chk & (typ > 0)
    cur = ix[sel]
    prev = ix[mdc[sel]]
    a = (w[sel] << np.uint64(2))
    ty = typ[sel]
    o = np.argsort(cur, kind="stable")
    return a[o], cur[o], prev[o], ty[o]


def bf_scratch_modes(events, nb, bd, sticky=False, tag_log2=0, last_k=1):
    """From-scratch evaluator of the paper-fidelity modes, same approach as
    bf_scratch -- every access rescans the history of its metadata entry:

    * ``sticky`` (reading A35): P3 and P4 also need the entry's sticky DevShared and BlkShared
      clear, P5 DevShared clear, as Table 2 writes them;
    * ``tag_log2`` (reading A36): word w uses entry w mod 2^tag_log2 whose 10-bit Tag is the next
      bits of w; the entry's history is the longest run of its most recent accesses that carry
      the current access's tag (an access with another tag claimed the entry, P1);
    * ``last_k`` (reading A37): the candidates are the last k writers (loads) or accessors,
      newest first; the first racy candidate is reported.
    Kernel boundaries (A31) end every history.  Returns the same tuples as bf_scratch."""
    geo = _Geo(nb, bd)
    addr, tid, kind, scope, mask, rawkind = _decode(events)
    L = lock_replay(events, nb, bd)
    C = (1 << tag_log2) if tag_log2 else None
    out = []
    hist = {}  # entry -> list of (access index, tag)
    for i in range(len(kind)):
        k = kind[i]
        if k == KERNEL_BOUNDARY:
            hist = {}
            continue
        if k not in ACCESS:
            continue
        a = addr[i] >> 2
        ent, tag = (a % C, (a // C) % 1024) if C else (a, 0)
        seq_all = hist.setdefault(ent, [])
        H = []
        for j, tj in reversed(seq_all):
            if tj != tag:
                break
            H.insert(0, j)
        if H:
            c = tid[i]
            writes = [j for j in H if kind[j] != LD]
            seq = H + [i]
            devS = any(geo.block(tid[x]) != geo.block(tid[y]) for x, y in zip(seq, seq[1:]))
            blkS = any(geo.block(tid[x]) == geo.block(tid[y]) and geo.warp(tid[x]) != geo.warp(tid[y])
                       for x, y in zip(seq, seq[1:]))
            ats = [j for j in H if kind[j] in ATOMICS]
            atomic = bool(ats)
            ascope = scope[ats[-1]] if ats else 0
            locks = L[H[-1]]
            LW = writes[-1] if writes else None
            if not (k == LD and LW is None):
                cands = (writes if k == LD else H)[::-1][:last_k]
                for md in cands:
                    p = tid[md]
                    same_w = geo.warp(p) == geo.warp(c)
                    same_b = geo.block(p) == geo.block(c)
                    P3 = p == c
                    P4 = same_w and (_sync_between(kind, tid, scope, geo, md, i, "warp_bar", geo.warp(c))
                                     or (mask[i] >> geo.lane(p)) & 1 == 1)
                    P5 = same_b and _sync_between(kind, tid, scope, geo, md, i, "block_bar", geo.block(c))
                    if sticky:
                        P3 = P3 and not devS and not blkS
                        P4 = P4 and not devS and not blkS
                        P5 = P5 and not devS
                    P6 = atomic and k in ATOMICS and (same_b or ascope == 2)
                    if P3 or P4 or P5 or P6:
                        continue
                    noAny = not _sync_between(kind, tid, scope, geo, md, i, "any_fence", p)
                    noDev = not _sync_between(kind, tid, scope, geo, md, i, "dev_fence", p)
                    typ = 0
                    if atomic and ascope == 1 and geo.block(tid[LW]) != geo.block(c):
                        typ = 1
                    elif same_w and noAny and not devS and not blkS:
                        typ = 2
                    elif same_b and noAny and not devS:
                        typ = 3
                    elif not same_b and noDev:
                        typ = 4
                    elif (locks | L[i]) != 0 and (locks & L[i]) == 0:
                        typ = 5
                    if typ:
                        out.append((a << 2, i, md, typ, rawkind[i], rawkind[md]))
                        break
        seq_all.append((i, tag))
    return out
