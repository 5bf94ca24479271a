"""Stage-level GPU tests: each kernel against a host reference of THAT stage.
a5 radix sort: stable by key == numpy stable argsort."""
import ctypes

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def gpu_sort(det, keys, vals, bits, mode):
    import torch

    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    lib.igd_debug_radix_sort.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                         ctypes.c_uint32, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
    k = torch.from_numpy(keys.view(np.int32)).cuda()
    v = torch.from_numpy(vals.view(np.int32)).cuda()
    ms = ctypes.c_float()
    rc = lib.igd_debug_radix_sort(det.ctx, k.data_ptr(), v.data_ptr(), len(keys), bits, mode, ctypes.byref(ms))
    assert rc == 0
    return k.cpu().numpy().view(np.uint32), v.cpu().numpy().view(np.uint32), ms.value


@pytest.mark.parametrize("mode", [1])
@pytest.mark.parametrize("n,dist", [(1, "u"), (2, "u"), (4095, "u"), (4097, "u"), (1_000_003, "u"),
                                    (777_777, "skew"), (300_000, "const"), (2_000_001, "hi")])
def test_radix_sort_stable(det, mode, n, dist):
    rng = np.random.default_rng(n + mode)
    if dist == "u":
        keys = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    elif dist == "skew":   # Zipf-like hot keys
        keys = (rng.zipf(1.3, n) % (1 << 30)).astype(np.uint32)
    elif dist == "const":
        keys = np.full(n, 12345, np.uint32)
    else:                  # only high digits vary
        keys = (rng.integers(0, 64, n).astype(np.uint32) << 24)
    vals = np.arange(n, dtype=np.uint32)
    ks, vs, _ = gpu_sort(det, keys, vals, 32, mode)
    order = np.argsort(keys, kind="stable")
    assert np.array_equal(ks, keys[order])
    assert np.array_equal(vs, vals[order])


# ---------------- a2: sync-epoch tables (CSR of per-entity timestamp lists) ----------------
def _entities(ev, nb, bd):
    """Host restatement of the a2 record layout (csrc/common.cuh KeySpace): one (entity,
    timestamp) record per synchronization role of each event, in trace order."""
    import tracegen as tg

    D, Wb = bd, (bd + 31) // 32
    T, W, B = nb * bd, nb * Wb, nb
    ANY, DEV, WB, BB = 0, T, 2 * T, 2 * T + W
    GRID = BB + B
    LOCK = GRID + 1
    KB = LOCK + W
    E = KB + 1
    tk = ev["tk"].astype(np.int64)
    tid, kind, scope = tk & 0xFFFFFF, (tk >> 24) & 0xF, (tk >> 28) & 3
    warp = (tid // D) * Wb + (tid % D) // 32
    blk = tid // D
    recs = []
    for i in range(len(ev)):
        k = int(kind[i])
        if k == tg.FENCE:
            recs.append((ANY + int(tid[i]), i))
            if scope[i] >= 2:
                recs.append((DEV + int(tid[i]), i))
        elif k in (tg.SYNCWARP, tg.CG_TILE_SYNC):
            recs.append((WB + int(warp[i]), i))
        elif k in (tg.SYNCTHREADS, tg.CG_BLOCK_SYNC):
            recs.append((BB + int(blk[i]), i))
        elif k in (tg.GRID_SYNC, tg.CG_GRID_SYNC):
            recs.append((GRID, i))
        elif k in (tg.CAS, tg.EXCH):
            recs.append((LOCK + int(warp[i]), i))
        elif k == tg.KERNEL_BOUNDARY:
            recs.append((KB, i))
    recs.sort(key=lambda r: r[0])  # stable: trace order inside an entity
    ent = np.array([r[0] for r in recs], np.int64)
    ts = np.array([r[1] for r in recs], np.uint32)
    off = np.searchsorted(ent, np.arange(E + 1), side="left").astype(np.uint32)
    return E, off, ts


def _tables(det):
    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    f = lib.igd_debug_sync_tables
    u64p = ctypes.POINTER(ctypes.c_uint64)
    f.argtypes = [ctypes.c_void_p, u64p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
    sizes = (ctypes.c_uint64 * 4)()
    assert f(det.ctx, sizes, None, None, None, None) == 0
    E, ns, T, npts = (int(x) for x in sizes)
    off = np.zeros(E + 1, np.uint32)
    ts = np.zeros(max(ns, 1), np.uint32)
    toff = np.zeros(T + 1, np.uint32)
    tpts = np.zeros(max(npts, 1), np.uint64)
    assert f(det.ctx, sizes, off.ctypes.data, ts.ctypes.data, toff.ctypes.data if npts else None,
             tpts.ctypes.data if npts else None) == 0
    return E, off, ts[:ns], (toff, tpts[:npts]) if npts else None


@pytest.mark.parametrize("seed,n,nb,bd", [(81, 50_000, 3, 96), (82, 200_000, 16, 128), (83, 30_000, 5, 48),
                                         (84, 80_000, 9, 16)])
def test_a2_sync_tables(det, seed, n, nb, bd):
    from test_gpu_parity import _fast_random

    w = [10, 8, 5, 6, 5, 14, 10, 8, 2, 3, 3, 2]
    ev, nb, bd = _fast_random(seed, n, 300, nb, bd, w)
    det.load(ev, nb, bd)
    det.detect()
    E, off, ts, _ = _tables(det)
    E2, off2, ts2 = _entities(ev, nb, bd)
    assert E == E2
    assert np.array_equal(off, off2)
    assert np.array_equal(ts, ts2)


# ---------------- a3: lock inference -> per-thread held-lock change points ----------------
def _change_points(ev, nb, bd):
    """Host restatement of §6.3 (readings A8-A10, A15, A31): replay the lock tables in
    trace order; after every event that can change a thread's held-lock Bloom, record
    (timestamp, Bloom) for each thread of the affected warp(s) whose Bloom changed."""
    import tracegen as tg
    from pins import _bloom, _h18

    D, Wb = bd, (bd + 31) // 32
    T = nb * bd
    tk = ev["tk"].astype(np.int64)
    tid, kind, scope = tk & 0xFFFFFF, (tk >> 24) & 0xF, (tk >> 28) & 3
    scope = np.where(scope == 3, 2, scope)

    def warp_of(t):
        return (t // D) * Wb + (t % D) // 32

    def threads_of(w):
        b, wi = divmod(w, Wb)
        return [b * D + wi * 32 + l for l in range(32) if wi * 32 + l < D]

    wt, tt, is_thread = {}, {}, set()
    held = [0] * T
    pts = [[] for _ in range(T)]
    lock_warps = {warp_of(int(tid[i])) for i in range(len(ev)) if kind[i] in (tg.CAS, tg.EXCH)}

    def table(t):
        w = warp_of(t)
        return tt.setdefault(t, []) if w in is_thread else wt.setdefault(w, [])

    def bloom_of(t):
        b = 0
        for h, s, act in table(t):
            if act:
                b |= _bloom(h)
        return b

    for i in range(len(ev)):
        k, t = int(kind[i]), int(tid[i])
        affected = []
        if k == tg.KERNEL_BOUNDARY:
            wt.clear(); tt.clear(); is_thread.clear()
            affected = sorted(lock_warps)
        elif k in (tg.GRID_SYNC, tg.CG_GRID_SYNC):
            for tab in list(wt.values()) + list(tt.values()):
                for e in tab:
                    e[2] = True
            affected = sorted(lock_warps)
        elif k == tg.FENCE:
            for e in table(t):
                if e[1] <= scope[i]:
                    e[2] = True
            affected = [warp_of(t)]
        elif k == tg.CAS:
            if bin(int(ev["mask"][i])).count("1") > 1:
                is_thread.add(warp_of(t))
            tab, h = table(t), _h18(int(ev["addr"][i]) >> 2)
            if not any(e[0] == h and e[1] == scope[i] for e in tab) and len(tab) < 3:
                tab.append([h, int(scope[i]), False])
            affected = [warp_of(t)]
        elif k == tg.EXCH:
            tab, h = table(t), _h18(int(ev["addr"][i]) >> 2)
            tab[:] = [e for e in tab if not (e[0] == h and e[1] == scope[i])]
            affected = [warp_of(t)]
        for w in affected:
            if w not in lock_warps:
                continue
            for u in threads_of(w):
                b = bloom_of(u)
                if b != held[u]:
                    held[u] = b
                    pts[u].append((i << 16) | b)
    toff = np.zeros(T + 1, np.uint32)
    toff[1:] = np.cumsum([len(p) for p in pts])
    flat = np.array([x for p in pts for x in p], np.uint64)
    return toff, flat


@pytest.mark.parametrize("seed,n,nb,bd", [(91, 20_000, 3, 64), (92, 60_000, 4, 96), (93, 15_000, 2, 48)])
def test_a3_lock_change_points(det, seed, n, nb, bd):
    from test_gpu_parity import _fast_random

    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, 200, nb, bd, w, lock_words=20)
    det.load(ev, nb, bd)
    det.detect()
    _, _, _, lk = _tables(det)
    toff2, pts2 = _change_points(ev, nb, bd)
    assert lk is not None and len(pts2) > 100
    toff, pts = lk
    assert np.array_equal(toff, toff2)
    assert np.array_equal(pts, pts2)


# ---------------- a6: segmented scan state of the shadow pass ----------------
@pytest.mark.parametrize("seed,n,words,nb,bd", [(95, 100_000, 40, 3, 96), (96, 400_000, 9_000, 16, 128),
                                               (97, 300_000, 3, 2, 64)])
def test_a6_scan_state(det, seed, n, words, nb, bd):
    # the ballot scan's per-access state (run in last-k mode, which leaves it in memory) against a
    # numpy segmented scan of the sorted accesses: last writer, scope of the last atomic, sticky
    # DevShared / BlkShared (A5, inclusive), segment heads
    import paper_conf_sosp_kamathb21_b200 as igd
    from test_gpu_parity import _fast_random

    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, words, nb, bd, w)
    det.load(ev, nb, bd)
    det.detect(last_k=2)
    kind_all = (ev["tk"] >> 24) & 0xF
    na = int((kind_all <= 4).sum())
    lib = igd.load_library()
    f = lib.igd_debug_scan_state
    f.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
    st = np.zeros(na, np.uint64)
    keys = np.zeros(na, np.uint32)
    pay = np.zeros(na, np.uint64)
    assert f(det.ctx, na, st.ctypes.data, keys.ctypes.data, pay.ctypes.data) == 0
    idx = (pay & np.uint64(0xFFFFFFFF)).astype(np.int64)
    acc = np.nonzero(kind_all <= 4)[0]
    word = (ev["addr"][acc] >> np.uint64(2)) & np.uint64(0xFFFFFFFF)
    order = np.lexsort((acc, word))
    assert np.array_equal(idx, acc[order]) and np.array_equal(keys, word[order].astype(np.uint32))
    tk = ev["tk"][idx].astype(np.int64)
    t, k, sc = tk & 0xFFFFFF, (tk >> 24) & 0xF, (tk >> 28) & 3
    sc = np.where(sc == 3, 2, sc)
    D, Wb = bd, (bd + 31) // 32
    b = t // D
    wp = b * Wb + (t % D) // 32
    pos = np.arange(na)
    head = np.ones(na, bool)
    head[1:] = keys[1:] != keys[:-1]
    seg = np.maximum.accumulate(np.where(head, pos, 0))
    wpos = np.maximum.accumulate(np.where(k != 0, pos, -1))
    lastw = np.full(na, -1)
    lastw[1:] = wpos[:-1]
    lastw = np.where(lastw >= seg, lastw, -1)
    apos = np.maximum.accumulate(np.where((k >= 2) & (k <= 4), pos, -1))
    lasta = np.full(na, -1)
    lasta[1:] = apos[:-1]
    lasta = np.where(lasta >= seg, lasta, -1)
    asc = np.where(lasta >= 0, sc[np.maximum(lasta, 0)], 0)
    devp = ~head & (np.roll(b, 1) != b)
    blkp = ~head & (np.roll(b, 1) == b) & (np.roll(wp, 1) != wp)

    def seg_or(x):
        c = np.cumsum(x.astype(np.int64))
        base = np.maximum.accumulate(np.where(head, c - x.astype(np.int64), -1))
        return (c - base) > 0

    dev, blk = seg_or(devp), seg_or(blkp)
    g_head = ((st >> np.uint64(36)) & np.uint64(1)).astype(bool)
    assert np.array_equal(g_head, head)
    nh = ~head
    g_lw = (st & np.uint64(0xFFFFFFFF)).astype(np.int64)
    assert np.array_equal(np.where(g_lw == 0xFFFFFFFF, -1, g_lw)[nh], lastw[nh])
    assert np.array_equal(((st >> np.uint64(32)) & np.uint64(3)).astype(np.int64)[nh], asc[nh])
    assert np.array_equal(((st >> np.uint64(34)) & np.uint64(1)).astype(bool)[nh], dev[nh])
    assert np.array_equal(((st >> np.uint64(35)) & np.uint64(1)).astype(bool)[nh], blk[nh])
