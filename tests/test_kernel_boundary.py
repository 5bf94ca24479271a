"""Multi-kernel traces (reading A31 in DESIGN.md): a KERNEL_BOUNDARY event
ends one kernel.  Its implicit all-thread barrier orders every access
before it before every access after it, and the locking protocol is inferred per kernel
(P:1163-1165), so a multi-kernel trace must report exactly the union of its kernels' reports.

Pins of the oracle (CPU, `-m "not gpu"`):
  * composition law: oracle(T1 | KB | T2 | ...) == union of oracle(Tk), each shifted to its
    position -- an identity between runs on different inputs, so a boundary that leaked state
    (shadow entries, lock tables, isThread, counters) across kernels fails it;
  * worked examples: a message-passing pair split by a boundary is race-free; a lock held
    at the end of kernel 1 does not protect or indict kernel 2;
  * field rules of the new kind.
GPU parity (`-m gpu`): libigd == oracle on multi-kernel traces, element by element.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import full_tuples

LOCKY = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]


def shifted_union(parts, nb, bd):
    """Reports of each kernel run alone, shifted to the kernel's position in the joined trace."""
    out, base = [], 0
    for t in parts:
        r = oracle.run(t, nb, bd).copy()
        r["cur"] += np.uint64(base)
        r["prev"] += np.uint64(base)
        out.append(r)
        base += len(t) + 1
    allr = np.concatenate(out) if out else np.zeros(0, oracle.REPORT_DTYPE)
    return allr[np.argsort(allr["cur"], kind="stable")]


def kernels_of(seed, k, n, nb, bd, **kw):
    parts = []
    for j in range(k):
        ev, _, _ = tg.random_trace(seed * 31 + j, n, n_blocks=nb, block_dim=bd, **kw)
        parts.append(ev)
    return parts


@pytest.mark.parametrize("batch", range(4))
def test_composition_law_random(batch):
    for seed in range(batch * 60, (batch + 1) * 60):
        rng = np.random.default_rng(seed)
        nb, bd = int(rng.integers(1, 4)), int(rng.choice([32, 64, 96]))
        kw = dict(weights=LOCKY, lock_words=3, p_lock_data=0.3) if seed % 2 else dict(n_words=6)
        parts = kernels_of(seed, int(rng.integers(2, 5)), int(rng.integers(1, 150)), nb, bd, **kw)
        joined = tg.concat_kernels(parts)
        assert full_tuples(oracle.run(joined, nb, bd)) == full_tuples(shifted_union(parts, nb, bd)), f"seed {seed}"


def test_composition_law_is_not_vacuous():
    # without the boundaries the same concatenation reports cross-kernel pairs
    diff = 0
    for seed in range(40):
        parts = kernels_of(seed, 3, 120, 2, 64, n_words=4)
        plain = np.concatenate(parts)
        diff += len(oracle.run(plain, 2, 64)) != len(shifted_union(parts, 2, 64))
    assert diff > 20


def test_families_joined():
    import tracegen.families as F

    a, nb, bd, _ = F.generate(1)               # C1 litmus: {R4, R2}
    b, _, _, _ = F.generate(1, fixed=True)     # race-free variant
    joined = tg.concat_kernels([a, b, a])
    r = oracle.run(joined, nb, bd)
    assert sorted(int(t) for t in r["type"]) == [2, 2, 4, 4]
    assert full_tuples(r) == full_tuples(shifted_union([a, b, a], nb, bd))


def test_message_passing_split_by_boundary():
    # W1 shape (Fig. 3): producer stores in block 0, consumer loads in block 1, no fence.
    b = tg.TraceBuilder(2, 64)
    b.st(0, 7)
    b.ld(64, 7)
    assert [int(x) for x in oracle.run(b.events(), 2, 64)["type"]] == [4]
    b = tg.TraceBuilder(2, 64)
    b.st(0, 7)
    b.kernel_boundary()
    b.ld(64, 7)
    assert len(oracle.run(b.events(), 2, 64)) == 0


def test_lock_state_resets():
    # kernel 1: thread 0 acquires lock L (CAS + device fence) and accesses x under it, never
    # releasing.  Kernel 2: thread 64 accesses x with no lock, then thread 0 again with no lock.
    def k1(b):
        b.cas(0, 900, mask=1)
        b.fence(0, tg.DEVICE, mask=1)
        b.st(0, 5, mask=1)

    b = tg.TraceBuilder(2, 64)
    k1(b)
    b.st(64, 5, mask=1)   # same kernel: R4 (block 1 vs block 0, no fence after md)
    same = oracle.run(b.events(), 2, 64)
    assert [int(x) for x in same["type"]] == [4]
    b = tg.TraceBuilder(2, 64)
    k1(b)
    b.kernel_boundary()
    b.st(64, 5, mask=1)   # first access of x in kernel 2: P1
    b.st(0, 5, mask=1)    # thread 0 holds no lock any more: lock sets {} vs {} -> no R5; R4 applies
    r = oracle.run(b.events(), 2, 64)
    assert [(int(x["type"]), int(x["cur"]), int(x["prev"])) for x in r] == [(4, 5, 4)]


@pytest.mark.parametrize("field", ["tid", "scope", "addr"])
def test_boundary_field_rules(field):
    ev = tg.concat_kernels([tg.random_trace(3, 20, n_blocks=2, block_dim=64)[0]] * 2)
    at = 20
    assert (ev["tk"][at] >> 24) & 0xF == tg.KERNEL_BOUNDARY
    if field == "tid":
        ev["tk"][at] = tg.pack_tk(1, tg.KERNEL_BOUNDARY, 0)
    elif field == "scope":
        ev["tk"][at] = tg.pack_tk(0, tg.KERNEL_BOUNDARY, tg.DEVICE)
    else:
        ev["addr"][at] = 64
    with pytest.raises(oracle.OracleError) as e:
        oracle.run(ev, 2, 64)
    assert e.value.bad_index == at


# ---------------------------------------------------------------- GPU parity
@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def _same(det, ev, nb, bd, what):
    want = oracle.run(ev, nb, bd)
    det.load(ev, nb, bd)
    det.detect()
    got = det.reports()
    assert len(got) == len(want), f"{what}: {len(got)} GPU vs {len(want)} oracle"
    assert np.array_equal(got, want), f"{what}"
    return len(want)


@pytest.mark.gpu
@pytest.mark.parametrize("batch", range(2))
def test_gpu_random_kernels(det, batch):
    for seed in range(batch * 100, (batch + 1) * 100):
        rng = np.random.default_rng(seed)
        nb, bd = int(rng.integers(1, 4)), int(rng.choice([32, 64, 96]))
        kw = dict(weights=LOCKY, lock_words=3, p_lock_data=0.3) if seed % 2 else dict(n_words=8)
        parts = kernels_of(seed, int(rng.integers(1, 6)), int(rng.integers(1, 200)), nb, bd, **kw)
        _same(det, tg.concat_kernels(parts), nb, bd, f"seed {seed}")


@pytest.mark.gpu
def test_gpu_boundaries_drawn_anywhere(det):
    # boundaries as a 13th kind drawn at random, several per trace, across tiles
    w = LOCKY + [2]
    for seed in range(50):
        ev, nb, bd = tg.random_trace(5000 + seed, 400, n_words=10, weights=w, lock_words=4, p_lock_data=0.2)
        _same(det, ev, nb, bd, f"seed {seed}")


@pytest.mark.gpu
def test_gpu_multi_tile_kernels(det):
    from test_gpu_parity import _fast_random

    parts = [_fast_random(100 + k, 60_000, 40 + 200 * k, 4, 64, LOCKY, lock_words=20)[0] for k in range(4)]
    ev = tg.concat_kernels(parts)
    assert _same(det, ev, 4, 64, "4 kernels x 60k") > 0


@pytest.mark.gpu
def test_gpu_families_joined(det):
    import tracegen.families as F

    p1 = F.Plan(3, n=300_000, seed=11)
    p2 = F.Plan(3, n=300_000, seed=12)
    a, b = p1.fill(), p2.fill()
    ev = tg.concat_kernels([a, b])
    assert _same(det, ev, p1.n_blocks, p1.block_dim, "C3 x 2") >= 0


@pytest.mark.gpu
def test_gpu_boundary_field_rules(det):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev = tg.concat_kernels([tg.random_trace(3, 20, n_blocks=2, block_dim=64)[0]] * 2)
    ev["tk"][20] = tg.pack_tk(1, tg.KERNEL_BOUNDARY, 0)
    det.load(ev, 2, 64)
    with pytest.raises(igd.IgdError) as e:
        det.detect()
    assert e.value.code == igd.igd.IGD_ETRACE and e.value.bad_index == 20


# ---- per-kernel geometry (reading A34: "the number of warps per threadblock remains
# constant for a kernel but can vary across kernels") ----------------------------------------------
def shifted_union_geo(parts, geoms):
    out, base = [], 0
    for t, (nb, bd) in zip(parts, geoms):
        r = oracle.run(t, nb, bd).copy()
        r["cur"] += np.uint64(base)
        r["prev"] += np.uint64(base)
        out.append(r)
        base += len(t) + 1
    allr = np.concatenate(out) if out else np.zeros(0, oracle.REPORT_DTYPE)
    return allr[np.argsort(allr["cur"], kind="stable")]


def mixed_geometry_kernels(seed, k, n):
    rng = np.random.default_rng(seed)
    parts, geoms = [], []
    for j in range(k):
        nb, bd = int(rng.integers(1, 5)), int(rng.choice([16, 32, 48, 64, 96, 128]))
        kw = dict(weights=LOCKY, lock_words=3, p_lock_data=0.3) if (seed + j) % 2 else dict(n_words=6)
        ev, _, _ = tg.random_trace(seed * 37 + j, int(rng.integers(1, n)), n_blocks=nb, block_dim=bd, **kw)
        parts.append(ev)
        geoms.append((nb, bd))
    return parts, geoms


@pytest.mark.parametrize("batch", range(4))
def test_composition_law_mixed_geometry(batch):
    # T1 on grid g1 | KB(g2) | T2 on grid g2 | ... == each kernel run alone on its own grid, shifted
    for seed in range(batch * 50, (batch + 1) * 50):
        parts, geoms = mixed_geometry_kernels(seed, 3, 150)
        joined = tg.concat_kernels(parts, geoms)
        got = full_tuples(oracle.run(joined, *geoms[0]))
        assert got == full_tuples(shifted_union_geo(parts, geoms)), f"seed {seed}"


def test_geometry_change_is_not_vacuous():
    # the same events read under the first kernel's grid would be judged differently: with 64-thread
    # blocks t0 and t40 share a block (R3 without a barrier); with 32-thread blocks they do not (R4)
    b = tg.TraceBuilder(1, 64)
    b.ld(0, 9)                      # kernel 1: nothing
    b.kernel_boundary(4, 32)        # kernel 2: 4 blocks x 32 threads
    b.st(0, 5)
    b.ld(40, 5)
    ev = b.events()
    r = oracle.run(ev, 1, 64)
    assert [(int(x["cur"]), int(x["prev"]), int(x["type"])) for x in r] == [(3, 2, 4)]
    same = ev.copy()
    same["addr"][1] = 0             # no geometry change: t40 is in t0's block -> R3
    assert [int(x["type"]) for x in oracle.run(same, 1, 64)] == [3]


@pytest.mark.parametrize("code,ok", [(0, True), ((2 << 32) | 64, True), ((1 << 32) | (1 << 24), True),
                                      (64, False), (2 << 32, False), ((2 << 32) | (1 << 24), False)])
def test_boundary_geometry_field_rule(code, ok):
    b = tg.TraceBuilder(1, 64)
    b.st(0, 1)
    b.ev(tg.KERNEL_BOUNDARY, 0, 0, tg.NONE, 0xFFFFFFFF, addr=code)
    b.st(0, 1)
    if ok:
        assert len(oracle.run(b.events(), 1, 64)) == 0
    else:
        with pytest.raises(oracle.OracleError) as e:
            oracle.run(b.events(), 1, 64)
        assert e.value.bad_index == 1


def test_validation_uses_each_kernels_grid():
    # tid 100 is out of range for 1 x 64 but valid after a boundary to 2 x 64, and vice versa
    b = tg.TraceBuilder(1, 64)
    b.st(0, 1)
    b.kernel_boundary(2, 64)
    b.st(100, 1)
    b.kernel_boundary(1, 32)
    b.st(40, 2)                     # 1 x 32 grid: tid 40 is invalid here
    with pytest.raises(oracle.OracleError) as e:
        oracle.run(b.events(), 1, 64)
    assert e.value.bad_index == 4


@pytest.mark.gpu
@pytest.mark.parametrize("batch", range(3))
def test_gpu_mixed_geometry_kernels(det, batch):
    # libigd runs the segments between grid changes on their own grids: identical to the oracle
    for seed in range(1000 + batch * 40, 1000 + (batch + 1) * 40):
        parts, geoms = mixed_geometry_kernels(seed, int(np.random.default_rng(seed).integers(2, 5)), 200)
        joined = tg.concat_kernels(parts, geoms)
        det.load(joined, *geoms[0])
        det.detect()
        assert np.array_equal(det.reports(), oracle.run(joined, *geoms[0])), f"seed {seed}"


@pytest.mark.gpu
def test_gpu_mixed_geometry_multi_tile(det):
    # large kernels on different grids (several check / sort tiles per segment), plain boundaries
    # inside a segment too
    from test_gpu_parity import _fast_random

    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    geoms = [(3, 96), (16, 128), (5, 48), (9, 16)]
    parts = [_fast_random(60 + k, 40_000 + 10_000 * k, 300, nb, bd, w)[0] for k, (nb, bd) in enumerate(geoms)]
    parts[1] = tg.concat_kernels([parts[1], parts[1][:5000]])  # a same-grid boundary inside
    joined = tg.concat_kernels(parts, geoms)
    det.load(joined, *geoms[0])
    det.detect()
    want = oracle.run(joined, *geoms[0])
    assert len(want) > 0 and np.array_equal(det.reports(), want)


@pytest.mark.gpu
@pytest.mark.parametrize("where", ["boundary_code", "tid_in_later_kernel", "first_kernel"])
def test_gpu_mixed_geometry_bad_event(det, where):
    import paper_conf_sosp_kamathb21_b200 as igd

    b = tg.TraceBuilder(1, 64)
    b.st(0, 1)
    b.st(60, 2)
    b.kernel_boundary(2, 64)
    b.st(100, 1)
    b.kernel_boundary(1, 32)
    b.st(20, 2)
    ev = b.events()
    if where == "boundary_code":
        ev["addr"][4] = 1 << 32            # block_dim 0
    elif where == "tid_in_later_kernel":
        ev["tk"][5] = tg.pack_tk(40, tg.ST, 0)   # tid 40 on a 1 x 32 grid
        ev["mask"][5] = 1 << 8
    else:
        ev["tk"][1] = tg.pack_tk(70, tg.ST, 0)   # tid 70 on the first 1 x 64 grid
        ev["mask"][1] = 1 << 6
    with pytest.raises(oracle.OracleError) as eo:
        oracle.run(ev, 1, 64)
    det.load(ev, 1, 64)
    with pytest.raises(igd.IgdError) as eg:
        det.detect()
    assert eg.value.code == igd.igd.IGD_ETRACE and eg.value.bad_index == eo.value.bad_index
