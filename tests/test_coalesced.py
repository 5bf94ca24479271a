"""Warp-coalesced check mode (§6.5; reading A32 in DESIGN.md):
when the active lanes of one warp instruction all load, or all atomically update (ATOM), one
word, only the first lane is checked and recorded on behalf of the group.

Pins of the oracle (CPU):
  * deletion equivalence: oracle(T, coalesce) == oracle(T without the non-first members), with
    report indices mapped back -- the group detection is restated here in numpy, independently
    of the oracle's C loop, and the right side is the plain (pinned) replay;
  * worked example: a warp-wide unfenced load of another block's flag is one R4, not 32;
  * traces without multi-lane same-word LD/ATOM instructions are unchanged.
GPU parity (`-m gpu`): libigd with IGD_DETECT_COALESCE == oracle(coalesce=True).
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import full_tuples


def members(ev, nb, bd):
    """Boolean array: event i is a non-first member of a coalesced group (A32), by a direct
    scan over warp instructions."""
    addr, tid, kind, scope, mask = tg.unpack(ev)
    g = tg.Geometry(nb, bd)
    n = len(ev)
    out = np.zeros(n, bool)
    i = 0
    while i < n:
        k = int(kind[i])
        m = int(mask[i])
        cnt = bin(m).count("1")
        lane0 = (m & -m).bit_length() - 1
        if k in (tg.LD, tg.ATOM) and cnt >= 2 and g.lane(int(tid[i])) == lane0 and i + cnt <= n:
            grp = slice(i, i + cnt)
            lanes = [g.lane(int(t)) for t in tid[grp]]
            warps = {g.warp(int(t)) for t in tid[grp]}
            if (np.all(kind[grp] == k) and np.all(scope[grp] == scope[i]) and np.all(mask[grp] == m)
                    and len(warps) == 1 and np.all((addr[grp] >> 2) == (addr[i] >> 2))
                    and all(a < b for a, b in zip(lanes, lanes[1:]))):
                out[i + 1:i + cnt] = True
                i += cnt
                continue
        i += 1
    return out


def deleted_replay(ev, nb, bd):
    keep = ~members(ev, nb, bd)
    idx = np.nonzero(keep)[0].astype(np.uint64)
    r = oracle.run(ev[keep], nb, bd).copy()
    r["cur"] = idx[r["cur"].astype(np.int64)]
    r["prev"] = idx[r["prev"].astype(np.int64)]
    return r


@pytest.mark.parametrize("batch", range(4))
def test_deletion_equivalence(batch):
    grouped = 0
    for seed in range(batch * 50, (batch + 1) * 50):
        rng = np.random.default_rng(seed)
        ev, nb, bd = tg.warp_instr_trace(seed, int(rng.integers(5, 120)), n_blocks=int(rng.integers(1, 4)),
                                         block_dim=int(rng.choice([32, 64, 96, 48])),
                                         n_words=int(rng.integers(2, 30)))
        grouped += int(members(ev, nb, bd).sum())
        assert full_tuples(oracle.run(ev, nb, bd, coalesce=True)) == full_tuples(deleted_replay(ev, nb, bd)), \
            f"seed {seed}"
    assert grouped > 100  # groups actually occur


def test_differs_from_per_lane_mode():
    diff = sum(len(oracle.run(*tg.warp_instr_trace(s, 80))) != len(oracle.run(*tg.warp_instr_trace(s, 80), coalesce=True))
               for s in range(30))
    assert diff > 10


def test_warp_wide_flag_read_is_one_report():
    b = tg.TraceBuilder(2, 64)
    b.st(0, 9, mask=1)                   # block 0 writes the flag, no fence
    for lane in range(32):               # block 1, warp 2: all 32 lanes load it together
        b.ld(64 + lane, 9, mask=0xFFFFFFFF)
    ev = b.events()
    per_lane = oracle.run(ev, 2, 64)
    assert [int(t) for t in per_lane["type"]] == [4] * 32
    co = oracle.run(ev, 2, 64, coalesce=True)
    assert [(int(r["type"]), int(r["cur"]), int(r["prev"])) for r in co] == [(4, 1, 0)]


def test_no_groups_no_change():
    for seed in range(40):
        ev, nb, bd = tg.random_trace(seed, 150, n_words=8)   # single-event instructions
        assert full_tuples(oracle.run(ev, nb, bd, coalesce=True)) == full_tuples(deleted_replay(ev, nb, bd))


def test_stores_and_lock_ops_not_coalesced():
    b = tg.TraceBuilder(1, 32)
    for lane in range(4):
        b.st(lane, 3, mask=0xF)
    for lane in range(4):
        b.cas(lane, 600, mask=0xF)
    assert not members(b.events(), 1, 32).any()
    assert full_tuples(oracle.run(b.events(), 1, 32, coalesce=True)) == full_tuples(oracle.run(b.events(), 1, 32))


# ---------------------------------------------------------------- GPU parity
@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def _same(det, ev, nb, bd, what):
    want = oracle.run(ev, nb, bd, coalesce=True)
    det.load(ev, nb, bd)
    det.detect(coalesce=True)
    got = det.reports()
    assert len(got) == len(want), f"{what}: {len(got)} GPU vs {len(want)} oracle"
    assert np.array_equal(got, want), what
    return len(want)


@pytest.mark.gpu
@pytest.mark.parametrize("batch", range(2))
def test_gpu_small(det, batch):
    for seed in range(batch * 100, (batch + 1) * 100):
        rng = np.random.default_rng(seed)
        ev, nb, bd = tg.warp_instr_trace(seed, int(rng.integers(1, 150)), n_blocks=int(rng.integers(1, 4)),
                                         block_dim=int(rng.choice([32, 64, 96, 48])),
                                         n_words=int(rng.integers(2, 30)))
        _same(det, ev, nb, bd, f"seed {seed}")


@pytest.mark.gpu
@pytest.mark.parametrize("seed,n_instr,nb,bd", [(1, 20_000, 4, 64), (2, 60_000, 8, 256), (3, 40_000, 3, 96)])
def test_gpu_multi_tile(det, seed, n_instr, nb, bd):
    ev, nb, bd = tg.warp_instr_trace(seed, n_instr, n_blocks=nb, block_dim=bd, n_words=400)
    assert _same(det, ev, nb, bd, f"seed {seed}") > 0


@pytest.mark.gpu
def test_gpu_families(det):
    import tracegen.families as F

    for fam, n in ((1, None), (3, 400_000), (4, 600_000)):
        ev, nb, bd, _ = F.generate(fam, n)
        _same(det, ev, nb, bd, f"C{fam}")


@pytest.mark.gpu
def test_gpu_kernel_boundaries_and_coalescing(det):
    parts = [tg.warp_instr_trace(70 + k, 300, n_blocks=2, block_dim=64)[0] for k in range(3)]
    _same(det, tg.concat_kernels(parts), 2, 64, "3 kernels")
