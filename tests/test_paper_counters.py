"""Paper-width synchronization IDs (first part; reading A33 in DESIGN.md):
the IDs iGUARD copies into a word's metadata are WarpBarID 6, BlkBarID 8, DevFenceID 6 and
BlkFenceID 6 bits wide (Fig. 4), so "unchanged since md" holds whenever a multiple of
2^width events of that ID's class happened in between -- the false-positive side of the paper's
bounded counters (§6.7).  Off by default (exact counters, A16).

Pins of the oracle (CPU): the from-scratch evaluator counting events modulo the widths
(tests/pins.py), identity with exact mode when no ID moves 2^width times, and worked examples
at exactly 64 / 256 events.  GPU parity (`-m gpu`): IGD_DETECT_PAPER_COUNTERS == oracle.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import full_tuples
from pins import bf_scratch

SYNCY = [14, 12, 6, 3, 2, 30, 20, 12, 3, 2, 2, 1]  # many fences and barriers


def _burst_trace(seed, n, nb=2, bd=64, threads=None):
    """Random trace with bursts of fences / barriers so IDs wrap between accesses.  ``threads``:
    draw every event's thread from this small set (so md's thread is often the fencing one)."""
    rng = np.random.default_rng(seed)
    b = tg.TraceBuilder(nb, bd)
    T = nb * bd
    for _ in range(n):
        r = rng.random()
        t = int(rng.choice(threads)) if threads else int(rng.integers(0, T))
        lane = t % bd % 32
        if r < 0.5:
            k = int(rng.choice([tg.LD, tg.ST, tg.ATOM]))
            b.ev(k, t, int(rng.integers(0, 4)), 0 if k != tg.ATOM else int(rng.integers(1, 3)),
                 1 << lane)
        else:
            reps = int(rng.choice([1, 63, 64, 65, 128, 256]))
            what = int(rng.integers(0, 4))
            for _ in range(reps):
                if what == 0:
                    b.fence(t, tg.DEVICE, mask=1 << lane)
                elif what == 1:
                    b.fence(t, tg.BLOCK, mask=1 << lane)
                elif what == 2:
                    b.syncwarp(t)
                else:
                    b.syncthreads(t // bd)
    return b.events(), nb, bd


@pytest.mark.parametrize("batch", range(4))
def test_bruteforce_random(batch):
    for seed in range(batch * 60, (batch + 1) * 60):
        rng = np.random.default_rng(seed)
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(5, 150)), n_words=int(rng.integers(1, 8)), weights=SYNCY)
        assert full_tuples(oracle.run(ev, nb, bd, paper_counters=True)) == bf_scratch(ev, nb, bd, paper_counters=True), seed


def test_bruteforce_bursts():
    differs = 0
    for seed in range(100):
        ev, nb, bd = _burst_trace(seed, 40)
        got = full_tuples(oracle.run(ev, nb, bd, paper_counters=True))
        assert got == bf_scratch(ev, nb, bd, paper_counters=True), seed
        differs += got != full_tuples(oracle.run(ev, nb, bd))
    assert differs > 8  # wrapping actually changes outcomes


def test_bruteforce_bursts_few_threads():
    for seed in range(100):
        ev, nb, bd = _burst_trace(seed, 30, threads=[0, 1, 33, 64])
        assert full_tuples(oracle.run(ev, nb, bd, paper_counters=True)) == bf_scratch(ev, nb, bd, paper_counters=True), seed


@pytest.mark.parametrize("reps,racy", [(1, False), (63, False), (64, True)])
def test_block_fence_wraps_at_64(reps, racy):
    # same block, other warp: md's thread fences at block scope `reps` times (R3 suppressed by
    # any fence of md's thread, A1/A30); a 6-bit BlkFenceID wraps at 64
    b = tg.TraceBuilder(1, 64)
    b.st(0, 3, mask=1)
    for _ in range(reps):
        b.fence(0, tg.BLOCK, mask=1)
    b.ld(32, 3, mask=1)
    assert len(oracle.run(b.events(), 1, 64)) == 0
    r = oracle.run(b.events(), 1, 64, paper_counters=True)
    assert [int(x) for x in r["type"]] == ([3] if racy else [])


def test_identity_below_widths():
    for seed in range(100):
        ev, nb, bd = tg.random_trace(seed, 120, n_words=6)   # far fewer than 64 syncs per entity
        assert full_tuples(oracle.run(ev, nb, bd, paper_counters=True)) == full_tuples(oracle.run(ev, nb, bd))


@pytest.mark.parametrize("reps,racy", [(63, False), (64, True), (65, False), (128, True)])
def test_device_fence_wraps_at_64(reps, racy):
    # Fig. 1-style message passing across blocks: producer stores, fences `reps` times at device
    # scope, consumer loads.  Exact counters: no race.  6-bit DevFenceID: 64k fences look like none.
    b = tg.TraceBuilder(2, 64)
    b.st(0, 3, mask=1)
    for _ in range(reps):
        b.fence(0, tg.DEVICE, mask=1)
    b.ld(64, 3, mask=1)
    ev = b.events()
    assert len(oracle.run(ev, 2, 64)) == 0
    r = oracle.run(ev, 2, 64, paper_counters=True)
    assert [int(x) for x in r["type"]] == ([4] if racy else [])


@pytest.mark.parametrize("reps,racy", [(255, False), (256, True)])
def test_block_barrier_wraps_at_256(reps, racy):
    b = tg.TraceBuilder(1, 64)
    b.st(0, 3, mask=1)
    for _ in range(reps):
        b.syncthreads(0)
    b.ld(32, 3, mask=1)   # same block, other warp
    r = oracle.run(b.events(), 1, 64, paper_counters=True)
    assert [int(x) for x in r["type"]] == ([3] if racy else [])


# ---------------------------------------------------------------- GPU parity
@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def _same(det, ev, nb, bd, what):
    want = oracle.run(ev, nb, bd, paper_counters=True)
    det.load(ev, nb, bd)
    det.detect(paper_counters=True)
    got = det.reports()
    assert len(got) == len(want), f"{what}: {len(got)} GPU vs {len(want)} oracle"
    assert np.array_equal(got, want), what
    return len(want)


@pytest.mark.gpu
def test_gpu_bursts(det):
    for seed in range(80):
        ev, nb, bd = _burst_trace(seed, 40)
        _same(det, ev, nb, bd, f"seed {seed}")


@pytest.mark.gpu
def test_gpu_random(det):
    for seed in range(150):
        rng = np.random.default_rng(seed)
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(1, 300)), n_words=int(rng.integers(1, 10)), weights=SYNCY)
        _same(det, ev, nb, bd, f"seed {seed}")


@pytest.mark.gpu
def test_gpu_families(det):
    import tracegen.families as F

    for fam, n in ((2, 2_000_000), (3, 2_000_000), (4, 3_000_000)):
        ev, nb, bd, _ = F.generate(fam, n)
        _same(det, ev, nb, bd, f"C{fam}")


@pytest.mark.gpu
@pytest.mark.parametrize("P", [2, 4])
def test_gpu_sharded(P):
    from test_gpu_multirank import sharded_stages_run

    for seed in range(30):
        ev, nb, bd = _burst_trace(seed, 40, threads=[0, 1, 33, 64] if seed % 2 else None)
        got = sharded_stages_run(ev, nb, bd, P, paper_counters=True)
        assert np.array_equal(got, oracle.run(ev, nb, bd, paper_counters=True)), f"seed {seed} P {P}"
