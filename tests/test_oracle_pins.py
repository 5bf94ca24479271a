"""Oracle vs independent evaluators: from-scratch brute force,
pairwise scoped happens-before, sync-free closed form, metamorphic invariants."""
import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import full_tuples, report_tuples
from pins import bf_scratch, closed_form_syncfree, pairwise

N_BF_SEEDS = 400


@pytest.mark.parametrize("batch", range(8))
def test_bruteforce_fuzz(batch):
    for seed in range(batch * N_BF_SEEDS // 8, (batch + 1) * N_BF_SEEDS // 8):
        rng = np.random.default_rng(seed)
        n = int(rng.integers(5, 160))
        ev, nb, bd = tg.random_trace(seed, n, n_words=int(rng.integers(1, 12)))
        got = full_tuples(oracle.run(ev, nb, bd))
        want = bf_scratch(ev, nb, bd)
        assert got == want, f"seed {seed}"


def test_bruteforce_lock_heavy():
    # CAS/EXCH/FENCE heavy mixes stress the lock replay and R5
    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    for seed in range(10_000, 10_150):
        ev, nb, bd = tg.random_trace(seed, 120, n_words=6, weights=w, lock_words=3 + seed % 30, p_lock_data=0.2)
        assert full_tuples(oracle.run(ev, nb, bd)) == bf_scratch(ev, nb, bd), f"seed {seed}"


def test_bruteforce_single_block_warp():
    # one warp: R2 / P4 dominate
    for seed in range(20_000, 20_150):
        ev, nb, bd = tg.random_trace(seed, 100, n_blocks=1, block_dim=32, n_words=4)
        assert full_tuples(oracle.run(ev, nb, bd)) == bf_scratch(ev, nb, bd), f"seed {seed}"


def test_pairwise_fuzz():
    hits = 0
    for seed in range(30_000, 30_400):
        ev, nb, bd = tg.random_trace(seed, 150, max_uses_per_word=2)
        want, eligible = pairwise(ev, nb, bd)
        got = [r for r in report_tuples(oracle.run(ev, nb, bd)) if (r[0] >> 2) in eligible]
        assert got == want, f"seed {seed}"
        hits += len(want)
    assert hits > 100  # the fuzz actually exercises races


def test_pairwise_covers_every_rule():
    seen = set()
    for seed in range(30_000, 30_400):
        ev, nb, bd = tg.random_trace(seed, 150, max_uses_per_word=2)
        seen |= {r[3] for r in pairwise(ev, nb, bd)[0]}
    assert seen == {1, 2, 3, 4, 5}


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_closed_form_syncfree(seed):
    rng = np.random.default_rng(seed)
    nb, bd = 8, 96
    n = 200_000
    threads = nb * bd
    kind = rng.choice([tg.LD, tg.ST, tg.ATOM], size=n, p=[0.5, 0.3, 0.2]).astype(np.uint32)
    tid = rng.integers(0, threads, n).astype(np.uint32)
    scope = np.where(kind == tg.ATOM, rng.integers(1, 4, n), 0).astype(np.uint32)
    word = rng.integers(0, 5000, n).astype(np.uint64)
    lane = (tid % bd) % 32
    mask = (rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32) | (1 << lane).astype(np.uint32))
    mask = np.where(rng.random(n) < 0.5, (1 << lane).astype(np.uint32), mask).astype(np.uint32)
    ev = np.zeros(n, tg.EVENT_DTYPE)
    ev["addr"] = word << np.uint64(2) | rng.integers(0, 4, n).astype(np.uint64)
    ev["tk"] = tg.pack_tk(tid, kind, scope)
    ev["mask"] = mask
    rep = oracle.run(ev, nb, bd)
    a, cur, prev, ty = closed_form_syncfree(ev, nb, bd)
    assert len(rep) == len(cur) and len(cur) > 1000
    assert np.array_equal(rep["addr"], a)
    assert np.array_equal(rep["cur"].astype(np.int64), cur)
    assert np.array_equal(rep["prev"].astype(np.int64), prev)
    assert np.array_equal(rep["type"].astype(np.int64), ty)


def test_metamorphic_word_renaming():
    # C.7 5(a): a bijection on data words permutes report addresses only
    for seed in range(40_000, 40_040):
        ev, nb, bd = tg.random_trace(seed, 200, n_words=10)
        rep = oracle.run(ev, nb, bd)
        ev2 = ev.copy()
        _, tid, kind, _, _ = tg.unpack(ev)
        data = np.isin(kind, [tg.LD, tg.ST, tg.ATOM])
        ev2["addr"][data] = (((ev["addr"][data] >> np.uint64(2)) * np.uint64(7919) + np.uint64(123456789))
                             << np.uint64(2))
        rep2 = oracle.run(ev2, nb, bd)
        assert [(r["cur"], r["prev"], r["type"]) for r in rep] == [(r["cur"], r["prev"], r["type"]) for r in rep2]


@pytest.mark.parametrize("K", [2, 3, 8])
def test_metamorphic_address_shards(K):
    # C.7 5(b): union over shards == full result
    for seed in range(50_000, 50_030):
        ev, nb, bd = tg.random_trace(seed, 300, n_words=40, lock_words=3)
        full = report_tuples(oracle.run(ev, nb, bd))
        parts = []
        for k in range(K):
            parts += report_tuples(oracle.run(ev, nb, bd, shard=(k, K)))
        assert sorted(parts, key=lambda r: r[1]) == full


def test_metamorphic_prefix_closure():
    # C.7 5(c)
    for seed in range(60_000, 60_030):
        ev, nb, bd = tg.random_trace(seed, 200, n_words=8)
        full = report_tuples(oracle.run(ev, nb, bd))
        for cut in (0, 17, 100, 199):
            assert report_tuples(oracle.run(ev[:cut], nb, bd)) == [r for r in full if r[1] < cut]


def test_metamorphic_delete_word():
    # C.7 5(d): deleting every event on a non-lock word deletes exactly its reports;
    # event indices shift, so compare (addr, type) multisets keyed by surviving indices
    for seed in range(70_000, 70_030):
        ev, nb, bd = tg.random_trace(seed, 200, n_words=8)
        full = report_tuples(oracle.run(ev, nb, bd))
        addr, _, kind, _, _ = tg.unpack(ev)
        acc = np.isin(kind, [tg.LD, tg.ST, tg.ATOM])
        victim = 3 << 2
        keep = ~(acc & ((addr >> np.uint64(2)) << np.uint64(2) == victim))
        newidx = np.cumsum(keep) - 1
        rep = report_tuples(oracle.run(ev[keep], nb, bd))
        want = [(a, int(newidx[c]), int(newidx[p]), t) for a, c, p, t in full if a != victim]
        assert rep == want
