"""Workload families C1..C5 vs the oracle: the injection ledgers (generator
intent, closed form per planted bug) and the zero-report invariant on race-free variants
("57 races ... without any false positives"; race-free apps give 0 reports, Tab. 5)."""
import hashlib

import numpy as np
import pytest

import oracle
import tracegen.families as F


def key4(a):
    return [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"])) for r in a]


def test_c1_litmus_exact():
    ev, nb, bd, led = F.generate(1)
    assert (nb, bd) == (2, 64) and 9_000 <= len(ev) <= 11_000
    rep = oracle.run(ev, nb, bd)
    # BASELINE configs[0]: block-scope-fence message passing (R4) + missing syncwarp (R2)
    assert sorted(r["type"] for r in rep) == [2, 4]
    assert key4(rep) == key4(led)


def test_c1_fixed_is_race_free():
    ev, nb, bd, led = F.generate(1, fixed=True)
    assert len(led) == 0 and len(oracle.run(ev, nb, bd)) == 0


@pytest.mark.parametrize("fam,n,rate", [(2, 3_000_000, 3.0), (3, 1_000_000, 100.0), (4, 3_000_000, 8.0),
                                        (5, 20_000_000, 50.0)])
def test_ledger_equals_oracle(fam, n, rate):
    ev, nb, bd, led = F.generate(fam, n, rate=rate)
    assert len(ev) == n
    rep = oracle.run(ev, nb, bd)
    assert len(led) > 0
    assert key4(rep) == key4(led)


@pytest.mark.parametrize("fam,n", [(2, 2_000_000), (3, 2_000_000), (4, 3_000_000), (5, 14_000_000)])
def test_race_free_variants_report_nothing(fam, n):
    ev, nb, bd, led = F.generate(fam, n, fixed=True)
    assert len(led) == 0
    assert len(oracle.run(ev, nb, bd)) == 0


def test_ledger_types_cover_rules():
    seen = set()
    for fam, n, rate in [(2, 3_000_000, 3.0), (3, 1_000_000, 100.0), (4, 6_000_000, 16.0)]:
        seen |= set(int(t) for t in F.generate(fam, n, rate=rate)[3]["type"])
    assert seen == {1, 2, 3, 4, 5}


def test_deterministic_and_seeded():
    a = F.generate(4, 1_000_000)[0]
    b = F.generate(4, 1_000_000)[0]
    c = F.generate(4, 1_000_000, seed=99)[0]
    assert hashlib.sha1(a.tobytes()).digest() == hashlib.sha1(b.tobytes()).digest()
    assert np.array_equal(a, b)
    d = F.generate(3, 500_000)[0]
    e = F.generate(3, 500_000, seed=7)[0]
    assert not np.array_equal(d["tk"], e["tk"]) or not np.array_equal(d["addr"], e["addr"]) or len(c)


@pytest.mark.parametrize("fam,n", [(2, 1_500_000), (4, 2_000_000), (5, 9_000_000)])
def test_range_fill_matches_full(fam, n):
    # per-rank chunks regenerate exactly their range (SURVEY 8(e) partitioning)
    p = F.Plan(fam, n)
    full = p.fill()
    for first, count in [(0, 1000), (123_457, 400_000), (n - 77_777, 77_777)]:
        assert np.array_equal(p.fill(first, count), full[first:first + count])
    P = 4
    parts = [p.fill(r * n // P, (r + 1) * n // P - r * n // P) for r in range(P)]
    assert np.array_equal(np.concatenate(parts), full)
    p.close()


def test_c5_exercises_every_radix_digit():
    ev = F.generate(5, 8_000_000)[0]
    kind = (ev["tk"] >> 24) & 0xF
    w = ev["addr"][kind <= 4] >> np.uint64(2)
    assert w.max() >= (1 << 29)
    for d in range(4):
        digits = np.unique(((w >> np.uint64(8 * d)) & np.uint64(255)))
        assert len(digits) >= (48 if d == 3 else 256)


# ---- the sync-heavy variant (f_acc ~0.9-0.95, fences ~5 %, spin-lock sections ~8 %) ----
@pytest.mark.parametrize("fam,n,rate", [(2, 3_000_000, 3.0), (5, 14_000_000, 30.0)])
def test_sync_heavy_ledger_equals_oracle(fam, n, rate):
    ev, nb, bd, led = F.generate(fam, n, rate=rate, **F.SYNC_HEAVY)
    kinds = np.bincount(((ev["tk"] >> 24) & 0xF).astype(np.int64), minlength=13)
    if fam == 2:
        assert kinds[5] / n > 0.04 and kinds[:5].sum() / n < 0.96  # fences, f_acc
        assert (kinds[3] + kinds[4]) / n > 0.02                      # lock CAS / EXCH
    rep = oracle.run(ev, nb, bd)
    assert len(led) > 0 and key4(rep) == key4(led)


def test_sync_heavy_race_free():
    ev, nb, bd, led = F.generate(2, 2_000_000, fixed=True, **F.SYNC_HEAVY)
    assert len(led) == 0 and len(oracle.run(ev, nb, bd)) == 0
