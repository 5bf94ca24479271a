"""Paper-fidelity modes of the oracle (readings A35-A37 in DESIGN.md).

* A35 sticky sharing flags: Table 2 writes "!md.DevShared AND !md.BlkShared" into P3 / P4 and
  "!md.DevShared" into P5; the literal reading takes them as the word's sticky flags
  (Fig. 4 has one Flags field).  SURVEY C.5 W8 fixes the outcome: exactly {X, 3, 2, R3}.
* A36 Tag aliasing: a metadata entry per word modulo the table size, identified by a 10-bit Tag
  (Fig. 4 bits 63-54): a word with another Tag claims the entry (its access
  is a first access), words equal modulo 2^10 table sizes share the entry.
* A37 last-k histories (§6.7: "tracking the last 2, 4, and 8 accessors"): the last k
  writers (loads) / accessors (stores, atomics) are checked newest first; the first racy one is
  reported.

Pins: the W8 / worked examples below, the from-scratch brute force (tests/pins.py
bf_scratch_modes) on random traces, and the mode laws (each mode equals the default where it
cannot apply; sticky and last-k only add reports, never change one)."""
import os

import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import GOLDEN_DIR, full_tuples, parse
from pins import bf_scratch_modes

LOCKY = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]


def rt(seed, n, **kw):
    return tg.random_trace(seed, n, **kw)


# ---------------- A35 sticky flags ----------------
def test_w8_sticky_reading_reports_r3():
    ev, nb, bd, exp = parse(os.path.join(GOLDEN_DIR, "W8_sharing_flag_reading.trace"))
    assert exp == []                                  # proposed reading (A4): no report
    r = oracle.run(ev, nb, bd, sticky_flags=True)
    assert [(int(x["addr"]) >> 2, int(x["cur"]), int(x["prev"]), int(x["type"])) for x in r] == \
           [(int(ev["addr"][0]) >> 2, 3, 2, 3)]       # {X, 3, 2, R3}


@pytest.mark.parametrize("batch", range(3))
def test_sticky_bruteforce(batch):
    for seed in range(40_000 + batch * 80, 40_000 + (batch + 1) * 80):
        rng = np.random.default_rng(seed)
        kw = dict(weights=LOCKY, lock_words=4, p_lock_data=0.2) if seed % 2 else {}
        ev, nb, bd = rt(seed, int(rng.integers(5, 150)), n_words=int(rng.integers(1, 8)), **kw)
        assert full_tuples(oracle.run(ev, nb, bd, sticky_flags=True)) == \
               bf_scratch_modes(ev, nb, bd, sticky=True), f"seed {seed}"


def test_sticky_only_adds_reports():
    added = 0
    for seed in range(300):
        ev, nb, bd = rt(seed, 120, n_words=5)
        base = {r[1]: r for r in full_tuples(oracle.run(ev, nb, bd))}
        st = {r[1]: r for r in full_tuples(oracle.run(ev, nb, bd, sticky_flags=True))}
        assert all(st.get(c) == r for c, r in base.items()), f"seed {seed}"
        added += len(st) - len(base)
    assert added > 20


def test_sticky_equals_default_within_one_warp():
    # one warp never sets DevShared / BlkShared: the two readings coincide
    for seed in range(100):
        ev, nb, bd = rt(seed, 150, n_blocks=1, block_dim=32, n_words=4)
        assert full_tuples(oracle.run(ev, nb, bd, sticky_flags=True)) == full_tuples(oracle.run(ev, nb, bd))


# ---------------- A36 tag aliasing ----------------
def test_tag_eviction_hides_a_race():
    # X and X + 2^8 share entry X mod 256 with different Tags: the access to the other word
    # claims the entry, so the unfenced cross-block read of X is a first access (false negative)
    b = tg.TraceBuilder(2, 64)
    b.st(0, 7)
    b.ld(64, 7)
    b.st(0, 9)
    b.st(1, 9 + 256)
    b.ld(64, 9)
    ev = b.events()
    exact = oracle.run(ev, 2, 64)
    tagged = oracle.run(ev, 2, 64, tag_log2=8)
    assert [int(r["cur"]) for r in exact] == [1, 4]
    assert [int(r["cur"]) for r in tagged] == [1]


def test_tag_alias_invents_a_race():
    # words 5 and 5 + 2^(8+10) have the same entry AND the same Tag: they share metadata, so t64's
    # load of the second word is checked against t0's store to the first (false positive)
    b = tg.TraceBuilder(2, 64)
    b.st(0, 5)
    b.ld(64, 5 + (1 << 18))
    ev = b.events()
    assert len(oracle.run(ev, 2, 64)) == 0
    r = oracle.run(ev, 2, 64, tag_log2=8)
    assert [(int(x["addr"]) >> 2, int(x["cur"]), int(x["prev"]), int(x["type"])) for x in r] == \
           [(5 + (1 << 18), 1, 0, 4)]


def _tag_trace(seed, n, log2):
    # words from a few entries, with several Tags and Tag aliases each
    ev, nb, bd = rt(seed, n, n_words=6, weights=LOCKY if seed % 2 else None, lock_words=3,
                    p_lock_data=0.2 if seed % 2 else 0.0)
    rng = np.random.default_rng(seed)
    acc = ((ev["tk"] >> 24) & 0xF) <= 2
    w = ev["addr"] >> np.uint64(2)
    bump = rng.choice([0, 1, 2, 1 << 9, 1 << 10, 1 << 10 | 1], size=len(ev)).astype(np.uint64) << np.uint64(log2)
    ev["addr"] = np.where(acc, (w + bump) << np.uint64(2), ev["addr"])
    return ev, nb, bd


@pytest.mark.parametrize("log2", [8, 12, 22])
def test_tag_bruteforce(log2):
    for seed in range(120):
        ev, nb, bd = _tag_trace(seed, 120, log2)
        assert full_tuples(oracle.run(ev, nb, bd, tag_log2=log2)) == \
               bf_scratch_modes(ev, nb, bd, tag_log2=log2), f"seed {seed}"


def test_tag_mode_equals_exact_without_collisions():
    for seed in range(100):
        ev, nb, bd = rt(seed, 150, n_words=40, weights=LOCKY, lock_words=5, p_lock_data=0.2)
        assert full_tuples(oracle.run(ev, nb, bd, tag_log2=10)) == full_tuples(oracle.run(ev, nb, bd))


# ---------------- A37 last-k ----------------
def test_last_k_finds_a_race_behind_a_synced_writer():
    # t1's store is warp-synchronous with t0's (lockstep mask) and t1 fences before t64 reads, so
    # the last writer is safe; t0 never fenced: only a 2-deep history sees the R4
    b = tg.TraceBuilder(2, 64)
    b.st(0, 3)
    b.st(1, 3, mask=0x3)
    b.fence(1)
    b.ld(64, 3)
    ev = b.events()
    assert len(oracle.run(ev, 2, 64)) == 0
    r = oracle.run(ev, 2, 64, last_k=2)
    assert [(int(x["cur"]), int(x["prev"]), int(x["type"])) for x in r] == [(3, 0, 4)]


@pytest.mark.parametrize("k", [2, 4, 8])
def test_last_k_bruteforce(k):
    for seed in range(50_000, 50_150):
        rng = np.random.default_rng(seed)
        kw = dict(weights=LOCKY, lock_words=4, p_lock_data=0.2) if seed % 2 else {}
        ev, nb, bd = rt(seed, int(rng.integers(5, 160)), n_words=int(rng.integers(1, 6)), **kw)
        assert full_tuples(oracle.run(ev, nb, bd, last_k=k)) == bf_scratch_modes(ev, nb, bd, last_k=k), \
            f"k {k} seed {seed}"


def test_last_k_is_monotone():
    grew = 0
    for seed in range(200):
        ev, nb, bd = rt(seed, 150, n_words=4)
        prev = None
        for k in (1, 2, 4, 8):
            cur = {r[1]: r for r in full_tuples(oracle.run(ev, nb, bd, last_k=k))}
            if prev is not None:
                assert all(cur.get(c) == r for c, r in prev.items()), f"seed {seed} k {k}"
                grew += len(cur) > len(prev)
            prev = cur
    assert grew > 10


def test_modes_reject_bad_parameters():
    ev = tg.TraceBuilder(1, 32).events()
    for kw in (dict(tag_log2=7), dict(tag_log2=23), dict(last_k=3)):
        with pytest.raises(oracle.OracleError):
            oracle.run(ev, 1, 32, **kw)


# ---------------- GPU parity of the modes (libigd through the C ABI) ----------------
@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def _gpu(det, ev, nb, bd, **kw):
    det.load(ev, nb, bd)
    det.detect(**kw)
    return det.reports()


@pytest.mark.gpu
def test_gpu_w8_sticky(det):
    ev, nb, bd, _ = parse(os.path.join(GOLDEN_DIR, "W8_sharing_flag_reading.trace"))
    assert np.array_equal(_gpu(det, ev, nb, bd, sticky_flags=True), oracle.run(ev, nb, bd, sticky_flags=True))


@pytest.mark.gpu
@pytest.mark.parametrize("mode", [dict(sticky_flags=True), dict(sticky_flags=True, paper_counters=True),
                                  dict(tag_log2=8), dict(tag_log2=12), dict(tag_log2=22),
                                  dict(tag_log2=10, sticky_flags=True), dict(last_k=2), dict(last_k=4),
                                  dict(last_k=8), dict(last_k=4, sticky_flags=True),
                                  dict(last_k=2, paper_counters=True), dict(last_k=4, tag_log2=12)],
                         ids=["sticky", "sticky+paper", "tag8", "tag12", "tag22", "tag10+sticky", "last2", "last4",
                              "last8", "last4+sticky", "last2+paper", "last4+tag12"])
def test_gpu_modes_vs_oracle(det, mode):
    from test_gpu_parity import _fast_random

    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    for seed, n, words, nb, bd in [(71, 30_000, 40, 3, 96), (72, 150_000, 3_000, 8, 128), (73, 80_000, 5, 2, 64),
                                   (74, 60_000, 700, 5, 48)]:
        ev, nb, bd = _fast_random(seed, n, words, nb, bd, w)
        if "tag_log2" in mode:
            # spread words over several tags / aliases of each entry
            rng = np.random.default_rng(seed)
            acc = ((ev["tk"] >> 24) & 0xF) <= 2
            bump = rng.choice([0, 1, 3, 1 << 9, 1 << 10, (1 << 10) | 1], size=len(ev)).astype(np.uint64)
            w_ = ev["addr"] >> np.uint64(2)
            ev["addr"] = np.where(acc, (w_ + (bump << np.uint64(mode["tag_log2"]))) << np.uint64(2), ev["addr"])
        want = oracle.run(ev, nb, bd, **mode)
        got = _gpu(det, ev, nb, bd, **mode)
        assert len(want) > 0 and np.array_equal(got, want), f"{mode} seed {seed}"


@pytest.mark.gpu
def test_gpu_sticky_lock_heavy_and_goldens(det):
    from golden_io import all_golden
    from test_gpu_parity import _fast_random

    for path in all_golden():
        ev, nb, bd, _ = parse(path)
        assert np.array_equal(_gpu(det, ev, nb, bd, sticky_flags=True), oracle.run(ev, nb, bd, sticky_flags=True)), path
    ev, nb, bd = _fast_random(75, 120_000, 300, 4, 64, LOCKY, lock_words=40)
    assert np.array_equal(_gpu(det, ev, nb, bd, sticky_flags=True), oracle.run(ev, nb, bd, sticky_flags=True))


@pytest.mark.gpu
def test_gpu_tag_mode_rejects_bad_sizes(det):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd, _ = parse(os.path.join(GOLDEN_DIR, "W1_mp_block_fence.trace"))
    det.load(ev, nb, bd)
    for b in (7, 23):
        with pytest.raises(igd.IgdError) as e:
            det.detect(tag_log2=b)
        assert e.value.code == igd.igd.IGD_EINVAL


@pytest.mark.gpu
def test_gpu_last_k_worked_example_and_kernels(det):
    b = tg.TraceBuilder(2, 64)
    b.st(0, 3)
    b.st(1, 3, mask=0x3)
    b.fence(1)
    b.ld(64, 3)
    ev = b.events()
    assert np.array_equal(_gpu(det, ev, 2, 64, last_k=2), oracle.run(ev, 2, 64, last_k=2))
    assert len(_gpu(det, ev, 2, 64, last_k=2)) == 1
    # kernel boundaries end the histories (A31)
    from test_gpu_parity import _fast_random

    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(76, 90_000, 60, 3, 64, w[:12])
    joined = tg.concat_kernels([ev[:40_000], ev[40_000:]])
    for k in (2, 8):
        assert np.array_equal(_gpu(det, joined, nb, bd, last_k=k), oracle.run(joined, nb, bd, last_k=k))
