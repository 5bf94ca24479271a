"""GPU parity: libigd (CUDA, through the C ABI) vs the CPU oracle, element by element on the
same seeded traces.  Bar: identical report arrays (bit-exact integers; A29: no tie-breaks)."""
import os

import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import all_golden, full_tuples, parse, report_tuples

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def gpu_run(det, ev, nb, bd):
    det.load(ev, nb, bd)
    det.detect()
    return det.reports()


def assert_same(det, ev, nb, bd, what=""):
    want = oracle.run(ev, nb, bd)
    got = gpu_run(det, ev, nb, bd)
    assert len(got) == len(want), f"{what}: {len(got)} GPU reports vs {len(want)} oracle"
    assert np.array_equal(got, want), f"{what}: first diff at {np.nonzero(got != want)[0][:5]}"
    return len(want)


@pytest.mark.parametrize("path", all_golden(), ids=[os.path.basename(p) for p in all_golden()])
def test_golden(det, path):
    ev, nb, bd, expects = parse(path)
    got = gpu_run(det, ev, nb, bd)
    assert report_tuples(got) == expects
    assert full_tuples(got) == full_tuples(oracle.run(ev, nb, bd))


def test_empty(det):
    assert len(gpu_run(det, tg.TraceBuilder(2, 64).events(), 2, 64)) == 0


@pytest.mark.parametrize("batch", range(4))
def test_random_small(det, batch):
    for seed in range(batch * 250, (batch + 1) * 250):
        rng = np.random.default_rng(seed)
        kw = {}
        if seed % 3 == 0:
            kw = dict(weights=[12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1], lock_words=3 + seed % 30, p_lock_data=0.2)
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(1, 300)), n_words=int(rng.integers(1, 20)), **kw)
        assert_same(det, ev, nb, bd, f"seed {seed}")


@pytest.mark.parametrize("seed,n,words,nb,bd", [
    (1, 20_000, 50, 3, 96),        # few words -> segments spanning many tiles
    (2, 100_000, 5_000, 8, 256),
    (3, 300_000, 1, 4, 64),        # one hot word: a single segment across ~300 tiles
    (4, 200_000, 70_000, 16, 128),
    (5, 150_000, 3, 1, 32),
    (6, 100_000, 500, 5, 48),      # block_dim not a power of two: the division geometry path
    (7, 80_000, 200, 9, 16),       # block_dim < 32: partial warps, one per block
    (8, 120_000, 2_000, 3, 1024),  # largest block: 32 warps per block on the shift path
])
def test_random_multi_tile(det, seed, n, words, nb, bd):
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, words, nb, bd, w)
    assert_same(det, ev, nb, bd, f"seed {seed}")


def _fast_random(seed, n, n_words, nb, bd, weights, lock_words=8):
    """Vectorised arbitrary-event generator (same distribution family as tg.random_trace)."""
    rng = np.random.default_rng(seed)
    T = nb * bd
    w = np.asarray(weights, float)
    kind = rng.choice(12, size=n, p=w / w.sum()).astype(np.uint32)
    tid = rng.integers(0, T, n).astype(np.uint32)
    lane = (tid % bd) % 32
    lb = (np.uint32(1) << lane).astype(np.uint32)
    mask = np.where(rng.random(n) < 0.5, lb, rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32) | lb)
    scope = rng.integers(1, 4, n).astype(np.uint32)
    word = rng.integers(0, n_words, n).astype(np.uint64)
    lockw = (500_000 + rng.integers(0, lock_words, n)).astype(np.uint64)
    is_lock = (kind == tg.CAS) | (kind == tg.EXCH)
    word = np.where(is_lock, lockw, word)
    plain = (kind == tg.LD) | (kind == tg.ST)
    sync_noscope = (kind >= tg.SYNCWARP)
    scope = np.where(plain | sync_noscope, 0, scope).astype(np.uint32)
    addr = np.where(kind <= tg.EXCH, word << np.uint64(2), 0).astype(np.uint64)
    grid = (kind == tg.GRID_SYNC) | (kind == tg.CG_GRID_SYNC)
    tid = np.where(grid, 0, tid).astype(np.uint32)
    mask = np.where(kind >= tg.SYNCTHREADS, 0xFFFFFFFF, mask).astype(np.uint32)
    ev = np.zeros(n, tg.EVENT_DTYPE)
    ev["addr"] = addr
    ev["tk"] = tg.pack_tk(tid, kind, scope)
    ev["mask"] = mask
    return ev, nb, bd


def test_lock_heavy_multi_tile(det):
    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(11, 120_000, 300, 4, 64, w, lock_words=40)
    assert assert_same(det, ev, nb, bd, "lock heavy") > 0


def test_sparse_high_addresses(det):
    # 45-bit virtual addresses, span < 2^32 words: the 32-bit key path is exact
    ev, nb, bd = _fast_random(12, 50_000, 2_000, 2, 64, [20, 18, 10, 0, 0, 8, 3, 3, 1, 1, 1, 1])
    acc = (ev["tk"] >> 24) & 0xF <= 4
    ev["addr"][acc] += np.uint64(0x7F3A_0000_0000)
    assert_same(det, ev, nb, bd, "high VA")


def test_word_span_wide_keys(det):
    # a4: accessed words spanning >= 2^32 words (sparse virtual addresses) take the u64-key path
    b = tg.TraceBuilder(2, 64)
    b.st(0, 1)
    b.st(0, 1 + (1 << 32))      # same low 32 bits, another word: must not collide
    b.ld(64, 1)                 # R4 on word 1 only
    b.ld(65, 1 + (1 << 32))     # R4 on the far word
    b.fence(0)
    b.ld(66, 7 << 40)
    b.st(67, 7 << 40)
    ev = b.events()
    want = oracle.run(ev, 2, 64)
    assert len(want) == 3
    assert np.array_equal(gpu_run(det, ev, 2, 64), want)


@pytest.mark.parametrize("seed,n,nb,bd,bits", [(41, 60_000, 4, 64, 45), (42, 300_000, 16, 128, 40),
                                               (43, 120_000, 3, 96, 62), (44, 50_000, 2, 64, 33)])
def test_wide_keys_vs_oracle(det, seed, n, nb, bd, bits):
    # random traces whose words are spread over 2^bits words (up to ceil(bits/8) radix passes);
    # lock words and data words both wide, few distinct words so histories are long
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, 3_000, nb, bd, w, lock_words=12)
    rng = np.random.default_rng(seed)
    acc = ((ev["tk"] >> 24) & 0xF) <= 4
    word = ev["addr"] >> np.uint64(2)
    uniq, inv = np.unique(word[acc], return_inverse=True)
    spread = rng.integers(0, 1 << bits, len(uniq), dtype=np.uint64)
    spread[0] = 0
    spread[-1] = (1 << bits) - 1
    ev["addr"][acc] = (spread[inv] << np.uint64(2)) | (ev["addr"][acc] & np.uint64(3))
    assert_same(det, ev, nb, bd, f"wide seed {seed}")


@pytest.mark.parametrize("seed,n,nb,bd,bits,words", [(51, 300_000, 16, 128, 30, 3_000), (52, 100_003, 4, 64, 25, 500),
                                                     (53, 250_000, 8, 96, 27, 60_000), (54, 70_001, 2, 64, 29, 20)])
def test_30bit_word_span_vs_oracle(det, seed, n, nb, bd, bits, words):
    # words spread over 2^25..2^30 words (C5's span): the u32-key path with every radix digit
    # non-trivial, many tiles, ragged tails
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, words, nb, bd, w, lock_words=12)
    rng = np.random.default_rng(seed)
    acc = ((ev["tk"] >> 24) & 0xF) <= 4
    word = ev["addr"] >> np.uint64(2)
    uniq, inv = np.unique(word[acc], return_inverse=True)
    spread = rng.integers(0, 1 << bits, len(uniq), dtype=np.uint64)
    spread[0] = 0x3FF  # digits 1..3 all occupied by more than one bin
    spread[-1] = (1 << bits) - 1
    ev["addr"][acc] = (spread[inv] << np.uint64(2)) | (ev["addr"][acc] & np.uint64(3))
    assert_same(det, ev, nb, bd, f"30-bit span seed {seed}")


@pytest.mark.parametrize("bad_at", [0, 5000, 99_999])
def test_invalid_event_index_matches_oracle(det, bad_at):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd = _fast_random(13, 100_000, 100, 2, 64, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    ev["tk"][bad_at] = tg.pack_tk(0, 13, 0)
    ev["tk"][min(bad_at + 7, len(ev) - 1)] = tg.pack_tk(0, 14, 0)
    with pytest.raises(oracle.OracleError) as eo:
        oracle.run(ev, nb, bd)
    det.load(ev, nb, bd)
    with pytest.raises(igd.IgdError) as eg:
        det.detect()
    assert eg.value.code == igd.igd.IGD_ETRACE and eg.value.bad_index == eo.value.bad_index == bad_at


def test_device_pointer_borrowed(det):
    import torch

    ev, nb, bd = _fast_random(14, 30_000, 500, 2, 96, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    t = torch.from_numpy(ev.view(np.uint8).copy()).cuda()
    det.load(t, nb, bd)
    det.detect()
    assert np.array_equal(det.reports(), oracle.run(ev, nb, bd))


def test_repeat_detect_is_deterministic(det):
    ev, nb, bd = _fast_random(15, 60_000, 50, 4, 64, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    det.load(ev, nb, bd)
    det.detect()
    a = det.reports()
    det.detect()
    assert np.array_equal(a, det.reports())


@pytest.mark.parametrize("seed", [21, 22])
def test_long_irregular_sync_lists(det, seed):
    # few entities with long, bursty synchronization lists: exercises the interpolation probes
    # and their binary-search fallback in every direction
    rng = np.random.default_rng(seed)
    n = 400_000
    w = np.array([20, 18, 10, 2, 2, 14, 12, 8, 1, 2, 2, 1], float)
    ev, nb, bd = _fast_random(seed, n, 40, 2, 64, w)
    # make the sync events bursty: shuffle blocks of the trace so syncs cluster
    kind = (ev["tk"] >> 24) & 0xF
    sync = kind >= 5
    burst = (np.arange(n) // 5000) % 3 == 0
    drop = sync & ~burst & (rng.random(n) < 0.9)
    ev = ev[~drop]
    assert_same(det, ev, nb, bd, f"bursty {seed}")


def test_c2_full_size_vs_oracle(det):
    # BASELINE configs[1] at its full size (10^7 events), element by element against the oracle
    import tracegen.families as F

    ev, nb, bd, led = F.generate(2)
    want = oracle.run(ev, nb, bd)
    det.load(ev, nb, bd)
    det.detect()
    got = det.reports()
    assert np.array_equal(got, want)
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def _shard_of(words, K):
    h = (words ^ (words >> np.uint64(32))).astype(np.uint64) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(16)
    h = (h * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(13)
    h = (h * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
    return (h ^ (h >> np.uint64(16))) % np.uint64(K)


def test_c4_full_size_sampled_words_vs_oracle(det):
    # configs[3] at its full size (5*10^8 events): the oracle replays every event but checks a 1/64
    # address shard; the GPU reports restricted to those words must be identical, and the whole GPU
    # report set must equal the generator's injection ledger
    import tracegen.families as F

    ev, nb, bd, led = F.generate(4)
    det.load(ev, nb, bd)
    det.detect()
    got = det.reports()
    want = oracle.run(ev, nb, bd, shard=(5, 64))
    mine = _shard_of(got["addr"] >> np.uint64(2), 64) == 5
    assert len(want) > 0 and np.array_equal(got[mine], want)
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def test_c5_prefix_sampled_words_vs_oracle(det):
    # configs[4]'s workload (the 4*10^9-event mix over 2^30 words): its first 4*10^8 events are a
    # valid trace (the check of access i depends only on events <= i); oracle on a 1/64 shard
    import tracegen.families as F

    plan = F.Plan(5)
    ev = plan.fill(0, 400_000_000)
    nb, bd = plan.n_blocks, plan.block_dim
    plan.close()
    det.load(ev, nb, bd)
    det.detect()
    got = det.reports()
    want = oracle.run(ev, nb, bd, shard=(9, 64))
    mine = _shard_of(got["addr"] >> np.uint64(2), 64) == 9
    assert len(want) > 0 and np.array_equal(got[mine], want)


def test_c3_full_size_sampled_words_vs_oracle(det):
    # configs[2] at full size (10^8 events): the oracle checks a 1/16 address shard (replaying every
    # synchronization event), the GPU result restricted to the same words must match exactly
    import tracegen.families as F

    ev, nb, bd, led = F.generate(3)
    det.load(ev, nb, bd)
    det.detect()
    got = det.reports()
    K = 16
    want = oracle.run(ev, nb, bd, shard=(5, K))

    def fmix(h):
        h = h & 0xFFFFFFFF
        h ^= h >> 16
        h = (h * 0x85EBCA6B) & 0xFFFFFFFF
        h ^= h >> 13
        h = (h * 0xC2B2AE35) & 0xFFFFFFFF
        return h ^ (h >> 16)

    words = got["addr"] >> np.uint64(2)
    mine = np.array([fmix(int(w) ^ (int(w) >> 32)) % K == 5 for w in words], bool)
    assert np.array_equal(got[mine], want)
    # the whole report array against the injection ledger, element by element
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


@pytest.mark.parametrize("env", [{"IGD_FUSED": "0"}], ids=["unfused_ingest"])
def test_pipeline_variants_vs_oracle(monkeypatch, env):
    """The alternate pipeline shape (unfused ingest write pass + radix pass 0, the one the sharded
    path uses) is selected per context from the environment: same report set."""
    import paper_conf_sosp_kamathb21_b200 as igd

    for k, v in env.items():
        monkeypatch.setenv(k, v)
    d = igd.Detector(0)
    try:
        w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
        for seed, n, words, nb, bd in [(21, 60_000, 40, 3, 96), (22, 200_000, 30_000, 16, 128)]:
            ev, nb, bd = _fast_random(seed, n, words, nb, bd, w)
            assert_same(d, ev, nb, bd, f"{env} seed {seed}")
    finally:
        d.close()
