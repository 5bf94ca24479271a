"""Streaming sessions (igd_stream_* in include/igd.h): a trace fed in
consecutive chunks, each checked on arrival with the shadow state carried between chunks.
Pin: the union of the chunks' reports equals the oracle's report set for the whole trace
(the oracle replays the whole trace at once; it has no notion of chunks), element by element,
for arbitrary cut points -- inside warp instructions, between a lock and its release, around
kernel boundaries, with empty and synchronization-only chunks."""
import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import all_golden, parse

pytestmark = pytest.mark.gpu

LOCKY = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]


@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def streamed(det, ev, nb, bd, cuts, **kw):
    det.stream_begin(nb, bd)
    parts = []
    bounds = [0] + sorted(cuts) + [len(ev)]
    for a, b in zip(bounds, bounds[1:]):
        parts.append(det.stream_feed(ev[a:b], **kw).copy())
    det.stream_end()
    allr = np.concatenate(parts) if parts else np.zeros(0, tg.REPORT_DTYPE)
    assert np.all(np.diff(allr["cur"].astype(np.int64)) > 0)  # chunks come out in order
    return allr


@pytest.mark.parametrize("path", all_golden()[:8])
def test_stream_goldens_every_cut(det, path):
    ev, nb, bd, _ = parse(path)
    want = oracle.run(ev, nb, bd)
    for cut in range(len(ev) + 1):
        assert np.array_equal(streamed(det, ev, nb, bd, [cut]), want), f"cut {cut}"


@pytest.mark.parametrize("seed", range(6))
def test_stream_random_chunks(det, seed):
    from test_gpu_parity import _fast_random

    rng = np.random.default_rng(seed)
    w = LOCKY if seed % 2 else [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(100 + seed, 120_000, [40, 3000, 5][seed % 3], 4, [64, 96, 128][seed % 3], w)
    cuts = sorted(set(rng.integers(0, len(ev), 1 + seed * 3).tolist()) | {0, len(ev) // 2})
    want = oracle.run(ev, nb, bd)
    assert len(want) > 0 and np.array_equal(streamed(det, ev, nb, bd, cuts), want)


@pytest.mark.parametrize("mode", [dict(paper_counters=True), dict(sticky_flags=True)])
def test_stream_modes(det, mode):
    from test_gpu_parity import _fast_random

    ev, nb, bd = _fast_random(120, 80_000, 200, 3, 64, LOCKY)
    want = oracle.run(ev, nb, bd, **mode)
    assert np.array_equal(streamed(det, ev, nb, bd, [10_000, 10_001, 50_000], **mode), want)


def test_stream_kernel_boundaries_and_families(det):
    import tracegen.families as F

    a, nb, bd, _ = F.generate(1)
    joined = tg.concat_kernels([a, a[:3000], a])
    want = oracle.run(joined, nb, bd)
    for cuts in ([len(a)], [len(a) + 1], [5, len(a) + 10, 2 * len(a)], list(range(0, len(joined), 997))):
        assert np.array_equal(streamed(det, joined, nb, bd, cuts), want)
    ev, nb, bd, led = F.generate(2)       # C2 at full size, 10 chunks
    got = streamed(det, ev, nb, bd, list(range(1_000_000, len(ev), 1_000_000)))
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def test_stream_bad_event_and_state(det):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd, _ = parse(all_golden()[0])
    ev = ev.copy()
    ev["tk"][3] = tg.pack_tk(0, 13, 0)
    det.stream_begin(nb, bd)
    det.stream_feed(ev[:2])
    with pytest.raises(igd.IgdError) as e:
        det.stream_feed(ev[2:])
    assert e.value.code == igd.igd.IGD_ETRACE and e.value.bad_index == 3
    with pytest.raises(igd.IgdError) as e:          # the failed chunk ended the session
        det.stream_feed(ev[:1])
    assert e.value.code == igd.igd.IGD_ESTATE
    det.stream_end()
