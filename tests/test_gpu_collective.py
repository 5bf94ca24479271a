"""GPU parity of the collective C-ABI path: a context created with an NCCL id
runs the multi-GPU pipeline inside libigd -- partition by owner, NCCL all-to-all of the access
records, all-gather of the synchronization streams, the sharded check, all-gather + merge of the
reports.  One GPU per box here, so the communicator has one rank (NCCL refuses two ranks on one
device); the multi-rank partition / exchange / merge semantics are covered by the loopback tests
(test_gpu_multirank.py, P = 1..8 logical ranks) and the gloo tests on CPU."""
import os

import numpy as np
import pytest

import oracle
import tracegen as tg
from golden_io import all_golden, full_tuples, parse
from test_gpu_parity import _fast_random

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cdet():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0, nranks=1, rank=0, nccl_id=igd.igd_nccl_unique_id())
    yield d
    d.close()


def run(d, ev, nb, bd):
    d.load(ev, nb, bd, first_event=0, n_events_total=len(ev))
    d.detect()
    return d.reports()


@pytest.mark.parametrize("path", all_golden(), ids=[os.path.basename(p) for p in all_golden()])
def test_collective_golden(cdet, path):
    ev, nb, bd, exp = parse(path)
    assert full_tuples(run(cdet, ev, nb, bd)) == full_tuples(oracle.run(ev, nb, bd))


@pytest.mark.parametrize("seed,n,words,nb,bd", [(31, 40_000, 60, 3, 96), (32, 250_000, 20_000, 16, 128),
                                                 (33, 120_000, 5, 2, 64), (34, 90_000, 800, 7, 48)])
def test_collective_random_vs_oracle(cdet, seed, n, words, nb, bd):
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(seed, n, words, nb, bd, w)
    got = run(cdet, ev, nb, bd)
    want = oracle.run(ev, nb, bd)
    assert len(want) > 0 and np.array_equal(got, want)


def test_collective_lock_heavy(cdet):
    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(35, 150_000, 300, 4, 64, w, lock_words=40)
    assert np.array_equal(run(cdet, ev, nb, bd), oracle.run(ev, nb, bd))


def test_collective_bad_event_index(cdet):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd = _fast_random(36, 50_000, 100, 2, 64, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    ev["tk"][12_345] = tg.pack_tk(0, 13, 0)
    cdet.load(ev, nb, bd, first_event=0, n_events_total=len(ev))
    with pytest.raises(igd.IgdError) as e:
        cdet.detect()
    assert e.value.code == igd.igd.IGD_ETRACE and e.value.bad_index == 12_345


def test_collective_c2_full_size(cdet):
    import tracegen.families as F

    ev, nb, bd, led = F.generate(2)
    got = run(cdet, ev, nb, bd)
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def test_collective_rejects_coalesce(cdet):
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd, _ = parse(all_golden()[0])
    cdet.load(ev, nb, bd, first_event=0, n_events_total=len(ev))
    with pytest.raises(igd.IgdError) as e:
        cdet.detect(coalesce=True)
    assert e.value.code == igd.igd.IGD_EINVAL


# ---- P > 1 ranks through the collective C ABI on one GPU: the in-process loopback transport ----
# ("IGDLOOP:<name>" ids; P contexts driven by P host threads exchange through device copies with
# the same count matrix, all-to-all and all-gathers as the NCCL transport)
def _loop_id(name):
    return (b"IGDLOOP:" + name.encode()).ljust(128, b"\0")


def run_ranks(ev, nb, bd, P, name, **kw):
    import threading

    import torch

    import paper_conf_sosp_kamathb21_b200 as igd

    n = len(ev)
    out, errs = [None] * P, [None] * P

    def rank(r):
        try:
            torch.cuda.set_device(0)
            d = igd.Detector(0, stream=torch.cuda.Stream(0), nranks=P, rank=r, nccl_id=_loop_id(name))
            lo, hi = n * r // P, n * (r + 1) // P
            d.load(ev[lo:hi], nb, bd, first_event=lo, n_events_total=n)
            d.detect(**kw)
            out[r] = d.reports()
            d.close()
        except Exception as e:  # noqa: BLE001 -- reported by the caller
            errs[r] = e

    ts = [threading.Thread(target=rank, args=(r,)) for r in range(P)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    return out, errs


@pytest.mark.parametrize("P", [2, 3, 4, 8])
def test_collective_loopback_ranks_vs_oracle(P):
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(40 + P, 150_000, 2_000, 6, 128, w)
    want = oracle.run(ev, nb, bd)
    out, errs = run_ranks(ev, nb, bd, P, f"ranks{P}")
    assert errs == [None] * P
    assert len(want) > 0
    for r in range(P):
        assert np.array_equal(out[r], want), f"rank {r}"


def test_collective_loopback_lock_heavy_and_families():
    import tracegen.families as F

    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(50, 100_000, 300, 4, 64, w, lock_words=40)
    out, errs = run_ranks(ev, nb, bd, 4, "locks4")
    assert errs == [None] * 4 and all(np.array_equal(o, oracle.run(ev, nb, bd)) for o in out)
    ev, nb, bd, led = F.generate(2)
    out, errs = run_ranks(ev, nb, bd, 3, "c2x3")
    assert errs == [None] * 3
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in out[2]] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def test_collective_loopback_paper_counters_and_sticky():
    w = [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1]
    ev, nb, bd = _fast_random(51, 80_000, 500, 3, 96, w)
    for kw, nm in ((dict(paper_counters=True), "pc"), (dict(sticky_flags=True), "st")):
        out, errs = run_ranks(ev, nb, bd, 2, nm, **kw)
        assert errs == [None, None] and all(np.array_equal(o, oracle.run(ev, nb, bd, **kw)) for o in out)


def test_collective_loopback_bad_event_agreed():
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd = _fast_random(52, 60_000, 100, 2, 64, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    ev["tk"][45_001] = tg.pack_tk(0, 13, 0)   # on rank 2 of 3
    out, errs = run_ranks(ev, nb, bd, 3, "bad3")
    assert all(isinstance(e, igd.IgdError) and e.code == igd.igd.IGD_ETRACE and e.bad_index == 45_001 for e in errs)
