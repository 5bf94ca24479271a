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
