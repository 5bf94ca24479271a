"""Sharded (multi-GPU) path on one GPU: P logical ranks, each with its own libigd context, the
exchange done in-process (LoopbackComm).  The merged reports must equal the single-GPU result and
the oracle for every P (address-shard invariance)."""
import numpy as np
import pytest

import oracle
import tracegen as tg
import tracegen.families as F
from test_gpu_parity import _fast_random

pytestmark = pytest.mark.gpu


def sharded_stages_run(ev, nb, bd, P, **kw):
    import paper_conf_sosp_kamathb21_b200 as igd
    from paper_conf_sosp_kamathb21_b200 import dist as D

    stages = []
    for r in range(P):
        lo, cnt = D.chunk_bounds(len(ev), P, r)
        s = D.GpuStage(igd.Detector(0))
        s.load(ev[lo:lo + cnt], lo, len(ev), nb, bd)
        stages.append(s)
    try:
        return D.LoopbackComm.run(stages, **kw)
    finally:
        for s in stages:
            s.det.close()


def sharded(ev, nb, bd, P):
    return sharded_stages_run(ev, nb, bd, P)


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_random_traces_all_P(P):
    for seed in range(40):
        rng = np.random.default_rng(seed)
        kw = {}
        if seed % 3 == 0:
            kw = dict(weights=[12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1], lock_words=3 + seed % 20, p_lock_data=0.2)
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(1, 400)), n_words=int(rng.integers(1, 30)), **kw)
        want = oracle.run(ev, nb, bd)
        got = sharded(ev, nb, bd, P)
        assert np.array_equal(got, want), f"seed {seed} P {P}"


@pytest.mark.parametrize("P", [2, 4, 8])
def test_multi_tile_trace(P):
    ev, nb, bd = _fast_random(77, 300_000, 3_000, 8, 128, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1], lock_words=20)
    assert np.array_equal(sharded(ev, nb, bd, P), oracle.run(ev, nb, bd))


@pytest.mark.parametrize("P,bd", [(3, 96), (2, 16)])
def test_multi_tile_trace_odd_geometry(P, bd):
    # block_dim not a power of two / below a warp: the sharded check on the division geometry path
    ev, nb, bd = _fast_random(78, 200_000, 2_000, 5, bd, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1], lock_words=20)
    assert np.array_equal(sharded(ev, nb, bd, P), oracle.run(ev, nb, bd))


@pytest.mark.parametrize("fam,n,rate", [(1, None, 1.0), (2, 2_000_000, 3.0), (4, 3_000_000, 8.0)])
def test_families_sharded_equal_ledger(fam, n, rate):
    ev, nb, bd, led = F.generate(fam, n, rate=rate)
    got = sharded(ev, nb, bd, 4)
    assert [(r["addr"], r["cur"], r["prev"], r["type"]) for r in got] == \
           [(r["addr"], r["cur"], r["prev"], r["type"]) for r in led]


def test_invalid_event_reported_globally():
    import paper_conf_sosp_kamathb21_b200 as igd

    ev, nb, bd = _fast_random(5, 50_000, 100, 2, 64, [20, 18, 10, 4, 3, 8, 3, 3, 1, 1, 1, 1])
    ev["tk"][31_337] = tg.pack_tk(0, 13, 0)
    with pytest.raises(igd.IgdError) as ei:
        sharded(ev, nb, bd, 4)
    assert ei.value.code == igd.igd.IGD_ETRACE and ei.value.bad_index == 31_337


@pytest.mark.parametrize("P", [2, 4])
def test_multi_kernel_sharded(P):
    # kernel boundaries (reading A31) travel with the synchronization stream to every rank
    w = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    for seed in range(30):
        parts = [tg.random_trace(seed * 7 + k, 150, n_blocks=2, block_dim=64, weights=w, lock_words=3,
                                 p_lock_data=0.3)[0] for k in range(3)]
        ev = tg.concat_kernels(parts)
        assert np.array_equal(sharded(ev, 2, 64, P), oracle.run(ev, 2, 64)), f"seed {seed} P {P}"
    big = tg.concat_kernels([_fast_random(90 + k, 80_000, 500, 4, 64, w, lock_words=16)[0] for k in range(3)])
    assert np.array_equal(sharded(big, 4, 64, P), oracle.run(big, 4, 64))
