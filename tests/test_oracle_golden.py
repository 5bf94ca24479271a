"""Oracle vs the paper's worked examples (fixtures in tests/golden/)."""
import os

import pytest

import oracle
import tracegen as tg
from golden_io import all_golden, parse, report_tuples

GOLDEN = all_golden()


@pytest.mark.parametrize("path", GOLDEN, ids=[os.path.basename(p) for p in GOLDEN])
def test_golden_exact(path):
    ev, nb, bd, expects = parse(path)
    rep = oracle.run(ev, nb, bd)
    assert report_tuples(rep) == expects


def test_golden_count():
    assert len(GOLDEN) >= 17


def test_w6_lock_words_have_disjoint_blooms():
    # the fixture's premise (reading A8): L0=200 and L1=201 summarise to disjoint Bloom bits
    def h18(w):
        return ((w & 0xFFFFFFFF) * 0x9E3779B1 & 0xFFFFFFFF) >> 14

    def bloom(h):
        return (1 << (h & 15)) | (1 << ((h >> 4) & 15))

    assert bloom(h18(200)) & bloom(h18(201)) == 0


def test_report_kinds_recorded():
    ev, nb, bd, _ = parse(os.path.join(os.path.dirname(GOLDEN[0]), "W7_block_scope_lock.trace"))
    rep = oracle.run(ev, nb, bd)
    assert [(r["cur_kind"], r["prev_kind"]) for r in rep] == [(tg.CAS, tg.EXCH), (tg.LD, tg.ST)]


def test_empty_trace():
    ev = tg.TraceBuilder(1, 32).events()
    assert len(oracle.run(ev, 1, 32)) == 0


def test_system_scope_equals_device():
    # A12: a SYSTEM fence publishes like a DEVICE fence (P:246-249 system scope ignored)
    for sc, expect in ((tg.SYSTEM, 0), (tg.DEVICE, 0), (tg.BLOCK, 1)):
        b = tg.TraceBuilder(2, 64)
        b.st(0, 5)
        b.fence(0, sc)
        b.ld(64, 5)
        assert len(oracle.run(b.events(), 2, 64)) == expect


@pytest.mark.parametrize("bad", ["kind", "tid", "lane", "scope_ld", "scope_atom", "fence_addr", "grid_tid", "hibits"])
def test_invalid_events_rejected(bad):
    b = tg.TraceBuilder(2, 64)
    b.st(0, 1)
    b.ld(1, 1)
    ev = b.events()
    bad_ev = ev.copy()
    row = bad_ev[1:2]
    if bad == "kind":
        row["tk"] = tg.pack_tk(1, 12, 0)
    elif bad == "tid":
        row["tk"] = tg.pack_tk(128, tg.LD, 0)
    elif bad == "lane":
        row["mask"] = 0x1  # tid 1 -> lane 1 not in mask
    elif bad == "scope_ld":
        row["tk"] = tg.pack_tk(1, tg.LD, tg.DEVICE)
    elif bad == "scope_atom":
        row["tk"] = tg.pack_tk(1, tg.ATOM, tg.NONE)
    elif bad == "fence_addr":
        row["tk"] = tg.pack_tk(1, tg.FENCE, tg.DEVICE)
    elif bad == "grid_tid":
        row["tk"] = tg.pack_tk(1, tg.GRID_SYNC, tg.NONE)
        row["addr"] = 0
    elif bad == "hibits":
        row["tk"] = tg.pack_tk(1, tg.LD, 0) | (1 << 30)
    bad_ev[1:2] = row
    with pytest.raises(oracle.OracleError) as ei:
        oracle.run(bad_ev, 2, 64)
    assert ei.value.code == oracle.O_ETRACE and ei.value.bad_index == 1
