"""Mutation check of the pins: each plausible one-line mistake in the oracle (a dropped term,
a wrong sign or index, a swapped operand) must be caught by the golden fixtures or by the
from-scratch brute force.  Builds mutated copies of oracle/igd_oracle.c with gcc."""
import ctypes
import os
import subprocess
import tempfile

import numpy as np
import pytest

import tracegen as tg
from golden_io import all_golden, full_tuples, parse
from pins import bf_scratch

SRC = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "oracle", "igd_oracle.c")
REPORT = np.dtype([("addr", "<u8"), ("cur", "<u8"), ("prev", "<u8"), ("type", "u1"),
                   ("cur_kind", "u1"), ("prev_kind", "u1"), ("pad", "u1", (5,))])

MUTANTS = {
    "noAny_uses_current_thread": ("noAny = (ANY(p) == md->sANY);", "noAny = (ANY(c) == md->sANY);"),
    "noDev_uses_any": ("noDev = (DEV(p) == md->sDEV);", "noDev = (ANY(p) == md->sDEV);"),
    "A33_devfence_width_7": ("noDev = (dDev & 63u) == 0;", "noDev = (dDev & 127u) == 0;"),
    "A33_blkfence_ignored": ("noAny = noDev && (dBlk & 63u) == 0;", "noAny = noDev;"),
    "A33_barrier_width_6": ("((dBB & 255u) != 0)", "((dBB & 63u) != 0)"),
    "md_always_last_accessor": ("(k == O_LD) ? &S->LW : &S->LA", "&S->LA"),
    "P4_drops_mask_clause": ("|| (e.mask >> g_lane(&g, p)) & 1u", "|| 0"),
    "P4_mask_uses_current_lane": ("(e.mask >> g_lane(&g, p))", "(e.mask >> g_lane(&g, c))"),
    "P5_drops_barrier": ("(BB(b_c) != md->sBB)", "1"),
    "P6_drops_scope": ("|| S->ascope == S_DEVICE)", ")"),
    "R1_uses_md_block": ("g_block(&g, S->LW.tid) != b_c", "b_p != b_c"),
    "R2_drops_blkShared": ("&& !S->devShared && !S->blkShared) type = R2", "&& !S->devShared) type = R2"),
    "R3_drops_devShared": ("noAny && !S->devShared) type = R3", "noAny) type = R3"),
    "R5_or_instead_of_and": ("(S->locks & L) == 0", "(S->locks | L) == 0"),
    "devShared_not_sticky": ("if (g_block(&g, la) != b_c) S->devShared = 1;", "S->devShared = 0; if (g_block(&g, la) != b_c) S->devShared = 1;"),
    "blkShared_not_sticky": ("else if (g_warp(&g, la) != w_c) S->blkShared = 1;", "else { S->blkShared = (g_warp(&g, la) != w_c); }"),
    "P2_for_stores_too": ("if (k == O_LD && !S->modified)", "if (!S->modified)"),
    "locks_field_last_writer": ("S->locks = L;", "if (isWrite) S->locks = L;"),
    "block_fence_counts_dev": ("if (s >= S_DEVICE) devF[c]++;", "devF[c]++;"),
    "activate_wider_scope": ("T->e[k].scope <= s", "T->e[k].scope >= s"),
    "isThread_never": ("__builtin_popcount(e.mask) > 1", "__builtin_popcount(e.mask) > 32"),
    "exch_ignores_scope": ("T->e[q].h18 == h && T->e[q].scope == s) {", "T->e[q].h18 == h) {"),
    "grid_no_lock_activation": ("o_activate(&wt[w], S_DEVICE);", ";"),
    "grid_not_barrier": ("#define BB(b) (bbar[b] + G)", "#define BB(b) (bbar[b])"),
    "system_not_device": ("(e.scope == S_SYSTEM) ? S_DEVICE : e.scope", "e.scope"),
    "ascope_first_atomic": ("if (isAtomic) { S->atomic = 1; S->ascope = (uint8_t)s; }",
                            "if (isAtomic) { if (!S->atomic) S->ascope = (uint8_t)s; S->atomic = 1; }"),
    "check_after_lock_update": ("uint16_t L = o_held_of(TABLE(c));", "uint16_t L = o_held_of(TABLE(c)) | (k == O_CAS ? o_bloom(o_h18(e.addr >> 2)) : 0);"),
    "bloom_single_bit": ("| (1u << ((h >> 4) & 15u))", ""),
    # reading A9 (lock-table capacity, duplicates, overflow): W10 / W11 discriminate
    "A9_no_dedup": ("T->e[q].scope == s) present = 1;", "T->e[q].scope == s) present = 0;"),
    "A9_evict_oldest": ("if (slot < 0) present = 1;",
                        "if (slot < 0) { T->e[0] = T->e[1]; T->e[1] = T->e[2]; T->e[2].valid = 0; slot = 2; }"),
    "A9_replace_last": ("if (slot < 0) present = 1;", "if (slot < 0) slot = 2;"),
    "A9_four_entries": ("if (slot < 0) present = 1;", "if (slot < 0) { memset(T, 0, sizeof(*T)); slot = 0; }"),
}


# paper-fidelity modes (A35-A37): caught by the mode brute force of tests/pins.py
MODE_MUTANTS = {
    "A35_P5_gated_on_blkShared_too": ("if (S->devShared) P5 = 0;", "if (S->devShared || S->blkShared) P5 = 0;"),
    "A35_P3_not_gated": ("if (S->devShared || S->blkShared) { P3 = 0; P4 = 0; }", "if (S->devShared || S->blkShared) { P4 = 0; }"),
    "A36_tag_ignored": ("(S->kernel != kernel || S->tag != tag)", "(S->kernel != kernel)"),
    "A36_tag_9_bits": ("(uint32_t)((word >> tag_log2) & 1023u)", "(uint32_t)((word >> tag_log2) & 511u)"),
    "A37_oldest_first": ("cands[q] = &S->hist[(k == O_LD ? 8 : 0) + q];",
                         "cands[q] = &S->hist[(k == O_LD ? 8 : 0) + ncand - 1 - q];"),
    "A37_writers_for_stores": ("cands[q] = &S->hist[(k == O_LD ? 8 : 0) + q];", "cands[q] = &S->hist[8 + q];"),
}


def _run_mode(lib, ev, nb, bd, flags, tag_log2, last_k):
    cap = 4096
    out = np.zeros(cap, REPORT)
    nrep, bad = ctypes.c_uint64(0), ctypes.c_uint64(0)
    rc = lib.igdo_run_ex3(ev.ctypes.data if len(ev) else None, len(ev), nb, bd, 0, 1, flags, tag_log2, last_k,
                          out.ctypes.data, cap, ctypes.byref(nrep), ctypes.byref(bad))
    assert rc == 0
    return full_tuples(out[: nrep.value])


def _caught_modes(lib):
    from pins import bf_scratch_modes
    from test_fidelity_modes import _tag_trace

    for seed in range(150):
        rng = np.random.default_rng(seed)
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(20, 150)), n_words=int(rng.integers(1, 6)))
        if _run_mode(lib, ev, nb, bd, 4, 0, 1) != bf_scratch_modes(ev, nb, bd, sticky=True):
            return f"sticky seed {seed}"
        if _run_mode(lib, ev, nb, bd, 0, 0, 4) != bf_scratch_modes(ev, nb, bd, last_k=4):
            return f"last-k seed {seed}"
        ev, nb, bd = _tag_trace(seed, 120, 8)
        if _run_mode(lib, ev, nb, bd, 0, 8, 1) != bf_scratch_modes(ev, nb, bd, tag_log2=8):
            return f"tag seed {seed}"
    return None


def _build(mutant_src, d):
    c = os.path.join(d, "m.c")
    so = os.path.join(d, "m.so")
    with open(c, "w") as f:
        f.write(mutant_src)
    subprocess.check_call(["gcc", "-O1", "-std=c11", "-w", "-fPIC", "-shared", "-o", so, c])
    lib = ctypes.CDLL(so)
    lib.igdo_run.restype = ctypes.c_int
    lib.igdo_run.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                             ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64,
                             ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
    lib.igdo_run_ex3.restype = ctypes.c_int
    lib.igdo_run_ex3.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                 ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p,
                                 ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
    lib.igdo_run_ex.restype = ctypes.c_int
    lib.igdo_run_ex.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64,
                                ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
    return lib


def _run_paper_counters(lib, ev, nb, bd):
    cap = 4096
    out = np.zeros(cap, REPORT)
    nrep, bad = ctypes.c_uint64(0), ctypes.c_uint64(0)
    rc = lib.igdo_run_ex(ev.ctypes.data if len(ev) else None, len(ev), nb, bd, 0, 1, 2, out.ctypes.data, cap,
                         ctypes.byref(nrep), ctypes.byref(bad))
    assert rc == 0
    return full_tuples(out[: nrep.value])


def _run(lib, ev, nb, bd):
    cap = 4096
    out = np.zeros(cap, REPORT)
    nrep, bad = ctypes.c_uint64(0), ctypes.c_uint64(0)
    rc = lib.igdo_run(ev.ctypes.data if len(ev) else None, len(ev), nb, bd, 0, 1, out.ctypes.data, cap,
                      ctypes.byref(nrep), ctypes.byref(bad))
    assert rc == 0
    return full_tuples(out[: nrep.value])


def _caught(lib):
    for path in all_golden():
        ev, nb, bd, exp = parse(path)
        if [r[:4] for r in _run(lib, ev, nb, bd)] != exp:
            return "golden:" + os.path.basename(path)
    w_lock = [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1]
    for seed in range(300):
        rng = np.random.default_rng(seed)
        kw = {"weights": w_lock, "lock_words": 5 + seed % 40, "p_lock_data": 0.2} if seed % 2 else {}
        ev, nb, bd = tg.random_trace(seed, int(rng.integers(20, 160)), n_words=int(rng.integers(1, 10)), **kw)
        if _run(lib, ev, nb, bd) != bf_scratch(ev, nb, bd):
            return f"bruteforce seed {seed}"
    from test_paper_counters import _burst_trace  # paper-width IDs (A33)
    for seed in range(100):
        ev, nb, bd = _burst_trace(seed, 40, threads=[0, 1, 33, 64] if seed % 2 else None)
        if _run_paper_counters(lib, ev, nb, bd) != bf_scratch(ev, nb, bd, paper_counters=True):
            return f"paper-counter bursts seed {seed}"
    return None


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_mutant_is_caught(name):
    src = open(SRC).read()
    old, new = MUTANTS[name]
    assert src.count(old) >= 1, f"mutation anchor vanished: {old!r}"
    with tempfile.TemporaryDirectory() as d:
        lib = _build(src.replace(old, new, 1), d)
        assert _caught(lib) is not None, f"mutant {name} survived every pin"


@pytest.mark.parametrize("name", sorted(MODE_MUTANTS))
def test_mode_mutant_is_caught(name):
    src = open(SRC).read()
    old, new = MODE_MUTANTS[name]
    assert src.count(old) >= 1, f"mutation anchor vanished: {old!r}"
    with tempfile.TemporaryDirectory() as d:
        lib = _build(src.replace(old, new, 1), d)
        assert _caught_modes(lib) is not None, f"mutant {name} survived every pin"
