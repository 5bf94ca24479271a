"""CPU oracle of the iGUARD race check -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product path
(``paper_conf_sosp_kamathb21_b200``) never imports it.

The oracle itself is plain C (``oracle/igd_oracle.c``): a sequential shadow-memory replay
of PAPER.md §6.2-§6.4 (Table 2) in the paper's order, with the readings
listed in DESIGN.md.  This module only marshals numpy arrays through ctypes.

Parity status per function:
  * igdo_run                -- pinned: worked examples W1-W9 (tests/golden), from-scratch
                               brute force, pairwise evaluator, sync-free closed form,
                               zero-report families, injection ledgers.
  * coalesced mode (A32)    -- pinned: equals the plain replay of the trace with the coalesced
                               members deleted (group detection restated in numpy in the
                               test), worked example (one report per warp instruction).
  * paper-width counters (A33) -- pinned: the from-scratch evaluator counting sync events
                               modulo the widths (tests/pins.py), equality with the exact
                               mode below the widths, a worked 64-fence example.
  * Bloom/hash constants    -- parity unpinned by the paper (reading A8): pinned only by
                               agreement with the brute force, which restates them.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "igd_oracle.c")
_LIB = os.path.join(_HERE, "libigd_oracle.so")

REPORT_DTYPE = np.dtype([("addr", "<u8"), ("cur", "<u8"), ("prev", "<u8"), ("type", "u1"),
                         ("cur_kind", "u1"), ("prev_kind", "u1"), ("pad", "u1", (5,))])

O_OK, O_EINVAL, O_ETRACE, O_ENOMEM = 0, -1, -2, -4


class OracleError(RuntimeError):
    def __init__(self, code, bad_index=None):
        super().__init__(f"oracle error {code} (bad event {bad_index})")
        self.code = code
        self.bad_index = bad_index


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (plain -O2, single-threaded)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-fPIC", "-shared",
                               "-o", _LIB, _SRC])
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.igdo_run.restype = ctypes.c_int
        lib.igdo_run.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                 ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64,
                                 ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
        lib.igdo_run_ex3.restype = ctypes.c_int
        lib.igdo_run_ex3.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                     ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                     ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
        lib.igdo_run_ex.restype = ctypes.c_int
        lib.igdo_run_ex.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                    ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p,
                                    ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
        _lib = lib
    return _lib


def run(events: np.ndarray, n_blocks: int, block_dim: int, shard=(0, 1), cap: int = None,
        coalesce: bool = False, paper_counters: bool = False, sticky_flags: bool = False,
        tag_log2: int = 0, last_k: int = 1):
    """Replay ``events`` (EVENT_DTYPE, 16 B each) and return the report array (REPORT_DTYPE),
    ascending by ``cur``.  ``shard=(k, K)`` checks only words owned by shard k (C.7 5(b)).
    ``coalesce``: warp-coalesced check mode (§6.5, reading A32).  ``paper_counters``: the
    synchronization IDs wrap at Fig. 4's widths (reading A33).  Paper-fidelity modes (SURVEY
    8(f) f3): ``sticky_flags`` -- P3-P5 gated on the word's sticky DevShared / BlkShared flags as
    Table 2 is written (reading A35); ``tag_log2`` -- metadata table of 2^tag_log2 entries with a
    10-bit Tag, aliasing words (reading A36); ``last_k`` -- the last k accessors / writers are
    checked (reading A37)."""
    lib = _load()
    ev = np.ascontiguousarray(events)
    assert ev.dtype.itemsize == 16
    n = int(ev.shape[0])
    if cap is None:
        cap = max(1024, n // 64)
    while True:
        out = np.zeros(cap, REPORT_DTYPE)
        nrep = ctypes.c_uint64(0)
        bad = ctypes.c_uint64(0)
        flags = (1 if coalesce else 0) | (2 if paper_counters else 0) | (4 if sticky_flags else 0)
        rc = lib.igdo_run_ex3(ev.ctypes.data if n else None, n, n_blocks, block_dim, shard[0], shard[1], flags,
                              tag_log2, last_k, out.ctypes.data, cap, ctypes.byref(nrep), ctypes.byref(bad))
        if rc != O_OK:
            raise OracleError(rc, bad.value if rc == O_ETRACE else None)
        if nrep.value <= cap:
            return out[: nrep.value].copy()
        cap = int(nrep.value)
