"""ctypes wrapper of tracegen/igdgen.c: the C1..C5 workload families.

Input generation only.  ``generate(family)`` returns the trace (EVENT_DTYPE), the grid
geometry and the injection ledger (REPORT-like records: addr, cur, prev, type) -- the races the
generator deliberately planted, written down when it planted them.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import EVENT_DTYPE

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "igdgen.c")
_LIB = os.path.join(_HERE, "libigdgen.so")

LEDGER_DTYPE = np.dtype([("addr", "<u8"), ("cur", "<u8"), ("prev", "<u8"), ("type", "<u4"), ("pad", "<u4")])
FAMILY_SEED = {k: 0x16D0000 + k for k in range(1, 6)}  # seed for config k
FAMILY_NAMES = {1: "C1-litmus", 2: "C2-graph-analytics", 3: "C3-warp-primitive", 4: "C4-cg-grid-sync",
                5: "C5-large-mixed"}
DEFAULT_N = {1: 10_000, 2: 10_000_000, 3: 100_000_000, 4: 500_000_000, 5: 4_000_000_000}


class _Cfg(ctypes.Structure):
    _fields_ = [("family", ctypes.c_uint32), ("fixed", ctypes.c_uint32), ("n_blocks", ctypes.c_uint32),
                ("block_dim", ctypes.c_uint32), ("seed", ctypes.c_uint64), ("n_target", ctypes.c_uint64),
                ("rate", ctypes.c_double), ("lock_frac", ctypes.c_double), ("fence_frac", ctypes.c_double)]


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fopenmp", "-fPIC", "-shared", "-Wall",
                               "-Wno-unused-function", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.igdgen_plan.restype = ctypes.c_void_p
        lib.igdgen_plan.argtypes = [ctypes.POINTER(_Cfg), ctypes.POINTER(ctypes.c_uint64),
                                    ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
        lib.igdgen_fill.restype = ctypes.c_int
        lib.igdgen_fill.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int]
        lib.igdgen_ledger.restype = ctypes.c_uint64
        lib.igdgen_ledger.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64]
        lib.igdgen_free.restype = None
        lib.igdgen_free.argtypes = [ctypes.c_void_p]
        _lib = lib
    return _lib


class Plan:
    """A planned trace: sizes and ledger known, events generated on demand (any range)."""

    def __init__(self, family: int, n: int = None, seed: int = None, fixed: bool = False, rate: float = 1.0,
                 lock_frac: float = 0.0, fence_frac: float = 0.0):
        """``lock_frac`` / ``fence_frac`` (C2, C5): the sync-heavy variant's share of spin-locked
        vertices (default 1 %) and per-warp release fences after each update round (default none)."""
        lib = _load()
        cfg = _Cfg(family, 1 if fixed else 0, 0, 0, FAMILY_SEED[family] if seed is None else seed,
                   0 if n is None else n, rate, lock_frac, fence_frac)
        ne, nb, bd = ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint32()
        self._p = lib.igdgen_plan(ctypes.byref(cfg), ctypes.byref(ne), ctypes.byref(nb), ctypes.byref(bd))
        if not self._p:
            raise ValueError(f"bad family {family}")
        self.family, self.n_events, self.n_blocks, self.block_dim = family, ne.value, nb.value, bd.value
        self.seed = cfg.seed
        self.fixed = fixed

    def fill(self, first: int = 0, count: int = None, out: np.ndarray = None, threads: int = 0) -> np.ndarray:
        if count is None:
            count = self.n_events - first
        if out is None:
            out = np.empty(count, EVENT_DTYPE)
        assert out.dtype.itemsize == 16 and out.flags.c_contiguous and len(out) >= count
        rc = _load().igdgen_fill(self._p, first, count, out.ctypes.data, threads)
        if rc != 0:
            raise ValueError("range outside the trace")
        return out

    def ledger(self) -> np.ndarray:
        lib = _load()
        n = lib.igdgen_ledger(self._p, None, 0)
        out = np.zeros(n, LEDGER_DTYPE)
        if n:
            lib.igdgen_ledger(self._p, out.ctypes.data, n)
        return out

    def close(self):
        if self._p:
            _load().igdgen_free(self._p)
            self._p = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass


# the sync-heavy variant of C2 / C5 (fences ~5 %, spin-lock sections ~8 %)
SYNC_HEAVY = {"lock_frac": 0.25, "fence_frac": 1.0}


def generate(family: int, n: int = None, seed: int = None, fixed: bool = False, rate: float = 1.0, **kw):
    """Whole trace in host memory: (events, n_blocks, block_dim, ledger)."""
    p = Plan(family, n, seed, fixed, rate, **kw)
    ev = p.fill()
    led = p.ledger()
    nb, bd = p.n_blocks, p.block_dim
    p.close()
    return ev, nb, bd, led
