"""Pins of the lock-summary reading A8 against what the paper fixes (§6.3):

* "an 18-bit hash of the variable's address": every hash value is < 2^18;
* "a 16-bit summary (2-way bloom filter)": every summary is a nonzero 16-bit
  word with at most two bits set, a function of the 18-bit hash alone, and the two bit positions
  are drawn from different parts of the hash (two ways: more than 16 distinct summaries occur);
* a lock table is one 64-bit structure (Fig. 7) holding 3 entries of {Valid, Active,
  Scope, 18-bit hash} = 3 x 21 bits plus the isThread bit: the capacity of reading A9, pinned by
  the W10 / W11 goldens.

The mixing constant itself is a reading (the paper defines no hash function); these tests pin
the oracle's lock summary to every property the paper does state."""
import ctypes

import numpy as np

import oracle


def _hash_fn():
    lib = oracle._load()
    f = lib.igdo_lock_hash
    f.restype = None
    f.argtypes = [ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]

    def h(word):
        a, b = ctypes.c_uint32(), ctypes.c_uint32()
        f(int(word), ctypes.byref(a), ctypes.byref(b))
        return a.value, b.value
    return h


def test_hash_is_18_bits_and_bloom_is_2way_16bit():
    h = _hash_fn()
    rng = np.random.default_rng(7)
    words = np.concatenate([np.arange(0, 4096, dtype=np.uint64),
                            rng.integers(0, 1 << 62, 20000, dtype=np.uint64)])
    by_hash = {}
    blooms = set()
    for w in words:
        hv, bl = h(w)
        assert 0 <= hv < (1 << 18)
        assert 0 < bl < (1 << 16)
        assert 1 <= bin(bl).count("1") <= 2
        assert by_hash.setdefault(hv, bl) == bl  # a function of the hash
        blooms.add(bl)
    assert len(blooms) > 16  # two hash functions, not one position
    assert len(by_hash) > 10000  # the 18-bit hash spreads words

