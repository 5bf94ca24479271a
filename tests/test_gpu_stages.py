"""Stage-level GPU tests: each kernel against a host reference of THAT stage.
a5 radix sort: stable by key == numpy stable argsort."""
import ctypes

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def det():
    import paper_conf_sosp_kamathb21_b200 as igd

    d = igd.Detector(0)
    yield d
    d.close()


def gpu_sort(det, keys, vals, bits, mode):
    import torch

    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    lib.igd_debug_radix_sort.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                         ctypes.c_uint32, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
    k = torch.from_numpy(keys.view(np.int32)).cuda()
    v = torch.from_numpy(vals.view(np.int32)).cuda()
    ms = ctypes.c_float()
    rc = lib.igd_debug_radix_sort(det.ctx, k.data_ptr(), v.data_ptr(), len(keys), bits, mode, ctypes.byref(ms))
    assert rc == 0
    return k.cpu().numpy().view(np.uint32), v.cpu().numpy().view(np.uint32), ms.value


@pytest.mark.parametrize("mode", [1])
@pytest.mark.parametrize("n,dist", [(1, "u"), (2, "u"), (4095, "u"), (4097, "u"), (1_000_003, "u"),
                                    (777_777, "skew"), (300_000, "const"), (2_000_001, "hi")])
def test_radix_sort_stable(det, mode, n, dist):
    rng = np.random.default_rng(n + mode)
    if dist == "u":
        keys = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    elif dist == "skew":   # Zipf-like hot keys
        keys = (rng.zipf(1.3, n) % (1 << 30)).astype(np.uint32)
    elif dist == "const":
        keys = np.full(n, 12345, np.uint32)
    else:                  # only high digits vary
        keys = (rng.integers(0, 64, n).astype(np.uint32) << 24)
    vals = np.arange(n, dtype=np.uint32)
    ks, vs, _ = gpu_sort(det, keys, vals, 32, mode)
    order = np.argsort(keys, kind="stable")
    assert np.array_equal(ks, keys[order])
    assert np.array_equal(vs, vals[order])
