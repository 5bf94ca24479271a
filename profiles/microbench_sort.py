"""Micro-benchmark of the a5 radix sort kernel alone (device-resident u32 pairs).
usage: python profiles/microbench_sort.py [n] ; prints G elements/s per pass and GB/s."""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sosp_kamathb21_b200 as igd  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 500_000_000
lib = igd.load_library()
lib.igd_debug_radix_sort.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.c_uint32, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
d = igd.Detector(0)
g = torch.Generator(device="cuda").manual_seed(1)
out = []
for dist in ("uniform32", "c5like30"):
    if dist == "uniform32":
        k0 = torch.randint(-2**31, 2**31 - 1, (n,), device="cuda", dtype=torch.int32, generator=g)
        bits = 32
    else:
        k0 = torch.randint(0, 2**30, (n,), device="cuda", dtype=torch.int32, generator=g)
        bits = 30
    v0 = torch.arange(n, device="cuda", dtype=torch.int32)
    for mode in (1, 0):
        best = 1e9
        for _ in range(3):
            k, v = k0.clone(), v0.clone()
            ms = ctypes.c_float()
            assert lib.igd_debug_radix_sort(d.ctx, k.data_ptr(), v.data_ptr(), n, bits, mode, ctypes.byref(ms)) == 0
            best = min(best, ms.value)
        passes = (bits + 7) // 8
        r = {"dist": dist, "mode": "ballot" if mode else "match_any", "n": n, "passes": passes, "ms": best,
             "ms_per_pass": best / passes, "Gelem_per_s_per_pass": n * passes / best / 1e6,
             "GBps": 16.0 * n * passes / best / 1e6}
        out.append(r)
        print(json.dumps(r), flush=True)
