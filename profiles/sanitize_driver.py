"""Drive libigd through the bare C ABI (no torch: cudaMallocAsync allocator, legacy stream) on
small traces, for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
    compute-sanitizer --tool racecheck python profiles/sanitize_driver.py
Checks every report set against the oracle too."""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import oracle  # noqa: E402
import tracegen as tg  # noqa: E402
import tracegen.families as F  # noqa: E402
from paper_conf_sosp_kamathb21_b200 import igd as I  # noqa: E402


def run(lib, ev, nb, bd, flags=0):
    ctx = ctypes.c_void_p()
    rc = lib.igd_ctx_create(ctypes.byref(ctx), 0, None, 1, 0, None, I.ALLOC_FN(), I.FREE_FN(), None)
    assert rc == 0, rc
    d = I.igd_trace_desc(nb, bd, len(ev), 0, len(ev), 0)
    assert lib.igd_trace_load(ctx, ctypes.byref(d), ctypes.c_void_p(ev.ctypes.data)) == 0
    n = ctypes.c_uint64()
    rc = lib.igd_detect(ctx, flags, ctypes.byref(n))
    assert rc == 0, (rc, lib.igd_last_error(ctx))
    out = np.zeros(max(n.value, 1), I.REPORT_DTYPE)
    w = ctypes.c_uint64()
    assert lib.igd_reports(ctx, out.ctypes.data, n.value, ctypes.byref(w)) == 0
    lib.igd_ctx_destroy(ctx)
    return out[: w.value]


def main():
    lib = I.load_library(build_if_missing=False)
    cases = []
    ev, nb, bd, _ = F.generate(1)
    cases.append(("C1", ev, nb, bd))
    plan = F.Plan(2)
    cases.append(("C2 prefix 2e5", plan.fill(0, 200_000), plan.n_blocks, plan.block_dim))
    plan.close()
    from test_gpu_parity import _fast_random
    e3, nb3, bd3 = _fast_random(5, 60_000, 200, 4, 64, [12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1], lock_words=20)
    cases.append(("lock-heavy random", e3, nb3, bd3))
    for name, ev, nb, bd in cases:
        got = run(lib, ev, nb, bd)
        want = oracle.run(ev, nb, bd)
        print(f"{name}: {len(ev)} events, {len(got)} reports, identical to the oracle: {np.array_equal(got, want)}",
              flush=True)
        assert np.array_equal(got, want)


if __name__ == "__main__":
    main()
