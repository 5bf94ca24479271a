"""Memory floor of the check's streaming phase: after one igd_detect on a workload, time
(a) streaming the sorted keys/indices and (b) the same plus the per-access event gather.
usage: python profiles/microbench_gather.py C4"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sosp_kamathb21_b200 as igd  # noqa: E402
import tracegen.families as F  # noqa: E402

fam = int(sys.argv[1][1:]) if len(sys.argv) > 1 else 4
plan = F.Plan(fam)
ev = plan.fill()
dev = torch.from_numpy(ev.view(np.uint8)).cuda()
d = igd.Detector(0)
d.load(dev, plan.n_blocks, plan.block_dim)
d.detect(timing=True)
check_ms = d.kernel_stats()["check"][1]
lib = igd.load_library()
lib.igd_debug_gather_probe.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
n_acc = int(((ev["tk"] >> 24) & 0xF <= 4).sum())
for gather in (0, 1, 0, 1):
    ms = ctypes.c_float()
    assert lib.igd_debug_gather_probe(d.ctx, gather, ctypes.byref(ms)) == 0
    print(json.dumps({"workload": F.FAMILY_NAMES[fam], "gather": gather, "ms": ms.value, "check_ms": check_ms,
                      "n_acc": n_acc, "stream_GBps": 8 * n_acc / ms.value / 1e6}), flush=True)
d.close()
