"""Event counters of the check kernel on a workload (what fraction of accesses reach which
Table-2 stage, how many list queries and how they are answered).
usage: python profiles/build_variants.py stats:IGD_CHECK_STATS=1
       IGD_LIB=variants/libigd_stats.so python profiles/check_stats.py C4 [events]
(counters not instrumented in the current kernel read 0)"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sosp_kamathb21_b200 as igd  # noqa: E402
import tracegen.families as F  # noqa: E402

NAMES = ["checked", "P2", "P3", "P6", "P4_lockstep", "mask_gather", "queued", "q_calls", "q_fast", "q_probe_hit",
         "q_bsearch", "reports", "ph2_P4_syncwarp", "ph2_P5", "ph2_fence_query", "ph2_R5_search"]
fam = int(sys.argv[1][1:]) if len(sys.argv) > 1 else 4
plan = F.Plan(fam, n=int(float(sys.argv[2])) if len(sys.argv) > 2 else None)
ev = plan.fill()
dev = torch.from_numpy(ev.view(np.uint8)).cuda()
d = igd.Detector(0)
lib = igd.load_library()
lib.igd_debug_check_stats.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
d.load(dev, plan.n_blocks, plan.block_dim)
lib.igd_debug_check_stats(d.ctx, 1, None)
d.detect()
out = np.zeros(16, np.uint64)
lib.igd_debug_check_stats(d.ctx, 0, out.ctypes.data)
n_acc = int((((ev["tk"] >> 24) & 0xF) <= 4).sum())
res = {"workload": F.FAMILY_NAMES[fam], "events": len(ev), "accesses": n_acc}
res.update({k: int(out[i]) for i, k in enumerate(NAMES)})
print(json.dumps(res))
d.close()
