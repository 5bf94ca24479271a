"""Does the GPU overlap the pipeline's memory-bound stages (ingest, radix passes) with its
ALU-bound check?  Two libigd contexts on two streams detect the same C4 trace: time K detects in
sequence on one context against K rounds of two concurrent detects (one host thread per context;
ctypes releases the GIL).  usage: python profiles/concurrency_probe.py [events] [K]"""
import json
import os
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sosp_kamathb21_b200 as igd  # noqa: E402
import tracegen.families as F  # noqa: E402

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 500_000_000
K = int(sys.argv[2]) if len(sys.argv) > 2 else 4
plan = F.Plan(4, n)
ev = plan.fill()
nb, bd = plan.n_blocks, plan.block_dim
plan.close()
dev = torch.from_numpy(ev.view(np.uint8)).cuda()
dets = [igd.Detector(0, stream=torch.cuda.Stream()) for _ in range(2)]
for d in dets:
    d.load(dev, nb, bd)
    d.detect()
ref = dets[0].reports()
torch.cuda.synchronize()


def run(d, k):
    for _ in range(k):
        d.detect()


def timed(fn):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


seq = timed(lambda: run(dets[0], 2 * K))


def conc():
    th = [threading.Thread(target=run, args=(d, K)) for d in dets]
    for t in th:
        t.start()
    for t in th:
        t.join()


par = timed(conc)
same = all(np.array_equal(d.reports(), ref) for d in dets)
print(json.dumps({"events": n, "detects": 2 * K, "sequential_ms_per_detect": seq / (2 * K),
                  "two_concurrent_ms_per_detect": par / (2 * K), "speedup": seq / par, "reports_equal": same}))
