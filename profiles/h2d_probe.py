"""H2D copy bandwidth from pinned host memory on this box: one stream vs two / four concurrent
streams (chunks of one buffer).  usage: python profiles/h2d_probe.py [GB]"""
import json
import sys
import time

import torch

gb = float(sys.argv[1]) if len(sys.argv) > 1 else 8.0
n = int(gb * (1 << 30))
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
host.fill_(1)
dev = torch.empty(n, dtype=torch.uint8, device="cuda")
out = {}
for ns in (1, 2, 4):
    streams = [torch.cuda.Stream() for _ in range(ns)]
    best = 0.0
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        step = n // ns
        for k, s in enumerate(streams):
            with torch.cuda.stream(s):
                dev[k * step:(k + 1) * step].copy_(host[k * step:(k + 1) * step], non_blocking=True)
        torch.cuda.synchronize()
        best = max(best, n / (time.perf_counter() - t0) / 1e9)
    out[f"{ns}_streams_GBps"] = best
print(json.dumps({"bytes": n, **out}))
