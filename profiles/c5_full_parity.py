"""Full-size C5 parity against the ORACLE itself (not only the injection ledger).

Generates the whole C5 trace (4e9 events, 64 GB), runs libigd on it, then runs the C oracle over
the WHOLE trace once per address shard k/K (C.7 5(b): every shard replays all synchronization and
lock events, shadow-checks only its own words) for the shards given, in parallel worker processes,
and compares the GPU reports on those shards' words element by element -- including every trace
index above 2^31.  Also checks the whole GPU report array against the injection ledger.

    python profiles/c5_full_parity.py --shards 0,17,33,50 --K 64 --out gpurun_out/c5_full_parity.json
"""
import argparse
import json
import multiprocessing as mp
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

_EV = None


def _shard_of(words, K):
    h = (words ^ (words >> np.uint64(32))).astype(np.uint64) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(16)
    h = (h * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(13)
    h = (h * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
    return (h ^ (h >> np.uint64(16))) % np.uint64(K)


def _oracle_shard(args):
    k, K, nb, bd = args
    import oracle
    t0 = time.time()
    rep = oracle.run(_EV, nb, bd, shard=(k, K), cap=1 << 20)
    return k, rep, time.time() - t0


def main():
    global _EV
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--events", type=int, default=0)
    ap.add_argument("--shards", default="0,17,33,50")
    ap.add_argument("--K", type=int, default=64)
    ap.add_argument("--out", default="gpurun_out/c5_full_parity.json")
    a = ap.parse_args()
    import torch
    import tracegen.families as F
    import paper_conf_sosp_kamathb21_b200 as igd

    plan = F.Plan(a.config, a.events or None)
    n, nb, bd = plan.n_events, plan.n_blocks, plan.block_dim
    ev = np.empty(n, igd.EVENT_DTYPE)
    plan.fill(out=ev)
    led = plan.ledger()
    plan.close()
    _EV = ev
    t0 = time.time()
    dev = torch.from_numpy(ev.view(np.uint8)).cuda()
    with igd.Detector(0) as d:
        d.load(dev, nb, bd)
        d.detect()
        got = d.reports()
    del dev
    torch.cuda.empty_cache()
    gpu_s = time.time() - t0
    ledger_ok = bool(len(led) == len(got) and np.array_equal(led["addr"], got["addr"])
                     and np.array_equal(led["cur"], got["cur"]) and np.array_equal(led["prev"], got["prev"])
                     and np.array_equal(led["type"].astype(np.uint8), got["type"]))
    shards = [int(x) for x in a.shards.split(",")]
    gsh = _shard_of(got["addr"] >> np.uint64(2), a.K)
    ctx = mp.get_context("fork")
    res = {}
    with ctx.Pool(len(shards)) as pool:
        for k, rep, dt in pool.imap_unordered(_oracle_shard, [(k, a.K, nb, bd) for k in shards]):
            mine = got[gsh == k]
            res[k] = {"oracle_reports": int(len(rep)), "gpu_reports": int(len(mine)),
                      "identical": bool(np.array_equal(mine, rep)), "oracle_s": round(dt, 1),
                      "max_cur": int(rep["cur"].max()) if len(rep) else None,
                      "above_2^31": int((rep["cur"] >= (1 << 31)).sum())}
            print(k, res[k], flush=True)
    out = {"workload": F.FAMILY_NAMES[a.config], "events": n, "K": a.K, "gpu_reports": int(len(got)),
           "ledger_reports": int(len(led)), "ledger_match": ledger_ok, "gpu_s": round(gpu_s, 1),
           "shards": res, "all_identical": all(v["identical"] for v in res.values())}
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    json.dump(out, open(a.out, "w"), indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
