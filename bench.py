#!/usr/bin/env python
"""bench.py -- G events race-checked/s on B200 (BASELINE.json metric).

One step = one ``igd_detect`` over the whole synthetic trace of the workload: ingest +
validation, sync-epoch tables, lock inference, radix sort by word, segmented shadow check,
report compaction and canonical ordering (every SURVEY 8(a) row).  The trace is resident in
HBM when the timed region starts (``value``); ``e2e`` repeats the measurement through the C
ABI with HOST buffers (H2D of the trace and D2H of the reports inside the timed region).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl igd|reference]

The default workload is C5 (4x10^9 events over 2^30 words; BASELINE.json configs[4], the
configuration the metric is quoted on at 1/2/4/8 GPUs).  Inputs (64 GB) are far larger than
L2 (126 MB), so no L2 flush is needed between steps.  ``cpu_baseline`` times the CPU oracle
(single thread) on a bounded prefix of the same trace; ``--impl reference`` times only the
oracle.  Data is synthetic (tracegen, seed 0x16D0000 + k).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "G events race-checked/s at 1/2/4/8 B200; achieved HBM GB/s vs peak"
CONFIGS = {"C1": 1, "C2": 2, "C3": 3, "C4": 4, "C5": 5}


def gen_kw(args):
    import tracegen.families as F

    return dict(F.SYNC_HEAVY) if getattr(args, "sync_heavy", False) else {}


def workload_name(args, fam):
    import tracegen.families as F

    return F.FAMILY_NAMES[fam] + ("-sync-heavy" if getattr(args, "sync_heavy", False) else "")


def log(*a):
    print(*a, file=sys.stderr, flush=True)


_JSON_OUT = None


def _claim_stdout():
    """Keep fd 1 for the one JSON line: libraries print to stdout from C (NCCL's version banner
    goes through printf when the communicator is created), so fd 1 is pointed at stderr for the
    rest of the run and the line is written to a private duplicate of the original stdout."""
    global _JSON_OUT
    if _JSON_OUT is None:
        sys.stdout.flush()
        _JSON_OUT = os.fdopen(os.dup(1), "w")
        os.dup2(2, 1)


def emit(line):
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    out.write(json.dumps(line) + "\n")
    out.flush()


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.t = threading.Thread(target=self._read, daemon=True)
        self.t.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                self.rows.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if r[5 + k].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except (OSError, KeyError, ValueError):
        return 6650.0, "fallback"


def host_info():
    """The host the oracle baseline ran on (nproc, CPU model, RAM)."""
    model, ram = None, None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                ram = round(int(line.split()[1]) / 1024 / 1024, 1)
                break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "ram_gib": ram}


def pin_one_core():
    """Pin this process to one host core for the oracle timing (the `taskset -c` of SURVEY 8(d));
    returns the previous affinity to restore, or None."""
    try:
        prev = os.sched_getaffinity(0)
        core = sorted(prev)[min(1, len(prev) - 1)]
        os.sched_setaffinity(0, {core})
        return prev
    except (AttributeError, OSError):
        return None


def oracle_baseline(ev, nb, bd, budget_s=15.0, coalesce=False, paper_counters=False):
    """Time the CPU oracle (as it stands, single-threaded, pinned to one core) on a bounded prefix
    of the trace."""
    import oracle

    prev = pin_one_core()
    try:
        return _oracle_baseline(oracle, ev, nb, bd, budget_s, coalesce, paper_counters)
    finally:
        if prev is not None:
            os.sched_setaffinity(0, prev)


ORACLE_SAMPLE = 12_000_000  # events of the bounded oracle sample (both the cpu_baseline and --impl reference)


def _oracle_baseline(oracle, ev, nb, bd, budget_s, coalesce, paper_counters):
    """The first ORACLE_SAMPLE events of the trace (the same sample --impl reference times), the
    best of up to three runs within the budget."""
    n = min(len(ev), ORACLE_SAMPLE)
    best = None
    t_start = time.perf_counter()
    for _ in range(3):
        t0 = time.perf_counter()
        oracle.run(ev[:n], nb, bd, coalesce=coalesce, paper_counters=paper_counters)
        dt = time.perf_counter() - t0
        best = dt if best is None else min(best, dt)
        if time.perf_counter() - t_start > budget_s:
            break
    return n, best


def run_reference(args, fam, rank, world):
    """--impl reference: the CPU oracle, timed as it stands on the host cores (rank 0 only)."""
    if rank != 0:
        return
    import tracegen.families as F
    import oracle

    plan = F.Plan(fam, **gen_kw(args))
    # each step checks a bounded prefix sample of the workload so the run ends in minutes
    sample = min(plan.n_events, args.oracle_events or ORACLE_SAMPLE)
    ev = plan.fill(0, sample)
    nb, bd, n_total = plan.n_blocks, plan.block_dim, plan.n_events
    plan.close()
    pin_one_core()
    for _ in range(args.warmup):
        oracle.run(ev[: min(sample, 1_000_000)], nb, bd)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.run(ev, nb, bd)
        times.append(time.perf_counter() - t0)
    t = sum(times) / len(times)
    value = sample / t / 1e9
    sample_desc = f"first {sample} of {n_total} events of {workload_name(args, fam)} (single-threaded oracle)"
    line = {"metric": METRIC, "value": value, "unit": "G events/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic", "impl": "reference",
            "config": {"workload": workload_name(args, fam), "events": n_total, "sample_events": sample,
                       "n_blocks": nb, "block_dim": bd},
            "cpu_baseline": {"value": value, "unit": "G events/s", "cores": 1, "kind": "oracle",
                             "sample": sample_desc, "host": host_info()},
            "e2e": {"value": value, "unit": "G events/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)


def run_sharded(args, fam, rank, world, local):
    """N GPUs (one process each) through the collective C ABI: every rank
    creates an igd context with the same NCCL unique id (torch.distributed only broadcasts the
    128-byte id and brackets the timed region), loads its contiguous chunk of the trace, and
    igd_detect runs the partition, the NCCL all-to-all / all-gathers, the sharded check and the
    report merge inside libigd.  The same global trace for every N (strong scaling); each rank
    generates only its chunk.  --sharded at N=1: the one-rank collective path."""
    import torch
    import torch.distributed as dist

    import paper_conf_sosp_kamathb21_b200 as igd
    import tracegen.families as F

    torch.cuda.set_device(local % torch.cuda.device_count())
    dev_index = torch.cuda.current_device()
    if world == 1:  # --sharded on one GPU: a one-rank process group
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", str(29500 + os.getpid() % 1000))
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
    if not dist.is_initialized():
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_index))
        else:
            dist.init_process_group(args.backend)
    tdev = f"cuda:{dev_index}" if args.backend == "nccl" else "cpu"
    idt = torch.zeros(128, dtype=torch.uint8, device=tdev)
    if rank == 0:
        idt.copy_(torch.frombuffer(bytearray(igd.igd_nccl_unique_id()), dtype=torch.uint8))
    dist.broadcast(idt, 0)
    nccl_id = bytes(idt.cpu().numpy().tobytes())

    t0 = time.time()
    plan = F.Plan(fam, args.events or None, **gen_kw(args))
    n, nb, bd = plan.n_events, plan.n_blocks, plan.block_dim
    lo = n * rank // world
    cnt = n * (rank + 1) // world - lo
    host = np.empty(cnt, igd.EVENT_DTYPE)
    plan.fill(lo, cnt, out=host, threads=args.threads)
    lg = plan.ledger()
    plan.close()
    if rank == 0:
        log(f"[bench] {workload_name(args, fam)}: {n} events over {world} ranks, chunk {cnt}, {time.time() - t0:.1f}s")
    cudart = torch.cuda.cudart()
    pinned = cudart.cudaHostRegister(host.ctypes.data, host.nbytes, 0) == 0
    chunk = torch.from_numpy(host.view(np.uint8)).to(f"cuda:{dev_index}")
    det = igd.Detector(dev_index, nranks=world, rank=rank, nccl_id=nccl_id)
    det.load(chunk, nb, bd, first_event=lo, n_events_total=n)
    for _ in range(args.warmup):
        nrep = det.detect()
    clocks = ClockSampler(dev_index)
    clocks.start()
    dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    kstats, launches = {}, 0
    e0.record(det.stream)
    for _ in range(args.steps):  # uninstrumented
        nrep = det.detect()
        launches += det.launch_count()
    e1.record(det.stream)
    torch.cuda.synchronize()
    dist.barrier()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1) / args.steps
    t = torch.tensor([ms], dtype=torch.float64, device=tdev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)  # slowest rank
    ms = float(t.item())
    value = n / (ms / 1e3) / 1e9
    rep = det.reports()
    for _ in range(args.steps):  # per-kernel breakdown from instrumented steps after the timed region
        det.detect(timing=True)
        for k, (c, ms_, b) in det.kernel_stats().items():
            c0, m0, b0 = kstats.get(k, (0, 0.0, 0.0))
            kstats[k] = (c0 + c, m0 + ms_, b0 + b)
    ledger_match = bool(len(lg) == len(rep) and np.array_equal(lg["addr"], rep["addr"])
                        and np.array_equal(lg["cur"], rep["cur"]) and np.array_equal(lg["prev"], rep["prev"])
                        and np.array_equal(lg["type"].astype(np.uint8), rep["type"]))
    # end to end: host chunk -> library H2D -> collective check -> global reports on the host
    del chunk
    det.load(np.zeros(0, igd.EVENT_DTYPE), nb, bd, first_event=lo, n_events_total=n)
    torch.cuda.empty_cache()
    e2e_times = []
    out = rep
    for s in range(0 if args.no_e2e else args.e2e_steps + 1):
        dist.barrier()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        det.load(host, nb, bd, first_event=lo, n_events_total=n)
        det.detect()
        out = det.reports()
        torch.cuda.synchronize()
        if s > 0:
            e2e_times.append(time.perf_counter() - t1)
    e2e_s = sum(e2e_times) / len(e2e_times) if e2e_times else 0.0
    t = torch.tensor([e2e_s], dtype=torch.float64, device=tdev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    e2e_s = float(t.item())
    if pinned:
        cudart.cudaHostUnregister(host.ctypes.data)
    peak, peak_kind = peaks()
    dom = max(kstats, key=lambda k: kstats[k][1])
    c, kms, kbytes = kstats[dom]
    achieved = kbytes / (kms / 1e3) / 1e9 if kms > 0 else 0.0
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "G events/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": {"workload": workload_name(args, fam), "events": n, "n_blocks": nb, "block_dim": bd,
                           "reports": int(nrep), "ledger_reports": int(len(lg)), "ledger_match": ledger_match,
                           "l2": "inputs larger than L2 (no flush)",
                           "parallelism": f"{world} ranks: contiguous trace chunks, words hash-sharded "
                                          "(fmix32 % P); NCCL all-to-all + all-gathers inside libigd "
                                          "(collective igd_detect)"},
                "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                             "frac": achieved / peak, "peak_source": peak_kind, "traffic": None,
                             "launches_per_step": c / args.steps, "rank": 0},
                "path": {"kernels": {k: {"launches": v[0] // args.steps, "ms": v[1] / args.steps}
                                     for k, v in kstats.items() if v[0]}},
                "cpu_baseline": None,
                "e2e": {"value": n / e2e_s / 1e9 if e2e_times else None, "unit": "G events/s",
                        "h2d_bytes_per_step": n * 16, "d2h_bytes_per_step": int(len(out)) * 32 * world,
                        "ms_per_step": e2e_s * 1e3},
                "gpu_launches": launches, "clocks": clk}
        emit(line)
    det.close()
    dist.destroy_process_group()


def run_stream(args, fam):
    """--stream-chunks K: each step is one streaming session over the device-resident
    trace cut into K equal chunks (igd_stream_begin / feed x K / end); the union of the chunks'
    reports is compared with the injection ledger."""
    import torch

    import paper_conf_sosp_kamathb21_b200 as igd
    import tracegen.families as F

    torch.cuda.set_device(0)
    plan = F.Plan(fam, args.events or None, **gen_kw(args))
    n, nb, bd = plan.n_events, plan.n_blocks, plan.block_dim
    host = np.empty(n, igd.EVENT_DTYPE)
    plan.fill(out=host, threads=args.threads)
    lg = plan.ledger()
    plan.close()
    dev = torch.from_numpy(host.view(np.uint8)).cuda()
    K = args.stream_chunks
    cuts = [n * k // K for k in range(K + 1)]
    chunks = [dev[cuts[k] * 16: cuts[k + 1] * 16] for k in range(K)]
    det = igd.Detector(0)

    def session():
        det.stream_begin(nb, bd)
        parts = [det.stream_feed(c) for c in chunks]
        det.stream_end()
        return np.concatenate(parts) if parts else np.zeros(0, igd.REPORT_DTYPE)

    for _ in range(args.warmup):
        rep = session()
    clocks = ClockSampler(0)
    clocks.start()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(det.stream)
    for _ in range(args.steps):
        rep = session()
    e1.record(det.stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1) / args.steps
    ledger_match = bool(len(lg) == len(rep) and np.array_equal(lg["cur"], rep["cur"])
                        and np.array_equal(lg["addr"], rep["addr"]) and np.array_equal(lg["prev"], rep["prev"])
                        and np.array_equal(lg["type"].astype(np.uint8), rep["type"]))
    line = {"metric": METRIC, "value": n / (ms / 1e3) / 1e9, "unit": "G events/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": workload_name(args, fam), "events": n, "n_blocks": nb, "block_dim": bd,
                       "check_mode": f"streaming session, {K} chunks (igd_stream_*)", "reports": int(len(rep)),
                       "ledger_reports": int(len(lg)), "ledger_match": ledger_match,
                       "l2": "inputs larger than L2 (no flush)" if n * 16 > 126e6 else "inputs smaller than L2"},
            "roofline": None, "cpu_baseline": None, "e2e": None, "gpu_launches": None, "clocks": clk}
    emit(line)
    det.close()


# kernel class -> the kernel ncu names for it (classes made of one kernel)
CLASS_KERNEL = {"sort_access": "rsort::k_onesweep<unsigned long, 0, unsigned int>",
                "check": "check::k_check4<0, 0, 0, 1, unsigned int>",
                "ingest_sort0": "fused::k_ingest_sort0<0, unsigned int>", "ingest": "ingest::k_count_fused<1, 0>"}
TRAFFIC_JSON = os.path.join(ROOT, "profiles", "traffic_r02.json")


def ncu_path_bytes(workload, n):
    """DRAM bytes of one whole igd_detect (every kernel) from the committed ncu launch list of this
    workload at this size (profiles/summarize_launches.py --detects), or None."""
    try:
        d = json.load(open(TRAFFIC_JSON)).get(f"{workload}@{n}", {})
    except (OSError, ValueError):
        return None
    return d.get("__dram_per_detect__")


def ncu_traffic(workload, n, kclass):
    """DRAM bytes per launch of the dominant kernel from the committed ncu launch list of this
    workload at this size (profiles/traffic_r01.json, written by profiles/summarize_launches.py
    from an `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum` run of this bench)."""
    k = CLASS_KERNEL.get(kclass)
    try:
        d = json.load(open(TRAFFIC_JSON)).get(f"{workload}@{n}", {})
    except (OSError, ValueError):
        return None, None
    if k in d:
        return d[k], f"ncu dram__bytes_read.sum + dram__bytes_write.sum, {os.path.basename(TRAFFIC_JSON)}"
    return None, None


def main():
    _claim_stdout()
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="igd", choices=["igd", "reference"])
    ap.add_argument("--events", type=int, default=0, help="override the trace length (testing)")
    ap.add_argument("--oracle-events", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the host-buffer run (profiling)")
    ap.add_argument("--threads", type=int, default=0, help="generator threads (0 = all cores)")
    ap.add_argument("--sharded", action="store_true", help="use the multi-GPU path even at N=1")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"], help="N>1 collectives")
    ap.add_argument("--paper-counters", action="store_true",
                    help="Fig. 4-width synchronization IDs (IGD_DETECT_PAPER_COUNTERS, reading A33)")
    ap.add_argument("--stream-chunks", type=int, default=0,
                    help="f4: time streaming sessions of this many chunks instead of igd_detect (1 GPU)")
    ap.add_argument("--sync-heavy", action="store_true",
                    help="C2 / C5 sync-heavy variant (spin-lock sections ~8 %%, fences ~5 %%; SURVEY 8(d))")
    ap.add_argument("--coalesce", action="store_true",
                    help="warp-coalesced check mode (IGD_DETECT_COALESCE, reading A32; 1 GPU)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    fam = CONFIGS[args.config]

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, fam, rank, world)
    if args.coalesce and (world > 1 or args.sharded):
        raise SystemExit("--coalesce is a single-context mode (reading A32)")
    if args.stream_chunks:
        return run_stream(args, fam)
    if world > 1 or args.sharded:
        return run_sharded(args, fam, rank, world, local)

    import torch
    import torch.distributed as dist

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import tracegen.families as F
    import paper_conf_sosp_kamathb21_b200 as igd

    # ---------------- workload ----------------
    t0 = time.time()
    plan = F.Plan(fam, args.events or None, **gen_kw(args))
    n, nb, bd = plan.n_events, plan.n_blocks, plan.block_dim
    host = np.empty(n, igd.EVENT_DTYPE)
    plan.fill(out=host, threads=args.threads)
    lg = plan.ledger()
    ledger_n = len(lg)
    plan.close()
    log(f"[bench] {workload_name(args, fam)}: {n} events, {nb}x{bd} threads, generated in {time.time() - t0:.1f}s")
    cudart = torch.cuda.cudart()
    pinned = cudart.cudaHostRegister(host.ctypes.data, host.nbytes, 0) == 0
    dev = torch.empty(host.nbytes, dtype=torch.uint8, device="cuda")
    dev.copy_(torch.from_numpy(host.view(np.uint8)), non_blocking=False)
    torch.cuda.synchronize()

    det = igd.Detector(local)
    stream = det.stream
    det.load(dev, nb, bd)
    co = args.coalesce
    pc = args.paper_counters
    for _ in range(args.warmup):
        nrep = det.detect(coalesce=co, paper_counters=pc)
    # ---------------- timed region (device-resident trace) ----------------
    clocks = ClockSampler(local)
    clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    launches = 0
    e0.record(stream)
    for _ in range(args.steps):  # uninstrumented: no per-kernel events inside the timed region
        nrep = det.detect(coalesce=co, paper_counters=pc)
        launches += det.launch_count()
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1) / args.steps
    if world > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    value = n * world / (ms / 1e3) / 1e9
    reports = det.reports()
    # per-kernel breakdown (CUDA events on the context stream around every launch) and stage times
    # from as many instrumented steps after the timed region
    kstats = {}
    for _ in range(args.steps):
        det.detect(timing=True, coalesce=co, paper_counters=pc)
        for k, (cnt, ms_, b) in det.kernel_stats().items():
            c0, m0, b0 = kstats.get(k, (0, 0.0, 0.0))
            kstats[k] = (c0 + cnt, m0 + ms_, b0 + b)
    stages = det.stage_times()
    assert np.array_equal(det.reports(), reports), "instrumented and timed runs disagree"

    # ---------------- roofline of the dominant kernel class ----------------
    peak, peak_kind = peaks()
    dom = max(kstats, key=lambda k: kstats[k][1])
    cnt, kms, kbytes = kstats[dom]
    achieved = kbytes / (kms / 1e3) / 1e9 if kms > 0 else 0.0
    total_alg = sum(v[2] for v in kstats.values()) / args.steps
    path_gbs = total_alg / (ms / 1e3) / 1e9
    f_acc = None
    traffic, tsrc = ncu_traffic(workload_name(args, fam), n, dom)
    path_bytes = ncu_path_bytes(workload_name(args, fam), n)
    # achieved = SURVEY 8(d)'s algorithmic bytes per unit x the units one launch processes:
    # a radix pass reads and writes 8 B per access; the check reads 8 B and gathers one 32-B sector
    # per access; the ingest reads every 16-B event and writes an 8-B key per access.  The design's
    # own element bytes (12-B sort elements) are reported beside it.
    kinds_all = np.bincount(((host["tk"] >> 24) & 0xF).astype(np.int64), minlength=13)
    n_acc = int(kinds_all[:5].sum())
    survey_bytes = {"sort_access": 16.0 * n_acc, "check": 40.0 * n_acc, "ingest_sort0": 16.0 * n + 8.0 * n_acc,
                    "ingest": 16.0 * n}
    per_launch = survey_bytes.get(dom)
    s_achieved = per_launch / (kms / max(cnt, 1) / 1e3) / 1e9 if (per_launch and kms > 0) else achieved
    roofline = {"bound": "hbm", "kernel": dom, "achieved": s_achieved, "peak": peak, "unit": "GB/s",
                "frac": s_achieved / peak, "peak_source": peak_kind, "traffic": traffic, "traffic_source": tsrc,
                "alg_bytes_basis": "SURVEY 8(d) per-unit bytes" if per_launch else "design bytes",
                "alg_bytes_per_launch": per_launch if per_launch else kbytes / max(cnt, 1),
                "launches_per_step": cnt / args.steps, "ms_per_launch": kms / max(cnt, 1),
                "achieved_design_bytes": achieved, "frac_design_bytes": achieved / peak,
                "design_bytes_per_launch": kbytes / max(cnt, 1)}
    breakdown = {k: {"launches": v[0] // args.steps, "ms": v[1] / args.steps,
                     "alg_GBps": (v[2] / (v[1] / 1e3) / 1e9) if v[1] > 0 else None}
                 for k, v in kstats.items() if v[0]}

    # ---------------- end to end through the C ABI with host buffers ----------------
    del dev
    det.load(np.zeros(0, igd.EVENT_DTYPE), nb, bd)  # drop the borrowed pointer
    torch.cuda.empty_cache()
    e2e_times = []
    h2d = host.nbytes
    d2h = 0
    nr, out = nrep, reports
    for s in range(0 if args.no_e2e else args.e2e_steps + 1):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        det.load(host, nb, bd)           # H2D copy of the trace inside the library
        nr = det.detect(coalesce=co, paper_counters=pc)
        out = det.reports()              # D2H of the reports
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        d2h = out.nbytes + 8
        if s > 0:                        # first pass allocates the owned trace buffer
            e2e_times.append(dt)
    e2e_s = sum(e2e_times) / len(e2e_times) if e2e_times else float("inf")
    if world > 1:
        t = torch.tensor([e2e_s], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e = {"value": n * world / e2e_s / 1e9, "unit": "G events/s", "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": d2h, "ms_per_step": e2e_s * 1e3, "pinned_host": bool(pinned)}
    assert nr == nrep and np.array_equal(out, reports), "e2e and device-resident runs disagree"
    det.close()

    # ---------------- CPU oracle baseline (rank 0, N=1) ----------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        sn, sdt = oracle_baseline(host, nb, bd, coalesce=co, paper_counters=pc)
        cpu = {"value": sn / sdt / 1e9, "unit": "G events/s", "cores": 1, "kind": "oracle",
               "sample": f"first {sn} events of {workload_name(args, fam)} (best of up to 3 runs, {sdt:.1f}s, "
                         f"single-threaded C oracle pinned to one core; the --impl reference sample)", "host": host_info()}
    if pinned:
        cudart.cudaHostUnregister(host.ctypes.data)

    # full-size parity against the generator's injection ledger, element by element on
    # (addr, cur, prev, type): the whole report array, not just its length
    ledger_match = None
    if not (co or pc):
        ledger_match = bool(len(lg) == len(reports)
                            and np.array_equal(lg["addr"], reports["addr"]) and np.array_equal(lg["cur"], reports["cur"])
                            and np.array_equal(lg["prev"], reports["prev"])
                            and np.array_equal(lg["type"].astype(np.uint8), reports["type"]))
    kinds = np.bincount(((host["tk"] >> 24) & 0xF).astype(np.int64), minlength=12)
    f_acc = float(kinds[:5].sum()) / max(n, 1)
    b_alg = 16 + 32 * f_acc  # read the event + read/write a 16-B metadata entry per access
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "G events/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": {"workload": workload_name(args, fam), "events": n, "n_blocks": nb, "block_dim": bd,
                           "f_acc": f_acc, "reports": int(nrep),
                           "ledger_reports": None if (co or pc) else ledger_n,  # ledger: per-lane, exact IDs
                           "ledger_match": ledger_match,
                           "check_mode": ("warp-coalesced (A32)" if co else "per-lane")
                           + (", paper-width IDs (A33)" if pc else ""),
                           "l2": "inputs larger than L2 (no flush)",
                           "parallelism": f"{world} GPU(s), one process per GPU"},
                "roofline": roofline,
                "path": {"alg_bytes_per_event_B_alg": b_alg, "alg_GBps_B_alg": value * b_alg,
                         "frac_B_alg": value * b_alg / peak, "kernel_alg_GBps": path_gbs,
                         # SURVEY 8(d) fraction 1 (north_star's gate): ncu DRAM bytes of a whole detect
                         # (committed launch list) over this run's step time
                         "ncu_dram_bytes_per_step": path_bytes,
                         "achieved_dram_GBps": (path_bytes / (ms / 1e3) / 1e9) if path_bytes else None,
                         "achieved_dram_frac": (path_bytes / (ms / 1e3) / 1e9 / peak) if path_bytes else None,
                         "stages_ms": stages, "kernels": breakdown},
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clk}
        emit(line)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
