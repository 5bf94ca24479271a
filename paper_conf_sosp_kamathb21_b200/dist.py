"""Multi-GPU sharded race check -- host orchestration over torch.distributed.

Rank r holds the contiguous global range [first_r, first_r + n_r) of the trace.  Words are
hash-sharded, owner(word) = fmix32(low 32 bits of word) % P, so each word's whole history lands
on one rank.  One check:

  1. ``igd_shard_prepare`` (GPU): validate, partition the chunk's access records by owner (each
     group in trace order) and extract its synchronization stream;
  2. collectives (NCCL on GPUs, gloo in the CPU tests): min-reduce of the first invalid event,
     min/max-reduce of the accessed word range, all-to-all of the record groups, all-gather of the
     synchronization streams in rank order (= trace order);
  3. ``igd_shard_detect`` (GPU): every rank rebuilds identical sync-epoch / lock tables from the
     global stream and checks the words it owns;
  4. all-gather of the reports, merged by ``cur``.  The union is the single-GPU report set (the
     address-shard invariance of SURVEY 8(c) C.7 5(b), tested against the oracle).

The exchange helpers are backend-agnostic; ``LoopbackComm`` runs P logical ranks in one process
(single-GPU tests of the partition / exchange / merge path).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch
import torch.distributed as dist

from . import igd as _igd

NONE64 = (1 << 64) - 1
RECORD_INTS = 4   # uint4 {key, global index, tk, mask}
EVENT_INTS = 4    # 16-byte event


def fmix32(x: np.ndarray) -> np.ndarray:
    """murmur3 finalizer on uint32 (the owner hash of include/igd.h)."""
    h = np.asarray(x, dtype=np.uint64) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(16)
    h = (h * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(13)
    h = (h * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
    h ^= h >> np.uint64(16)
    return h


def owner_of(words: np.ndarray, nranks: int) -> np.ndarray:
    return (fmix32(np.asarray(words, np.uint64) & np.uint64(0xFFFFFFFF)) % np.uint64(nranks)).astype(np.int64)


def chunk_bounds(n_total: int, nranks: int, rank: int):
    """Contiguous timestamp range of a rank: [r*N/P, (r+1)*N/P)."""
    lo = n_total * rank // nranks
    hi = n_total * (rank + 1) // nranks
    return lo, hi - lo


def merge_reports(parts) -> np.ndarray:
    """Union of per-rank report arrays in canonical order (ascending cur; cur is unique)."""
    parts = [p.cpu().numpy().reshape(-1).view(_igd.REPORT_DTYPE) if isinstance(p, torch.Tensor) else p
             for p in parts]
    parts = [p for p in parts if len(p)]
    if not parts:
        return np.zeros(0, _igd.REPORT_DTYPE)
    allr = np.concatenate(parts)
    return allr[np.argsort(allr["cur"], kind="stable")]


# ---- communication ------------------------------------------------------------------------------
class TorchComm:
    """Collectives over a torch.distributed process group: NCCL on GPUs (device tensors move over
    NVLink / NVSwitch); with gloo, device tensors are staged through host memory."""

    def __init__(self, group=None):
        self.group = group
        self.rank = dist.get_rank(group)
        self.size = dist.get_world_size(group)
        self.host_staged = dist.get_backend(group) == "gloo"

    def _in(self, t: torch.Tensor) -> torch.Tensor:
        return t.cpu() if self.host_staged else t

    def allreduce_u64(self, value: int, op: str, device) -> int:
        """min / max of a non-negative int over ranks; "min_none" treats NONE64 as absent."""
        if op == "min_none":
            v = (1 << 62) if value == NONE64 else int(value)
            t = self._in(torch.tensor([v], dtype=torch.int64, device=device))
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=self.group)
            r = int(t.item())
            return NONE64 if r == (1 << 62) else r
        t = self._in(torch.tensor([int(value)], dtype=torch.int64, device=device))
        dist.all_reduce(t, op=dist.ReduceOp.MIN if op == "min" else dist.ReduceOp.MAX, group=self.group)
        return int(t.item())

    def all_to_all_var(self, send: torch.Tensor, counts) -> torch.Tensor:
        """Rows of `send` grouped by destination rank (counts[d] rows for rank d) -> rows received
        from every rank, concatenated in source-rank order."""
        dev = send.device
        send = self._in(send)
        cnt = torch.tensor([int(c) for c in counts], dtype=torch.int64, device=send.device)
        rcnt = torch.empty_like(cnt)
        dist.all_to_all_single(rcnt, cnt, group=self.group)
        rc = [int(x) for x in rcnt.tolist()]
        recv = torch.empty((sum(rc),) + tuple(send.shape[1:]), dtype=send.dtype, device=send.device)
        dist.all_to_all_single(recv, send, output_split_sizes=rc, input_split_sizes=[int(c) for c in counts],
                               group=self.group)
        return recv.to(dev)

    def all_gather_var(self, t: torch.Tensor) -> torch.Tensor:
        """Concatenation over ranks (rank order) of variable-length tensors."""
        dev = t.device
        t = self._in(t)
        n = torch.tensor([t.shape[0]], dtype=torch.int64, device=t.device)
        ns = [torch.empty_like(n) for _ in range(self.size)]
        dist.all_gather(ns, n, group=self.group)
        sizes = [int(x.item()) for x in ns]
        m = max(sizes) if sizes else 0
        pad = torch.zeros((m,) + tuple(t.shape[1:]), dtype=t.dtype, device=t.device)
        pad[: t.shape[0]] = t
        outs = [torch.empty_like(pad) for _ in range(self.size)]
        dist.all_gather(outs, pad, group=self.group)
        return torch.cat([o[:s] for o, s in zip(outs, sizes)]).to(dev)


# ---- device stage (libigd) ----------------------------------------------------------------------
class _CudaArray:
    def __init__(self, ptr, shape, typestr="<i4"):
        self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3}


def _wrap(ptr, rows, cols, device):
    if rows == 0 or not ptr:
        return torch.zeros((0, cols), dtype=torch.int32, device=device)
    return torch.as_tensor(_CudaArray(ptr, (rows, cols)), device=device)


class GpuStage:
    """One rank's libigd context (stage 1 and stage 2 of the sharded check)."""

    def __init__(self, det: "_igd.Detector"):
        self.det = det
        self.device = torch.device("cuda", det.device)

    def _order(self):
        """libigd runs on the Detector's stream: make it wait for the work the caller queued on
        the current torch stream (e.g. the NCCL exchange that fills recv / sync buffers)."""
        if self.device.type == "cuda":
            self.det.stream.wait_stream(torch.cuda.current_stream(self.device))

    def load(self, chunk, first_event: int, n_total: int, n_blocks: int, block_dim: int):
        lib = _igd.load_library()
        self._order()
        if isinstance(chunk, torch.Tensor):
            n = chunk.numel() * chunk.element_size() // 16
            ptr, flags = (chunk.data_ptr() if n else 0), _igd.IGD_TRACE_DEVICE_PTR
            self._borrow = chunk
        else:
            ev = np.ascontiguousarray(chunk)
            n = len(ev)
            ptr, flags = (ev.ctypes.data if n else 0), 0
            self._borrow = None
        d = _igd.igd_trace_desc(n_blocks, block_dim, n_total, first_event, n, flags)
        rc = lib.igd_trace_load(self.det.ctx, ctypes.byref(d), ctypes.c_void_p(ptr or None))
        if rc != _igd.IGD_OK:
            raise _igd.IgdError(rc, lib.igd_last_error(self.det.ctx).decode())

    def prepare(self, nranks: int):
        lib = _igd.load_library()
        self._order()
        counts = (ctypes.c_uint64 * nranks)()
        nsync, bad = ctypes.c_uint64(), ctypes.c_uint64()
        mm = (ctypes.c_uint64 * 2)()
        rc = lib.igd_shard_prepare(self.det.ctx, nranks, counts, ctypes.byref(nsync), ctypes.byref(bad), mm)
        if rc != _igd.IGD_OK:
            raise _igd.IgdError(rc, lib.igd_last_error(self.det.ctx).decode())
        rec, sidx, sev = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
        lib.igd_shard_buffers(self.det.ctx, ctypes.byref(rec), ctypes.byref(sidx), ctypes.byref(sev))
        nrec = int(sum(counts))
        return {"records": _wrap(rec.value, nrec, RECORD_INTS, self.device), "counts": [int(c) for c in counts],
                "sync_idx": _wrap(sidx.value, nsync.value, 1, self.device).reshape(-1),
                "sync_ev": _wrap(sev.value, nsync.value, EVENT_INTS, self.device),
                "bad": int(bad.value), "min_word": int(mm[0]), "max_word": int(mm[1])}

    def detect(self, recv, sync_idx, sync_ev, min_word: int, timing: bool = False,
               paper_counters: bool = False) -> np.ndarray:
        lib = _igd.load_library()
        recv = recv.contiguous()
        self._order()
        sync_idx = sync_idx.contiguous()
        sync_ev = sync_ev.contiguous()
        nrep = ctypes.c_uint64()
        rc = lib.igd_shard_detect(self.det.ctx, ctypes.c_void_p(recv.data_ptr() if recv.numel() else None),
                                  recv.shape[0], ctypes.c_void_p(sync_idx.data_ptr() if sync_idx.numel() else None),
                                  ctypes.c_void_p(sync_ev.data_ptr() if sync_ev.numel() else None), sync_idx.shape[0],
                                  min_word, (_igd.IGD_DETECT_TIMING if timing else 0)
                                  | (_igd.IGD_DETECT_PAPER_COUNTERS if paper_counters else 0), ctypes.byref(nrep))
        if rc != _igd.IGD_OK:
            raise _igd.IgdError(rc, lib.igd_last_error(self.det.ctx).decode())
        self.det.n_reports = n = int(nrep.value)
        if n == 0:
            return torch.zeros((0, 32), dtype=torch.uint8, device=self.device)
        ptr, cnt = ctypes.c_void_p(), ctypes.c_uint64()
        lib.igd_reports_device(self.det.ctx, ctypes.byref(ptr), ctypes.byref(cnt))
        # device copy of the context-owned reports ([n, 32] bytes, ascending cur)
        return torch.as_tensor(_CudaArray(ptr.value, (n, 32), "|u1"), device=self.device).clone()


# ---- orchestration --------------------------------------------------------------------------------
def _check_prepared(bad: int, lo: int, hi: int, any_access: bool):
    if bad != NONE64:
        raise _igd.IgdError(_igd.IGD_ETRACE, f"invalid event at global index {bad}", bad)
    if any_access and hi - lo >= (1 << 32):
        raise _igd.IgdError(_igd.IGD_ETOOBIG, "accessed word range spans >= 2^32 words")


def sharded_detect(stage, comm: TorchComm, timing: bool = False, paper_counters: bool = False) -> np.ndarray:
    """One rank's part of the distributed check (the chunk is already loaded in `stage`).
    Returns the global report set (identical on every rank)."""
    prep = stage.prepare(comm.size)
    dev = prep["records"].device
    bad = comm.allreduce_u64(prep["bad"], "min_none", dev)
    has = prep["min_word"] != NONE64
    lo = comm.allreduce_u64(prep["min_word"] if has else (1 << 62), "min", dev)
    hi = comm.allreduce_u64(prep["max_word"] if has else 0, "max", dev)
    _check_prepared(bad, lo, hi, lo != (1 << 62))
    recv = comm.all_to_all_var(prep["records"], prep["counts"])
    sidx = comm.all_gather_var(prep["sync_idx"].reshape(-1, 1)).reshape(-1)
    sev = comm.all_gather_var(prep["sync_ev"])
    local = stage.detect(recv, sidx, sev, lo if lo != (1 << 62) else 0, timing, paper_counters)
    if isinstance(local, np.ndarray):
        local = torch.from_numpy(local.view(np.uint8).reshape(-1, 32).copy()).to(dev)
    everything = comm.all_gather_var(local)           # [n, 32] bytes, rank order
    if everything.shape[0] > 1:                       # merge by cur on the device (cur is unique)
        cur = everything.view(torch.int64)[:, 1]
        everything = everything[torch.argsort(cur)]
    return everything.cpu().numpy().reshape(-1).view(_igd.REPORT_DTYPE)


class LoopbackComm:
    """P logical ranks in one process: the same exchange semantics as TorchComm, evaluated for all
    ranks at once (single-GPU tests of the sharded path)."""

    @staticmethod
    def run(stages, timing: bool = False, paper_counters: bool = False) -> np.ndarray:
        P = len(stages)
        preps = [s.prepare(P) for s in stages]
        bad = min((p["bad"] for p in preps), default=NONE64)
        has = [p for p in preps if p["min_word"] != NONE64]
        lo = min((p["min_word"] for p in has), default=0)
        hi = max((p["max_word"] for p in has), default=0)
        _check_prepared(bad, lo, hi, bool(has))
        offs = [np.concatenate([[0], np.cumsum(p["counts"])]) for p in preps]
        sidx = torch.cat([p["sync_idx"] for p in preps])
        sev = torch.cat([p["sync_ev"] for p in preps])
        # all exchanges first: a stage's detect releases its send buffer
        recvs = [torch.cat([p["records"][int(o[d]):int(o[d + 1])] for p, o in zip(preps, offs)])
                 for d in range(P)]
        parts = [s.detect(recv, sidx, sev, lo, timing, paper_counters) for s, recv in zip(stages, recvs)]
        return merge_reports(parts)
