"""ctypes binding of libigd (include/igd.h): argument marshalling only.

Functions keep the C names (``igd_ctx_create``, ``igd_trace_load``, ``igd_detect``,
``igd_reports``, ``igd_ctx_destroy``, ``igd_strerror``).  :class:`Detector` wires them to
PyTorch for device memory (caching-allocator callbacks) and the current CUDA stream.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

EVENT_DTYPE = np.dtype([("addr", "<u8"), ("tk", "<u4"), ("mask", "<u4")])
REPORT_DTYPE = np.dtype([("addr", "<u8"), ("cur", "<u8"), ("prev", "<u8"), ("type", "u1"),
                         ("cur_kind", "u1"), ("prev_kind", "u1"), ("pad", "u1", (5,))])
IGD_OK, IGD_EINVAL, IGD_ETRACE, IGD_ETOOBIG, IGD_ENOMEM, IGD_ECUDA, IGD_ENCCL, IGD_ESTATE = 0, -1, -2, -3, -4, -5, -6, -7
IGD_TRACE_DEVICE_PTR = 1
IGD_DETECT_TIMING = 1
IGD_DETECT_COALESCE = 2
IGD_DETECT_PAPER_COUNTERS = 4
IGD_DETECT_STICKY_FLAGS = 8
IGD_DETECT_TAG_SHIFT = 8
IGD_DETECT_LAST_K_SHIFT = 16
IGD_N_STAGES = 8
IGD_N_KCLASS = 9


class igd_trace_desc(ctypes.Structure):
    _fields_ = [("n_blocks", ctypes.c_uint32), ("block_dim", ctypes.c_uint32),
                ("n_events_total", ctypes.c_uint64), ("first_event", ctypes.c_uint64),
                ("n_events", ctypes.c_uint64), ("flags", ctypes.c_uint32)]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)

_lib = None


def lib_path() -> str:
    return _build.LIB


def load_library(build_if_missing: bool = True):
    """Load libigd.so (building it with nvcc first if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("IGD_LIB", _build.LIB)  # tuning variants (profiles/) only
    if path == _build.LIB and build_if_missing and _build.needs_build():
        _build.build()
    if not os.path.exists(path):
        raise ImportError(f"libigd.so not built at {path}")
    lib = ctypes.CDLL(path)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    lib.igd_ctx_create.argtypes = [ctypes.POINTER(vp), i32, vp, i32, i32, vp, ALLOC_FN, FREE_FN, vp]
    lib.igd_ctx_create.restype = i32
    lib.igd_trace_load.argtypes = [vp, ctypes.POINTER(igd_trace_desc), vp]
    lib.igd_trace_load.restype = i32
    lib.igd_detect.argtypes = [vp, u32, ctypes.POINTER(u64)]
    lib.igd_detect.restype = i32
    lib.igd_reports.argtypes = [vp, vp, u64, ctypes.POINTER(u64)]
    lib.igd_reports.restype = i32
    lib.igd_reports_device.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(u64)]
    lib.igd_reports_device.restype = i32
    lib.igd_bad_event.argtypes = [vp]
    lib.igd_bad_event.restype = u64
    lib.igd_stage_times.argtypes = [vp, ctypes.POINTER(ctypes.c_float)]
    lib.igd_stage_times.restype = i32
    lib.igd_stage_name.argtypes = [i32]
    lib.igd_stage_name.restype = ctypes.c_char_p
    lib.igd_last_launch_count.argtypes = [vp]
    lib.igd_last_launch_count.restype = u64
    lib.igd_kernel_stats.argtypes = [vp, i32, ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(u32),
                                     ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_double)]
    lib.igd_kernel_stats.restype = i32
    lib.igd_shard_prepare.argtypes = [vp, u32, ctypes.POINTER(u64), ctypes.POINTER(u64), ctypes.POINTER(u64),
                                      ctypes.POINTER(u64)]
    lib.igd_shard_prepare.restype = i32
    lib.igd_shard_buffers.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp)]
    lib.igd_shard_buffers.restype = i32
    lib.igd_shard_detect.argtypes = [vp, vp, u64, vp, vp, u64, u64, u32, ctypes.POINTER(u64)]
    lib.igd_shard_detect.restype = i32
    lib.igd_stream_begin.argtypes = [vp, u32, u32]
    lib.igd_stream_begin.restype = i32
    lib.igd_stream_feed.argtypes = [vp, vp, u64, u32, u32, ctypes.POINTER(u64)]
    lib.igd_stream_feed.restype = i32
    lib.igd_stream_end.argtypes = [vp]
    lib.igd_stream_end.restype = i32
    lib.igd_nccl_unique_id.argtypes = [vp]
    lib.igd_nccl_unique_id.restype = i32
    lib.igd_ctx_destroy.argtypes = [vp]
    lib.igd_ctx_destroy.restype = None
    lib.igd_strerror.argtypes = [i32]
    lib.igd_strerror.restype = ctypes.c_char_p
    lib.igd_last_error.argtypes = [vp]
    lib.igd_last_error.restype = ctypes.c_char_p
    _lib = lib
    return lib


class IgdError(RuntimeError):
    def __init__(self, code: int, msg: str = "", bad_index=None):
        super().__init__(f"igd error {code} ({igd_strerror(code)}): {msg}")
        self.code = code
        self.bad_index = bad_index


# ---- thin same-name wrappers ---------------------------------------------------------------
def igd_strerror(code: int) -> str:
    return load_library().igd_strerror(code).decode()


def igd_nccl_unique_id() -> bytes:
    """A fresh 128-byte NCCL unique id (rank 0 creates it, the caller shares it with the others)."""
    _prefer_torch_nccl()
    buf = (ctypes.c_uint8 * 128)()
    rc = load_library().igd_nccl_unique_id(buf)
    if rc != IGD_OK:
        raise IgdError(rc, "igd_nccl_unique_id")
    return bytes(buf)


def _prefer_torch_nccl():
    """libigd resolves libnccl.so.2 at run time and reuses a copy already in the process: load
    torch first so its NCCL (the one torch.distributed uses) is that copy."""
    try:
        import torch  # noqa: F401
    except ImportError:
        pass


def igd_ctx_create(cuda_device: int, cuda_stream: int, alloc_fn=None, free_fn=None, nranks: int = 1,
                   rank: int = 0, nccl_id: bytes = None):
    lib = load_library()
    ctx = ctypes.c_void_p()
    idbuf = None
    if nccl_id is not None:
        _prefer_torch_nccl()
        assert len(nccl_id) == 128
        idbuf = (ctypes.c_uint8 * 128).from_buffer_copy(nccl_id)
    rc = lib.igd_ctx_create(ctypes.byref(ctx), cuda_device, ctypes.c_void_p(cuda_stream), nranks, rank,
                            ctypes.cast(idbuf, ctypes.c_void_p) if idbuf is not None else None,
                            alloc_fn or ALLOC_FN(), free_fn or FREE_FN(), None)
    if rc != IGD_OK:
        raise IgdError(rc, "igd_ctx_create")
    return ctx


def igd_trace_load(ctx, n_blocks: int, block_dim: int, events_ptr: int, n_events: int, device_ptr: bool,
                   first_event: int = 0, n_events_total: int = None):
    lib = load_library()
    d = igd_trace_desc(n_blocks, block_dim, n_events if n_events_total is None else n_events_total, first_event,
                       n_events, IGD_TRACE_DEVICE_PTR if device_ptr else 0)
    rc = lib.igd_trace_load(ctx, ctypes.byref(d), ctypes.c_void_p(events_ptr or None))
    if rc != IGD_OK:
        raise IgdError(rc, lib.igd_last_error(ctx).decode())


def igd_detect(ctx, flags: int = 0) -> int:
    lib = load_library()
    n = ctypes.c_uint64(0)
    rc = lib.igd_detect(ctx, flags, ctypes.byref(n))
    if rc != IGD_OK:
        bad = lib.igd_bad_event(ctx) if rc == IGD_ETRACE else None
        raise IgdError(rc, lib.igd_last_error(ctx).decode(), bad)
    return int(n.value)


def igd_reports(ctx, cap: int) -> np.ndarray:
    lib = load_library()
    out = np.zeros(cap, REPORT_DTYPE)
    n = ctypes.c_uint64(0)
    rc = lib.igd_reports(ctx, out.ctypes.data if cap else None, cap, ctypes.byref(n))
    if rc != IGD_OK:
        raise IgdError(rc, lib.igd_last_error(ctx).decode())
    return out[: n.value]


def igd_ctx_destroy(ctx) -> None:
    load_library().igd_ctx_destroy(ctx)


# ---- torch plumbing ------------------------------------------------------------------------
class Detector:
    """One libigd context on a CUDA device, using torch's caching allocator and stream.

    ``load`` accepts a host numpy EVENT_DTYPE array (copied by the library) or a CUDA
    tensor of the same bytes (borrowed: kept alive here until the next load)."""

    def __init__(self, device: int = 0, stream=None, nranks: int = 1, rank: int = 0, nccl_id: bytes = None):
        """``nranks`` / ``rank`` / ``nccl_id``: a collective context (one process per GPU, the same
        id on every rank; igd_nccl_unique_id on one of them) -- detect() is then collective and
        returns the global report set on every rank.  nranks == 1 with an id: the collective path
        on one GPU."""
        import torch

        if not torch.cuda.is_available():
            raise RuntimeError("libigd needs a CUDA device; there is no CPU fallback")
        self._torch = torch
        self.device = device
        self.stream = stream if stream is not None else torch.cuda.current_stream(device)
        dev = device

        def _alloc(nbytes, stream, user):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), dev, stream or 0)
            except Exception:  # noqa: BLE001 -- reported to the library as NULL (IGD_ENOMEM)
                return None

        cdelete = torch.cuda.caching_allocator_delete  # bound now: survives interpreter teardown

        def _free(p, stream, user):
            try:
                cdelete(p)
            except Exception:  # noqa: BLE001 -- process exit: the driver reclaims the memory
                pass

        self._afn = ALLOC_FN(_alloc)
        self._ffn = FREE_FN(_free)
        self.nranks, self.rank = nranks, rank
        self.ctx = igd_ctx_create(device, self.stream.cuda_stream, self._afn, self._ffn, nranks, rank, nccl_id)
        self._borrowed = None
        self.n_reports = 0

    def load(self, events, n_blocks: int, block_dim: int, first_event: int = 0, n_events_total: int = None):
        """Attach a trace (or, on a collective context, this rank's chunk starting at global index
        ``first_event`` of an ``n_events_total``-event trace)."""
        torch = self._torch
        if isinstance(events, torch.Tensor):
            assert events.is_cuda and events.is_contiguous() and events.numel() * events.element_size() % 16 == 0
            assert events.data_ptr() % 16 == 0, "device events must be 16-byte aligned"
            n = events.numel() * events.element_size() // 16
            self._borrowed = events
            igd_trace_load(self.ctx, n_blocks, block_dim, events.data_ptr() if n else 0, n, True, first_event,
                           n_events_total)
        else:
            ev = np.ascontiguousarray(events)
            assert ev.dtype.itemsize == 16
            self._borrowed = None
            igd_trace_load(self.ctx, n_blocks, block_dim, ev.ctypes.data if len(ev) else 0, len(ev), False,
                           first_event, n_events_total)

    def detect(self, timing: bool = False, coalesce: bool = False, paper_counters: bool = False,
               sticky_flags: bool = False, tag_log2: int = 0, last_k: int = 1) -> int:
        """igd_detect; ``coalesce``: warp-coalesced check mode (IGD_DETECT_COALESCE, reading A32);
        ``paper_counters``: Fig. 4-width synchronization IDs (IGD_DETECT_PAPER_COUNTERS, A33);
        ``sticky_flags``: Table 2's sticky sharing flags in P3-P5 (IGD_DETECT_STICKY_FLAGS, A35);
        ``tag_log2``: a 2^tag_log2-entry metadata table with 10-bit Tags (IGD_DETECT_TAG_LOG2, A36);
        ``last_k``: the last k writers / accessors are checked (IGD_DETECT_LAST_K, A37)."""
        flags = ((IGD_DETECT_TIMING if timing else 0) | (IGD_DETECT_COALESCE if coalesce else 0)
                 | (IGD_DETECT_PAPER_COUNTERS if paper_counters else 0)
                 | (IGD_DETECT_STICKY_FLAGS if sticky_flags else 0) | (int(tag_log2) << IGD_DETECT_TAG_SHIFT)
                 | ((int(last_k) if last_k > 1 else 0) << IGD_DETECT_LAST_K_SHIFT))
        self.n_reports = igd_detect(self.ctx, flags)
        return self.n_reports

    def reports(self) -> np.ndarray:
        return igd_reports(self.ctx, self.n_reports)

    # ---- streaming sessions (igd_stream_*) ----
    def stream_begin(self, n_blocks: int, block_dim: int):
        rc = load_library().igd_stream_begin(self.ctx, n_blocks, block_dim)
        if rc != IGD_OK:
            raise IgdError(rc, load_library().igd_last_error(self.ctx).decode())

    def stream_feed(self, events, paper_counters: bool = False, sticky_flags: bool = False,
                    timing: bool = False) -> np.ndarray:
        """Check the next chunk (host EVENT_DTYPE array or CUDA tensor); returns its reports."""
        lib = load_library()
        torch = self._torch
        if isinstance(events, torch.Tensor):
            assert events.is_cuda and events.is_contiguous() and events.data_ptr() % 16 == 0
            n = events.numel() * events.element_size() // 16
            ptr, fl, keep = events.data_ptr() if n else 0, IGD_TRACE_DEVICE_PTR, events
        else:
            keep = np.ascontiguousarray(events)
            n = len(keep)
            ptr, fl = keep.ctypes.data if n else 0, 0
        flags = ((IGD_DETECT_TIMING if timing else 0) | (IGD_DETECT_PAPER_COUNTERS if paper_counters else 0)
                 | (IGD_DETECT_STICKY_FLAGS if sticky_flags else 0))
        nr = ctypes.c_uint64(0)
        rc = lib.igd_stream_feed(self.ctx, ctypes.c_void_p(ptr or None), n, fl, flags, ctypes.byref(nr))
        del keep
        if rc != IGD_OK:
            bad = lib.igd_bad_event(self.ctx) if rc == IGD_ETRACE else None
            raise IgdError(rc, lib.igd_last_error(self.ctx).decode(), bad)
        self.n_reports = int(nr.value)
        return self.reports()

    def stream_end(self):
        load_library().igd_stream_end(self.ctx)

    def stage_times(self) -> dict:
        lib = load_library()
        arr = (ctypes.c_float * IGD_N_STAGES)()
        lib.igd_stage_times(self.ctx, arr)
        return {lib.igd_stage_name(i).decode(): float(arr[i]) for i in range(IGD_N_STAGES)}

    def kernel_stats(self) -> dict:
        """{class: (launches, ms, algorithmic bytes)} of the last detect(timing=True)."""
        lib = load_library()
        out = {}
        for k in range(IGD_N_KCLASS):
            nm, n, ms, b = ctypes.c_char_p(), ctypes.c_uint32(), ctypes.c_float(), ctypes.c_double()
            lib.igd_kernel_stats(self.ctx, k, ctypes.byref(nm), ctypes.byref(n), ctypes.byref(ms), ctypes.byref(b))
            out[nm.value.decode()] = (int(n.value), float(ms.value), float(b.value))
        return out

    def launch_count(self) -> int:
        return int(load_library().igd_last_launch_count(self.ctx))

    def close(self):
        if self.ctx is not None:
            igd_ctx_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def detect(events, n_blocks: int, block_dim: int, device: int = 0) -> np.ndarray:
    """One-shot convenience: load, detect, fetch reports (ascending ``cur``)."""
    with Detector(device) as d:
        d.load(events, n_blocks, block_dim)
        d.detect()
        return d.reports()
