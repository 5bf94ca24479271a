"""B200-native deterministic race check of iGUARD (SOSP'21) traces.

The product is the C-ABI library ``libigd.so`` (include/igd.h, kernels in ``csrc/``);
:mod:`.igd` is a thin ctypes binding with the same names.  There is no CPU fallback:
every step of the check runs in the CUDA kernels, and loading fails loudly when the
library or a GPU is missing.
"""
from .igd import (EVENT_DTYPE, REPORT_DTYPE, Detector, IgdError, igd_ctx_create, igd_ctx_destroy,  # noqa: F401
                  igd_detect, igd_nccl_unique_id, igd_reports, igd_strerror, igd_trace_load, lib_path,
                  load_library)
