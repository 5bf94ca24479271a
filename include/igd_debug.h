/*
 * igd_debug.h -- stage-level test and micro-benchmark hooks of libigd (not part of the
 * product API of igd.h; used by tests/test_gpu_stages.py and profiling runs).
 */
#ifndef IGD_DEBUG_H
#define IGD_DEBUG_H
#include "igd.h"
#ifdef __cplusplus
extern "C" {
#endif

/* Stable LSD radix sort (the a5 kernel) of n (key, value) u32 pairs held in DEVICE memory,
   in place, over the low max_bits key bits.  mode: ignored (one multisplit policy, rows ranked
   alternately by ballots and match.any; kept for ABI stability).
   *ms = device time of the sort passes (CUDA events on the context stream). */
int igd_debug_radix_sort(igd_ctx* ctx, uint32_t* d_keys, uint32_t* d_vals, uint64_t n, uint32_t max_bits, int mode,
                         float* ms);

/* Memory-floor probe of the check's streaming phase on the last igd_detect's sorted accesses:
   stream keys + indices, and (gather != 0) gather every access's 16-byte event. */
int igd_debug_gather_probe(igd_ctx* ctx, int gather, float* ms);

/* Check-kernel event counters: returns the counters accumulated since the last call in out16
   (may be NULL), resets them, and enables (1) or disables (0) counting for later igd_detect
   calls.  Slot meaning: see check.cuh (CSTAT). */
int igd_debug_check_stats(igd_ctx* ctx, int enable, uint64_t* out16);

#ifdef __cplusplus
}
#endif
#endif
