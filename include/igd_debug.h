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
   in place, over the low max_bits key bits.  mode: 1 = ballot multisplit, 0 = match.any.
   *ms = device time of the sort passes (CUDA events on the context stream). */
int igd_debug_radix_sort(igd_ctx* ctx, uint32_t* d_keys, uint32_t* d_vals, uint64_t n, uint32_t max_bits, int mode,
                         float* ms);

#ifdef __cplusplus
}
#endif
#endif
