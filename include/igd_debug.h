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

/* a2 / a3 tables of the last igd_detect (single GPU).  sizes[0..3] = entities E, sync records,
   threads T, lock change points; then (any pointer may be NULL) off[E+1] = CSR offsets of the
   entity-sorted sync timestamps ts[n_sync] (entity layout: csrc/common.cuh KeySpace), and when
   the trace has lock events toff[T+1] / tpts[n_points] = per-thread change points
   (timestamp << 16 | held-lock Bloom). */
int igd_debug_sync_tables(igd_ctx* ctx, uint64_t* sizes, uint32_t* off, uint32_t* ts, uint32_t* toff,
                          uint64_t* tpts);

/* a6 scan state of the last igd_detect run with IGD_DETECT_LAST_K (n = its accesses): per sorted
   access the packed state before it (check.cuh st_make: [31:0] last-writer position, [33:32]
   scope of the last atomic, [34] DevShared, [35] BlkShared, inclusive; [36] = segment head),
   the sorted u32 keys and u64 payloads (trace index | tk << 32). */
int igd_debug_scan_state(igd_ctx* ctx, uint64_t n, uint64_t* state, uint32_t* keys, uint64_t* payload);

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
