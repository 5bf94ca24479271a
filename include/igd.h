/*
 * igd.h -- C ABI of libigd, the B200-native race check of iGUARD (Kamath & Basu, SOSP'21),
 * restated as deterministic replay of a fixed-order trace.  PAPER.md lines are cited P:<n>.
 *
 * The operation (§6.2-§6.4): for every load/store/atomic of a kernel, compare it
 * with the last writer (loads) or last accessor (stores/atomics) of the same 4-byte word
 * (P:1097-1099), skip it if one of the preliminary checks P1-P6 holds, and otherwise
 * report the first of the race conditions R1-R5 that holds (Table 2, P:1093-1151;
 * "checked in the order given in the table").  Synchronization metadata
 * comes from fences, __syncwarp, __syncthreads and grid syncs (Fig. 5); locks are
 * inferred from atomicCAS + fence / atomicExch (§6.3).  Cooperative-group syncs
 * are checked through their constituents.  Readings where the paper is
 * silent are listed in DESIGN.md ("Readings", A1-A30); they bind this library.
 *
 * All arithmetic is integer; results are a deterministic function of the trace.
 * No C++ types cross this ABI; every call returns an int status (IGD_OK = 0, < 0 = error)
 * except igd_ctx_destroy / igd_strerror.  Nothing throws.  One context per stream;
 * contexts are not thread-safe.
 */
#ifndef IGD_H
#define IGD_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes --------------------------------------------------------------- */
#define IGD_OK 0
#define IGD_EINVAL (-1)  /* bad argument or geometry (threads must be 1..2^24) */
#define IGD_ETRACE (-2)  /* an event violates the field rules below; see igd_bad_event() */
#define IGD_ETOOBIG (-3) /* n_events >= 2^32 - 8192 (32-bit trace indices), or -- sharded / collective
                            contexts only -- the accessed word range spans >= 2^32 words */
#define IGD_ENOMEM (-4)  /* device allocation failed */
#define IGD_ECUDA (-5)   /* a CUDA runtime call failed; see igd_last_error() */
#define IGD_ENCCL (-6)   /* an NCCL call failed, or libnccl.so.2 could not be loaded (multi-GPU) */
#define IGD_ESTATE (-7)  /* call out of order (e.g. igd_detect before igd_trace_load) */

/* ---- trace event: 16 bytes, little-endian, arrays 16-byte aligned ---------------- */
typedef struct {
    uint64_t addr; /* accesses: byte address, checked at the 4-byte word addr>>2;
                      synchronization events: 0 */
    uint32_t tk;   /* bits [0,24) tid = global linear thread id; [24,28) kind; [28,30) scope;
                      [30,32) must be 0 */
    uint32_t mask; /* active mask of the warp instruction the event belongs to (P4, P:1115-1119;
                      isThread inference); SYNCWARP: member lanes (ignored) */
} igd_event;

/* kind (tk bits 24..27) */
#define IGD_LD 0
#define IGD_ST 1
#define IGD_ATOM 2         /* any other atomic RMW / atomic load or store */
#define IGD_CAS 3          /* atomicCAS: also a lock-acquire candidate */
#define IGD_EXCH 4         /* atomicExch: also a lock release */
#define IGD_FENCE 5        /* __threadfence{_block,,_system} (Fig. 5b) */
#define IGD_SYNCWARP 6     /* __syncwarp */
#define IGD_SYNCTHREADS 7  /* __syncthreads (Fig. 5a) */
#define IGD_GRID_SYNC 8    /* grid-wide barrier: device fence by every thread + barrier (reading A15) */
#define IGD_CG_TILE_SYNC 9 /* == SYNCWARP */
#define IGD_CG_BLOCK_SYNC 10 /* == SYNCTHREADS */
#define IGD_CG_GRID_SYNC 11  /* == GRID_SYNC */
#define IGD_KERNEL_BOUNDARY 12 /* end of one kernel, start of the next (reading A31):
                                  the implicit all-thread barrier at kernel end
                                  orders everything before it before everything after it, so every
                                  word's shadow state is discarded (its next access is P1), and the
                                  locking protocol is inferred per kernel: every lock
                                  table and isThread bit is reset.  One geometry for all kernels. */
/* scope (tk bits 28..29) */
#define IGD_SCOPE_NONE 0
#define IGD_SCOPE_BLOCK 1
#define IGD_SCOPE_DEVICE 2
#define IGD_SCOPE_SYSTEM 3 /* treated as DEVICE: the paper ignores system scope */

/*
 * Field rules (violations -> IGD_ETRACE, first offending index via igd_bad_event):
 *   LD, ST            : tid < threads, mask contains lane(tid), scope NONE
 *   ATOM, CAS, EXCH   : tid < threads, mask contains lane(tid), scope BLOCK/DEVICE/SYSTEM
 *   FENCE             : addr 0, tid < threads, mask contains lane(tid), scope != NONE
 *   SYNCWARP, CG_TILE : addr 0, tid = any thread of the warp (< threads), scope NONE
 *   SYNCTHREADS, CG_BLOCK : addr 0, tid = any thread of the block (< threads), scope NONE
 *   GRID_SYNC, CG_GRID: addr 0, tid 0, scope NONE
 *   KERNEL_BOUNDARY   : addr 0, tid 0, scope NONE
 *   kind > 12 or tk bits 30..31 set: invalid.
 * Geometry: block(t) = t / block_dim, warps per block
 * Wb = ceil(block_dim/32), warp(t) = block(t)*Wb + (t % block_dim)/32,
 * lane(t) = (t % block_dim) % 32.
 * Conventions: the trace order is the execution order; per-lane events of one warp
 * instruction are contiguous in ascending lane order; one SYNCTHREADS per (block, barrier
 * instance), one SYNCWARP per (warp, instance), one GRID_SYNC per instance.
 */

typedef struct {
    uint32_t n_blocks, block_dim; /* geometry of the traced kernel */
    uint64_t n_events_total;      /* global trace length (all ranks) */
    uint64_t first_event;         /* global index of events[0] on this rank (0 on one GPU) */
    uint64_t n_events;            /* events in this buffer */
    uint32_t flags;               /* IGD_TRACE_DEVICE_PTR: `events` is a device pointer */
} igd_trace_desc;
#define IGD_TRACE_DEVICE_PTR 1u

/* ---- report: 32 bytes ------------------------------------------------------------ */
typedef struct {
    uint64_t addr;    /* byte address of the racy 4-byte word (word << 2) */
    uint64_t cur;     /* global index of the access at which the race is declared */
    uint64_t prev;    /* global index of md: the last writer for a load, else the last accessor */
    uint8_t type;     /* 1 R1 scoped atomic, 2 R2 intra-warp (ITS), 3 R3 intra-block,
                         4 R4 inter-block, 5 R5 missing lock (Table 2) */
    uint8_t cur_kind, prev_kind; /* igd kinds of the two accesses */
    uint8_t pad[5];
} igd_report;
#define IGD_R1 1
#define IGD_R2 2
#define IGD_R3 3
#define IGD_R4 4
#define IGD_R5 5

/* Device allocator callbacks (e.g. a shim over torch's caching allocator).  May be NULL,
   then cudaMallocAsync / cudaFreeAsync on the context stream are used. */
typedef void* (*igd_alloc_fn)(size_t bytes, void* stream, void* user);
typedef void (*igd_free_fn)(void* p, void* stream, void* user);

typedef struct igd_ctx igd_ctx; /* opaque; owns every device buffer it allocates */

/* Create a context on `cuda_device`, issuing all work on `cuda_stream` (a cudaStream_t;
   NULL = the legacy default stream).  The context also owns a greatest-priority side stream that
   igd_detect forks from and joins back into `cuda_stream` (the a2 / a3 stages beside the access
   sort on lock-heavy traces), so every result is ordered on `cuda_stream` as before.
   Multi-GPU: nranks > 1 processes (one per GPU) each create a context with their
   rank in [0, nranks) and the SAME 128-byte NCCL unique id (igd_nccl_unique_id on one rank,
   shared by the caller, e.g. a torch.distributed broadcast).  The call initialises an NCCL
   communicator (ncclCommInitRank: blocks until every rank joins) and makes igd_detect collective.
   nranks == 1 with a non-NULL id gives a one-rank communicator (the collective path on one GPU);
   nranks == 1 with NULL is the single-GPU pipeline.  An id whose first 8 bytes are "IGDLOOP:"
   (followed by a NUL-terminated group name) selects the in-process loopback transport instead of
   NCCL: the nranks contexts of one process, driven by one host thread each, exchange through
   device copies with the same collectives (the test transport of one-GPU boxes, where NCCL
   refuses two ranks on one device).  IGD_EINVAL: rank out of range, nranks > 1
   without an id, one of alloc_fn / free_fn NULL; IGD_ENCCL: libnccl unavailable or the
   communicator could not be created. */
int igd_ctx_create(igd_ctx** out, int cuda_device, void* cuda_stream, int nranks, int rank,
                   const uint8_t* nccl_unique_id, igd_alloc_fn alloc_fn, igd_free_fn free_fn,
                   void* alloc_user);

/* Attach a trace.  Host `events` (flags without IGD_TRACE_DEVICE_PTR) are copied to device
   memory owned by the context, asynchronously on the context stream from the caller's
   buffer; the call synchronizes the stream before returning, so the caller may free the
   buffer afterwards.  Device `events` are BORROWED: they must stay valid and unmodified until
   igd_detect returns, and be 16-byte aligned.  Returns IGD_EINVAL on bad geometry / desc or a
   misaligned device pointer, IGD_ETOOBIG when
   n_events >= 2^32 - 1.  Field validation happens in igd_detect. */
int igd_trace_load(igd_ctx* ctx, const igd_trace_desc* desc, const igd_event* events);

/* Run the race check over the attached trace.  On success *n_reports_global holds the number
   of reports; the reports stay in context-owned device memory until the next igd_detect or
   igd_ctx_destroy.  Returns IGD_ETRACE (igd_bad_event gives the index) on an ill-formed
   event.  Word keys (a4): the low 32 bits of the word when the accessed words span < 2^32
   words, else u64 keys word - (min word rounded down to 256) sorted over ceil(bits(span)/8)
   radix passes -- any 62-bit word range (e.g. sparse 48-bit virtual addresses) is exact.
   flags: IGD_DETECT_TIMING (per-stage timings, below) | IGD_DETECT_COALESCE (warp-coalesced
   check, §6.5, reading A32: of a warp instruction whose >= 2 active lanes all LD, or
   all ATOM, one word -- consecutive events, same warp / kind / scope / mask / word, lanes
   ascending from the mask's lowest -- only the first lane is checked and recorded; the
   reports then differ from the per-lane default).  Single-context (not sharded) only. */
#define IGD_DETECT_COALESCE 2u
/* IGD_DETECT_PAPER_COUNTERS (reading A33): the synchronization IDs copied into a
   word's metadata keep Fig. 4's widths -- WarpBarID 6, BlkBarID 8, DevFenceID 6,
   BlkFenceID 6 bits -- so an ID whose events since md number a multiple of 2^width reads as
   unchanged (the paper's bounded-counter false positives, §6.7).  Default: exact counters (A16).
   Also accepted by igd_shard_detect. */
#define IGD_DETECT_PAPER_COUNTERS 4u
/* Paper-fidelity modes (off by default, combinable):
   IGD_DETECT_STICKY_FLAGS (reading A35): Table 2 as written -- P3 and P4 also need the word's
     sticky DevShared and BlkShared flags clear, P5 DevShared clear.  The default
     reading A4 derives them from md and the current access.  Also accepted by igd_shard_detect
     and collective contexts.
   IGD_DETECT_TAG_LOG2(b), 8 <= b <= 22 (reading A36): the metadata of Fig. 4 as a table of 2^b
     entries with a 10-bit Tag: word w uses entry w mod 2^b with Tag
     (w >> b) mod 2^10; an access whose Tag differs from the entry's claims it (a first access),
     words with equal entry and Tag share it.  Reports carry the accessed word's address.
     Single-GPU contexts only (IGD_EINVAL otherwise). */
/* IGD_DETECT_LAST_K(k), k in {2, 4, 8} (reading A37, §6.7): the last k writers (loads)
     or accessors (stores, atomics) of the word are checked newest first with Table 2, and the
     first racy one is reported.  k = 1 (or 0) is the default.  Single-GPU contexts only. */
#define IGD_DETECT_LAST_K_SHIFT 16
#define IGD_DETECT_LAST_K(k) ((uint32_t)(k) << IGD_DETECT_LAST_K_SHIFT)
#define IGD_DETECT_STICKY_FLAGS 8u
#define IGD_DETECT_TAG_SHIFT 8
#define IGD_DETECT_TAG_LOG2(b) ((uint32_t)(b) << IGD_DETECT_TAG_SHIFT)
int igd_detect(igd_ctx* ctx, uint32_t flags, uint64_t* n_reports_global);
/* Collective contexts (created with an NCCL id): every rank calls igd_detect after loading its
   contiguous chunk [desc.first_event, desc.first_event + desc.n_events) of one global trace of
   desc.n_events_total events (chunks in rank order, covering the trace).  Words are
   hash-sharded (owner = fmix32(low 32 bits of the word) % nranks); the access records move to
   their owner by an NCCL all-to-all, the synchronization streams are all-gathered, each rank
   checks the words it owns, and the reports are all-gathered and merged: every rank returns the
   identical global report set (igd_reports), equal to the single-GPU result.  Errors are agreed
   across ranks (the first invalid GLOBAL index for IGD_ETRACE), so every rank returns the same
   code.  IGD_DETECT_COALESCE is rejected (IGD_EINVAL). */

/* A fresh 128-byte NCCL unique id for igd_ctx_create (call on one rank, share with the others).
   IGD_ENCCL when libnccl cannot be loaded. */
int igd_nccl_unique_id(uint8_t* out128);

/* ---- multi-GPU sharding, driven by the host over torch.distributed / NCCL ----
   Each rank loads its contiguous chunk with igd_trace_load (desc.first_event = global index of
   events[0], desc.n_events_total = global length).  Words are hash-sharded:
   owner(word) = fmix32(low 32 bits of word) % nranks (murmur3 finalizer).

   Stage 1, igd_shard_prepare: partitions the chunk.  counts[o] = access records destined to rank o;
   *n_sync_stream = synchronization-stream events (FENCE, SYNCWARP, SYNCTHREADS, GRID_SYNC, the CG
   kinds, CAS, EXCH); *bad_event = first invalid GLOBAL index (~0 if none; the caller reduces it over
   ranks and must not continue if any rank has one); word_minmax = min / max accessed word of the chunk
   (the caller reduces them; the global span must be < 2^32 words).  Returns IGD_OK even when
   *bad_event is set.
   igd_shard_buffers: device pointers (context-owned, valid until the next prepare or until
   igd_shard_detect returns, which releases the record buffer -- after the check when the
   caller passes it back as d_records) to the records
   (uint4 {low 32 bits of the word, global index, tk, active mask}, grouped by owner in rank order,
   trace order inside a group), the sync-stream global indices (u32) and events (16 B).
   Exchange (caller): all-to-all of the record groups; all-gather of the sync streams concatenated
   in rank order (= trace order).

   Stage 2, igd_shard_detect: checks the words this rank owns.  d_records = the records received from
   all ranks concatenated in source-rank order; d_sync_idx / d_sync_events = the global sync stream;
   min_word = global minimum accessed word.  Device pointers are borrowed for the call.  Reports (global
   indices) are read with igd_reports / igd_reports_device; the union over ranks is the single-GPU
   report set (address-shard invariance).  flags: IGD_DETECT_TIMING | IGD_DETECT_PAPER_COUNTERS (IGD_DETECT_COALESCE:
   IGD_EINVAL, a coalesced group may straddle two ranks' chunks). */
int igd_shard_prepare(igd_ctx* ctx, uint32_t nranks, uint64_t* counts, uint64_t* n_sync_stream,
                      uint64_t* bad_event, uint64_t* word_minmax);
int igd_shard_buffers(igd_ctx* ctx, void** d_records, void** d_sync_idx, void** d_sync_events);
int igd_shard_detect(igd_ctx* ctx, const void* d_records, uint64_t n_records, const uint32_t* d_sync_idx,
                     const void* d_sync_events, uint64_t n_sync_stream, uint64_t min_word, uint32_t flags,
                     uint64_t* n_reports);

/* ---- streaming sessions (the paper's online setting) ----
   A trace arrives in consecutive chunks (e.g. drained from an instrumentation buffer) and each
   chunk is checked on arrival: its reports (global trace indices, ascending cur, read with
   igd_reports) are final, and their union over the session equals igd_detect of the whole trace.
   The context carries the synchronization stream so far and, per accessed word, its last writer,
   last accessor, sticky sharing flags and scope of its last atomic.  Single-GPU contexts; the
   session's words must span < 2^32 words (IGD_ETOOBIG); grid-changing kernel boundaries are
   rejected (IGD_EINVAL).
   igd_stream_begin: start (or restart) a session for kernels of grid (n_blocks, block_dim).
   igd_stream_feed: check the next n_events events (event_flags: IGD_TRACE_DEVICE_PTR for a
     device pointer, borrowed for the call, else host memory, copied); detect_flags:
     IGD_DETECT_TIMING | IGD_DETECT_PAPER_COUNTERS | IGD_DETECT_STICKY_FLAGS.  *n_reports = this
     chunk's reports.  IGD_ETRACE (igd_bad_event = global index) and other errors end the session.
     IGD_ESTATE without an active session.  igd_detect / igd_shard_detect return IGD_ESTATE
     while a session is active.
   igd_stream_end: end the session and release its carried state. */
int igd_stream_begin(igd_ctx* ctx, uint32_t n_blocks, uint32_t block_dim);
int igd_stream_feed(igd_ctx* ctx, const igd_event* events, uint64_t n_events, uint32_t event_flags,
                    uint32_t detect_flags, uint64_t* n_reports);
int igd_stream_end(igd_ctx* ctx);

/* Copy min(cap, total) reports, ascending by `cur` (at most one report per access, so the
   order is total), to host memory `host_out`; *n_written = number copied. */
int igd_reports(igd_ctx* ctx, igd_report* host_out, uint64_t cap, uint64_t* n_written);

/* Device pointer to the report array of the last igd_detect (context-owned; same order). */
int igd_reports_device(igd_ctx* ctx, const igd_report** dev_ptr, uint64_t* n);

/* Index of the first invalid event found by the last igd_detect (valid after IGD_ETRACE). */
uint64_t igd_bad_event(const igd_ctx* ctx);

/* Per-stage device timings (milliseconds, CUDA events on the context stream) of the last
   igd_detect when IGD_DETECT_TIMING was passed; stage order: see igd_stage_name. */
#define IGD_DETECT_TIMING 1u
#define IGD_N_STAGES 8
int igd_stage_times(const igd_ctx* ctx, float* ms_out /* [IGD_N_STAGES] */);
const char* igd_stage_name(int stage);

/* Number of kernel launches the last igd_detect issued (evidence for gpu_launches). */
uint64_t igd_last_launch_count(const igd_ctx* ctx);

/* Per kernel class (0..IGD_N_KCLASS-1: ingest, sort_sync, csr_offsets, lock_infer, sort_access,
   check, report, misc, ingest_sort0 = the ingest write pass fused with radix pass 0) of the last igd_detect run with IGD_DETECT_TIMING: launch count, summed
   device time (CUDA events on the context stream around each launch) and the algorithmic bytes
   those launches must move.  Any output pointer may be NULL. */
#define IGD_N_KCLASS 9
int igd_kernel_stats(const igd_ctx* ctx, int kclass, const char** name, uint32_t* launches, float* ms,
                     double* alg_bytes);

void igd_ctx_destroy(igd_ctx* ctx);
const char* igd_strerror(int code);
const char* igd_last_error(const igd_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* IGD_H */
