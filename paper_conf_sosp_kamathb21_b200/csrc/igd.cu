// igd.cu -- host orchestration of the race-check pipeline and the C ABI of include/igd.h.
//
// Pipeline (one stream, kernels in csrc/*.cuh):
//   a1+a2+a4  ingest::k_ingest      validate, compact accesses / sync records, digit histograms
//   a2        rsort::k_onesweep     stable radix sort of sync records by entity
//             syncx::k_csr_offsets  CSR offsets of the per-entity timestamp lists
//   a3        syncx::k_lock_infer   per-warp lock-table replay -> held-lock change points
//   a5        rsort::k_onesweep     stable radix sort of accesses by word (trace order kept)
//   a6        check::k_check        segmented shadow-metadata scan + Table 2 check
//   a7        report sort by `cur`  canonical order
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "check.cuh"
#include "check4.cuh"
#include "coalesce.cuh"
#include "common.cuh"
#include "fused.cuh"
#include "ingest.cuh"
#include "lastk.cuh"
#include "sort.cuh"
#include "shard.cuh"
#include "sync.cuh"
#include <dlfcn.h>
#include <nvtx3/nvToolsExt.h>
#include <nccl.h>  // types and prototypes only: the library is resolved at run time (NcclApi)
#include <algorithm>
#include <condition_variable>
#include <map>
#include <mutex>
#include <vector>

#ifndef IGD_PASS0_GENERIC
#define IGD_PASS0_GENERIC 0  // 1: the fused pipeline's pass 0 through the generic k_ingest<0> (A/B)
#endif

namespace {
struct LoopGroup;  // in-process loopback transport (defined with the collectives)

enum KClass { KC_INGEST = 0, KC_SORT_SYNC, KC_CSR, KC_LOCK, KC_SORT_ACC, KC_CHECK, KC_REPORT, KC_MISC, KC_FUSED };

struct Buf {
    void* p = nullptr;
    size_t cap = 0;
};

enum Stage { S_INGEST = 0, S_SYNC_SORT, S_TABLES, S_ACC_SORT, S_CHECK, S_REPORT, S_HOST, S_TOTAL };
const char* kClassNames[IGD_N_KCLASS] = {"ingest", "sort_sync", "csr_offsets", "lock_infer",
                                         "sort_access", "check", "report", "misc", "ingest_sort0"};
constexpr int kMaxTimed = 128;
const char* kStageNames[IGD_N_STAGES] = {"ingest", "sync_sort", "epoch_lock_tables", "access_sort",
                                         "check", "report_sort", "host_sync", "total"};

// ---- NCCL, resolved at run time -------------------------------------------------------------
// A process that uses torch.distributed already has torch's libnccl loaded: RTLD_NOLOAD finds that
// copy, so libigd's communicator and torch's come from one library.  Otherwise the system
// libnccl.so.2 is loaded.  Only multi-rank contexts need it (igd_ctx_create with an NCCL id).
struct NcclApi {
    bool ok = false;
    std::string why;
    decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
    decltype(&ncclCommInitRank) CommInitRank = nullptr;
    decltype(&ncclCommDestroy) CommDestroy = nullptr;
    decltype(&ncclAllReduce) AllReduce = nullptr;
    decltype(&ncclAllGather) AllGather = nullptr;
    decltype(&ncclBroadcast) Broadcast = nullptr;
    decltype(&ncclSend) Send = nullptr;
    decltype(&ncclRecv) Recv = nullptr;
    decltype(&ncclGroupStart) GroupStart = nullptr;
    decltype(&ncclGroupEnd) GroupEnd = nullptr;
    decltype(&ncclGetErrorString) GetErrorString = nullptr;
};
NcclApi load_nccl() {
    NcclApi a;
    // RTLD_LOCAL: a copy loaded here must not satisfy another library's later symbol lookups
    // (torch resolves its own, newer NCCL symbols against the global namespace)
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_LOCAL);
    if (!h) {
        const char* e = dlerror();
        a.why = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
        return a;
    }
#define IGD_NCCL_SYM(F)                                                  \
    a.F = reinterpret_cast<decltype(a.F)>(dlsym(h, "nccl" #F));          \
    if (!a.F) {                                                          \
        a.why = "libnccl lacks nccl" #F;                                 \
        return a;                                                        \
    }
    IGD_NCCL_SYM(GetUniqueId)
    IGD_NCCL_SYM(CommInitRank)
    IGD_NCCL_SYM(CommDestroy)
    IGD_NCCL_SYM(AllReduce)
    IGD_NCCL_SYM(AllGather)
    IGD_NCCL_SYM(Broadcast)
    IGD_NCCL_SYM(Send)
    IGD_NCCL_SYM(Recv)
    IGD_NCCL_SYM(GroupStart)
    IGD_NCCL_SYM(GroupEnd)
    IGD_NCCL_SYM(GetErrorString)
#undef IGD_NCCL_SYM
    a.ok = true;
    return a;
}
NcclApi& nccl() {
    static NcclApi api = load_nccl();
    return api;
}

}  // namespace

struct igd_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    // multi-GPU: an NCCL communicator makes igd_detect collective
    int nranks = 1, rank = 0;
    ncclComm_t comm = nullptr;
    LoopGroup* loop = nullptr;  // in-process loopback transport (tests), instead of comm
    Buf cl_small, cl_mat, cl_recv, cl_sidx, cl_sev, cl_nrep, cl_rep;
    // per-kernel geometry (reading A34): the trace runs as segments between grid-changing
    // kernel boundaries, each on its own grid
    bool in_segment = false;
    const igd_event* seg_ev = nullptr;
    u64 seg_n = 0, seg_first = 0;
    u32 seg_nb = 0, seg_bd = 0;
    Buf gkb, seg_rep;
    // streaming sessions: chunks of one trace checked in order, the shadow state
    // carried between them as two records per word, the synchronization stream accumulated
    bool str_active = false;
    u64 str_n = 0, str_wmin = ~0ull, str_wmax = 0, str_nsync = 0, str_ncarry = 0;
    u32 str_nb = 0, str_bd = 0;
    Buf str_sidx, str_sev, str_carry[2], str_rec, str_co, str_flags;
    int str_cur = 0;
    igd_alloc_fn afn = nullptr;
    igd_free_fn ffn = nullptr;
    void* auser = nullptr;
    std::string err;

    igd_trace_desc desc{};
    const igd_event* events = nullptr;
    bool loaded = false;
    Buf owned_events;

    Buf acc_k[2], acc_v[2], syn_k[2], syn_v[2];
    Buf st_in_a, st_in_s, status, stats, hist, base, ctr;
    Buf dstatus;        // digit statuses of the radix passes, epoch-tagged (never cleared per pass)
    u32 ds_epoch = 0;   // tag of the last radix pass
    // a2 / a3 run on a side stream concurrently with the a5 access sort (SideSection): their own
    // scan / radix workspaces, swapped in for the section
    cudaStream_t side = nullptr;
    cudaEvent_t side_ev[2] = {nullptr, nullptr};
    Buf sw_base, sw_dstatus, sw_status, sw_ctr;
    u32 sw_epoch = 0;
    bool in_side = false;
    Buf off, ldesc, gtab, tcnt, tpts, tbits, fdev, skipb;
    Buf rep_raw, rep_k[2], rep_v[2], rep_out, rep_ctr, rep_hist;
    u64 sync_cap = 0;
    u64 rep_cap = 0;
    bool coalesce = false;  // IGD_DETECT_COALESCE of the running igd_detect (reading A32)
    bool paper_counters = false;  // IGD_DETECT_PAPER_COUNTERS (reading A33)
    bool sticky = false;          // IGD_DETECT_STICKY_FLAGS (reading A35)
    u32 tag_log2 = 0;             // IGD_DETECT_TAG_LOG2 (reading A36): 0 = exact per-word state
    u32 last_k = 1;               // IGD_DETECT_LAST_K (reading A37): history depth
    Buf lk_state;
    int fused = 1;      // single GPU: ingest write pass fused with radix pass 0 (IGD_FUSED=0: unfused)
    // sharded mode: stage-1 outputs, stage-2 inputs
    bool shard = false;
    Buf sh_cnt, sh_obase, sh_send, sh_sidx_buf, sh_sev_buf;
    u64 sh_send_n = 0, sh_sync_n = 0;
    const void* sh_rec = nullptr;
    u64 sh_nrec = 0;
    const u32* sh_sidx = nullptr;
    const void* sh_sev = nullptr;
    u64 sh_ns = 0, sh_wbase = 0, sh_ntotal = 0;
    int last_acur = 0;  // buffer holding the sorted accesses of the last igd_detect (debug hooks)
    int last_scur = 0;  // ... the sorted sync records
    u64 last_nsync = 0, last_npts = 0;  // sync records, lock change points
    u32 last_E = 0, last_T = 0;         // entities, threads
    u64 last_nacc = 0;
    u64 n_reports = 0;
    u64 bad_event = 0;
    u64 launches = 0;

    // pinned host mirrors
    u64* h_stats = nullptr;  // 8
    u32* h_hist = nullptr;   // 2 x 1024 (+ report hist 1024, + wide-key digits 4..7)
    u64* h_small = nullptr;  // 8

    bool timing = false;
    int nvtx_depth = 0;
    cudaEvent_t ev[IGD_N_STAGES + 1];
    float stage_ms[IGD_N_STAGES];
    // per-launch timing (IGD_DETECT_TIMING): events around every kernel launch
    cudaEvent_t kev[2 * kMaxTimed];
    int kcls[kMaxTimed];
    double kbytes[kMaxTimed];
    int nk = 0;
    float cls_ms[IGD_N_KCLASS];
    uint32_t cls_n[IGD_N_KCLASS];
    double cls_bytes[IGD_N_KCLASS];
};

// Launch bracket: records CUDA events on the context stream around one kernel launch.
struct KTimer {
    igd_ctx* ctx;
    int slot;
    KTimer(igd_ctx* c, int cls, double alg_bytes) : ctx(c), slot(-1) {
        c->launches++;
        if (c->timing && c->nk < kMaxTimed) {
            slot = c->nk++;
            c->kcls[slot] = cls;
            c->kbytes[slot] = alg_bytes;
            cudaEventRecord(c->kev[2 * slot], c->stream);
        }
    }
    ~KTimer() {
        if (slot >= 0) cudaEventRecord(ctx->kev[2 * slot + 1], ctx->stream);
    }
};

#define CK(call)                                                                               \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess) {                                                               \
            ctx->err = std::string(#call) + ": " + cudaGetErrorString(e_);                     \
            return e_ == cudaErrorMemoryAllocation ? IGD_ENOMEM : IGD_ECUDA;                   \
        }                                                                                      \
    } while (0)
#define RET(x)                   \
    do {                         \
        int r_ = (x);            \
        if (r_ != IGD_OK) return r_; \
    } while (0)
#define NK(call)                                                                               \
    do {                                                                                       \
        ncclResult_t e_ = (call);                                                              \
        if (e_ != ncclSuccess) {                                                               \
            ctx->err = std::string(#call) + ": " + nccl().GetErrorString(e_);                  \
            return IGD_ENCCL;                                                                  \
        }                                                                                      \
    } while (0)

static int buf_free(igd_ctx* ctx, Buf& b) {
    if (b.p) {
        if (ctx->ffn) ctx->ffn(b.p, (void*)ctx->stream, ctx->auser);
        else CK(cudaFreeAsync(b.p, ctx->stream));
    }
    b.p = nullptr;
    b.cap = 0;
    return IGD_OK;
}

static int ensure(igd_ctx* ctx, Buf& b, size_t bytes) {
    if (bytes == 0) bytes = 16;
    if (b.cap >= bytes) return IGD_OK;
    RET(buf_free(ctx, b));
    size_t want = bytes < (1ull << 30) ? bytes + bytes / 8 : bytes;  // headroom for small buffers only
    void* p = nullptr;
    if (ctx->afn) {
        p = ctx->afn(want, (void*)ctx->stream, ctx->auser);
        if (!p) {
            ctx->err = "allocator callback returned NULL for " + std::to_string(want) + " bytes";
            return IGD_ENOMEM;
        }
    } else {
        cudaError_t e = cudaMallocAsync(&p, want, ctx->stream);
        if (e != cudaSuccess) {
            ctx->err = std::string("cudaMallocAsync: ") + cudaGetErrorString(e);
            (void)cudaGetLastError();
            return IGD_ENOMEM;
        }
    }
    b.p = p;
    b.cap = want;
    return IGD_OK;
}

// The digit-status buffer for a radix pass over `tiles` tiles and the pass's epoch tag: cleared
// only when (re)allocated or when the 22-bit epoch wraps.
static int next_digit_epoch(igd_ctx* ctx, u64 tiles, u32* epoch) {
    const size_t bytes = tiles * 256 * sizeof(u64);
    const size_t old_cap = ctx->dstatus.cap;
    RET(ensure(ctx, ctx->dstatus, bytes));
    if (ctx->dstatus.cap != old_cap || ctx->ds_epoch >= 0x3FFFFFu) {
        CK(cudaMemsetAsync(ctx->dstatus.p, 0, ctx->dstatus.cap, ctx->stream));
        ctx->ds_epoch = 0;
    }
    *epoch = ++ctx->ds_epoch;
    return IGD_OK;
}

template <class T>
static T* P_(Buf& b) {
    return reinterpret_cast<T*>(b.p);
}

static u32 bits_needed(u64 maxval) {
    u32 b = 0;
    while (b < 64 && (maxval >> b)) b++;
    return b;
}

static void geo_init(Geo& g, u32 nb, u32 bd) { g.init(nb, bd); }

static int sm_count(igd_ctx* ctx) {
    int v = 148;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, ctx->device);
    return v;
}

// Stage boundaries: CUDA events (IGD_DETECT_TIMING) and an NVTX range per stage
// ("igd:<stage>", visible to Nsight Systems / ncu --nvtx; a no-op without a tool attached).
static void mark(igd_ctx* ctx, int stage) {
    if (ctx->timing) cudaEventRecord(ctx->ev[stage], ctx->stream);
    while (ctx->nvtx_depth > 0) {
        nvtxRangePop();
        ctx->nvtx_depth--;
    }
    if (stage < IGD_N_STAGES - 1) {
        static const char* names[IGD_N_STAGES - 1] = {"igd:a1-a4 ingest", "igd:a2 sync sort", "igd:a2-a3 tables+locks",
                                                      "igd:a5 access sort", "igd:a6 check", "igd:a7 reports",
                                                      "igd:host sync"};
        nvtxRangePushA(names[stage]);
        ctx->nvtx_depth++;
    }
}

// a2 / a3 concurrently with a5: the host enqueues the access sort on the context stream, then
// runs the a2 / a3 code with the side stream (forked from the context stream) as ctx->stream and
// the scan / radix workspaces swapped for the side copies, so the two sorts never share a tile
// counter, digit-status buffer or digit-base table; end() (or the destructor on an error path)
// swaps back and joins: the context stream waits for everything the section enqueued.
struct SideSection {
    igd_ctx* ctx;
    bool on = false;
    explicit SideSection(igd_ctx* c) : ctx(c) {}
    void swap_all() {
        std::swap(ctx->stream, ctx->side);
        std::swap(ctx->base, ctx->sw_base);
        std::swap(ctx->dstatus, ctx->sw_dstatus);
        std::swap(ctx->status, ctx->sw_status);
        std::swap(ctx->ctr, ctx->sw_ctr);
        std::swap(ctx->ds_epoch, ctx->sw_epoch);
        ctx->in_side = !ctx->in_side;
    }
    // the fork point: recorded on the context stream before the work the section overlaps
    bool use = false;
    int fork(bool want) {
        use = want && ctx->side;
        if (use) CK(cudaEventRecord(ctx->side_ev[0], ctx->stream));
        return IGD_OK;
    }
    int begin() {
        if (!use) return IGD_OK;
        CK(cudaStreamWaitEvent(ctx->side, ctx->side_ev[0], 0));
        swap_all();
        on = true;
        // the side copies of the fixed-size workspaces (the others grow on demand)
        RET(ensure(ctx, ctx->ctr, 64));
        RET(ensure(ctx, ctx->base, 8 * 256 * sizeof(u32)));
        return IGD_OK;
    }
    int end() {
        if (!on) return IGD_OK;
        on = false;
        cudaError_t e = cudaEventRecord(ctx->side_ev[1], ctx->stream);  // the side stream
        swap_all();
        if (e == cudaSuccess) e = cudaStreamWaitEvent(ctx->stream, ctx->side_ev[1], 0);
        if (e != cudaSuccess) {
            ctx->err = std::string("side stream join: ") + cudaGetErrorString(e);
            return IGD_ECUDA;
        }
        return IGD_OK;
    }
    ~SideSection() {
        if (on) {
            cudaStreamSynchronize(ctx->stream);  // error path: the side work must not outlive its buffers' owner
            end();
        }
    }
};

// One radix pass over n keys: the full tiles, then (if any) the partial last tile (same tile
// counter: the tail's ticket is the last tile).
template <typename VT, typename KT = u32>
static void launch_pass(u64 n, cudaStream_t st, const rsort::PassParams& pp) {
    const size_t smem = rsort::onesweep_smem<VT, KT>();
    const u64 full = n / rsort::TILE;
    if (full) rsort::k_onesweep<VT, false, KT><<<(unsigned)full, rsort::THREADS, smem, st>>>(pp);
    if (n % rsort::TILE) rsort::k_onesweep<VT, true, KT><<<1u, rsort::THREADS, smem, st>>>(pp);
}
template <typename VT, typename KT = u32>
static void set_pass_smem() {
    const int b = (int)rsort::onesweep_smem<VT, KT>();
    cudaFuncSetAttribute(rsort::k_onesweep<VT, false, KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
    cudaFuncSetAttribute(rsort::k_onesweep<VT, true, KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
}

// Stable LSD radix sort of n (key, value) pairs in buffers k[cur], v[cur]; h_hist is the host
// copy of the 4x256 (u32 keys) or 8x256 (kbytes = 8: u64 keys) digit histogram (device copy
// d_hist).  Digits above max_bits and digits with one occupied bin are skipped.  Returns the
// buffer index holding the result.
// vin_first: values of the input (instead of v[first_cur]) for the first pass that runs -- the
// sharded path sorts the received records in place of a split copy.
static int radix_sort(igd_ctx* ctx, int cls, Buf* k, Buf* v, u64 n, const u32* d_hist, const u32* h_hist,
                      u32 max_bits, int* out_cur, int vbytes = 4, u32 first_pass = 0, int first_cur = 0,
                      const void* vin_first = nullptr, int kbytes = 4) {
    const u32 ndig = kbytes == 8 ? 8u : 4u;
    int cur = first_cur;
    *out_cur = cur;
    bool ran = false;
    if (n <= 1) {
        if (n == 1 && vin_first) CK(cudaMemcpyAsync(v[cur].p, vin_first, vbytes, cudaMemcpyDeviceToDevice, ctx->stream));
        return IGD_OK;
    }
    if (n > 0xFFFFFFFFull - 2 * rsort::TILE) return IGD_ETOOBIG;  // 32-bit tile indexing
    {
        KTimer kt(ctx, KC_MISC, 0);
        rsort::k_digit_base<<<ndig, rsort::RADIX, 0, ctx->stream>>>(d_hist, P_<u32>(ctx->base));
    }
    const u64 tiles = (n + rsort::TILE - 1) / rsort::TILE;
    for (u32 p = first_pass; p < ndig; p++) {
        if (p * 8 >= max_bits) break;
        bool trivial = false;
        for (int d = 0; d < 256; d++)
            if (h_hist[p * 256 + d] == n) trivial = true;
        if (trivial) continue;
        rsort::PassParams pp;
        RET(next_digit_epoch(ctx, tiles, &pp.epoch));
        CK(cudaMemsetAsync(P_<u32>(ctx->ctr), 0, sizeof(u32), ctx->stream));
        pp.kin = k[cur].p;
        pp.vin = (!ran && vin_first) ? vin_first : v[cur].p;
        ran = true;
        pp.kout = k[cur ^ 1].p;
        pp.vout = v[cur ^ 1].p;
        pp.n = (u32)n;
        pp.shift = p * 8;
        pp.dmask = max_bits >= p * 8 + 8 ? 255u : (1u << (max_bits - p * 8)) - 1u;
        pp.digit_base = P_<u32>(ctx->base) + p * 256;
        pp.status = P_<u64>(ctx->dstatus);
        pp.tile_ctr = P_<u32>(ctx->ctr);
        {
            KTimer kt(ctx, cls, 2.0 * (kbytes + vbytes) * (double)n);  // read + write the key and the value
            if (kbytes == 8) launch_pass<u64, u64>(n, ctx->stream, pp);
            else if (vbytes == 16) launch_pass<uint4>(n, ctx->stream, pp);
            else if (vbytes == 8) launch_pass<u64>(n, ctx->stream, pp);
            else launch_pass<u32>(n, ctx->stream, pp);
        }
        if (n > rsort::TILE && n % rsort::TILE) ctx->launches++;  // the partial-tile launch
        CK(cudaGetLastError());
        cur ^= 1;
    }
    if (!ran && vin_first)  // every digit trivial: the values still have to land in v[cur]
        CK(cudaMemcpyAsync(v[cur].p, vin_first, n * vbytes, cudaMemcpyDeviceToDevice, ctx->stream));
    *out_cur = cur;
    return IGD_OK;
}

// a6 kernel instantiation: sharded payload (MV), kernel boundaries (KB), paper-fidelity bits
// (FID: 1 = Fig. 4-width IDs, A33; 2 = sticky sharing flags, A35), power-of-two geometry (GEO2),
// u64 keys (a4's wide path).  The fidelity modes and the wide path use the general-geometry
// instantiation only (fewer kernels to build; they are not the timed path).
template <bool MV, bool KB>
static void launch_check_w(int fid, unsigned tb, cudaStream_t st, const check::Params& cp) {
    // power-of-two geometry (block_dim >= 32): shift / mask instead of divisions (common case)
    const bool geo2 = cp.g.dlog < 32 && cp.g.D >= 32;
    if constexpr (MV) {
        if (fid & 8) {  // streaming mode (f4): carried records, state out
            switch (fid & 3) {
                case 0: check::k_check4<MV, KB, 8, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
                case 1: check::k_check4<MV, KB, 9, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
                case 2: check::k_check4<MV, KB, 10, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
                default: check::k_check4<MV, KB, 11, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
            }
            return;
        }
    }
    switch (fid) {
        case 0:
            if (geo2) check::k_check4<MV, KB, 0, true><<<tb, check::C4_THREADS, 0, st>>>(cp);
            else check::k_check4<MV, KB, 0, false><<<tb, check::C4_THREADS, 0, st>>>(cp);
            break;
        case 1: check::k_check4<MV, KB, 1, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 2: check::k_check4<MV, KB, 2, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 3: check::k_check4<MV, KB, 3, false><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        default:  // last-k state out (single context only)
            if constexpr (!MV) {
                if (fid == 4) check::k_check4<MV, KB, 4, false><<<tb, check::C4_THREADS, 0, st>>>(cp);
                else if (fid == 5) check::k_check4<MV, KB, 5, false><<<tb, check::C4_THREADS, 0, st>>>(cp);
                else if (fid == 6) check::k_check4<MV, KB, 6, false><<<tb, check::C4_THREADS, 0, st>>>(cp);
                else check::k_check4<MV, KB, 7, false><<<tb, check::C4_THREADS, 0, st>>>(cp);
            }
            break;
    }
}
template <bool KB>
static void launch_check_64(int fid, unsigned tb, cudaStream_t st, const check::Params& cp) {
    switch (fid) {
        case 0: check::k_check4<false, KB, 0, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 1: check::k_check4<false, KB, 1, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 2: check::k_check4<false, KB, 2, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 3: check::k_check4<false, KB, 3, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 4: check::k_check4<false, KB, 4, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 5: check::k_check4<false, KB, 5, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        case 6: check::k_check4<false, KB, 6, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
        default: check::k_check4<false, KB, 7, false, u64><<<tb, check::C4_THREADS, 0, st>>>(cp); break;
    }
}
static void launch_check(bool mv, bool kb, int fid, bool key64, unsigned tb, cudaStream_t st,
                         const check::Params& cp) {
    if (key64) {  // a4's wide path (single GPU)
        if (kb) launch_check_64<true>(fid, tb, st, cp);
        else launch_check_64<false>(fid, tb, st, cp);
        return;
    }
    if (mv && kb) launch_check_w<true, true>(fid, tb, st, cp);
    else if (mv) launch_check_w<true, false>(fid, tb, st, cp);
    else if (kb) launch_check_w<false, true>(fid, tb, st, cp);
    else launch_check_w<false, false>(fid, tb, st, cp);
}

static int scan_excl(igd_ctx* ctx, u32* data, u64 n) {
    const u64 per = (u64)syncx::SCAN_THREADS * syncx::SCAN_ITEMS;
    const u64 tiles = (n + per - 1) / per;
    RET(ensure(ctx, ctx->status, tiles * sizeof(u64)));
    CK(cudaMemsetAsync(ctx->status.p, 0, tiles * sizeof(u64), ctx->stream));
    CK(cudaMemsetAsync(P_<u32>(ctx->ctr), 0, sizeof(u32), ctx->stream));
    {
        KTimer kt(ctx, KC_LOCK, 8.0 * (double)n);
        syncx::k_scan_excl<<<(unsigned)tiles, syncx::SCAN_THREADS, 0, ctx->stream>>>(data, data, (u32)n,
                                                                                     P_<u64>(ctx->status),
                                                                                     P_<u32>(ctx->ctr));
    }
    CK(cudaGetLastError());
    return IGD_OK;
}

// a7: reports `in[0..n)` (one per access, unique `cur` < n_time) in ascending `cur` order into
// ctx->rep_out: a radix sort of the u32 keys cur, then a gather.
static int canon_reports(igd_ctx* ctx, const igd_report* in, u64 n, u64 n_time) {
    RET(ensure(ctx, ctx->rep_out, (n ? n : 1) * sizeof(igd_report)));
    if (n == 1 && in != P_<igd_report>(ctx->rep_out)) {
        CK(cudaMemcpyAsync(ctx->rep_out.p, in, sizeof(igd_report), cudaMemcpyDeviceToDevice, ctx->stream));
    } else if (n > 1 && n <= (u64)check::SMALL_REP && n_time <= 0xFFFFFFFFull) {
        // small sets (the latency-bound configs): one CTA, no host round trip
        KTimer kt(ctx, KC_REPORT, 64.0 * (double)n);
        check::k_report_sort_small<<<1, 1024, 0, ctx->stream>>>(in, (u32)n, P_<igd_report>(ctx->rep_out));
        CK(cudaGetLastError());
    } else if (n > 1) {
        const int sms = sm_count(ctx);
        for (int b = 0; b < 2; b++) {
            RET(ensure(ctx, ctx->rep_k[b], n * sizeof(u32)));
            RET(ensure(ctx, ctx->rep_v[b], n * sizeof(u32)));
        }
        RET(ensure(ctx, ctx->rep_hist, 1024 * sizeof(u32)));
        unsigned blocks = (unsigned)std::min<u64>((n + 255) / 256, (u64)sms * 8);
        {
            KTimer kt(ctx, KC_REPORT, 40.0 * (double)n);
            check::k_report_keys<<<blocks, 256, 0, ctx->stream>>>(in, (u32)n, 0, P_<u32>(ctx->rep_k[0]),
                                                                P_<u32>(ctx->rep_v[0]));
        }
        CK(cudaMemsetAsync(ctx->rep_hist.p, 0, 1024 * sizeof(u32), ctx->stream));
        {
            KTimer kt(ctx, KC_REPORT, 4.0 * (double)n);
            rsort::k_hist4<<<blocks, 256, 0, ctx->stream>>>(P_<u32>(ctx->rep_k[0]), n, P_<u32>(ctx->rep_hist));
        }
        CK(cudaMemcpyAsync(ctx->h_hist + 2048, ctx->rep_hist.p, 1024 * sizeof(u32), cudaMemcpyDeviceToHost,
                           ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        u32 hh[1024];
        memcpy(hh, ctx->h_hist + 2048, sizeof(hh));
        int rcur = 0;
        RET(radix_sort(ctx, KC_REPORT, ctx->rep_k, ctx->rep_v, n, P_<u32>(ctx->rep_hist), hh,
                       bits_needed(n_time ? n_time - 1 : 0), &rcur));
        {
            KTimer kt(ctx, KC_REPORT, 68.0 * (double)n);
            check::k_report_gather<<<blocks, 256, 0, ctx->stream>>>(in, P_<u32>(ctx->rep_v[rcur]), (u32)n,
                                                                   P_<igd_report>(ctx->rep_out));
        }
        CK(cudaGetLastError());
    }
    return IGD_OK;
}

// The pipeline.  Single GPU: the trace is `ctx->events`.  Sharded (ctx->shard): the
// synchronization side runs over the all-gathered sync stream (global timestamps in sh_sidx),
// the access side over the records this rank received in the all-to-all.
// Segment mode (ctx->in_segment, reading A34): the events [seg_first, seg_first + seg_n) of one
// kernel run on their own grid; reports and error indices are shifted to global indices.
constexpr int IGD_SEGMENTS_NEEDED = 1;  // internal: the trace changes grids, run it per segment
static int detect_impl(igd_ctx* ctx, u64* n_out) {
    const igd_trace_desc& D = ctx->desc;
    const bool SH = ctx->shard;
    const bool SEG = ctx->in_segment && !SH;
    const igd_event* ev0 = SEG ? ctx->seg_ev : ctx->events;
    const u64 n_ev = SEG ? ctx->seg_n : D.n_events;
    const u64 first = SEG ? ctx->seg_first : 0;
    const u64 n = SH ? ctx->sh_ntotal : n_ev;                      // timestamp domain [0, n)
    const igd_event* src_ev = SH ? (const igd_event*)ctx->sh_sev : ev0;
    const u64 n_src = SH ? ctx->sh_ns : n_ev;                      // events the ingest reads
    ctx->n_reports = 0;
    ctx->bad_event = 0;
    if (!SH && !SEG) {  // sharded / segments: keep the earlier launches in the same accounting
        ctx->launches = 0;
        ctx->nk = 0;
    }
    *n_out = 0;
    mark(ctx, 0);
    if (n == 0 || (n_src == 0 && (!SH || ctx->sh_nrec == 0))) {
        for (int s = 1; s <= IGD_N_STAGES; s++) mark(ctx, s);
        return IGD_OK;
    }
    Geo g;
    geo_init(g, SEG ? ctx->seg_nb : D.n_blocks, SEG ? ctx->seg_bd : D.block_dim);
    KeySpace ks;
    ks.init(g);
    const int sms = sm_count(ctx);

    // ---------------- a1 + a2 + a4: ingest ----------------
    const u64 in_tiles = (n_src + ingest::TILE - 1) / ingest::TILE;
    RET(ensure(ctx, ctx->stats, 8 * sizeof(u64)));
    // hist: [0, 1024) access-key digits 0..3, [1024, 2048) sync-key digits, [2048, 4096) the
    // 8 digits of wide (u64) access keys
    RET(ensure(ctx, ctx->hist, 4 * 1024 * sizeof(u32)));
    RET(ensure(ctx, ctx->base, 8 * 256 * sizeof(u32)));
    RET(ensure(ctx, ctx->ctr, 64));
    RET(ensure(ctx, ctx->st_in_a, (in_tiles + 1) * sizeof(u32)));
    RET(ensure(ctx, ctx->st_in_s, (in_tiles + 1) * sizeof(u32)));
    const u64 acc_cap = SH ? ctx->sh_nrec : n_ev;
    RET(ensure(ctx, ctx->gkb, 1024 * sizeof(u64)));
    // sharded payload: the single-GPU (index | tk) u64 -- the received records stay resident for
    // the rare active-mask lookups (SPLIT) -- or, in streaming sessions, the 16-byte record itself
    // (its mask field carries the carried state)
    const bool SPLIT = SH && !ctx->str_active;
    const int vbytes = (SH && !SPLIT) ? 16 : 8;
    for (int b = 0; b < 2; b++) {
        RET(ensure(ctx, ctx->acc_k[b], acc_cap * sizeof(u32)));
        RET(ensure(ctx, ctx->acc_v[b], acc_cap * vbytes));
    }
    u64 init[8] = {~0ull, 0, ~0ull, 0, 0, 0, 0, 0};
    memcpy(ctx->h_small, init, sizeof(init));
    CK(cudaMemcpyAsync(ctx->stats.p, ctx->h_small, sizeof(init), cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaMemsetAsync(ctx->hist.p, 0, 2 * 1024 * sizeof(u32), ctx->stream));
    CK(cudaMemsetAsync(ctx->st_in_a.p, 0, (in_tiles + 1) * sizeof(u32), ctx->stream));
    CK(cudaMemsetAsync(ctx->st_in_s.p, 0, (in_tiles + 1) * sizeof(u32), ctx->stream));
    ingest::Params ip;
    memset(&ip, 0, sizeof(ip));
    ip.ev = src_ev;
    ip.n = n_src;
    ip.g = g;
    ip.ks = ks;
    ip.gidx = SH ? ctx->sh_sidx : nullptr;
    ip.tile_acc = P_<u32>(ctx->st_in_a);
    ip.tile_sync = P_<u32>(ctx->st_in_s);
    ip.hist_acc = P_<u32>(ctx->hist);
    ip.hist_sync = P_<u32>(ctx->hist) + 1024;
    ip.gkb = P_<u64>(ctx->gkb);
    ip.gkb_cap = (u32)(ctx->gkb.cap / sizeof(u64));
    ip.stats = P_<u64>(ctx->stats);
    ip.n_tiles = (u32)in_tiles;
    ip.skip_bits = nullptr;
    if (ctx->coalesce && !SH && n_src > 0) {
        // warp-coalesced mode (A32): mark the events checked by their group's first lane
        const u64 rows = (n_src + 31) / 32;
        RET(ensure(ctx, ctx->skipb, rows * sizeof(u32)));
        const u64 warps = (rows + coal::ROWS - 1) / coal::ROWS;
        KTimer kt(ctx, KC_INGEST, 16.0 * (double)n_src);
        coal::k_coalesce_marks<<<(unsigned)((warps * 32 + coal::THREADS - 1) / coal::THREADS), coal::THREADS, 0,
                                 ctx->stream>>>(src_ev, n_src, g, P_<u32>(ctx->skipb));
        CK(cudaGetLastError());
        ip.skip_bits = P_<u32>(ctx->skipb);
    }
    const bool FUSED = !SH && ctx->fused;
    ip.hist0 = FUSED ? 1 : 0;
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ingest::k_ingest<0>, ingest::THREADS, 0);
    const u64 grid = std::max<u64>(1, std::min<u64>((u64)sms * (occ > 0 ? occ : 1), in_tiles));
    if (n_src > 0) {
        KTimer kt(ctx, KC_INGEST, 16.0 * (double)n_src);  // pass 0 reads every event
        if (FUSED && !IGD_PASS0_GENERIC) {
            // the timed path: branch-free rules, compile-time geometry / coalescing variants
            const bool geo2 = g.dlog < 32 && g.D >= 32;
            if (geo2 && !ip.skip_bits) ingest::k_count_fused<true, false><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
            else if (geo2) ingest::k_count_fused<true, true><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
            else if (!ip.skip_bits) ingest::k_count_fused<false, false><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
            else ingest::k_count_fused<false, true><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
        } else {
            ingest::k_ingest<0><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
        }
    }
    CK(cudaGetLastError());
    RET(scan_excl(ctx, P_<u32>(ctx->st_in_a), in_tiles + 1));
    RET(scan_excl(ctx, P_<u32>(ctx->st_in_s), in_tiles + 1));
    CK(cudaMemcpyAsync(ctx->h_stats, ctx->stats.p, 8 * sizeof(u64), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_hist, ctx->hist.p, 2 * 1024 * sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(&ctx->h_small[0], P_<u32>(ctx->st_in_a) + in_tiles, sizeof(u32), cudaMemcpyDeviceToHost,
                       ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    // grid-changing kernel boundaries (A34): the caller reruns the trace segment by segment (the
    // events of later kernels were validated against the first kernel's grid here)
    if (!SH && !SEG && ctx->h_stats[6] > 0) return IGD_SEGMENTS_NEEDED;
    if (ctx->h_stats[2] != ~0ull) {
        ctx->bad_event = ctx->h_stats[2] + first;
        ctx->err = "invalid event at index " + std::to_string(ctx->bad_event);
        return IGD_ETRACE;
    }
    const u64 n_acc = SH ? ctx->sh_nrec : (ctx->h_small[0] & 0xFFFFFFFFull);
    const u64 n_sync = ctx->h_stats[4];
    const u64 n_lock = ctx->h_stats[5];
    const u64 wbase = SH ? ctx->sh_wbase : ctx->h_stats[0];
    if (n_sync + 64 > 0xFFFFFFFFull) return IGD_ETOOBIG;  // 32-bit record positions
    // a4: accessed words spanning >= 2^32 words (sparse virtual addresses) take the wide path:
    // u64 keys word - kbase, sorted over ceil(bits(span) / 8) digit passes
    // A36 tag mode: keys = low (tag_log2 + 10) bits of the word (entry + Tag), sorted by the entry
    const u32 TG = SH ? 0u : ctx->tag_log2;
    const bool key64 = !SH && !TG && n_acc > 0 && ctx->h_stats[1] - ctx->h_stats[0] >= (1ull << 32);
    if (TG && !FUSED) {
        ctx->err = "the tag-aliasing mode needs the fused ingest pipeline";
        return IGD_EINVAL;
    }
    const u64 kbase = key64 ? (ctx->h_stats[0] & ~255ull) : 0;  // low digit unchanged: pass 0's histogram holds
    if (key64) {
        if (!FUSED) {
            ctx->err = "word spans >= 2^32 words need the fused ingest pipeline (IGD_FUSED=1)";
            return IGD_ETOOBIG;
        }
        for (int b = 0; b < 2; b++) RET(ensure(ctx, ctx->acc_k[b], acc_cap * sizeof(u64)));
    }
    if (ctx->sync_cap < n_sync) ctx->sync_cap = n_sync + n_sync / 8 + 4096;
    for (int b = 0; b < 2; b++) {
        // +64 entries: the check's 32-byte timestamp probes may read past the last list
        RET(ensure(ctx, ctx->syn_k[b], (ctx->sync_cap + 64) * sizeof(u32)));
        RET(ensure(ctx, ctx->syn_v[b], (ctx->sync_cap + 64) * sizeof(u32)));
    }
    ip.acc_key = SH ? nullptr : P_<u32>(ctx->acc_k[0]);
    ip.acc_val = SH ? nullptr : P_<u64>(ctx->acc_v[0]);
    ip.sync_key = P_<u32>(ctx->syn_k[0]);
    ip.sync_val = P_<u32>(ctx->syn_v[0]);
    ip.sync_cap = ctx->sync_cap;
    if (FUSED) {
        // one pass: sync records + accesses sorted by digit 0 (fused.cuh) into acc_*[1]
        const u64 ft = (n_src + fused::TILE - 1) / fused::TILE;
        {
            KTimer kt(ctx, KC_MISC, 0);
            rsort::k_digit_base<<<1, rsort::RADIX, 0, ctx->stream>>>(P_<u32>(ctx->hist), P_<u32>(ctx->base));
        }
        fused::Params fp;
        RET(next_digit_epoch(ctx, ft, &fp.epoch));
        CK(cudaMemsetAsync(ctx->ctr.p, 0, sizeof(u32), ctx->stream));
        fp.ev = src_ev;
        fp.n = n_src;
        fp.g = g;
        fp.ks = ks;
        fp.tile_sync = P_<u32>(ctx->st_in_s);
        fp.sync_key = P_<u32>(ctx->syn_k[0]);
        fp.sync_val = P_<u32>(ctx->syn_v[0]);
        fp.sync_cap = ctx->sync_cap;
        fp.digit_base = P_<u32>(ctx->base);
        fp.status = P_<u64>(ctx->dstatus);
        fp.tile_ctr = P_<u32>(ctx->ctr);
        fp.kout = ctx->acc_k[1].p;
        fp.kbase = kbase;
        fp.keymask = TG ? (u32)((1ull << (TG + 10)) - 1) : 0xFFFFFFFFu;
        fp.vout = P_<u64>(ctx->acc_v[1]);
        fp.skip_bits = ip.skip_bits;
        {
            // reads every event once, writes the 12-byte access records and 8-byte sync records
            KTimer kt(ctx, KC_FUSED, 16.0 * (double)n_src + 12.0 * (double)n_acc + 8.0 * (double)n_sync);
            if (key64) {
                const size_t sm64 = fused::smem_bytes<u64>();
                if (fp.skip_bits) fused::k_ingest_sort0<true, u64><<<(unsigned)ft, fused::THREADS, sm64, ctx->stream>>>(fp);
                else fused::k_ingest_sort0<false, u64><<<(unsigned)ft, fused::THREADS, sm64, ctx->stream>>>(fp);
            } else if (fp.skip_bits) {
                fused::k_ingest_sort0<true><<<(unsigned)ft, fused::THREADS, fused::smem_bytes(), ctx->stream>>>(fp);
            } else if (g.dlog < 32 && g.D >= 32) {  // power-of-two geometry (common case)
                fused::k_ingest_sort0<false, u32, true><<<(unsigned)ft, fused::THREADS, fused::smem_bytes(),
                                                          ctx->stream>>>(fp);
            } else {
                fused::k_ingest_sort0<false><<<(unsigned)ft, fused::THREADS, fused::smem_bytes(), ctx->stream>>>(fp);
            }
        }
        CK(cudaGetLastError());
    }
    if (n_src > 0 && !FUSED) {
        // pass 1 re-reads the events and writes the (key, value) records
        KTimer kt(ctx, KC_INGEST, 16.0 * (double)n_src + (SH ? 0.0 : 12.0 * (double)n_acc) + 8.0 * (double)n_sync);
        ingest::k_ingest<1><<<(unsigned)grid, ingest::THREADS, 0, ctx->stream>>>(ip);
    }
    CK(cudaGetLastError());
    if (SH && n_acc > 0) {
        const unsigned sb = (unsigned)std::min<u64>((n_acc + 255) / 256, (u64)sms * 8);
        if (SPLIT) {
            // received records {key, index, tk, mask} -> sort keys + (index | tk) payload and the
            // keys' digit histograms (12-byte sort elements, as on one GPU)
            KTimer kt(ctx, KC_INGEST, 28.0 * (double)n_acc);
            shard::k_record_split<<<sb, 256, 0, ctx->stream>>>((const uint4*)ctx->sh_rec, (u32)n_acc,
                                                              P_<u32>(ctx->acc_k[0]), P_<u64>(ctx->acc_v[0]),
                                                              P_<u32>(ctx->hist));
        } else {
            // the sort keys and their digit histograms; the records themselves are the payload
            // of the first radix pass
            KTimer kt(ctx, KC_INGEST, 20.0 * (double)n_acc);
            shard::k_record_keys<<<sb, 256, 0, ctx->stream>>>((const uint4*)ctx->sh_rec, (u32)n_acc,
                                                             P_<u32>(ctx->acc_k[0]), P_<u32>(ctx->hist));
        }
    }
    if (FUSED && IGD_HIST_UP_LATE && n_acc > 0) {
        KTimer kt(ctx, KC_INGEST, 4.0 * (double)n_acc);  // access-key digits 1..3
        const unsigned hb = (unsigned)std::min<u64>((n_acc / 4 + 255) / 256 + 1, (u64)sms * 8);
        ingest::k_hist_keys<<<hb, 256, 0, ctx->stream>>>(P_<u32>(ctx->acc_k[1]), (u32)n_acc, P_<u32>(ctx->hist), 1);
    }
    if (key64) {
        // wide keys: digit 0 is pass 0's (kbase has a zero low digit); digits 1..7 over the keys
        // the fused pass wrote
        CK(cudaMemsetAsync(P_<u32>(ctx->hist) + 2048, 0, 2048 * sizeof(u32), ctx->stream));
        CK(cudaMemcpyAsync(P_<u32>(ctx->hist) + 2048, ctx->hist.p, 256 * sizeof(u32), cudaMemcpyDeviceToDevice,
                           ctx->stream));
        KTimer kt(ctx, KC_INGEST, 8.0 * (double)n_acc);
        const unsigned hb = (unsigned)std::min<u64>((n_acc + 255) / 256, (u64)sms * 8);
        rsort::k_hist8<<<hb, 256, 0, ctx->stream>>>(P_<u64>(ctx->acc_k[1]), n_acc, P_<u32>(ctx->hist) + 2048, 1);
    }
    if (TG && n_acc > 0) {
        // tag mode: the sort runs over the entry bits only; digits 1..3 of the masked keys
        CK(cudaMemsetAsync(P_<u32>(ctx->hist) + 256, 0, 768 * sizeof(u32), ctx->stream));
        KTimer kt(ctx, KC_INGEST, 4.0 * (double)n_acc);
        const unsigned hb = (unsigned)std::min<u64>((n_acc / 4 + 255) / 256 + 1, (u64)sms * 8);
        ingest::k_hist_keys<<<hb, 256, 0, ctx->stream>>>(P_<u32>(ctx->acc_k[1]), (u32)n_acc, P_<u32>(ctx->hist), 1,
                                                         (u32)((1ull << TG) - 1));
    }
    if (FUSED && n_sync > 0) {
        // sync-key digit histograms over the records the fused pass wrote (trace order)
        KTimer kt(ctx, KC_INGEST, 4.0 * (double)n_sync);
        const unsigned hb = (unsigned)std::min<u64>((n_sync / 4 + 255) / 256 + 1, (u64)sms * 8);
        ingest::k_hist_keys<<<hb, 256, 0, ctx->stream>>>(P_<u32>(ctx->syn_k[0]), (u32)n_sync,
                                                         P_<u32>(ctx->hist) + 1024, 0);
    }
    if (n_acc > 0 && !FUSED && !SH) {  // fused: ingest pass 0 built them; sharded: k_record_keys
        KTimer kt(ctx, KC_INGEST, 4.0 * (double)n_acc);  // access-key digit histograms
        const unsigned hb = (unsigned)std::min<u64>((n_acc / 4 + 255) / 256 + 1, (u64)sms * 8);
        ingest::k_hist_keys<<<hb, 256, 0, ctx->stream>>>(P_<u32>(ctx->acc_k[0]), (u32)n_acc, P_<u32>(ctx->hist), 0);
    }
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(ctx->h_hist, ctx->hist.p, (FUSED ? 2048 : 1024) * sizeof(u32), cudaMemcpyDeviceToHost,
                       ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    mark(ctx, 1);
    u32 h_hist_acc[1024], h_hist_sync[1024];
    memcpy(h_hist_acc, ctx->h_hist, sizeof(h_hist_acc));
    memcpy(h_hist_sync, ctx->h_hist + 1024, sizeof(h_hist_sync));
    std::vector<u32> h_hist64;
    if (key64) {
        h_hist64.resize(2048);
        CK(cudaMemcpyAsync(ctx->h_hist + 2048, P_<u32>(ctx->hist) + 2048, 2048 * sizeof(u32), cudaMemcpyDeviceToHost,
                           ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        memcpy(h_hist64.data(), ctx->h_hist + 2048, 2048 * sizeof(u32));
    }

    // the a2 / a3 stages run concurrently with a5 (SideSection): their stage marks are taken
    // here on the context stream, so the "a5" stage time covers a2 + a3 + a5 (the per-kernel
    // class times still separate them)
    mark(ctx, 2);
    mark(ctx, 3);
    // Overlap only when the lock replay is substantial (>= 1 lock event per 1024 events, e.g. the
    // sync-heavy C5: 223 -> 216 ms): the overlapped kernels take SM slots from the sort, so for a
    // light a2 / a3 (default C5: 0.05 % lock events) the gain is ~1 ms and the sort runs 5 % slower
    // (r02s9); IGD_SIDE_STREAM=0 / 1 forces it off / on.
    static int side_env = -2;
    if (side_env == -2) {
        const char* e = getenv("IGD_SIDE_STREAM");
        side_env = e ? atoi(e) : -1;
    }
    SideSection side(ctx);
    RET(side.fork(side_env >= 0 ? side_env != 0 : n_lock * 1024 >= n_src));
    // ---------------- a5: accesses sorted by word, stable ----------------
    int acur = 0;
    if (key64)
        RET(radix_sort(ctx, KC_SORT_ACC, ctx->acc_k, ctx->acc_v, n_acc, P_<u32>(ctx->hist) + 2048, h_hist64.data(),
                       bits_needed(ctx->h_stats[1] - kbase), &acur, vbytes, 1, 1, nullptr, 8));
    else
        RET(radix_sort(ctx, KC_SORT_ACC, ctx->acc_k, ctx->acc_v, n_acc, P_<u32>(ctx->hist), h_hist_acc,
                       TG ? TG : 32u, &acur, vbytes, FUSED ? 1 : 0, FUSED ? 1 : 0,
                       (SH && !SPLIT) ? ctx->sh_rec : nullptr));
    RET(side.begin());
    // ---------------- a2: sync records sorted by entity, CSR offsets ----------------
    int scur = 0;
    ctx->last_nsync = 0;
    ctx->last_npts = 0;
    RET(radix_sort(ctx, KC_SORT_SYNC, ctx->syn_k, ctx->syn_v, n_sync, P_<u32>(ctx->hist) + 1024, h_hist_sync,
                   bits_needed(ks.E), &scur));
    // the check's 32-byte timestamp probes may read up to 64 entries past the last list: defined
    // values there (they are masked out of every decision; compute-sanitizer initcheck is clean)
    CK(cudaMemsetAsync(P_<u32>(ctx->syn_v[scur]) + n_sync, 0xFF, 64 * sizeof(u32), ctx->stream));
    RET(ensure(ctx, ctx->off, ((u64)ks.E + 2) * sizeof(u32)));
    {
        u64 work = (u64)ks.E + 1;
        unsigned blocks = (unsigned)std::min<u64>((work + 255) / 256, (u64)sms * 16);
        KTimer kt(ctx, KC_CSR, 4.0 * (double)work);
        syncx::k_csr_offsets<<<blocks, 256, 0, ctx->stream>>>(P_<u32>(ctx->syn_k[scur]), (u32)n_sync, ks.E,
                                                             P_<u32>(ctx->off));
        CK(cudaGetLastError());
    }
    RET(ensure(ctx, ctx->ldesc, ((u64)ks.E + 1) * sizeof(uint4)));
    {
        unsigned blocks = (unsigned)std::min<u64>(((u64)ks.E + 255) / 256, (u64)sms * 16);
        KTimer kt(ctx, KC_CSR, 24.0 * (double)ks.E);
        check::k_list_desc<<<blocks, 256, 0, ctx->stream>>>(P_<u32>(ctx->off), P_<u32>(ctx->syn_v[scur]), ks.E,
                                                           P_<uint4>(ctx->ldesc));
        CK(cudaGetLastError());
    }
    // grid-sync bucket table (<= 2^22 buckets, L2-resident)
    u32 glims[2] = {0, 0}, klims[2] = {0, 0};  // grid-sync list, kernel-boundary list
    CK(cudaMemcpyAsync(glims, P_<u32>(ctx->off) + ks.grid, 2 * sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(klims, P_<u32>(ctx->off) + ks.kb, 2 * sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    const u32 gshift = std::max<u32>(8, bits_needed(n) > 22 ? bits_needed(n) - 22 : 0);
    const u32 gnb = (u32)((n >> gshift) + 2);
    RET(ensure(ctx, ctx->gtab, (u64)gnb * sizeof(u64)));
    if (glims[1] > glims[0]) {
        unsigned blocks = (unsigned)std::min<u64>((gnb + 255) / 256, (u64)sms * 16);
        KTimer kt(ctx, KC_CSR, 8.0 * (double)gnb);
        check::k_grid_table<<<blocks, 256, 0, ctx->stream>>>(P_<u32>(ctx->syn_v[scur]), glims[0], glims[1], gshift,
                                                            gnb, P_<u64>(ctx->gtab));
        CK(cudaGetLastError());
    }
    // ---------------- a3: lock inference ----------------
    syncx::LockView lv;
    memset(&lv, 0, sizeof(lv));
    if (n_lock > 0) {
        RET(ensure(ctx, ctx->tcnt, ((u64)g.T + 1) * sizeof(u32)));
        CK(cudaMemsetAsync(ctx->tcnt.p, 0, ((u64)g.T + 1) * sizeof(u32), ctx->stream));
        syncx::LockParams lp;
        memset(&lp, 0, sizeof(lp));
        lp.ev = src_ev;
        lp.gidx = SH ? ctx->sh_sidx : nullptr;
        lp.gn = (u32)n_src;
        lp.g = g;
        lp.ks = ks;
        lp.off = P_<u32>(ctx->off);
        lp.sts = P_<u32>(ctx->syn_v[scur]);
        lp.tcnt = P_<u32>(ctx->tcnt);
        RET(ensure(ctx, ctx->fdev, n_sync + 64));
        {
            KTimer kt(ctx, KC_LOCK, 0);
            syncx::k_fence_scopes<<<(g.T + 255) / 256, 256, 0, ctx->stream>>>(P_<u32>(ctx->off),
                                                                             P_<u32>(ctx->syn_v[scur]), ks, g.T,
                                                                             P_<uint8_t>(ctx->fdev));
        }
        CK(cudaGetLastError());
        lp.fdev = P_<uint8_t>(ctx->fdev);
        const unsigned lblocks = (unsigned)(((u64)g.W * 32 + 255) / 256);
        {
            KTimer kt(ctx, KC_LOCK, 0);
            syncx::k_lock_infer<false><<<lblocks, 256, 0, ctx->stream>>>(lp);
        }
        CK(cudaGetLastError());
        RET(scan_excl(ctx, P_<u32>(ctx->tcnt), (u64)g.T + 1));
        u32 tot = 0;
        CK(cudaMemcpyAsync(&tot, P_<u32>(ctx->tcnt) + g.T, sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        RET(ensure(ctx, ctx->tpts, ((u64)tot + 1) * sizeof(u64)));
        lp.toff = P_<u32>(ctx->tcnt);
        lp.tpts = P_<u64>(ctx->tpts);
        {
            KTimer kt(ctx, KC_LOCK, 0);
            syncx::k_lock_infer<true><<<lblocks, 256, 0, ctx->stream>>>(lp);
        }
        CK(cudaGetLastError());
        lv.toff = P_<u32>(ctx->tcnt);
        lv.tpts = P_<u64>(ctx->tpts);
        lv.any = 1;
        RET(ensure(ctx, ctx->tbits, ((u64)g.T / 32 + 1) * sizeof(u32)));
        {
            KTimer kt(ctx, KC_LOCK, 4.0 * (double)g.T);
            const u32 nw = (g.T + 31) / 32;
            syncx::k_lock_bits<<<(nw + 255) / 256, 256, 0, ctx->stream>>>(P_<u32>(ctx->tcnt), g.T, P_<u32>(ctx->tbits));
        }
        CK(cudaGetLastError());
        lv.tbits = P_<u32>(ctx->tbits);
        ctx->last_npts = tot;
    }
    RET(side.end());
    ctx->last_acur = acur;
    ctx->last_scur = scur;
    ctx->last_nsync = n_sync;
    ctx->last_E = ks.E;
    ctx->last_T = g.T;
    ctx->last_nacc = SH ? 0 : n_acc;
    mark(ctx, 4);
    // ---------------- a6: segmented shadow pass + check ----------------
    if (ctx->rep_cap == 0) ctx->rep_cap = 1 << 20;
    u64 n_rep = 0;
    if (n_acc > 0) {
        const u64 ctile = check::C4_TILE;
        const u64 tiles = (n_acc + ctile - 1) / ctile;
        for (int attempt = 0;; attempt++) {
            RET(ensure(ctx, ctx->rep_raw, ctx->rep_cap * sizeof(igd_report)));
            RET(ensure(ctx, ctx->rep_ctr, 2 * sizeof(u64)));
            RET(ensure(ctx, ctx->status, tiles * sizeof(u64)));
            CK(cudaMemsetAsync(ctx->status.p, 0, tiles * sizeof(u64), ctx->stream));
            CK(cudaMemsetAsync(ctx->ctr.p, 0, sizeof(u32), ctx->stream));
            CK(cudaMemsetAsync(ctx->rep_ctr.p, 0, sizeof(u64), ctx->stream));
            check::Params cp;
            memset(&cp, 0, sizeof(cp));
            cp.key = ctx->acc_k[acur].p;
            cp.val = ctx->acc_v[acur].p;
            cp.wbase = key64 ? kbase : wbase;
            cp.n = (u32)n_acc;
            cp.ev = ev0;
            cp.g = g;
            cp.ks = ks;
            cp.desc = P_<uint4>(ctx->ldesc);
            cp.gtab = P_<u64>(ctx->gtab);
            cp.gshift = gshift;
            cp.glo = glims[0];
            cp.ghi = glims[1];
            cp.has_kb = klims[1] > klims[0] ? 1u : 0u;
            cp.sts = P_<u32>(ctx->syn_v[scur]);
            cp.lv = lv;
            cp.status = P_<u64>(ctx->status);
            cp.tile_ctr = P_<u32>(ctx->ctr);
            cp.rep = P_<igd_report>(ctx->rep_raw);
            cp.rep_cap = ctx->rep_cap;
            cp.rep_ctr = P_<unsigned long long>(ctx->rep_ctr);
            cp.first_event = first;
            cp.addr_from_ev = TG ? 1u : 0u;
            const u32 LK = SH ? 1u : ctx->last_k;
            if (LK > 1) {  // A37: the scan state per access, then the candidates per access
                RET(ensure(ctx, ctx->lk_state, n_acc * sizeof(u64)));
                cp.st_out = P_<u64>(ctx->lk_state);
            }
            {
                // key + payload streamed (12 or 20 bytes per access)
                KTimer kt(ctx, KC_CHECK, (4.0 + vbytes) * (double)n_acc);
                if (SH && ctx->str_active) {  // streaming mode (f4)
                    cp.carry_before = (u32)ctx->str_n;
                    cp.carry_out = ctx->str_co.p;
                }
                if (SPLIT) {  // the active mask of an access, when needed, from the received records
                    cp.rec = reinterpret_cast<const uint4*>(ctx->sh_rec);
                    cp.nrec = (u32)n_acc;
                }
                launch_check(SH && !SPLIT, cp.has_kb != 0,
                             (ctx->paper_counters ? 1 : 0) | (ctx->sticky ? 2 : 0) | (LK > 1 ? 4 : 0) |
                                 (SH && ctx->str_active ? 8 : 0),
                             key64, (unsigned)tiles, ctx->stream, cp);
            }
            CK(cudaGetLastError());
            if (LK > 1) {
                lastk::Params lp2;
                lp2.C = cp;
                lp2.C.st_out = nullptr;
                lp2.st = P_<u64>(ctx->lk_state);
                lp2.k = LK;
                const unsigned lb = (unsigned)((n_acc + 255) / 256);
                KTimer kt(ctx, KC_CHECK, 20.0 * (double)n_acc);
                const bool W = ctx->paper_counters, T = ctx->sticky;
                if (key64) {
                    if (W && T) lastk::k_lastk<true, true, u64><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else if (W) lastk::k_lastk<true, false, u64><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else if (T) lastk::k_lastk<false, true, u64><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else lastk::k_lastk<false, false, u64><<<lb, 256, 0, ctx->stream>>>(lp2);
                } else {
                    if (W && T) lastk::k_lastk<true, true, u32><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else if (W) lastk::k_lastk<true, false, u32><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else if (T) lastk::k_lastk<false, true, u32><<<lb, 256, 0, ctx->stream>>>(lp2);
                    else lastk::k_lastk<false, false, u32><<<lb, 256, 0, ctx->stream>>>(lp2);
                }
                CK(cudaGetLastError());
            }
            CK(cudaMemcpyAsync(ctx->h_small, ctx->rep_ctr.p, sizeof(u64), cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaStreamSynchronize(ctx->stream));
            n_rep = ctx->h_small[0];
            if (n_rep <= ctx->rep_cap) break;
            ctx->rep_cap = n_rep + n_rep / 8;
            if (attempt > 2) return IGD_ECUDA;
        }
    }
    mark(ctx, 5);
    // ---------------- a7: canonical order (ascending cur) ----------------
    RET(canon_reports(ctx, P_<igd_report>(ctx->rep_raw), n_rep, first + n));
    mark(ctx, 6);
    CK(cudaStreamSynchronize(ctx->stream));
    mark(ctx, 7);
    mark(ctx, 8);
    ctx->n_reports = n_rep;
    *n_out = n_rep;
    return IGD_OK;
}

// ---------------- sharded mode, stage 1: partition one rank's chunk ----------------
static int shard_prepare_impl(igd_ctx* ctx, u32 P, u64* counts, u64* n_sync_stream, u64* bad, u64* minmax) {
    const igd_trace_desc& D = ctx->desc;
    const u64 n = D.n_events;
    Geo g;
    geo_init(g, D.n_blocks, D.block_dim);
    KeySpace ks;
    ks.init(g);
    const int sms = sm_count(ctx);
    const u64 tiles = (n + shard::TILE - 1) / shard::TILE;
    const u64 row = tiles + 1;
    RET(ensure(ctx, ctx->stats, 8 * sizeof(u64)));
    RET(ensure(ctx, ctx->ctr, 64));
    RET(ensure(ctx, ctx->sh_cnt, (P + 1) * row * sizeof(u32)));
    RET(ensure(ctx, ctx->sh_obase, (P + 1) * sizeof(u64)));
    u64 init[8] = {~0ull, 0, ~0ull, 0, 0, 0, 0, 0};
    memcpy(ctx->h_small, init, sizeof(init));
    CK(cudaMemcpyAsync(ctx->stats.p, ctx->h_small, sizeof(init), cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaMemsetAsync(ctx->sh_cnt.p, 0, (P + 1) * row * sizeof(u32), ctx->stream));
    shard::Params sp;
    memset(&sp, 0, sizeof(sp));
    sp.ev = ctx->events;
    sp.n = n;
    sp.first = D.first_event;
    sp.g = g;
    sp.ks = ks;
    sp.P = P;
    sp.n_tiles = (u32)tiles;
    sp.cnt = P_<u32>(ctx->sh_cnt);
    sp.stats = P_<u64>(ctx->stats);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, shard::k_shard<0>, shard::THREADS, 0);
    const u64 grid = std::max<u64>(1, std::min<u64>((u64)sms * (occ > 0 ? occ : 1), tiles));
    if (n > 0) {
        KTimer kt(ctx, KC_INGEST, 16.0 * (double)n);
        shard::k_shard<0><<<(unsigned)grid, shard::THREADS, 0, ctx->stream>>>(sp);
    }
    CK(cudaGetLastError());
    for (u32 o = 0; o <= P; o++) RET(scan_excl(ctx, P_<u32>(ctx->sh_cnt) + (u64)o * row, row));
    std::vector<u32> tot(P + 1);
    for (u32 o = 0; o <= P; o++)
        CK(cudaMemcpyAsync(&tot[o], P_<u32>(ctx->sh_cnt) + (u64)o * row + tiles, sizeof(u32), cudaMemcpyDeviceToHost,
                           ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_stats, ctx->stats.p, 8 * sizeof(u64), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    bad[0] = ctx->h_stats[2];
    minmax[0] = ctx->h_stats[0];
    minmax[1] = ctx->h_stats[1];
    if (ctx->h_stats[3] && bad[0] == ~0ull) {
        ctx->err = "kernel boundaries that change the grid (reading A34) need a single-GPU context";
        return IGD_EINVAL;
    }
    std::vector<u64> ob(P + 1, 0);
    u64 nrec = 0;
    for (u32 o = 0; o < P; o++) {
        counts[o] = tot[o];
        ob[o] = nrec;
        nrec += tot[o];
    }
    *n_sync_stream = tot[P];
    ctx->sh_send_n = nrec;
    ctx->sh_sync_n = tot[P];
    RET(ensure(ctx, ctx->sh_send, (nrec + 1) * sizeof(uint4)));
    RET(ensure(ctx, ctx->sh_sidx_buf, ((u64)tot[P] + 1) * sizeof(u32)));
    RET(ensure(ctx, ctx->sh_sev_buf, ((u64)tot[P] + 1) * sizeof(uint4)));
    if (bad[0] != ~0ull) return IGD_OK;  // the caller reduces the error across ranks
    CK(cudaMemcpyAsync(ctx->sh_obase.p, ob.data(), (P + 1) * sizeof(u64), cudaMemcpyHostToDevice, ctx->stream));
    sp.obase = P_<u64>(ctx->sh_obase);
    sp.send = P_<uint4>(ctx->sh_send);
    sp.sync_idx = P_<u32>(ctx->sh_sidx_buf);
    sp.sync_ev = P_<uint4>(ctx->sh_sev_buf);
    if (n > 0) {
        KTimer kt(ctx, KC_INGEST, 16.0 * (double)n + 16.0 * (double)nrec + 20.0 * (double)tot[P]);
        shard::k_shard<1><<<(unsigned)grid, shard::THREADS, 0, ctx->stream>>>(sp);
    }
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(ctx->stream));
    return IGD_OK;
}

// ---------------- per-kernel geometry (reading A34) ----------------
// A KERNEL_BOUNDARY with a nonzero addr starts a kernel on another grid.  Every word's shadow
// state and every lock table end at a boundary (A31), so the trace is exactly the concatenation
// of its segments between such boundaries, each checked on its own grid (the composition law the
// oracle is pinned by).  Pass 0 of the whole-trace run listed the boundaries; each segment is then
// a full pipeline run with shifted indices, its reports appended in order (canonical by
// construction).  The boundary events themselves are validated here, in trace order with the
// segments, so the first invalid index is the oracle's.
static int segmented_detect(igd_ctx* ctx, u64* n_out) {
    const u64 ng = ctx->h_stats[6];
    const u64 cap = ctx->gkb.cap / sizeof(u64);
    if (ng > cap) {  // more grid changes than the list holds: a larger list, one more pass 0
        RET(ensure(ctx, ctx->gkb, (ng + 1) * sizeof(u64)));
        ctx->in_segment = false;
        u64 dummy = 0;
        int rc = detect_impl(ctx, &dummy);
        if (rc != IGD_SEGMENTS_NEEDED) return rc == IGD_OK ? IGD_ECUDA : rc;
    }
    std::vector<u64> kb(ng);
    CK(cudaMemcpyAsync(kb.data(), ctx->gkb.p, ng * sizeof(u64), cudaMemcpyDeviceToHost, ctx->stream));
    std::vector<igd_event> kev(ng);
    CK(cudaStreamSynchronize(ctx->stream));
    std::sort(kb.begin(), kb.end());
    for (u64 k = 0; k < ng; k++)
        CK(cudaMemcpyAsync(&kev[k], ctx->events + kb[k], sizeof(igd_event), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    const u64 N = ctx->desc.n_events;
    u32 nb = ctx->desc.n_blocks, bd = ctx->desc.block_dim;
    u64 total = 0, start = 0;
    for (u64 k = 0; k <= ng; k++) {
        const u64 end = k < ng ? kb[k] : N;
        if (end > start) {
            ctx->in_segment = true;
            ctx->seg_ev = ctx->events + start;
            ctx->seg_n = end - start;
            ctx->seg_first = start;
            ctx->seg_nb = nb;
            ctx->seg_bd = bd;
            u64 nk = 0;
            int rc = detect_impl(ctx, &nk);
            ctx->in_segment = false;
            if (rc != IGD_OK) return rc;
            if (nk) {
                // append (a grown buffer keeps the earlier segments' reports)
                if (ctx->seg_rep.cap < (total + nk) * sizeof(igd_report)) {
                    Buf nb2;
                    std::swap(nb2, ctx->seg_rep);
                    RET(ensure(ctx, ctx->seg_rep, (total + nk) * 2 * sizeof(igd_report)));
                    if (total)
                        CK(cudaMemcpyAsync(ctx->seg_rep.p, nb2.p, total * sizeof(igd_report), cudaMemcpyDeviceToDevice,
                                           ctx->stream));
                    RET(buf_free(ctx, nb2));
                }
                CK(cudaMemcpyAsync((char*)ctx->seg_rep.p + total * sizeof(igd_report), ctx->rep_out.p,
                                   nk * sizeof(igd_report), cudaMemcpyDeviceToDevice, ctx->stream));
                total += nk;
            }
        }
        if (k == ng) break;
        // the boundary itself: KERNEL_BOUNDARY, tid 0, scope NONE, a valid grid code
        const igd_event& e = kev[k];
        const u32 kind = (e.tk >> 24) & 0xFu, tid = e.tk & 0xFFFFFFu, scope = (e.tk >> 28) & 3u;
        const u32 nnb = (u32)(e.addr >> 32), nbd = (u32)e.addr;
        if ((e.tk >> 30) || kind != IGD_KERNEL_BOUNDARY || tid != 0 || scope != 0 || !geo_code_ok(nnb, nbd)) {
            ctx->bad_event = kb[k];
            ctx->err = "invalid event at index " + std::to_string(kb[k]);
            return IGD_ETRACE;
        }
        nb = nnb;
        bd = nbd;
        start = kb[k] + 1;
    }
    std::swap(ctx->seg_rep, ctx->rep_out);  // rep_out: all segments' reports, ascending cur
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->n_reports = total;
    *n_out = total;
    return IGD_OK;
}

// ---------------- streaming sessions ----------------
// A producer (e.g. an instrumentation runtime draining per-warp buffers)
// hands over a trace in consecutive chunks.  Each chunk is checked as soon as it arrives and its
// reports are final: the union over the chunks is exactly the whole-trace result.  Carried
// between chunks: the synchronization stream so far (epoch tables and lock replay are rebuilt
// over it, so interval queries reaching into earlier chunks stay exact), and per accessed word
// two records {a head record (its last writer when that is not its last accessor, else a
// neutral load), its last accessor with the word's sticky DevShared / BlkShared and the scope of
// its last atomic}.  The chunk's access records follow the carried ones into the sharded-mode
// pipeline (stable sort by word keeps carried state before new accesses), the check skips the
// carried records and writes the next carried pairs.
static int grow_keep(igd_ctx* ctx, Buf& b, size_t used, size_t want) {
    if (b.cap >= want) return IGD_OK;
    Buf nb;
    RET(ensure(ctx, nb, want + want / 2));
    if (used) CK(cudaMemcpyAsync(nb.p, b.p, used, cudaMemcpyDeviceToDevice, ctx->stream));
    RET(buf_free(ctx, b));
    b = nb;
    return IGD_OK;
}

static int stream_feed_impl(igd_ctx* ctx, const igd_event* events, u64 n, u32 ev_flags, u64* n_out) {
    *n_out = 0;
    ctx->n_reports = 0;
    ctx->launches = 0;
    ctx->nk = 0;
    igd_trace_desc d{};
    d.n_blocks = ctx->str_nb;
    d.block_dim = ctx->str_bd;
    d.first_event = ctx->str_n;
    d.n_events = n;
    d.n_events_total = ctx->str_n + n;
    d.flags = ev_flags;
    if (d.n_events_total > 0xFFFFFFFFull - 2 * rsort::TILE) return IGD_ETOOBIG;
    RET(igd_trace_load(ctx, &d, events));
    u64 counts[2] = {0, 0}, nsync = 0, bad = ~0ull, mm[2] = {~0ull, 0};
    RET(shard_prepare_impl(ctx, 1, counts, &nsync, &bad, mm));
    if (bad != ~0ull) {
        ctx->bad_event = bad;
        ctx->err = "invalid event at index " + std::to_string(bad);
        return IGD_ETRACE;
    }
    const u64 nrec = counts[0];
    const u64 wmin = std::min(ctx->str_wmin, mm[0]), wmax = nrec ? std::max(ctx->str_wmax, mm[1]) : ctx->str_wmax;
    if (wmin != ~0ull && wmax - wmin >= (1ull << 32)) {
        ctx->err = "a streaming session's words must span < 2^32 words";
        return IGD_ETOOBIG;
    }
    // the synchronization stream so far
    RET(grow_keep(ctx, ctx->str_sidx, ctx->str_nsync * sizeof(u32), (ctx->str_nsync + nsync + 1) * sizeof(u32)));
    RET(grow_keep(ctx, ctx->str_sev, ctx->str_nsync * 16, (ctx->str_nsync + nsync + 1) * 16));
    if (nsync) {
        CK(cudaMemcpyAsync(P_<u32>(ctx->str_sidx) + ctx->str_nsync, ctx->sh_sidx_buf.p, nsync * sizeof(u32),
                           cudaMemcpyDeviceToDevice, ctx->stream));
        CK(cudaMemcpyAsync((char*)ctx->str_sev.p + ctx->str_nsync * 16, ctx->sh_sev_buf.p, nsync * 16,
                           cudaMemcpyDeviceToDevice, ctx->stream));
    }
    const u64 nsy = ctx->str_nsync + nsync;
    // carried records, then the chunk's records (trace order)
    const u64 nc = ctx->str_ncarry, nall = nc + nrec;
    if (nall > 0xFFFFFFFFull - 2 * rsort::TILE || nsy + 64 > 0xFFFFFFFFull) return IGD_ETOOBIG;
    RET(ensure(ctx, ctx->str_rec, (nall + 1) * 16));
    if (nc) CK(cudaMemcpyAsync(ctx->str_rec.p, ctx->str_carry[ctx->str_cur].p, nc * 16, cudaMemcpyDeviceToDevice,
                               ctx->stream));
    if (nrec) CK(cudaMemcpyAsync((char*)ctx->str_rec.p + nc * 16, ctx->sh_send.p, nrec * 16, cudaMemcpyDeviceToDevice,
                                 ctx->stream));
    RET(buf_free(ctx, ctx->sh_send));
    RET(ensure(ctx, ctx->str_co, (2 * nall + 2) * 16));
    ctx->shard = true;
    ctx->sh_rec = ctx->str_rec.p;
    ctx->sh_nrec = nall;
    ctx->sh_sidx = P_<u32>(ctx->str_sidx);
    ctx->sh_sev = ctx->str_sev.p;
    ctx->sh_ns = nsy;
    ctx->sh_wbase = wmin == ~0ull ? 0 : wmin;
    ctx->sh_ntotal = d.n_events_total;
    u64 nrep = 0;
    int rc = detect_impl(ctx, &nrep);
    ctx->shard = false;
    if (rc != IGD_OK) return rc;
    // the next carried pairs (in key order)
    if (nall) {
        RET(ensure(ctx, ctx->str_flags, (nall + 1) * sizeof(u32)));
        const int sms = sm_count(ctx);
        const unsigned blocks = (unsigned)std::min<u64>((nall + 256) / 256, (u64)sms * 16);
        {
            KTimer kt(ctx, KC_MISC, 0);
            check::k_carry_flags<<<blocks, 256, 0, ctx->stream>>>(reinterpret_cast<const uint4*>(ctx->str_co.p),
                                                                 (u32)nall, P_<u32>(ctx->str_flags));
        }
        RET(scan_excl(ctx, P_<u32>(ctx->str_flags), nall + 1));
        u32 kept = 0;
        CK(cudaMemcpyAsync(&kept, P_<u32>(ctx->str_flags) + nall, sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        Buf& out = ctx->str_carry[ctx->str_cur ^ 1];
        RET(ensure(ctx, out, ((u64)kept * 2 + 1) * 16));
        {
            KTimer kt(ctx, KC_MISC, 0);
            check::k_carry_scatter<<<blocks, 256, 0, ctx->stream>>>(reinterpret_cast<const uint4*>(ctx->str_co.p),
                                                                   P_<u32>(ctx->str_flags), (u32)nall,
                                                                   reinterpret_cast<uint4*>(out.p));
        }
        CK(cudaGetLastError());
        ctx->str_cur ^= 1;
        ctx->str_ncarry = (u64)kept * 2;
    }
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->str_nsync = nsy;
    ctx->str_n += n;
    ctx->str_wmin = wmin;
    ctx->str_wmax = wmax;
    ctx->n_reports = nrep;
    *n_out = nrep;
    return IGD_OK;
}

// ---------------- the collective transport ----------------
// Four collectives carry the multi-GPU check.  With an NCCL communicator they are NCCL calls on
// the context stream.  An id starting with "IGDLOOP:" instead selects the in-process loopback
// transport: the P contexts of one process (driven by P host threads) meet at a barrier and copy
// from each other's device buffers -- the same exchange pattern, testable on a one-GPU box, where
// NCCL refuses two ranks on one device.
namespace {
struct LoopGroup {
    int P = 0, refs = 0;
    std::mutex m;
    std::condition_variable cv;
    int arrived = 0;
    u64 gen = 0;
    std::vector<const char*> base;      // per rank: the posted send buffer
    std::vector<std::vector<u64>> off, len;  // per rank: per peer offset / bytes in that buffer
    std::vector<u64> red;               // per rank x 8: all-reduce contributions
};
std::mutex g_loop_m;
std::map<std::string, LoopGroup*> g_loops;

LoopGroup* loop_join(const std::string& name, int P) {
    std::lock_guard<std::mutex> lk(g_loop_m);
    LoopGroup*& g = g_loops[name];
    if (!g) {
        g = new LoopGroup();
        g->P = P;
        g->base.assign(P, nullptr);
        g->off.assign(P, std::vector<u64>(P, 0));
        g->len.assign(P, std::vector<u64>(P, 0));
        g->red.assign((size_t)P * 8, 0);
    }
    if (g->P != P) return nullptr;
    g->refs++;
    return g;
}
void loop_leave(LoopGroup* g) {
    std::lock_guard<std::mutex> lk(g_loop_m);
    if (--g->refs == 0) {
        for (auto it = g_loops.begin(); it != g_loops.end(); ++it)
            if (it->second == g) {
                g_loops.erase(it);
                break;
            }
        delete g;
    }
}
void loop_barrier(LoopGroup* g) {
    std::unique_lock<std::mutex> lk(g->m);
    const u64 my = g->gen;
    if (++g->arrived == g->P) {
        g->arrived = 0;
        g->gen++;
        g->cv.notify_all();
    } else {
        g->cv.wait(lk, [&] { return g->gen != my; });
    }
}
}  // namespace

// min-all-reduce of n <= 8 u64 values in device memory (in place)
static int coll_allreduce_min(igd_ctx* ctx, u64* dbuf, int n) {
    if (ctx->comm) {
        NK(nccl().AllReduce(dbuf, dbuf, n, ncclUint64, ncclMin, ctx->comm, ctx->stream));
        return IGD_OK;
    }
    LoopGroup* g = ctx->loop;
    u64 v[8];
    CK(cudaMemcpyAsync(v, dbuf, n * sizeof(u64), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    for (int k = 0; k < n; k++) g->red[(size_t)ctx->rank * 8 + k] = v[k];
    loop_barrier(g);
    for (int k = 0; k < n; k++) {
        u64 m = ~0ull;
        for (int r = 0; r < g->P; r++) m = std::min(m, g->red[(size_t)r * 8 + k]);
        v[k] = m;
    }
    loop_barrier(g);  // every rank has read the contributions
    CK(cudaMemcpyAsync(dbuf, v, n * sizeof(u64), cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return IGD_OK;
}

// all-to-all(v): send[q] = bytes [soff[q], soff[q] + slen[q]) of sbase for rank q; the bytes from
// rank q land at rbase + roff[q] (rlen[q] of them).  Every buffer is device memory.
static int coll_alltoallv(igd_ctx* ctx, const void* sbase, const u64* soff, const u64* slen, void* rbase,
                          const u64* roff, const u64* rlen) {
    const int P = ctx->nranks, me = ctx->rank;
    if (ctx->comm) {
        NcclApi& N = nccl();
        NK(N.GroupStart());
        for (int q = 0; q < P; q++) {
            if (slen[q]) NK(N.Send((const char*)sbase + soff[q], slen[q], ncclUint8, q, ctx->comm, ctx->stream));
            if (rlen[q]) NK(N.Recv((char*)rbase + roff[q], rlen[q], ncclUint8, q, ctx->comm, ctx->stream));
        }
        NK(N.GroupEnd());
        return IGD_OK;
    }
    LoopGroup* g = ctx->loop;
    CK(cudaStreamSynchronize(ctx->stream));  // the send buffer is complete
    g->base[me] = (const char*)sbase;
    for (int q = 0; q < P; q++) {
        g->off[me][q] = soff[q];
        g->len[me][q] = slen[q];
    }
    loop_barrier(g);
    int rc = IGD_OK;
    for (int q = 0; q < P && rc == IGD_OK; q++) {
        if (g->len[q][me] != rlen[q]) rc = IGD_ECUDA;  // counts disagree: a transport bug
        else if (rlen[q] && cudaMemcpyAsync((char*)rbase + roff[q], g->base[q] + g->off[q][me], rlen[q],
                                            cudaMemcpyDefault, ctx->stream) != cudaSuccess)
            rc = IGD_ECUDA;
    }
    if (cudaStreamSynchronize(ctx->stream) != cudaSuccess) rc = IGD_ECUDA;
    loop_barrier(g);  // every rank has copied out of the posted buffers
    if (rc != IGD_OK) ctx->err = "loopback all-to-all failed";
    return rc;
}

// all-gather(v): rank q's slen bytes at sbase land at rbase + roff[q] on every rank (rlen[q] each)
static int coll_allgatherv(igd_ctx* ctx, const void* sbase, u64 slen, void* rbase, const u64* roff,
                           const u64* rlen) {
    const int P = ctx->nranks, me = ctx->rank;
    if (ctx->comm) {
        NcclApi& N = nccl();
        NK(N.GroupStart());
        for (int q = 0; q < P; q++) {
            if (!rlen[q]) continue;
            char* d = (char*)rbase + roff[q];
            NK(N.Broadcast(q == me ? sbase : d, d, rlen[q], ncclUint8, q, ctx->comm, ctx->stream));
        }
        NK(N.GroupEnd());
        return IGD_OK;
    }
    std::vector<u64> so(P, 0), sl(P, slen), ro(roff, roff + P), rl(rlen, rlen + P);
    return coll_alltoallv(ctx, sbase, so.data(), sl.data(), rbase, ro.data(), rl.data());
}

// ---------------- multi-GPU collective check ----------------
// Every rank holds the contiguous global range [first_event, first_event + n_events) of one trace.
// 1. partition the chunk: access records grouped by owner rank fmix32(word) % P, and the
//    synchronization stream (shard_prepare_impl);
// 2. NCCL: one all-reduce of {first bad index, min word, ~max word, local error} (min), an
//    all-gather of every rank's per-owner record counts and sync-stream length;
// 3. NCCL: all-to-all of the record groups (grouped send / recv: received groups land in
//    source-rank order = trace order, so the stable radix sort keeps (word, time) order) and the
//    sync streams of all ranks broadcast into one global stream (rank order = trace order);
// 4. the words this rank owns are checked against the rebuilt global sync / lock tables
//    (detect_impl, sharded mode);
// 5. NCCL: every rank's reports are broadcast to all, then merged by `cur` (a7).
// Every rank returns the same global report set.  Errors found by any rank (bad event, word span,
// a local allocation failure) are agreed through step 2, so no rank is left inside a collective.
static int collective_detect(igd_ctx* ctx, u64* n_out) {
    const u32 P = (u32)ctx->nranks, me = (u32)ctx->rank;
    cudaStream_t st = ctx->stream;
    *n_out = 0;
    ctx->n_reports = 0;
    ctx->launches = 0;
    ctx->nk = 0;
    std::vector<u64> counts(P + 1, 0);
    u64 nsync = 0, bad = ~0ull, mm[2] = {~0ull, 0};
    RET(ensure(ctx, ctx->cl_small, 8 * sizeof(u64)));
    int lrc = shard_prepare_impl(ctx, P, counts.data(), &nsync, &bad, mm);
    u64 small[4] = {bad, mm[0], mm[0] == ~0ull ? ~0ull : ~mm[1], lrc == IGD_OK ? ~0ull : (u64)(-lrc)};
    CK(cudaMemcpyAsync(ctx->cl_small.p, small, sizeof(small), cudaMemcpyHostToDevice, st));
    RET(coll_allreduce_min(ctx, P_<u64>(ctx->cl_small), 4));
    CK(cudaMemcpyAsync(small, ctx->cl_small.p, sizeof(small), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (small[3] != ~0ull) {
        if (lrc == IGD_OK) ctx->err = "another rank failed in the partition stage (" + std::to_string(-(int64_t)small[3]) + ")";
        return -(int)small[3];
    }
    if (small[0] != ~0ull) {
        ctx->bad_event = small[0];
        ctx->err = "invalid event at global index " + std::to_string(small[0]);
        return IGD_ETRACE;
    }
    const bool any_acc = small[1] != ~0ull;
    const u64 wmin = any_acc ? small[1] : 0, wmax = any_acc ? ~small[2] : 0;
    if (any_acc && wmax - wmin >= (1ull << 32)) {
        ctx->err = "accessed word range spans >= 2^32 words";
        return IGD_ETOOBIG;
    }
    // count matrix: row r = rank r's records per owner, then its sync-stream length
    const u64 W = P + 1;
    RET(ensure(ctx, ctx->cl_mat, (W * P + W) * sizeof(u64)));
    counts[P] = nsync;
    CK(cudaMemcpyAsync(P_<u64>(ctx->cl_mat) + W * P, counts.data(), W * sizeof(u64), cudaMemcpyHostToDevice, st));
    {
        std::vector<u64> ro(P), rl(P, W * sizeof(u64));
        for (u32 r = 0; r < P; r++) ro[r] = (u64)r * W * sizeof(u64);
        RET(coll_allgatherv(ctx, P_<u64>(ctx->cl_mat) + W * P, W * sizeof(u64), ctx->cl_mat.p, ro.data(), rl.data()));
    }
    std::vector<u64> M(W * P);
    CK(cudaMemcpyAsync(M.data(), ctx->cl_mat.p, W * P * sizeof(u64), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    std::vector<u64> soff(P + 1, 0), roff(P + 1, 0), yoff(P + 1, 0);
    for (u32 r = 0; r < P; r++) {
        soff[r + 1] = soff[r] + M[me * W + r];  // my records for owner r
        roff[r + 1] = roff[r] + M[r * W + me];  // records rank r sends me
        yoff[r + 1] = yoff[r] + M[r * W + P];   // rank r's sync stream
    }
    const u64 nrecv = roff[P], nsy = yoff[P];
    if (nsy + 64 > 0xFFFFFFFFull || nrecv > 0xFFFFFFFFull - 2 * rsort::TILE) return IGD_ETOOBIG;
    RET(ensure(ctx, ctx->cl_recv, (nrecv + 1) * 16));
    RET(ensure(ctx, ctx->cl_sidx, (nsy + 1) * sizeof(u32)));
    RET(ensure(ctx, ctx->cl_sev, (nsy + 1) * 16));
    {
        // all-to-all of the access records (received groups in source-rank order = trace order)
        std::vector<u64> so(P), sl(P), rof(P), rl(P);
        for (u32 r = 0; r < P; r++) {
            so[r] = soff[r] * 16;
            sl[r] = M[me * W + r] * 16;
            rof[r] = roff[r] * 16;
            rl[r] = M[r * W + me] * 16;
        }
        RET(coll_alltoallv(ctx, ctx->sh_send.p, so.data(), sl.data(), ctx->cl_recv.p, rof.data(), rl.data()));
        // the synchronization streams, concatenated in rank order (a variable all-gather)
        std::vector<u64> io(P), il(P), eo(P), el(P);
        for (u32 r = 0; r < P; r++) {
            io[r] = yoff[r] * sizeof(u32);
            il[r] = M[r * W + P] * sizeof(u32);
            eo[r] = yoff[r] * 16;
            el[r] = M[r * W + P] * 16;
        }
        RET(coll_allgatherv(ctx, ctx->sh_sidx_buf.p, nsync * sizeof(u32), ctx->cl_sidx.p, io.data(), il.data()));
        RET(coll_allgatherv(ctx, ctx->sh_sev_buf.p, nsync * 16, ctx->cl_sev.p, eo.data(), el.data()));
    }
    RET(buf_free(ctx, ctx->sh_send));  // stream-ordered: after the sends
    // the words this rank owns
    ctx->shard = true;
    ctx->sh_rec = ctx->cl_recv.p;
    ctx->sh_nrec = nrecv;
    ctx->sh_sidx = P_<u32>(ctx->cl_sidx);
    ctx->sh_sev = ctx->cl_sev.p;
    ctx->sh_ns = nsy;
    ctx->sh_wbase = wmin;
    ctx->sh_ntotal = ctx->desc.n_events_total ? ctx->desc.n_events_total : ctx->desc.n_events;
    u64 nloc = 0;
    lrc = detect_impl(ctx, &nloc);
    ctx->shard = false;
    // agree on success, then every rank's reports to every rank
    RET(ensure(ctx, ctx->cl_nrep, 2 * P * sizeof(u64)));
    u64 mine[2] = {lrc == IGD_OK ? nloc : 0, lrc == IGD_OK ? 0 : (u64)(-lrc)};
    CK(cudaMemcpyAsync(P_<u64>(ctx->cl_nrep) + 2 * me, mine, sizeof(mine), cudaMemcpyHostToDevice, st));
    {
        std::vector<u64> ro(P), rl(P, 2 * sizeof(u64));
        for (u32 r = 0; r < P; r++) ro[r] = (u64)r * 2 * sizeof(u64);
        RET(coll_allgatherv(ctx, P_<u64>(ctx->cl_nrep) + 2 * me, 2 * sizeof(u64), ctx->cl_nrep.p, ro.data(),
                            rl.data()));
    }
    std::vector<u64> NR(2 * P);
    CK(cudaMemcpyAsync(NR.data(), ctx->cl_nrep.p, 2 * P * sizeof(u64), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    for (u32 r = 0; r < P; r++)
        if (NR[2 * r + 1]) {
            if (lrc == IGD_OK) ctx->err = "rank " + std::to_string(r) + " failed in the check stage";
            return -(int)NR[2 * r + 1];
        }
    std::vector<u64> off(P + 1, 0);
    for (u32 r = 0; r < P; r++) off[r + 1] = off[r] + NR[2 * r];
    const u64 total = off[P];
    if (P > 1) {
        RET(ensure(ctx, ctx->cl_rep, (total ? total : 1) * sizeof(igd_report)));
        std::vector<u64> ro(P), rl(P);
        for (u32 r = 0; r < P; r++) {
            ro[r] = off[r] * sizeof(igd_report);
            rl[r] = NR[2 * r] * sizeof(igd_report);
        }
        RET(coll_allgatherv(ctx, ctx->rep_out.p, nloc * sizeof(igd_report), ctx->cl_rep.p, ro.data(), rl.data()));
        RET(canon_reports(ctx, P_<igd_report>(ctx->cl_rep), total, ctx->sh_ntotal));
    }
    CK(cudaStreamSynchronize(st));
    ctx->n_reports = total;
    *n_out = total;
    return IGD_OK;
}

// ================================ C ABI =====================================================
extern "C" {

int igd_ctx_create(igd_ctx** out, int cuda_device, void* cuda_stream, int nranks, int rank,
                   const uint8_t* nccl_unique_id, igd_alloc_fn alloc_fn, igd_free_fn free_fn, void* alloc_user) {
    if (!out) return IGD_EINVAL;
    *out = nullptr;
    if (nranks < 1 || rank < 0 || rank >= nranks) return IGD_EINVAL;
    if (nranks > 1 && !nccl_unique_id) return IGD_EINVAL;
    if ((alloc_fn == nullptr) != (free_fn == nullptr)) return IGD_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || cuda_device < 0 || cuda_device >= ndev) {
        (void)cudaGetLastError();
        return IGD_ECUDA;
    }
    if (cudaSetDevice(cuda_device) != cudaSuccess) return IGD_ECUDA;
    igd_ctx* ctx = new igd_ctx();
    ctx->device = cuda_device;
    ctx->stream = (cudaStream_t)cuda_stream;
    ctx->afn = alloc_fn;
    ctx->ffn = free_fn;
    ctx->auser = alloc_user;
    if (const char* m = getenv("IGD_FUSED")) ctx->fused = atoi(m) != 0;
    cudaFuncSetAttribute(fused::k_ingest_sort0<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)fused::smem_bytes());
    cudaFuncSetAttribute(fused::k_ingest_sort0<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)fused::smem_bytes());
    cudaFuncSetAttribute(fused::k_ingest_sort0<false, u32, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)fused::smem_bytes());
    cudaFuncSetAttribute(fused::k_ingest_sort0<false, u64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)fused::smem_bytes<u64>());
    cudaFuncSetAttribute(fused::k_ingest_sort0<true, u64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)fused::smem_bytes<u64>());
    set_pass_smem<u32>();
    set_pass_smem<u64>();
    set_pass_smem<uint4>();
    set_pass_smem<u64, u64>();
    if (cudaMallocHost(&ctx->h_stats, 8 * sizeof(u64)) != cudaSuccess ||
        cudaMallocHost(&ctx->h_hist, 4 * 1024 * sizeof(u32)) != cudaSuccess ||
        cudaMallocHost(&ctx->h_small, 8 * sizeof(u64)) != cudaSuccess) {
        delete ctx;
        return IGD_ENOMEM;
    }
    for (int i = 0; i <= IGD_N_STAGES; i++) cudaEventCreate(&ctx->ev[i]);
    // the side stream at the greatest priority: its small a2 / a3 kernels take SM slots as the
    // access sort's CTAs retire instead of queueing behind all of the sort's passes
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    if (cudaStreamCreateWithPriority(&ctx->side, cudaStreamNonBlocking, prio_hi) != cudaSuccess ||
        cudaEventCreateWithFlags(&ctx->side_ev[0], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&ctx->side_ev[1], cudaEventDisableTiming) != cudaSuccess) {
        (void)cudaGetLastError();
        igd_ctx_destroy(ctx);
        return IGD_ECUDA;
    }
    for (int i = 0; i < 2 * kMaxTimed; i++) cudaEventCreate(&ctx->kev[i]);
    for (int i = 0; i < IGD_N_STAGES; i++) ctx->stage_ms[i] = 0.f;
    for (int i = 0; i < IGD_N_KCLASS; i++) {
        ctx->cls_ms[i] = 0.f;
        ctx->cls_n[i] = 0;
        ctx->cls_bytes[i] = 0;
    }
    ctx->nranks = nranks;
    ctx->rank = rank;
    if (nccl_unique_id && memcmp(nccl_unique_id, "IGDLOOP:", 8) == 0) {
        // in-process loopback transport (tests): ranks of one process meet by the id's name
        char name[121];
        memcpy(name, nccl_unique_id + 8, 120);
        name[120] = 0;
        ctx->loop = loop_join(name, nranks);
        if (!ctx->loop) {
            igd_ctx_destroy(ctx);
            return IGD_EINVAL;
        }
    } else if (nccl_unique_id) {
        // a communicator (also for nranks == 1: the collective path on one GPU); blocks until
        // every rank has joined
        NcclApi& N = nccl();
        if (!N.ok) {
            igd_ctx_destroy(ctx);
            return IGD_ENCCL;
        }
        ncclUniqueId id;
        memcpy(&id, nccl_unique_id, sizeof(id));
        if (N.CommInitRank(&ctx->comm, nranks, id, rank) != ncclSuccess) {
            ctx->comm = nullptr;
            igd_ctx_destroy(ctx);
            return IGD_ENCCL;
        }
    }
    *out = ctx;
    return IGD_OK;
}

int igd_trace_load(igd_ctx* ctx, const igd_trace_desc* desc, const igd_event* events) {
    if (!ctx || !desc) return IGD_EINVAL;
    if (desc->n_blocks == 0 || desc->block_dim == 0) return IGD_EINVAL;
    if ((u64)desc->n_blocks * desc->block_dim > (1ull << 24)) return IGD_EINVAL;
    if (desc->n_events > 0xFFFFFFFFull - 2 * rsort::TILE) return IGD_ETOOBIG;
    if (desc->n_events > 0 && !events) return IGD_EINVAL;
    if (desc->n_events_total != 0 && desc->first_event + desc->n_events > desc->n_events_total) {
        ctx->err = "first_event + n_events exceeds n_events_total";
        return IGD_EINVAL;
    }
    if ((desc->n_events_total ? desc->n_events_total : desc->n_events) > 0xFFFFFFFFull - 2 * rsort::TILE)
        return IGD_ETOOBIG;
    cudaSetDevice(ctx->device);
    ctx->desc = *desc;
    ctx->loaded = false;
    if (desc->flags & IGD_TRACE_DEVICE_PTR) {
        // the kernels read events with 16-byte vector loads and TMA bulk copies
        if (((uintptr_t)events & 15u) != 0) {
            ctx->err = "device events must be 16-byte aligned";
            return IGD_EINVAL;
        }
        ctx->events = events;
    } else {
        const size_t bytes = desc->n_events * sizeof(igd_event);
        RET(ensure(ctx, ctx->owned_events, bytes));
        if (bytes) CK(cudaMemcpyAsync(ctx->owned_events.p, events, bytes, cudaMemcpyHostToDevice, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        ctx->events = P_<igd_event>(ctx->owned_events);
    }
    ctx->loaded = true;
    return IGD_OK;
}

static void collect_timing(igd_ctx* ctx);

int igd_detect(igd_ctx* ctx, uint32_t flags, uint64_t* n_reports_global) {
    if (!ctx || !n_reports_global) return IGD_EINVAL;
    if (!ctx->loaded || ctx->str_active) return IGD_ESTATE;
    const u32 tag_log2 = (flags >> IGD_DETECT_TAG_SHIFT) & 31u;
    if (tag_log2 && (tag_log2 < 8 || tag_log2 > 22)) {
        ctx->err = "IGD_DETECT_TAG_LOG2 must be 8..22";
        return IGD_EINVAL;
    }
    u32 last_k = (flags >> IGD_DETECT_LAST_K_SHIFT) & 15u;
    if (last_k == 0) last_k = 1;
    if (last_k != 1 && last_k != 2 && last_k != 4 && last_k != 8) {
        ctx->err = "IGD_DETECT_LAST_K must be 1, 2, 4 or 8";
        return IGD_EINVAL;
    }
    if (ctx->comm || ctx->loop) {  // collective over the communicator's ranks
        if (flags & IGD_DETECT_COALESCE) {  // reading A32: a group may straddle two ranks' chunks
            ctx->err = "IGD_DETECT_COALESCE is a single-context mode";
            return IGD_EINVAL;
        }
        if (tag_log2 || last_k > 1) {  // A36: the owner hash would have to be over metadata entries
            ctx->err = "the tag-aliasing and last-k modes are single-context modes";
            return IGD_EINVAL;
        }
        cudaSetDevice(ctx->device);
        ctx->timing = (flags & IGD_DETECT_TIMING) != 0;
        ctx->paper_counters = (flags & IGD_DETECT_PAPER_COUNTERS) != 0;
        ctx->sticky = (flags & IGD_DETECT_STICKY_FLAGS) != 0;
        int rc = collective_detect(ctx, n_reports_global);
        ctx->paper_counters = false;
        ctx->sticky = false;
        if (rc == IGD_OK && ctx->timing) collect_timing(ctx);
        return rc;
    }
    if (ctx->desc.first_event != 0 ||
        (ctx->desc.n_events_total != 0 && ctx->desc.n_events_total != ctx->desc.n_events)) {
        ctx->err = "igd_detect checks a whole trace; a rank's chunk goes through igd_shard_*";
        return IGD_EINVAL;
    }
    cudaSetDevice(ctx->device);
    ctx->timing = (flags & IGD_DETECT_TIMING) != 0;
    ctx->coalesce = (flags & IGD_DETECT_COALESCE) != 0;
    ctx->paper_counters = (flags & IGD_DETECT_PAPER_COUNTERS) != 0;
    ctx->sticky = (flags & IGD_DETECT_STICKY_FLAGS) != 0;
    ctx->tag_log2 = tag_log2;
    ctx->last_k = last_k;
    ctx->shard = false;
    ctx->in_segment = false;
    int rc = detect_impl(ctx, n_reports_global);
    if (rc == IGD_SEGMENTS_NEEDED) rc = segmented_detect(ctx, n_reports_global);
    ctx->coalesce = false;
    ctx->paper_counters = false;
    ctx->sticky = false;
    ctx->tag_log2 = 0;
    ctx->last_k = 1;
    if (rc == IGD_OK && ctx->timing) collect_timing(ctx);
    return rc;
}

int igd_shard_prepare(igd_ctx* ctx, uint32_t nranks, uint64_t* counts, uint64_t* n_sync_stream,
                      uint64_t* bad_event, uint64_t* word_minmax) {
    if (!ctx || !counts || !n_sync_stream || !bad_event || !word_minmax) return IGD_EINVAL;
    if (nranks == 0 || nranks > (uint32_t)shard::MAXP) return IGD_EINVAL;
    if (!ctx->loaded) return IGD_ESTATE;
    cudaSetDevice(ctx->device);
    ctx->launches = 0;
    ctx->nk = 0;
    ctx->timing = true;  // per-launch events are cheap; igd_shard_detect reports them with its own
    return shard_prepare_impl(ctx, nranks, counts, n_sync_stream, bad_event, word_minmax);
}

int igd_shard_buffers(igd_ctx* ctx, void** d_records, void** d_sync_idx, void** d_sync_events) {
    if (!ctx || !d_records || !d_sync_idx || !d_sync_events) return IGD_EINVAL;
    *d_records = ctx->sh_send.p;
    *d_sync_idx = ctx->sh_sidx_buf.p;
    *d_sync_events = ctx->sh_sev_buf.p;
    return IGD_OK;
}

int igd_shard_detect(igd_ctx* ctx, const void* d_records, uint64_t n_records, const uint32_t* d_sync_idx,
                     const void* d_sync_events, uint64_t n_sync_stream, uint64_t min_word, uint32_t flags,
                     uint64_t* n_reports) {
    if (!ctx || !n_reports) return IGD_EINVAL;
    if ((n_records && !d_records) || (n_sync_stream && (!d_sync_idx || !d_sync_events))) return IGD_EINVAL;
    if ((((uintptr_t)d_records | (uintptr_t)d_sync_events) & 15u) != 0) {
        ctx->err = "records and sync events must be 16-byte aligned";
        return IGD_EINVAL;
    }
    if (!ctx->loaded) return IGD_ESTATE;
    if (flags & IGD_DETECT_COALESCE) {  // reading A32: a group may straddle two ranks' chunks
        ctx->err = "IGD_DETECT_COALESCE is a single-context mode";
        return IGD_EINVAL;
    }
    if (ctx->str_active) return IGD_ESTATE;  // a streaming session owns the sharded-mode state
    cudaSetDevice(ctx->device);
    ctx->timing = (flags & IGD_DETECT_TIMING) != 0;
    ctx->paper_counters = (flags & IGD_DETECT_PAPER_COUNTERS) != 0;
    ctx->sticky = (flags & IGD_DETECT_STICKY_FLAGS) != 0;
    if (((flags >> IGD_DETECT_TAG_SHIFT) & 31u) || ((flags >> IGD_DETECT_LAST_K_SHIFT) & 15u) > 1) {
        ctx->err = "the tag-aliasing and last-k modes are single-context modes";
        return IGD_EINVAL;
    }
    ctx->shard = true;
    ctx->sh_rec = d_records;
    ctx->sh_nrec = n_records;
    ctx->sh_sidx = d_sync_idx;
    ctx->sh_sev = d_sync_events;
    ctx->sh_ns = n_sync_stream;
    ctx->sh_wbase = min_word;
    ctx->sh_ntotal = ctx->desc.n_events_total ? ctx->desc.n_events_total : ctx->desc.n_events;
    // the exchange is done: release the send buffer first, unless the caller passes (part of) it
    // back as the received records (one rank, or an in-place exchange) -- then after the check
    const char* sb = (const char*)ctx->sh_send.p;
    const char* rb = (const char*)d_records;
    const bool aliased = sb && rb && rb < sb + ctx->sh_send.cap && rb + n_records * 16 > sb;
    if (!aliased) RET(buf_free(ctx, ctx->sh_send));
    int rc = detect_impl(ctx, n_reports);
    if (aliased) buf_free(ctx, ctx->sh_send);
    ctx->shard = false;
    ctx->paper_counters = false;
    ctx->sticky = false;
    if (rc == IGD_OK && ctx->timing) collect_timing(ctx);
    return rc;
}

static void collect_timing(igd_ctx* ctx) {
    {
        cudaEventSynchronize(ctx->ev[8]);
        for (int s = 0; s < IGD_N_STAGES - 1; s++) cudaEventElapsedTime(&ctx->stage_ms[s], ctx->ev[s], ctx->ev[s + 1]);
        cudaEventElapsedTime(&ctx->stage_ms[IGD_N_STAGES - 1], ctx->ev[0], ctx->ev[7]);
        for (int i = 0; i < IGD_N_KCLASS; i++) {
            ctx->cls_ms[i] = 0.f;
            ctx->cls_n[i] = 0;
            ctx->cls_bytes[i] = 0;
        }
        for (int q = 0; q < ctx->nk; q++) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, ctx->kev[2 * q], ctx->kev[2 * q + 1]);
            ctx->cls_ms[ctx->kcls[q]] += ms;
            ctx->cls_n[ctx->kcls[q]] += 1;
            ctx->cls_bytes[ctx->kcls[q]] += ctx->kbytes[q];
        }
    }
}

int igd_reports(igd_ctx* ctx, igd_report* host_out, uint64_t cap, uint64_t* n_written) {
    if (!ctx || !n_written || (cap > 0 && !host_out)) return IGD_EINVAL;
    u64 k = ctx->n_reports < cap ? ctx->n_reports : cap;
    *n_written = k;
    if (k) {
        CK(cudaMemcpyAsync(host_out, ctx->rep_out.p, k * sizeof(igd_report), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
    }
    return IGD_OK;
}

int igd_reports_device(igd_ctx* ctx, const igd_report** dev_ptr, uint64_t* n) {
    if (!ctx || !dev_ptr || !n) return IGD_EINVAL;
    *dev_ptr = P_<igd_report>(ctx->rep_out);
    *n = ctx->n_reports;
    return IGD_OK;
}

uint64_t igd_bad_event(const igd_ctx* ctx) { return ctx ? ctx->bad_event : 0; }

int igd_stage_times(const igd_ctx* ctx, float* ms_out) {
    if (!ctx || !ms_out) return IGD_EINVAL;
    for (int i = 0; i < IGD_N_STAGES; i++) ms_out[i] = ctx->stage_ms[i];
    return IGD_OK;
}

const char* igd_stage_name(int stage) {
    return (stage >= 0 && stage < IGD_N_STAGES) ? kStageNames[stage] : "?";
}

uint64_t igd_last_launch_count(const igd_ctx* ctx) { return ctx ? ctx->launches : 0; }

int igd_kernel_stats(const igd_ctx* ctx, int kclass, const char** name, uint32_t* launches, float* ms,
                     double* alg_bytes) {
    if (!ctx || kclass < 0 || kclass >= IGD_N_KCLASS) return IGD_EINVAL;
    if (name) *name = kClassNames[kclass];
    if (launches) *launches = ctx->cls_n[kclass];
    if (ms) *ms = ctx->cls_ms[kclass];
    if (alg_bytes) *alg_bytes = ctx->cls_bytes[kclass];
    return IGD_OK;
}

int igd_stream_begin(igd_ctx* ctx, uint32_t n_blocks, uint32_t block_dim) {
    if (!ctx || n_blocks == 0 || block_dim == 0 || (u64)n_blocks * block_dim > (1ull << 24)) return IGD_EINVAL;
    if (ctx->comm || ctx->loop) {
        ctx->err = "streaming sessions are single-context";
        return IGD_EINVAL;
    }
    ctx->str_active = true;
    ctx->str_n = ctx->str_nsync = ctx->str_ncarry = 0;
    ctx->str_wmin = ~0ull;
    ctx->str_wmax = 0;
    ctx->str_nb = n_blocks;
    ctx->str_bd = block_dim;
    ctx->str_cur = 0;
    return IGD_OK;
}

int igd_stream_feed(igd_ctx* ctx, const igd_event* events, uint64_t n_events, uint32_t event_flags,
                    uint32_t detect_flags, uint64_t* n_reports) {
    if (!ctx || !n_reports) return IGD_EINVAL;
    if (!ctx->str_active) return IGD_ESTATE;
    if (detect_flags & (IGD_DETECT_COALESCE | (31u << IGD_DETECT_TAG_SHIFT) | (15u << IGD_DETECT_LAST_K_SHIFT))) {
        ctx->err = "streaming sessions support IGD_DETECT_TIMING, _PAPER_COUNTERS and _STICKY_FLAGS";
        return IGD_EINVAL;
    }
    cudaSetDevice(ctx->device);
    ctx->timing = (detect_flags & IGD_DETECT_TIMING) != 0;
    ctx->paper_counters = (detect_flags & IGD_DETECT_PAPER_COUNTERS) != 0;
    ctx->sticky = (detect_flags & IGD_DETECT_STICKY_FLAGS) != 0;
    int rc = stream_feed_impl(ctx, events, n_events, event_flags, n_reports);
    ctx->paper_counters = false;
    ctx->sticky = false;
    if (rc != IGD_OK) ctx->str_active = false;  // a failed chunk ends the session
    if (rc == IGD_OK && ctx->timing) collect_timing(ctx);
    return rc;
}

int igd_stream_end(igd_ctx* ctx) {
    if (!ctx) return IGD_EINVAL;
    cudaSetDevice(ctx->device);
    ctx->str_active = false;
    Buf* all[] = {&ctx->str_sidx, &ctx->str_sev, &ctx->str_carry[0], &ctx->str_carry[1], &ctx->str_rec,
                  &ctx->str_co, &ctx->str_flags};
    for (Buf* b : all) RET(buf_free(ctx, *b));
    return IGD_OK;
}

int igd_nccl_unique_id(uint8_t* out128) {
    if (!out128) return IGD_EINVAL;
    NcclApi& N = nccl();
    if (!N.ok) return IGD_ENCCL;
    ncclUniqueId id;
    if (N.GetUniqueId(&id) != ncclSuccess) return IGD_ENCCL;
    memcpy(out128, &id, sizeof(id));
    return IGD_OK;
}

void igd_ctx_destroy(igd_ctx* ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    if (ctx->comm) {
        nccl().CommDestroy(ctx->comm);
        ctx->comm = nullptr;
    }
    if (ctx->loop) {
        loop_leave(ctx->loop);
        ctx->loop = nullptr;
    }
    Buf* all[] = {&ctx->owned_events, &ctx->acc_k[0], &ctx->acc_k[1], &ctx->acc_v[0], &ctx->acc_v[1],
                  &ctx->syn_k[0],     &ctx->syn_k[1], &ctx->syn_v[0], &ctx->syn_v[1], &ctx->st_in_a,
                  &ctx->st_in_s,      &ctx->status,   &ctx->dstatus,  &ctx->stats,    &ctx->hist,     &ctx->base,
                  &ctx->ctr,          &ctx->off,      &ctx->ldesc,    &ctx->gtab,     &ctx->tcnt,
                  &ctx->tpts,         &ctx->tbits,    &ctx->fdev,     &ctx->skipb,    &ctx->rep_raw,  &ctx->rep_k[0], &ctx->rep_k[1],
                  &ctx->rep_v[0],     &ctx->rep_v[1], &ctx->rep_out,  &ctx->rep_ctr,  &ctx->rep_hist,
                  &ctx->sh_cnt,       &ctx->sh_obase, &ctx->sh_send,  &ctx->sh_sidx_buf, &ctx->sh_sev_buf,
                  &ctx->cl_small,     &ctx->cl_mat,   &ctx->cl_recv,  &ctx->cl_sidx,  &ctx->cl_sev,
                  &ctx->cl_nrep,      &ctx->cl_rep,   &ctx->gkb,      &ctx->seg_rep,  &ctx->lk_state,
                  &ctx->str_sidx,     &ctx->str_sev,  &ctx->str_carry[0], &ctx->str_carry[1], &ctx->str_rec,
                  &ctx->str_co,       &ctx->str_flags, &ctx->sw_base, &ctx->sw_dstatus, &ctx->sw_status,
                  &ctx->sw_ctr};
    for (Buf* b : all) buf_free(ctx, *b);
    cudaStreamSynchronize(ctx->stream);
    if (ctx->side) {
        cudaStreamSynchronize(ctx->side);
        cudaStreamDestroy(ctx->side);
    }
    for (cudaEvent_t e : ctx->side_ev)
        if (e) cudaEventDestroy(e);
    cudaFreeHost(ctx->h_stats);
    cudaFreeHost(ctx->h_hist);
    cudaFreeHost(ctx->h_small);
    for (int i = 0; i <= IGD_N_STAGES; i++) cudaEventDestroy(ctx->ev[i]);
    for (int i = 0; i < 2 * kMaxTimed; i++) cudaEventDestroy(ctx->kev[i]);
    delete ctx;
}

const char* igd_strerror(int code) {
    switch (code) {
        case IGD_OK: return "ok";
        case IGD_EINVAL: return "invalid argument or geometry";
        case IGD_ETRACE: return "ill-formed trace event";
        case IGD_ETOOBIG: return "trace too large for the 32-bit index path";
        case IGD_ENOMEM: return "device out of memory";
        case IGD_ECUDA: return "CUDA error";
        case IGD_ENCCL: return "NCCL error (or libnccl unavailable)";
        case IGD_ESTATE: return "call out of order";
        default: return "unknown error";
    }
}

const char* igd_last_error(const igd_ctx* ctx) { return ctx ? ctx->err.c_str() : ""; }

// ---- stage-level test / micro-benchmark hooks (include/igd_debug.h) ----
int igd_debug_check_stats(igd_ctx* ctx, int enable, uint64_t* out16) {
    if (!ctx) return IGD_EINVAL;
    cudaSetDevice(ctx->device);
    if (out16) CK(cudaMemcpyFromSymbol(out16, check::g_chk_stats, 16 * sizeof(u64)));
    const unsigned long long zero[16] = {0};
    CK(cudaMemcpyToSymbol(check::g_chk_stats, zero, sizeof(zero)));
    CK(cudaMemcpyToSymbol(check::g_chk_stats_on, &enable, sizeof(int)));
    return IGD_OK;
}

int igd_debug_sync_tables(igd_ctx* ctx, uint64_t* sizes, uint32_t* off, uint32_t* ts, uint32_t* toff,
                          uint64_t* tpts) {
    if (!ctx || !sizes) return IGD_EINVAL;
    if (!ctx->loaded) return IGD_ESTATE;
    sizes[0] = ctx->last_E;
    sizes[1] = ctx->last_nsync;
    sizes[2] = ctx->last_T;
    sizes[3] = ctx->last_npts;
    cudaSetDevice(ctx->device);
    if (off && ctx->last_E) CK(cudaMemcpy(off, ctx->off.p, ((u64)ctx->last_E + 1) * sizeof(u32), cudaMemcpyDeviceToHost));
    if (ts && ctx->last_nsync)
        CK(cudaMemcpy(ts, ctx->syn_v[ctx->last_scur].p, ctx->last_nsync * sizeof(u32), cudaMemcpyDeviceToHost));
    if (toff && ctx->last_npts)
        CK(cudaMemcpy(toff, ctx->tcnt.p, ((u64)ctx->last_T + 1) * sizeof(u32), cudaMemcpyDeviceToHost));
    if (tpts && ctx->last_npts) CK(cudaMemcpy(tpts, ctx->tpts.p, ctx->last_npts * sizeof(u64), cudaMemcpyDeviceToHost));
    return IGD_OK;
}

int igd_debug_scan_state(igd_ctx* ctx, uint64_t n, uint64_t* state, uint32_t* keys, uint64_t* payload) {
    if (!ctx || n != ctx->last_nacc) return IGD_EINVAL;
    cudaSetDevice(ctx->device);
    if (state && n) CK(cudaMemcpy(state, ctx->lk_state.p, n * sizeof(u64), cudaMemcpyDeviceToHost));
    if (keys && n) CK(cudaMemcpy(keys, ctx->acc_k[ctx->last_acur].p, n * sizeof(u32), cudaMemcpyDeviceToHost));
    if (payload && n) CK(cudaMemcpy(payload, ctx->acc_v[ctx->last_acur].p, n * sizeof(u64), cudaMemcpyDeviceToHost));
    return IGD_OK;
}

int igd_debug_gather_probe(igd_ctx* ctx, int gather, float* ms) {
    if (!ctx || !ctx->loaded || ctx->last_nacc == 0) return IGD_ESTATE;
    cudaSetDevice(ctx->device);
    RET(ensure(ctx, ctx->ctr, 64));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int sms = sm_count(ctx);
    cudaEventRecord(a, ctx->stream);
    check::k_gather_probe<<<sms * 8, 256, 0, ctx->stream>>>(P_<u32>(ctx->acc_k[ctx->last_acur]),
                                                          P_<u64>(ctx->acc_v[ctx->last_acur]), (u32)ctx->last_nacc,
                                                          ctx->events, P_<u32>(ctx->ctr), gather);
    cudaEventRecord(b, ctx->stream);
    cudaEventSynchronize(b);
    if (ms) cudaEventElapsedTime(ms, a, b);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    CK(cudaGetLastError());
    return IGD_OK;
}

int igd_debug_radix_sort(igd_ctx* ctx, uint32_t* d_keys, uint32_t* d_vals, uint64_t n, uint32_t max_bits, int mode,
                         float* ms) {
    if (!ctx || n >= 0xFFFFFFFFull || (n && (!d_keys || !d_vals))) return IGD_EINVAL;
    cudaSetDevice(ctx->device);
    (void)mode;  // one multisplit policy (IGD_SORT_MIX); kept in the signature for the hook's callers
    for (int b = 0; b < 2; b++) {
        RET(ensure(ctx, ctx->acc_k[b], n * sizeof(u32)));
        RET(ensure(ctx, ctx->acc_v[b], n * sizeof(u32)));
    }
    RET(ensure(ctx, ctx->hist, 3 * 1024 * sizeof(u32)));
    RET(ensure(ctx, ctx->base, 4 * 256 * sizeof(u32)));
    RET(ensure(ctx, ctx->ctr, 64));
    CK(cudaMemcpyAsync(ctx->acc_k[0].p, d_keys, n * 4, cudaMemcpyDeviceToDevice, ctx->stream));
    CK(cudaMemcpyAsync(ctx->acc_v[0].p, d_vals, n * 4, cudaMemcpyDeviceToDevice, ctx->stream));
    CK(cudaMemsetAsync(ctx->hist.p, 0, 1024 * sizeof(u32), ctx->stream));
    const int sms = sm_count(ctx);
    rsort::k_hist4<<<sms * 8, 256, 0, ctx->stream>>>(P_<u32>(ctx->acc_k[0]), n, P_<u32>(ctx->hist));
    CK(cudaMemcpyAsync(ctx->h_hist, ctx->hist.p, 1024 * sizeof(u32), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    u32 hh[1024];
    memcpy(hh, ctx->h_hist, sizeof(hh));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a, ctx->stream);
    int cur = 0;
    int rc = radix_sort(ctx, KC_SORT_ACC, ctx->acc_k, ctx->acc_v, n, P_<u32>(ctx->hist), hh, max_bits, &cur);
    cudaEventRecord(b, ctx->stream);
    cudaEventSynchronize(b);
    if (ms) cudaEventElapsedTime(ms, a, b);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    if (rc != IGD_OK) return rc;
    CK(cudaMemcpyAsync(d_keys, ctx->acc_k[cur].p, n * 4, cudaMemcpyDeviceToDevice, ctx->stream));
    CK(cudaMemcpyAsync(d_vals, ctx->acc_v[cur].p, n * 4, cudaMemcpyDeviceToDevice, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return IGD_OK;
}

}  // extern "C"
