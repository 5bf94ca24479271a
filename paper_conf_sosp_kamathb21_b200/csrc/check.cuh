// check.cuh -- a6 building blocks shared by the check kernel (check4.cuh) and the report stage:
//
// * the packed per-word shadow state carried across warps and tiles by the decoupled look-back
//   (last-writer position, scope of the last atomic, DevShared, BlkShared, segment-head bit) and
//   its segmented "last-of / OR" combine -- the state the paper keeps per 4-byte word (Fig. 4,
//   P:763-829; updates P:1000-1058) as a function of the word's access prefix;
// * interval queries on the a2 timestamp lists: "is there a sync of entity e in (a, b)?" -- the
//   exact replacement of Table 2's counter comparisons (reading A16) -- answered from a per-list
//   descriptor {lo, hi, first, last} and interpolation-guided 32-byte probes, and for grid syncs
//   an L2-resident bucket table;
// * report canonicalisation kernels (a7) and a gather micro-benchmark probe.
#pragma once
#include "common.cuh"
#include "sync.cuh"

namespace check {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
constexpr int ITEMS = 4;
constexpr int TILE = THREADS * ITEMS;

// Packed scan state (37 bits): [31:0] lastW position (NONE = 0xFFFFFFFF), [33:32] scope of the
// last atomic (0 none, 1 block, 2 device), [34] devShared, [35] blkShared, [36] segment head seen.
__device__ __forceinline__ u64 st_make(u32 lastW, u32 as, u32 dev, u32 blk, u32 head) {
    return (u64)lastW | ((u64)as << 32) | ((u64)dev << 34) | ((u64)blk << 35) | ((u64)head << 36);
}
__device__ __forceinline__ u32 st_lastW(u64 s) { return (u32)s; }
__device__ __forceinline__ u32 st_as(u64 s) { return (u32)(s >> 32) & 3u; }
__device__ __forceinline__ u32 st_dev(u64 s) { return (u32)(s >> 34) & 1u; }
__device__ __forceinline__ u32 st_blk(u64 s) { return (u32)(s >> 35) & 1u; }
__device__ __forceinline__ u32 st_head(u64 s) { return (u32)(s >> 36) & 1u; }
#define ST_IDENTITY (0xFFFFFFFFull)
#define ST_HEAD_MARK (ST_IDENTITY | (1ull << 36))  // last-k mode: the access starts its segment

// a then b (b later): segmented "last-of" / OR combine
__device__ __forceinline__ u64 combine(u64 a, u64 b) {
    if (st_head(b)) return b;
    const u32 lw = st_lastW(b) != IGD_NONE32 ? st_lastW(b) : st_lastW(a);
    const u32 as = st_as(b) ? st_as(b) : st_as(a);
    return st_make(lw, as, st_dev(a) | st_dev(b), st_blk(a) | st_blk(b), st_head(a));
}

// List descriptors: desc[e] = {lo, hi, ts[lo], ts[hi-1]} of entity e's timestamp list.
__global__ void k_list_desc(const u32* __restrict__ off, const u32* __restrict__ ts, u32 E, uint4* __restrict__ desc) {
    for (u64 e = (u64)blockIdx.x * blockDim.x + threadIdx.x; e < E; e += (u64)gridDim.x * blockDim.x) {
        const u32 lo = off[e], hi = off[e + 1];
        desc[e] = make_uint4(lo, hi, lo < hi ? ts[lo] : 0u, lo < hi ? ts[hi - 1] : 0u);
    }
}

// Optional event counters (igd_debug_check_stats): a debug aid, off unless enabled.
__device__ int g_chk_stats_on;
__device__ unsigned long long g_chk_stats[16];
#ifndef IGD_CHECK_STATS
#define IGD_CHECK_STATS 0  // build a variant with -DIGD_CHECK_STATS=1 for profiles/check_stats.py
#endif
#define CSTAT(k)                                                            \
    do {                                                                    \
        if (IGD_CHECK_STATS && g_chk_stats_on) atomicAdd(&g_chk_stats[k], 1ull); \
    } while (0)

// Is there an element x of entity e's list with a < x < b ?
#ifndef IGD_QB_INLINE
#define IGD_QB_INLINE 1  // inlined into the check: C5 55.9 -> 54.1 ms (r02t); 0 = a call
#endif
#if IGD_QB_INLINE
#define IGD_QB_ATTR __forceinline__
#else
#define IGD_QB_ATTR __noinline__
#endif
__device__ IGD_QB_ATTR bool q_between(const uint4* __restrict__ desc, const u32* __restrict__ ts, u32 e, u32 a,
                                       u32 b) {
    const uint4 d = __ldg(desc + e);
    CSTAT(7);
    if (d.x == d.y || d.w <= a) {  // empty, or every element <= a
        CSTAT(8);
        return false;
    }
    if (d.z > a) {  // the first element is the first one > a
        CSTAT(8);
        return d.z < b;
    }
    // first <= a < last: the successor of a lies in [lo, hi]; guess its position by
    // interpolation and probe aligned 32-byte sectors (8 timestamps) around the guess
    u32 lo = d.x + 1, hi = d.y - 1;
    // single-precision guess (a hint only: it is clamped and verified by the probes)
    u32 g = d.x + 1 + (u32)(__fdividef((float)(a - d.z), (float)(d.w - d.z)) * (float)(d.y - 1 - d.x));
    g = min(max(g, lo), hi);
#pragma unroll 1
    for (int probe = 0; probe < 3 && lo < hi; probe++) {
        g = min(max(g, lo), hi);  // the probe always covers a position of [lo, hi]
        const u32 g0 = g & ~7u;
        const uint4* p = reinterpret_cast<const uint4*>(ts + g0);
        const uint4 v0 = __ldg(p), v1 = __ldg(p + 1);
        const u32 s0 = max(g0, lo), s1 = min(g0 + 8, hi + 1);  // probed positions inside [lo, hi]
        const u32 lem = (u32)(v0.x <= a) | ((u32)(v0.y <= a) << 1) | ((u32)(v0.z <= a) << 2) |
                        ((u32)(v0.w <= a) << 3) | ((u32)(v1.x <= a) << 4) | ((u32)(v1.y <= a) << 5) |
                        ((u32)(v1.z <= a) << 6) | ((u32)(v1.w <= a) << 7);
        const u32 rng = ((1u << (s1 - g0)) - 1u) & ~((1u << (s0 - g0)) - 1u);
        const u32 le = __popc(lem & rng);
        if (le == s1 - s0) {          // all <= a: successor after the probe
            lo = s1;
            g = s1;
        } else if (le == 0) {         // all > a: successor is s0 or before
            hi = s0;
            g = s0 > 8 ? s0 - 8 : 0;
        } else {                      // successor inside the probe (L1-resident)
            CSTAT(9);
            return __ldg(ts + s0 + le) < b;
        }
    }
    CSTAT(10);
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(ts + mid) <= a) lo = mid + 1;
        else hi = mid;
    }
    return __ldg(ts + lo) < b;
}

struct Params {
    const void* key; // sorted word keys: u32 low 32 bits of the word, or u64 word - wbase (wide path)
    const void* val; // sorted payload: u64 (index | tk << 32), or uint4 {key, index, tk, mask} (MV)
    u64 wbase;       // u32 keys: smallest accessed word (reports rebuild the 64-bit word from the
                     // key); u64 keys: the key base
    u32 n;           // number of accesses
    const igd_event* ev;
    Geo g;
    KeySpace ks;
    const uint4* desc;  // per-entity list descriptors
    const u64* gtab;    // grid-sync bucket table: {first grid-list index at or after the bucket start, its timestamp}
    u32 gshift;         // bucket = t >> gshift
    u32 glo, ghi;       // the grid list inside sts
    u32 has_kb;         // the trace has kernel boundaries (reading A31)
    const u32* sts;     // sync timestamps (sorted by entity, then time)
    syncx::LockView lv;
    u64* status;     // [n_tiles] zeroed
    u32* tile_ctr;   // zeroed: tile tickets
    igd_report* rep;
    u64 rep_cap;
    unsigned long long* rep_ctr;
    u64 first_event; // global index offset (multi-rank)
    u32 addr_from_ev;  // tag-aliasing mode (A36): keys hold entry + tag, report addresses come from the trace
    u64* st_out;       // last-k mode (A37): per-access scan state out, no checks here (NULL otherwise)
    const uint4* rec;  // sharded mode: the received records, ascending by index (active-mask lookups)
    u32 nrec;
    u32 carry_before;  // streaming mode (f4): records with index < carry_before are carried state
    void* carry_out;   // streaming mode: 2 uint4 per access (carried pair at each word's last access)
};

// The active mask of the access with trace index i: from the trace on one GPU, else from the
// received records of a sharded check (ascending by index: a binary search -- the mask is read
// only when no syncwarp decides P4, rarely)
__device__ __forceinline__ u32 mask_of(const Params& P, u32 i) {
    if (!P.rec) return ld_event(P.ev, i).w;
    u32 lo = 0, hi = P.nrec;
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(&P.rec[mid].y) < i) lo = mid + 1;
        else hi = mid;
    }
    return __ldg(&P.rec[lo].w);
}

// Streaming mode: keep the carried pairs written at each word's last access (compaction by
// flag, exclusive scan, scatter; the survivors stay in key order)
__global__ void k_carry_flags(const uint4* __restrict__ co, u32 n, u32* __restrict__ flags) {
    for (u32 x = blockIdx.x * blockDim.x + threadIdx.x; x <= n; x += gridDim.x * blockDim.x)
        flags[x] = x < n && co[2 * (u64)x + 1].y != IGD_NONE32 ? 1u : 0u;
}
__global__ void k_carry_scatter(const uint4* __restrict__ co, const u32* __restrict__ pos, u32 n,
                                uint4* __restrict__ out) {
    for (u32 x = blockIdx.x * blockDim.x + threadIdx.x; x < n; x += gridDim.x * blockDim.x)
        if (pos[x + 1] != pos[x]) {
            out[2 * (u64)pos[x]] = co[2 * (u64)x];
            out[2 * (u64)pos[x] + 1] = co[2 * (u64)x + 1];
        }
}

// Grid-sync bucket table: gtab[b] = {index, timestamp} of the first grid sync with timestamp >=
// b << shift (timestamp NONE past the last).  The grid list is global and short, so "a grid sync
// in (a, b)?" -- the most frequent query of P5 / R2..R4 -- is one L2-resident 8-byte load in the
// common case (no grid sync between the bucket start and a), else a step or two along the list.
__global__ void k_grid_table(const u32* __restrict__ ts, u32 glo, u32 ghi, u32 shift, u32 nb, u64* __restrict__ gtab) {
    for (u64 b = (u64)blockIdx.x * blockDim.x + threadIdx.x; b < nb; b += (u64)gridDim.x * blockDim.x) {
        const u64 start = b << shift;
        u32 lo = glo, hi = ghi;
        while (lo < hi) {
            const u32 mid = (lo + hi) >> 1;
            if ((u64)ts[mid] < start) lo = mid + 1;
            else hi = mid;
        }
        gtab[b] = (u64)lo | ((u64)(lo < ghi ? ts[lo] : IGD_NONE32) << 32);
    }
}

template <class PP>
__device__ __forceinline__ bool q_grid(const PP& P, u32 a, u32 b) {
    if (P.glo == P.ghi) return false;
    const u64 e = __ldg(P.gtab + ((a + 1) >> P.gshift));  // first grid sync at or after a's bucket
    u32 x = (u32)e;
    const u32 v0 = (u32)(e >> 32);
    if (x >= P.ghi) return false;
    if (v0 > a) return v0 < b;
    x++;
#pragma unroll 1
    for (int step = 0; x < P.ghi; step++, x++) {
        const u32 v = __ldg(P.sts + x);
        if (v > a) return v < b;
        if (step == 8) return q_between(P.desc, P.sts, P.ks.grid, a, b);  // dense grid syncs
    }
    return false;
}

// queue entry flags
#define QF_SAME_W 1u
#define QF_SAME_B 2u
#define QF_DEV 4u
#define QF_BLK 8u
#define QF_R1 16u
#define QF_MASK 32u  // P4's lockstep clause still needs the active mask (read from the trace)

// Sorted payload of one access: single GPU = u64 (trace index | tk << 32), the active mask is
// gathered from the trace when needed; sharded = the record uint4 {key, index, tk, mask} (the events of
// other ranks are not resident).
struct Acc {
    u32 idx, tk, mask;
};
template <bool MV>
__device__ __forceinline__ Acc acc_at(const void* val, u32 k) {
    Acc a;
    if (MV) {  // the received record {key, idx, tk, mask}
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(val) + k);
        a.idx = v.y;
        a.tk = v.z;
        a.mask = v.w;
    } else {
        const unsigned long long v = __ldg(reinterpret_cast<const unsigned long long*>(val) + k);
        a.idx = (u32)v;
        a.tk = (u32)(v >> 32);
        a.mask = 0;
    }
    return a;
}

// Micro-benchmark probe: stream the sorted keys / indices and gather each access's event,
// nothing else (the memory floor of phase 1).
__global__ void k_gather_probe(const u32* __restrict__ key, const u64* __restrict__ val, u32 n,
                               const igd_event* __restrict__ ev, u32* __restrict__ sink, int gather) {
    u32 acc = 0;
    for (u32 k = (blockIdx.x * blockDim.x + threadIdx.x) * 4; k < n; k += gridDim.x * blockDim.x * 4) {
        if (k + 4 <= n) {
            const uint4 k4 = __ldcs(reinterpret_cast<const uint4*>(key + k));
            const uint4 va = __ldcs(reinterpret_cast<const uint4*>(val + k));
            const uint4 vb = __ldcs(reinterpret_cast<const uint4*>(val + k + 2));
            acc ^= k4.x ^ k4.y ^ k4.z ^ k4.w;
            if (gather) {
                const uint4 e0 = ld_event(ev, va.x), e1 = ld_event(ev, va.z), e2 = ld_event(ev, vb.x),
                            e3 = ld_event(ev, vb.z);
                acc ^= e0.z ^ e1.z ^ e2.z ^ e3.z;
            } else {
                acc ^= va.x ^ va.y ^ vb.z ^ vb.w;
            }
        }
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

// a7 for small report sets (n <= 2048, one CTA, no host round trip): bitonic sort of (cur, index)
// pairs in shared memory, then the gather.  cur is unique (one report per access, A21).
constexpr int SMALL_REP = 2048;
__global__ void __launch_bounds__(1024) k_report_sort_small(const igd_report* __restrict__ in, u32 n,
                                                            igd_report* __restrict__ out) {
    __shared__ u64 s[SMALL_REP];
    for (u32 i = threadIdx.x; i < SMALL_REP; i += blockDim.x)
        s[i] = i < n ? ((u64)(u32)in[i].cur << 32) | i : ~0ull;
    __syncthreads();
    for (u32 k = 2; k <= SMALL_REP; k <<= 1)
        for (u32 j = k >> 1; j > 0; j >>= 1) {
            for (u32 i = threadIdx.x; i < SMALL_REP; i += blockDim.x) {
                const u32 l = i ^ j;
                if (l > i) {
                    const u64 a = s[i], b = s[l];
                    const bool up = (i & k) == 0;
                    if ((a > b) == up) {
                        s[i] = b;
                        s[l] = a;
                    }
                }
            }
            __syncthreads();
        }
    for (u32 i = threadIdx.x; i < n; i += blockDim.x) out[i] = in[(u32)s[i]];
}

// reports: key = cur (u32 trace index) for the canonical-order sort
__global__ void k_report_keys(const igd_report* __restrict__ rep, u32 n, u64 first_event, u32* keys, u32* vals) {
    for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        keys[i] = (u32)(rep[i].cur - first_event);
        vals[i] = i;
    }
}
__global__ void k_report_gather(const igd_report* __restrict__ in, const u32* __restrict__ perm, u32 n,
                                igd_report* __restrict__ out) {
    for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = in[perm[i]];
}

}  // namespace check
