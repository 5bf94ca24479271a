// check.cuh -- a6: per-address segmented shadow-metadata pass + Table 2 race check.
//
// Input: accesses sorted by (word key, trace index).  Within one word's segment the shadow
// state the paper keeps per 4-byte word (Fig. 4; updates P:1000-1058) before access
// j is a pure function of the segment prefix ("equivalent formulation"):
//   valid      = j is not the segment head                         (P1)
//   LA         = access j-1                                          (last accessor)
//   LW         = last write before j             -> segmented last-of scan
//   Atomic/Scope = any atomic before j / scope of the last one       (reading A6)
//   DevShared / BlkShared = OR of adjacent-pair predicates up to j   (A5)
//   Locks      = held-lock Bloom of LA at LA's time                  (A7)
//
// Two phases per 1024-access tile (256 threads x 4 consecutive accesses):
//  1. streaming: coalesced key/index loads, one 16-byte event gather per access, thread-local
//     + warp-shuffle + block scans of the packed shadow state, decoupled look-back across tiles
//     (a tile containing a segment head publishes its inclusive state at once, so only tiles
//     inside one long hot-word segment wait), then the checks that need no synchronization
//     history: P1, P2, P3, P6 and P4's lockstep clause.
//  2. the accesses still undecided are queued in shared memory and processed densely by the
//     whole CTA: P4 (syncwarp), P5, R1..R5.  The synchronization-counter comparisons of Table 2
//     become interval queries on the a2 lists ("did md's thread fence in (md.idx, i)?", reading
//     A1), answered by a per-list descriptor {lo, hi, first, last} and interpolation-guided
//     32-byte probes (two dependent loads for the periodic lists of real kernels).
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
#define CSTAT(k)                                                \
    do {                                                        \
        if (g_chk_stats_on) atomicAdd(&g_chk_stats[k], 1ull);   \
    } while (0)

// Is there an element x of entity e's list with a < x < b ?
__device__ __noinline__ bool q_between(const uint4* __restrict__ desc, const u32* __restrict__ ts, u32 e, u32 a,
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
    const u32* key;  // sorted word keys
    const void* val; // sorted payload: u64 (index | tk << 32), or uint4 {index, tk, mask, 0} (MV)
    u64 wbase;       // smallest accessed word (reports rebuild the 64-bit word from the key)
    u32 n;           // number of accesses
    const igd_event* ev;
    Geo g;
    KeySpace ks;
    const uint4* desc;  // per-entity list descriptors
    const u32* gtab;    // grid-sync bucket table: first grid-list index at or after bucket start
    u32 gshift;         // bucket = t >> gshift
    u32 glo, ghi;       // the grid list inside sts
    const u32* sts;     // sync timestamps (sorted by entity, then time)
    syncx::LockView lv;
    u64* status;     // [n_tiles] zeroed
    u32* tile_ctr;   // zeroed
    igd_report* rep;
    u64 rep_cap;
    unsigned long long* rep_ctr;
    u64 first_event; // global index offset (multi-rank)
    int debug_stop;  // profiling only (IGD_CHECK_STOP): 1 = stop after the scans, 2 = after phase 1
};

// Grid-sync bucket table: gtab[b] = index of the first grid sync with timestamp >= b << shift.
// The grid list is global and short, so "a grid sync in (a, b)?" -- the most frequent query of
// P5 / R2..R4 -- becomes one L2-resident table load plus a step or two along the list.
__global__ void k_grid_table(const u32* __restrict__ ts, u32 glo, u32 ghi, u32 shift, u32 nb, u32* __restrict__ gtab) {
    for (u64 b = (u64)blockIdx.x * blockDim.x + threadIdx.x; b < nb; b += (u64)gridDim.x * blockDim.x) {
        const u64 start = b << shift;
        u32 lo = glo, hi = ghi;
        while (lo < hi) {
            const u32 mid = (lo + hi) >> 1;
            if ((u64)ts[mid] < start) lo = mid + 1;
            else hi = mid;
        }
        gtab[b] = lo;
    }
}

template <class PP>
__device__ __forceinline__ bool q_grid(const PP& P, u32 a, u32 b) {
    if (P.glo == P.ghi) return false;
    u32 x = __ldg(P.gtab + ((a + 1) >> P.gshift));  // first grid sync at or after a's bucket
#pragma unroll 1
    for (int step = 0; x < P.ghi; step++, x++) {
        const u32 v = __ldg(P.sts + x);
        if (v > a) return v < b;
        if (step == 8) return q_between(P.desc, P.sts, P.ks.grid, a, b);  // dense grid syncs
    }
    return false;
}

#ifndef IGD_CHECK_WARPQ
#define IGD_CHECK_WARPQ 1
#endif

// queue entry flags
#define QF_SAME_W 1u
#define QF_SAME_B 2u
#define QF_DEV 4u
#define QF_BLK 8u
#define QF_R1 16u

// Sorted payload of one access: single GPU = u64 (trace index | tk << 32), the active mask is
// gathered from the trace when needed; sharded = uint4 {index, tk, mask, 0} (the events of
// other ranks are not resident).
struct Acc {
    u32 idx, tk, mask;
};
template <bool MV>
__device__ __forceinline__ Acc acc_at(const void* val, u32 k) {
    Acc a;
    if (MV) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(val) + k);
        a.idx = v.x;
        a.tk = v.y;
        a.mask = v.z;
    } else {
        const unsigned long long v = __ldg(reinterpret_cast<const unsigned long long*>(val) + k);
        a.idx = (u32)v;
        a.tk = (u32)(v >> 32);
        a.mask = 0;
    }
    return a;
}

template <bool MV>
#ifndef IGD_CHECK_MINB
#define IGD_CHECK_MINB 6
#endif
__global__ void __launch_bounds__(THREADS, IGD_CHECK_MINB) k_check(Params P) {
    __shared__ u32 s_tile;
    __shared__ u64 s_wagg[WARPS];
    __shared__ u64 s_prefix;
    __shared__ u32 s_ready;
    __shared__ u32 s_qn;
    // queue of undecided accesses (SoA)
    // per-warp queues of undecided accesses (SoA; q_pos: sorted position): each warp answers
    // its own queue right after its phase 1, with no CTA-wide barrier in between
#if IGD_CHECK_WARPQ
    constexpr int QCAP = 32 * ITEMS;
    __shared__ u32 s_wqn[WARPS];
#else
    constexpr int QCAP = TILE;
#endif
    __shared__ u32 q_i[TILE], q_md[TILE], q_c[TILE], q_p[TILE], q_pos[TILE];

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) {
        // tiles in launch order (the block scheduler dispatches CTAs in blockIdx order, as
        // decoupled look-back scans rely on); no atomic round trip before the loads
        s_tile = blockIdx.x;
        s_qn = 0;
#if IGD_CHECK_WARPQ
        for (int w = 0; w < WARPS; w++) s_wqn[w] = 0;
#endif
        s_ready = 0;
    }
    __syncthreads();
    const u32 tile = s_tile;
    const u32 first = tile * TILE + t * ITEMS;  // n <= 2^32 - 2^13
    const Geo g = P.g;

    // K: word key, V: trace index, Z: the event's tk word (tid | kind | scope), carried by the sort
    u32 K[ITEMS], V[ITEMS], Z[ITEMS], M[ITEMS];
    if (!MV && first + ITEMS <= P.n) {
#pragma unroll
        for (int q = 0; q < ITEMS / 4; q++) {
            const uint4 k4 = __ldcs(reinterpret_cast<const uint4*>(P.key + first) + q);
            K[4 * q] = k4.x; K[4 * q + 1] = k4.y; K[4 * q + 2] = k4.z; K[4 * q + 3] = k4.w;
        }
#pragma unroll
        for (int q = 0; q < ITEMS / 2; q++) {
            const uint4 v = __ldcs(reinterpret_cast<const uint4*>(P.val) + first / 2 + q);
            V[2 * q] = v.x; Z[2 * q] = v.y; V[2 * q + 1] = v.z; Z[2 * q + 1] = v.w;
        }
#pragma unroll
        for (int j = 0; j < ITEMS; j++) M[j] = 0;
    } else {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const bool in = first + j < P.n;
            const Acc a = in ? acc_at<MV>(P.val, first + j) : Acc{0, 0, 0};
            K[j] = in ? P.key[first + j] : 0;
            V[j] = a.idx;
            Z[j] = a.tk;
            M[j] = a.mask;
        }
    }

    // previous element (first - 1): from the neighbour lane; lane 0 reads it
    u32 pK = __shfl_up_sync(IGD_FULL, K[ITEMS - 1], 1);
    u32 pV = __shfl_up_sync(IGD_FULL, V[ITEMS - 1], 1);
    u32 pZ = __shfl_up_sync(IGD_FULL, Z[ITEMS - 1], 1);
    if (lane == 0 && first > 0 && first - 1 < P.n) {
        pK = __ldg(P.key + first - 1);
        const Acc a = acc_at<MV>(P.val, first - 1);
        pV = a.idx;
        pZ = a.tk;
    }

    // per-access scan contributions
    u64 contrib[ITEMS];
    {
        u32 prevTid = pZ & 0xFFFFFFu, prevKey = pK;
        bool prevValid = first > 0;
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const bool inr = first + j < P.n;
            const u32 c = Z[j] & 0xFFFFFFu, kind = (Z[j] >> 24) & 0xFu;
            const bool head = !prevValid || prevKey != K[j];
            u32 dev = 0, blk = 0;
            if (!head) {
                const u32 bp = g.block(prevTid), bc = g.block(c);
                if (bp != bc) dev = 1;
                else if (g.warp(prevTid) != g.warp(c)) blk = 1;
            }
            const u32 lw = kind != IGD_LD ? first + j : IGD_NONE32;
            const u32 as = (kind >= IGD_ATOM && kind <= IGD_EXCH) ? norm_scope((Z[j] >> 28) & 3u) : 0u;
            contrib[j] = inr ? st_make(lw, as, dev, blk, head ? 1u : 0u) : ST_IDENTITY;
            prevTid = c;
            prevKey = K[j];
            prevValid = true;
        }
    }
    u64 agg = contrib[0];
#pragma unroll
    for (int j = 1; j < ITEMS; j++) agg = combine(agg, contrib[j]);
    u64 inc = agg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const u64 x = __shfl_up_sync(IGD_FULL, inc, o);
        if (lane >= (u32)o) inc = combine(x, inc);
    }
    if (lane == 31) s_wagg[warp] = inc;
    u64 wexcl = __shfl_up_sync(IGD_FULL, inc, 1);
    if (lane == 0) wexcl = ST_IDENTITY;
    __syncthreads();
    // Tile-relative state.  Only accesses of the segment that continues from the previous tile
    // (no head before them in this tile) need the look-back prefix; warp 0 lane 0 computes it
    // while every other access proceeds.
    if (t == 0) {
        u64 tagg = s_wagg[0];
#pragma unroll
        for (int w = 1; w < WARPS; w++) tagg = combine(tagg, s_wagg[w]);
        u64 prefix = ST_IDENTITY;
        st_relaxed(&P.status[tile], ((tile == 0 || st_head(tagg)) ? ST_INC : ST_AGG) | tagg);
        if (tile > 0) {
            // combine predecessors back to an inclusive status or a head-containing aggregate
            long tt = (long)tile - 1;
            u64 acc = ST_IDENTITY;
            bool have = false;
            while (tt >= 0) {
                u64 s;
                do {
                    s = ld_relaxed(&P.status[tt]);
                } while ((s >> 62) == 0);
                const u64 v = s & ST_VAL_MASK;
                acc = have ? combine(v, acc) : v;
                have = true;
                if ((s >> 62) == 2 || st_head(v)) break;
                tt--;
            }
            prefix = acc;
            if (!st_head(tagg)) st_relaxed(&P.status[tile], ST_INC | combine(prefix, tagg));
        }
        s_prefix = prefix;
        __threadfence_block();
        *(volatile u32*)&s_ready = 1u;
    }
    u64 run = ST_IDENTITY;
    for (u32 w = 0; w < warp; w++) run = combine(run, s_wagg[w]);
    run = combine(run, wexcl);  // tile-relative shadow state before this thread's first access

    if (P.debug_stop == 1) {
        if (run == 0x123456789ull) P.rep_ctr[1] = run;  // keep the scans alive
        return;
    }
    // ---- phase 1: history-free checks; queue the rest ----
    u32 laIdx = pV, laTid = pZ & 0xFFFFFFu, laKind = (pZ >> 24) & 0xFu;
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        u64 before = run;
        run = combine(run, contrib[j]);
        if (!st_head(before) && first + j < P.n && !st_head(contrib[j])) {
            // continues the previous tile's segment: wait for the look-back prefix
            CSTAT(12);
            while (*(volatile u32*)&s_ready == 0u) __nanosleep(64);
            before = combine(*(volatile u64*)&s_prefix, before);
        }
        const u32 i = V[j];
        const u32 c = Z[j] & 0xFFFFFFu, kind = (Z[j] >> 24) & 0xFu;
        bool queue = false;
        u32 mdIdx = laIdx, p = laTid, mdKind = laKind, flags = 0;
        if (first + j < P.n && !st_head(contrib[j])) {
            const u32 lastW = st_lastW(before), as = st_as(before);
            CSTAT(0);
            do {
                if (kind == IGD_LD && lastW == IGD_NONE32) {  // P2: never written
                    CSTAT(1);
                    break;
                }
                if (kind == IGD_LD && lastW != first + j - 1) {  // md = last writer, further back
                    CSTAT(13);
                    const Acc mv = acc_at<MV>(P.val, lastW);
                    mdIdx = mv.idx;
                    p = mv.tk & 0xFFFFFFu;
                    mdKind = (mv.tk >> 24) & 0xFu;
                }
                if (p == c) {  // P3: program order
                    CSTAT(2);
                    break;
                }
                const bool isA = kind >= IGD_ATOM && kind <= IGD_EXCH;
                const u32 bc = g.block(c);
                const bool same_b = g.block(p) == bc;
                if (as && isA && (same_b || as == IGD_SCOPE_DEVICE)) {  // P6
                    CSTAT(3);
                    break;
                }
                const bool same_w = same_b && g.warp(p) == g.warp(c);
                // P4, lockstep clause: md's lane is in this instruction's active mask.  The sort
                // carries two mask summaries in tk bits 31 (full warp) and 30 (own lane only); the
                // mask itself is gathered only for other partial masks
                if (same_w && !(Z[j] >> 30)) CSTAT(5);
                if (same_w && ((Z[j] >> 31) ||
                               (!((Z[j] >> 30) & 1u) &&
                                (((MV ? M[j] : ld_event(P.ev, i).w) >> g.lane(p)) & 1u)))) {
                    CSTAT(4);
                    break;
                }
                flags = (same_w ? QF_SAME_W : 0u) | (same_b ? QF_SAME_B : 0u) |
                        ((st_dev(before) | st_dev(contrib[j])) ? QF_DEV : 0u) |
                        ((st_blk(before) | st_blk(contrib[j])) ? QF_BLK : 0u);
                if (as == IGD_SCOPE_BLOCK) {  // R1 candidate: block-scope atomic, writer elsewhere
                    u32 lwTid = p;
                    if (kind != IGD_LD && lastW != first + j - 1)
                        lwTid = acc_at<MV>(P.val, lastW).tk & 0xFFFFFFu;
                    if (g.block(lwTid) != bc) flags |= QF_R1;
                }
                queue = true;
                CSTAT(6);
            } while (0);
        }
        const u32 qmask = __ballot_sync(IGD_FULL, queue);
        if (qmask) {
            u32 qbase = 0;
#if IGD_CHECK_WARPQ
            if (lane == 0) {
                qbase = warp * QCAP + s_wqn[warp];
                s_wqn[warp] += __popc(qmask);
            }
#else
            if (lane == 0) qbase = atomicAdd(&s_qn, __popc(qmask));
#endif
            qbase = __shfl_sync(IGD_FULL, qbase, 0);
            if (queue) {
                const u32 q = qbase + __popc(qmask & lanemask_lt());
                q_i[q] = i;
                q_md[q] = mdIdx;
                q_c[q] = c | (flags << 24);
                q_p[q] = p | (kind << 24) | (mdKind << 28);
                q_pos[q] = first + j;
            }
        }
        laIdx = i;
        laTid = c;
        laKind = kind;
    }
#if IGD_CHECK_WARPQ
    __syncwarp();
    if (P.debug_stop == 2) return;
    // ---- phase 2: the warp's queued accesses, densely over its lanes ----
    const u32 qn = warp * QCAP + *(volatile u32*)&s_wqn[warp];
    const KeySpace ks = P.ks;
    for (u32 q = warp * QCAP + lane; q < qn; q += 32) {
#else
    __syncthreads();
    if (P.debug_stop == 2) return;
    // ---- phase 2: the queued accesses, densely over the CTA ----
    const u32 qn = s_qn;
    const KeySpace ks = P.ks;
    for (u32 q = t; q < qn; q += THREADS) {
#endif
        const u32 i = q_i[q], mdIdx = q_md[q];
        const u32 c = q_c[q] & 0xFFFFFFu, flags = q_c[q] >> 24;
        const u32 p = q_p[q] & 0xFFFFFFu;
        const bool same_w = flags & QF_SAME_W, same_b = flags & QF_SAME_B;
        if (same_w && q_between(P.desc, P.sts, ks.wb + g.warp(c), mdIdx, i)) continue;  // P4: syncwarp
        const bool grid = q_grid(P, mdIdx, i);
        if (same_b && (grid || q_between(P.desc, P.sts, ks.bb + g.block(c), mdIdx, i))) continue;  // P5
        u32 type = (flags & QF_R1) ? IGD_R1 : 0u;
        if (!type) {
            if (same_b) {
                // R2 (same warp, no sharing) then R3 (same block, no DevShared): md's thread must
                // not have fenced since md (A1, A30)
                if (!(flags & QF_DEV) && !grid && !q_between(P.desc, P.sts, ks.any + p, mdIdx, i))
                    type = (same_w && !(flags & QF_BLK)) ? IGD_R2 : IGD_R3;
            } else if (!grid && !q_between(P.desc, P.sts, ks.dev + p, mdIdx, i)) {
                type = IGD_R4;  // R4: other block, no device fence by md's thread
            }
        }
        if (!type && P.lv.any) {  // R5: lock sets of the last accessor and of this access
            const u32 L = syncx::held_before(P.lv, g, c, i);
            const Acc la = acc_at<MV>(P.val, q_pos[q] - 1);  // the last accessor (rare path)
            const u32 locks = syncx::held_before(P.lv, g, la.tk & 0xFFFFFFu, la.idx);
            if ((locks | L) != 0 && (locks & L) == 0) type = IGD_R5;
        }
        if (type) {
            CSTAT(11);
            const unsigned long long slot = atomicAdd(P.rep_ctr, 1ull);
            if (slot < P.rep_cap) {
                igd_report r;
                // full word from the 32-bit key: the accessed words span < 2^32 from wbase
                r.addr = (P.wbase + (u32)(__ldg(P.key + q_pos[q]) - (u32)P.wbase)) << 2;
                r.cur = P.first_event + i;
                r.prev = P.first_event + mdIdx;
                r.type = (uint8_t)type;
                r.cur_kind = (uint8_t)((q_p[q] >> 24) & 0xFu);
                r.prev_kind = (uint8_t)(q_p[q] >> 28);
                for (int z = 0; z < 5; z++) r.pad[z] = 0;
                P.rep[slot] = r;
            }
        }
    }
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
