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
// The scans run per tile (256 threads x 4 accesses) and across tiles with decoupled look-back;
// a tile that contains a segment head publishes its inclusive state immediately, so only
// tiles inside one long (hot-word) segment ever wait.  The synchronization-counter comparisons
// of Table 2 become interval queries on the a2 CSR lists ("did md's thread fence in
// (md.idx, i)?", reading A1), lock sets come from the a3 change points.
#pragma once
#include "common.cuh"
#include "sync.cuh"

namespace check {

constexpr int THREADS = 256;
constexpr int ITEMS = 4;
constexpr int TILE = THREADS * ITEMS;

// Packed scan state (39 bits): [31:0] lastW position (NONE = 0xFFFFFFFF), [33:32] scope of the
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
    u32 lw = st_lastW(b) != IGD_NONE32 ? st_lastW(b) : st_lastW(a);
    u32 as = st_as(b) ? st_as(b) : st_as(a);
    return st_make(lw, as, st_dev(a) | st_dev(b), st_blk(a) | st_blk(b), st_head(a));
}

struct Params {
    const u32* key;  // sorted word keys
    const u32* val;  // sorted trace indices
    u32 n;           // number of accesses
    const igd_event* ev;
    Geo g;
    KeySpace ks;
    const u32* off;  // sync CSR offsets
    const u32* sts;  // sync timestamps
    syncx::LockView lv;
    u64* status;     // [n_tiles] zeroed
    u32* tile_ctr;   // zeroed
    igd_report* rep;
    u64 rep_cap;
    unsigned long long* rep_ctr;
    u64 first_event; // global index offset (multi-rank)
};

__device__ __forceinline__ bool sync_between(const Params& P, u32 key, u32 a, u32 b) {
    const u32 lo = __ldg(P.off + key), hi = __ldg(P.off + key + 1);
    if (lo == hi) return false;
    return between(P.sts, lo, hi, a, b);
}

__global__ void __launch_bounds__(THREADS) k_check(Params P) {
    __shared__ u32 s_tile;
    __shared__ u64 s_wagg[THREADS / 32];
    __shared__ u64 s_prefix;
    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) s_tile = atomicAdd(P.tile_ctr, 1u);
    __syncthreads();
    const u32 tile = s_tile;
    const u64 first = (u64)tile * TILE + (u64)t * ITEMS;
    const Geo g = P.g;

    u32 K[ITEMS], V[ITEMS];
    if (first + ITEMS <= P.n) {
        uint4 k4 = __ldcs(reinterpret_cast<const uint4*>(P.key + first));
        uint4 v4 = __ldcs(reinterpret_cast<const uint4*>(P.val + first));
        K[0] = k4.x; K[1] = k4.y; K[2] = k4.z; K[3] = k4.w;
        V[0] = v4.x; V[1] = v4.y; V[2] = v4.z; V[3] = v4.w;
    } else {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            K[j] = (first + j < P.n) ? P.key[first + j] : 0;
            V[j] = (first + j < P.n) ? P.val[first + j] : 0;
        }
    }
    uint4 E[ITEMS];
#pragma unroll
    for (int j = 0; j < ITEMS; j++) E[j] = (first + j < P.n) ? ld_event(P.ev, V[j]) : make_uint4(0, 0, 0, 0);

    // previous element (first - 1): from the neighbour lane, lane 0 reads it
    u32 pK = __shfl_up_sync(IGD_FULL, K[ITEMS - 1], 1);
    u32 pV = __shfl_up_sync(IGD_FULL, V[ITEMS - 1], 1);
    u32 pZ = __shfl_up_sync(IGD_FULL, E[ITEMS - 1].z, 1);
    bool has_prev = first > 0;
    if (lane == 0 && has_prev && first - 1 < P.n) {
        pK = P.key[first - 1];
        pV = P.val[first - 1];
        pZ = ld_event(P.ev, pV).z;
    }

    // per-element scan contributions
    u64 contrib[ITEMS];
    u32 prevTid = pZ & 0xFFFFFFu;
    u32 prevKey = pK;
    bool prevValid = has_prev;
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const bool inr = first + j < P.n;
        const u32 c = ev_tid(E[j]);
        const u32 kind = ev_kind(E[j]);
        const bool head = !prevValid || prevKey != K[j];
        u32 dev = 0, blk = 0;
        if (!head) {
            u32 bp = g.block(prevTid), bc = g.block(c);
            if (bp != bc) dev = 1;
            else if (g.warp(prevTid) != g.warp(c)) blk = 1;
        }
        u32 lw = (inr && kind != IGD_LD) ? (u32)(first + j) : IGD_NONE32;
        u32 as = (inr && kind >= IGD_ATOM && kind <= IGD_EXCH) ? norm_scope(ev_scope(E[j])) : 0u;
        contrib[j] = inr ? st_make(lw, as, dev, blk, head ? 1u : 0u) : st_make(IGD_NONE32, 0, 0, 0, 0);
        prevTid = c;
        prevKey = K[j];
        prevValid = true;
    }
    // thread aggregate
    u64 agg = contrib[0];
#pragma unroll
    for (int j = 1; j < ITEMS; j++) agg = combine(agg, contrib[j]);
    // warp inclusive scan
    u64 inc = agg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        u64 x = __shfl_up_sync(IGD_FULL, inc, o);
        if (lane >= (u32)o) inc = combine(x, inc);
    }
    if (lane == 31) s_wagg[warp] = inc;
    u64 wexcl = __shfl_up_sync(IGD_FULL, inc, 1);
    if (lane == 0) wexcl = ST_IDENTITY;
    __syncthreads();
    if (warp == 0) {
        // scan warp aggregates (8) -> tile aggregate, look back
        u64 tagg = s_wagg[0];
#pragma unroll
        for (int w = 1; w < THREADS / 32; w++) tagg = combine(tagg, s_wagg[w]);
        u64 prefix = ST_IDENTITY;
        if (tile == 0 || st_head(tagg)) {
            if (lane == 0) st_relaxed(&P.status[tile], ST_INC | tagg);
            // the tile prefix is still needed for the elements before the first head
        } else {
            if (lane == 0) st_relaxed(&P.status[tile], ST_AGG | tagg);
        }
        if (tile > 0) {
            // walk back: combine predecessors until an inclusive status or a head-containing aggregate
            if (lane == 0) {
                long tt = (long)tile - 1;
                u64 acc = ST_IDENTITY;
                bool have = false;
                while (tt >= 0) {
                    u64 s;
                    do {
                        s = ld_relaxed(&P.status[tt]);
                    } while ((s >> 62) == 0);
                    u64 v = s & ST_VAL_MASK;
                    acc = have ? combine(v, acc) : v;
                    have = true;
                    if ((s >> 62) == 2 || st_head(v)) break;
                    tt--;
                }
                prefix = acc;
                if (!st_head(tagg)) st_relaxed(&P.status[tile], ST_INC | combine(prefix, tagg));
            }
        }
        if (lane == 0) s_prefix = prefix;
    }
    __syncthreads();
    u64 wpre = ST_IDENTITY;
    for (u32 w = 0; w < warp; w++) wpre = (w == 0) ? s_wagg[0] : combine(wpre, s_wagg[w]);
    u64 run = combine(combine(s_prefix, wpre), wexcl);  // state before this thread's first element

    // evaluate each access
    u32 laIdx = pV, laTid = pZ & 0xFFFFFFu, laKind = (pZ >> 24) & 0xFu;
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const bool inr = first + j < P.n;
        const u64 before = run;
        run = combine(run, contrib[j]);
        const u32 i = V[j];
        const u32 c = ev_tid(E[j]), kind = ev_kind(E[j]);
        if (inr && !st_head(contrib[j])) {
            const u32 lastW = st_lastW(before), as = st_as(before);
            const u32 dev = st_dev(before) | st_dev(contrib[j]);
            const u32 blk = st_blk(before) | st_blk(contrib[j]);
            do {
                if (kind == IGD_LD && lastW == IGD_NONE32) break;  // P2
                u32 mdIdx, p, mdKind;
                if (kind == IGD_LD && lastW != (u32)(first + j - 1)) {
                    mdIdx = __ldg(P.val + lastW);
                    uint4 me = ld_event(P.ev, mdIdx);
                    p = ev_tid(me);
                    mdKind = ev_kind(me);
                } else {
                    mdIdx = laIdx;
                    p = laTid;
                    mdKind = laKind;
                }
                if (p == c) break;  // P3
                const bool isA = kind >= IGD_ATOM && kind <= IGD_EXCH;
                const u32 bp = g.block(p), bc = g.block(c);
                const bool same_b = bp == bc;
                if (as && isA && (same_b || as == IGD_SCOPE_DEVICE)) break;  // P6
                const u32 wp = g.warp(p), wc = g.warp(c);
                const bool same_w = wp == wc;
                if (same_w && ((E[j].w >> g.lane(p)) & 1u)) break;                      // P4 (lockstep)
                if (same_w && sync_between(P, P.ks.wb + wc, mdIdx, i)) break;           // P4 (syncwarp)
                bool grid = false, grid_known = false;
                if (same_b) {
                    if (sync_between(P, P.ks.bb + bc, mdIdx, i)) break;                 // P5
                    grid = sync_between(P, P.ks.grid, mdIdx, i);
                    grid_known = true;
                    if (grid) break;                                                    // P5 (grid)
                }
                u32 type = 0;
                if (as == IGD_SCOPE_BLOCK) {  // R1
                    u32 lwTid = (lastW == (u32)(first + j - 1)) ? laTid : ev_tid(ld_event(P.ev, __ldg(P.val + lastW)));
                    if (g.block(lwTid) != bc) type = IGD_R1;
                }
                if (!type) {
                    if (!grid_known) grid = sync_between(P, P.ks.grid, mdIdx, i);
                    if (same_b) {
                        // R2 (same warp, no sharing) then R3 (same block, no DevShared); both
                        // need md's thread not to have fenced since md (A1, A30)
                        if (!dev) {
                            bool noAny = !grid && !sync_between(P, P.ks.any + p, mdIdx, i);
                            if (noAny) type = (same_w && !blk) ? IGD_R2 : IGD_R3;
                        }
                    } else {
                        bool noDev = !grid && !sync_between(P, P.ks.dev + p, mdIdx, i);
                        if (noDev) type = IGD_R4;  // R4: other block, no device fence by md's thread
                    }
                }
                if (!type) {
                    const u32 L = syncx::held_before(P.lv, g, c, i);
                    const u32 locks = syncx::held_before(P.lv, g, laTid, laIdx);
                    if ((locks | L) != 0 && (locks & L) == 0) type = IGD_R5;
                }
                if (type) {
                    unsigned long long slot = atomicAdd(P.rep_ctr, 1ull);
                    if (slot < P.rep_cap) {
                        igd_report r;
                        r.addr = (ev_addr(E[j]) >> 2) << 2;
                        r.cur = P.first_event + i;
                        r.prev = P.first_event + mdIdx;
                        r.type = (uint8_t)type;
                        r.cur_kind = (uint8_t)kind;
                        r.prev_kind = (uint8_t)mdKind;
                        for (int q = 0; q < 5; q++) r.pad[q] = 0;
                        P.rep[slot] = r;
                    }
                }
            } while (0);
        }
        laIdx = i;
        laTid = c;
        laKind = kind;
    }
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
