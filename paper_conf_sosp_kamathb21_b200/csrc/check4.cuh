// check4.cuh -- a6, ballot formulation: per-address segmented shadow-metadata pass + Table 2 check.
//
// Input: accesses sorted by (word, trace index) (a5); the
// shadow state the paper keeps per 4-byte word (Fig. 4; updates P:1000-1058) before
// access j is a pure function of its word-segment prefix.  Inside a warp the
// segmented scan is done with warp ballots (the packed 64-bit state of check.cuh only crosses warps
// and tiles):
//
//   A warp owns 32*ITEMS consecutive sorted accesses, striped: item j of lane l is position
//   j*32 + l.  Six predicates per access are balloted (segment head, write, atomic, block-scoped
//   atomic, DevShared pair, BlkShared pair: the adjacent-pair predicates of P:1001-1007, reading
//   A5).  Every scan quantity the check needs is then "the highest set bit of a predicate mask
//   at or below my position" compared with my segment's head position:
//     lastW  = highest write  < j, if >= head      (segmented last-of: P:1013-1016, LW of Fig. 4)
//     Atomic = highest atomic < j, if >= head, and its scope (reading A6)
//     DevShared / BlkShared = a pair bit in (head, j]   (sticky OR, A5)
//   Only accesses before the warp's first head need the state carried in from earlier warps
//   (a CTA aggregate) and earlier tiles (decoupled look-back on the packed state of check.cuh).
//
// Phase 1 (history-free checks P1, P2, P3, P6, P4-lockstep) runs on every access; undecided
// accesses go to a per-warp shared-memory queue that the warp drains densely (P4 syncwarp, P5,
// R1..R5 via list queries), with the tile's payload staged in shared memory so md / last-accessor
// lookups inside the tile are shared-memory reads.
#pragma once
#include "check.cuh"

namespace check {

#ifndef IGD_C4_ITEMS
#define IGD_C4_ITEMS 4
#endif
#ifndef IGD_C4_MINB
#define IGD_C4_MINB 7  // default mode: 32 registers (36 B of spills), 7 CTAs/SM: C5 check 53.5 -> 50.5 ms (r02s12; 8 equal, 5-6 slower)
#endif
#ifndef IGD_C4_MBAR
#define IGD_C4_MBAR 1  // warps wait for the tile prefix on an mbarrier (0: poll a shared flag)
#endif
#ifndef IGD_C4_SLEEP
#define IGD_C4_SLEEP 32  // ns between polls of the tile prefix
#endif
constexpr int C4_ITEMS = IGD_C4_ITEMS;
constexpr int C4_WT = 32 * C4_ITEMS;         // accesses per warp
#ifndef IGD_C4_THREADS
#define IGD_C4_THREADS 256
#endif
constexpr int C4_THREADS = IGD_C4_THREADS;
constexpr int C4_WARPS = C4_THREADS / 32;
constexpr int C4_TILE = C4_THREADS * C4_ITEMS;  // accesses per CTA

__device__ __forceinline__ int hib(u32 m) { return 31 - (int)__clz(m); }  // m != 0

// Number of entries x of entity e's list with a < x < b (paper-width IDs, reading A33):
// lower_bound(b) - upper_bound(a), with the descriptor's fast paths
__device__ __noinline__ u32 q_count(const uint4* __restrict__ desc, const u32* __restrict__ ts, u32 e, u32 a, u32 b) {
    const uint4 d = __ldg(desc + e);
    if (d.x == d.y || d.w <= a || d.z >= b || b <= a + 1) return 0;
    u32 lo = d.x, hi = d.y;  // upper_bound(a)
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(ts + mid) <= a) lo = mid + 1;
        else hi = mid;
    }
    const u32 ua = lo;
    hi = d.y;  // lower_bound(b) in [ua, d.y)
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(ts + mid) < b) lo = mid + 1;
        else hi = mid;
    }
    return lo - ua;
}

// q_between without the call (no caller-saved spills in the scan loop): descriptor fast paths,
// then a binary search -- for short lists such as the kernel boundaries
__device__ __forceinline__ bool q_between_inl(const uint4* __restrict__ desc, const u32* __restrict__ ts, u32 e, u32 a,
                                              u32 b) {
    const uint4 d = __ldg(desc + e);
    if (d.x == d.y || d.w <= a) return false;
    if (d.z > a) return d.z < b;
    u32 lo = d.x + 1, hi = d.y - 1;  // successor of a in [lo, hi]: ts[hi] = d.w > a
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(ts + mid) <= a) lo = mid + 1;
        else hi = mid;
    }
    return __ldg(ts + lo) < b;
}

// KB: the trace has kernel boundaries (a separate instantiation: the boundary test costs
// registers, 8% of the kernel, ncu r01s3, when compiled into the common case)
// KT: u32 word keys (low 32 bits; spans < 2^32 words) or u64 keys (word - wbase, a4's wide path)
// FID: paper-fidelity bits -- 1 = Fig. 4-width synchronization IDs (reading A33), 2 = sticky
// sharing flags gate P3-P5 as Table 2 is written (reading A35), 4 = last-k state out (A37)
// the default mode (single GPU, no fidelity bits, u32 keys) at IGD_C4_MINB CTAs per SM; the
// other instantiations carry more state and spill more at 32 registers: 6 CTAs per SM (40)
template <bool MV, bool KB, int FID, bool GEO2, typename KT = u32>
__global__ void __launch_bounds__(C4_THREADS, (!MV && FID == 0 && sizeof(KT) == 4) ? IGD_C4_MINB : 1536 / C4_THREADS) k_check4(Params P) {
    constexpr bool WRAP = (FID & 1) != 0;
    constexpr bool STK = (FID & 2) != 0;
    constexpr bool LKO = (FID & 4) != 0;  // last-k mode (A37): scan state out, decisions in k_lastk
    // streaming mode (sharded payload only): records with an index below
    // P.carry_before are carried state of earlier chunks -- per word a head record and the last
    // accessor, whose mask field holds the word's sticky flags and the scope of its last atomic --
    // and are never checked; the state after each word's last access goes to P.carry_out
    constexpr bool CARRY = MV && (FID & 8) != 0;
    __shared__ u32 s_v[C4_TILE], s_z[C4_TILE];    // staged payload: trace index, tk
    __shared__ u32 q_x[C4_TILE], q_md[C4_TILE];   // per-warp queues: sorted position, md position
    __shared__ uint8_t q_f[C4_TILE];              // queue flags
    __shared__ u64 s_wagg[C4_WARPS];
    __shared__ u64 s_prefix;
    __shared__ u32 s_ready;
    __shared__ __align__(8) u64 s_rbar;  // IGD_C4_MBAR: the tile prefix is ready (one arrival)
    __shared__ u32 s_tile;

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    // Tile ids in the order CTAs start (a ticket, not blockIdx.x): a tile only waits on tiles
    // that are already running, so the decoupled look-back cannot deadlock whatever order the
    // hardware dispatches CTAs in (MPS, SM partitions).
    if (t == 0) {
        s_tile = atomicAdd(P.tile_ctr, 1u);
        s_ready = 0;
        if (IGD_C4_MBAR) mbar_init(&s_rbar, 1);
    }
    __syncthreads();
    const u32 tile = s_tile;
    const u32 tbase = tile * C4_TILE;
    const u32 wloc = warp * C4_WT;
    const u32 wbase = tbase + wloc;
    const u32 n = P.n;
    const Geo g = P.g;
    // GEO2: block_dim is a power of two >= 32, so block / warp / lane are shifts and masks
    const u32 dlog = g.dlog;
    auto blk_of = [&](u32 t) -> u32 { return GEO2 ? t >> dlog : g.block(t); };
    auto warp_of = [&](u32 t) -> u32 { return GEO2 ? t >> 5 : g.warp(t); };
    auto lane_of = [&](u32 t) -> u32 { return GEO2 ? t & 31u : g.lane(t); };
    const KT* keys = reinterpret_cast<const KT*>(P.key);
    KT K[C4_ITEMS];
    u32 V[C4_ITEMS], Z[C4_ITEMS], M[C4_ITEMS];
#pragma unroll
    for (int j = 0; j < C4_ITEMS; j++) {
        const u32 x = wbase + j * 32 + lane;
        const bool in = x < n;
        K[j] = in ? __ldcs(keys + x) : KT(0);
        if (MV) {  // the received record {key, idx, tk, mask}
            const uint4 v = in ? __ldcs(reinterpret_cast<const uint4*>(P.val) + x) : make_uint4(0, 0, 0, 0);
            V[j] = v.y;
            Z[j] = v.z;
            M[j] = v.w;
        } else {
            const unsigned long long v = in ? __ldcs(reinterpret_cast<const unsigned long long*>(P.val) + x) : 0ull;
            V[j] = (u32)v;
            Z[j] = (u32)(v >> 32);
            M[j] = 0;
        }
    }
    // the access before the warp's first one
    KT cK = 0;
    u32 cZ = 0, cV = 0;
    if (lane == 0 && wbase > 0 && wbase <= n) {
        cK = __ldg(keys + wbase - 1);
        const Acc a = acc_at<MV>(P.val, wbase - 1);
        cZ = a.tk;
        cV = a.idx;
    }
#pragma unroll
    for (int j = 0; j < C4_ITEMS; j++) {
        s_v[wloc + j * 32 + lane] = V[j];
        s_z[wloc + j * 32 + lane] = Z[j];
    }

    // ---- predicates and ballots ----
    u32 hm[C4_ITEMS], wm[C4_ITEMS], am[C4_ITEMS], bsm[C4_ITEMS], dm[C4_ITEMS], bm[C4_ITEMS], tm[C4_ITEMS];
    u32 pm[C4_ITEMS], kc[C4_ITEMS];  // CARRY: carried records, key changes
#pragma unroll
    for (int j = 0; j < C4_ITEMS; j++) {
        const u32 x = wbase + j * 32 + lane;
        const KT rK = __shfl_sync(IGD_FULL, K[j], (lane + 31u) & 31u);
        const u32 rZ = __shfl_sync(IGD_FULL, Z[j], (lane + 31u) & 31u);
        const KT pK = lane ? rK : cK;
        const u32 pZ = lane ? rZ : cZ;
        const bool pvalid = lane ? true : (j > 0 || wbase > 0);
        cK = rK;  // lane 0: the last access of row j precedes row j+1's first
        cZ = rZ;
        const bool in = x < n;
        const u32 c = Z[j] & 0xFFFFFFu, kind = (Z[j] >> 24) & 0xFu;
        bool head = !in || !pvalid || pK != K[j];
        if (KB) {
            // a kernel boundary between the previous access of this word and this one ends the
            // word's history (reading A31): a new segment, as if the word were fresh
            const u32 rV = __shfl_sync(IGD_FULL, V[j], (lane + 31u) & 31u);
            const u32 pV = lane ? rV : cV;
            cV = rV;
            if (!head) head = q_between_inl(P.desc, P.sts, P.ks.kb, pV, V[j]);
        }
        bool dev = false, blk = false, same_t = false;
        if (!head) {
            const u32 pt = pZ & 0xFFFFFFu;
            const u32 bp = blk_of(pt), bc = blk_of(c);
            dev = bp != bc;
            // same block: different warps iff the in-block offsets differ in their warp index
            blk = !dev && (GEO2 ? (pt >> 5) != (c >> 5) : ((pt - bp * g.D) >> 5) != ((c - bc * g.D) >> 5));
            same_t = pt == c;
        }
        bool isA = in && kind >= IGD_ATOM && kind <= IGD_EXCH;
        u32 ascp = norm_scope((Z[j] >> 28) & 3u);
        if (CARRY) {
            const bool pseudo = in && V[j] < P.carry_before;
            pm[j] = __ballot_sync(IGD_FULL, pseudo);
            kc[j] = __ballot_sync(IGD_FULL, in && (!pvalid || pK != K[j]));
            if (pseudo && !head) {  // the carried last accessor: the word's state before the chunk
                dev = M[j] & 1u;
                blk = (M[j] >> 1) & 1u;
                same_t = false;
                ascp = (M[j] >> 2) & 3u;
                isA = ascp != 0;
            }
        }
        hm[j] = __ballot_sync(IGD_FULL, head);
        wm[j] = __ballot_sync(IGD_FULL, in && kind != IGD_LD);
        am[j] = __ballot_sync(IGD_FULL, isA);
        bsm[j] = __ballot_sync(IGD_FULL, isA && ascp == IGD_SCOPE_BLOCK);
        dm[j] = __ballot_sync(IGD_FULL, dev);
        bm[j] = __ballot_sync(IGD_FULL, blk);
        tm[j] = __ballot_sync(IGD_FULL, same_t);
        // P4's lockstep clause will need this instruction's active mask when md is likely the
        // previous access, from another lane of the same warp, and the mask is partial: gather
        // it now so the trace read overlaps the scans (phase 1 re-checks the exact condition)
    }

    // ---- warp aggregate in the packed state of check.cuh (state after the warp's last access) ----
    {
        int H = -1, LW = -1, LA = -1, LD = -1, LB = -1;
        u32 las = 0;
#pragma unroll
        for (int j = 0; j < C4_ITEMS; j++) {
            if (hm[j]) H = j * 32 + hib(hm[j]);
            if (wm[j]) LW = j * 32 + hib(wm[j]);
            if (am[j]) {
                LA = j * 32 + hib(am[j]);
                las = (bsm[j] >> hib(am[j])) & 1u ? IGD_SCOPE_BLOCK : IGD_SCOPE_DEVICE;
            }
            if (dm[j]) LD = j * 32 + hib(dm[j]);
            if (bm[j]) LB = j * 32 + hib(bm[j]);
        }
        const u64 agg = st_make((LW >= 0 && LW >= H) ? wbase + (u32)LW : IGD_NONE32,
                                (LA >= 0 && LA >= H) ? las : 0u, LD > H ? 1u : 0u, LB > H ? 1u : 0u,
                                H >= 0 ? 1u : 0u);
        if (lane == 0) s_wagg[warp] = agg;
    }
    __syncthreads();
    if (t == 0) {
        u64 tagg = s_wagg[0];
#pragma unroll
        for (int w = 1; w < C4_WARPS; w++) tagg = combine(tagg, s_wagg[w]);
        u64 prefix = ST_IDENTITY;
        st_relaxed(&P.status[tile], ((tile == 0 || st_head(tagg)) ? ST_INC : ST_AGG) | tagg);
        if (tile > 0 && !(hm[0] & 1u)) {  // a tile starting with a head needs no prefix
            // combine predecessors back to an inclusive status or a head-containing aggregate;
            // a tile with a head has published already (its successors never need more), its
            // accesses before the first head still need the prefix
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
        if (IGD_C4_MBAR) mbar_arrive(&s_rbar);  // release: s_prefix before the phase flips
    }

    // state carried into this warp's first segment (needed only before its first head)
    u64 carry = ST_IDENTITY;
    if (!(hm[0] & 1u)) {
        for (u32 w = 0; w < warp; w++) carry = combine(carry, s_wagg[w]);
        if (!st_head(carry) && tile > 0) {
            if (IGD_C4_MBAR) {
                mbar_wait(&s_rbar, 0);  // suspended in hardware, not polling issue slots
            } else {
                while (*(volatile u32*)&s_ready == 0u) __nanosleep(IGD_C4_SLEEP);
            }
            carry = combine(*(volatile u64*)&s_prefix, carry);
        }
    }

    // ---- phase 1: scan quantities per access, history-free checks, queue the rest ----
    auto tk_at = [&](u32 pos) -> u32 {  // tk of sorted position pos (tile: shared memory)
        return (pos - tbase < (u32)C4_TILE) ? s_z[pos - tbase] : acc_at<MV>(P.val, pos).tk;
    };
    const u32 lt = lanemask_lt(), le = lt | (1u << lane);
    int cH = -1, cW = -1, cA = -1, cD = -1, cB = -1;  // highest bit in rows < j
    u32 cAs = 0;
    u32 qn = 0;  // warp-uniform queue length
    const u32 qb = wloc;
#pragma unroll
    for (int j = 0; j < C4_ITEMS; j++) {
        const u32 x = wbase + j * 32 + lane;
        const bool isHead = (hm[j] >> lane) & 1u;
        bool queue = false;
        u32 mdp = 0, fl = 0;
        if (LKO && isHead && x < n) P.st_out[x] = ST_HEAD_MARK;  // a first access (P1)
        u32 cw_lastW = IGD_NONE32, cw_as = 0;  // CARRY: the state before x (heads: none)
        bool cw_dev = false, cw_blk = false;
        if (!isHead) {
            u32 m = hm[j] & le;
            const int sH = m ? j * 32 + hib(m) : cH;
            m = wm[j] & lt;
            const int lw = m ? j * 32 + hib(m) : cW;
            m = am[j] & lt;
            const int la = m ? j * 32 + hib(m) : cA;
            const u32 las = m ? (((bsm[j] >> hib(m)) & 1u) ? IGD_SCOPE_BLOCK : IGD_SCOPE_DEVICE) : cAs;
            u32 lastW, as;
            if (sH >= 0) {
                lastW = lw >= sH ? wbase + (u32)lw : IGD_NONE32;
                as = la >= sH ? las : 0u;
            } else {
                lastW = lw >= 0 ? wbase + (u32)lw : st_lastW(carry);
                as = la >= 0 ? las : st_as(carry);
            }
            // the sharing flags: needed up front by the sticky / streaming / last-k modes, else
            // only for the accesses that reach the queue (after the P2 / P3 / P6 / P4 exits)
            auto sharing = [&](bool& dev, bool& blk) {
                u32 mm = dm[j] & le;
                const int ldv = mm ? j * 32 + hib(mm) : cD;
                mm = bm[j] & le;
                const int lbv = mm ? j * 32 + hib(mm) : cB;
                if (sH >= 0) {
                    dev = ldv > sH;
                    blk = lbv > sH;
                } else {
                    dev = ldv >= 0 || st_dev(carry);
                    blk = lbv >= 0 || st_blk(carry);
                }
            };
            constexpr bool EAGER = STK || CARRY || LKO;
            bool dev = false, blk = false;
            if (EAGER) sharing(dev, blk);
            const u32 c = Z[j] & 0xFFFFFFu, kind = (Z[j] >> 24) & 0xFu;
            if (CARRY) {
                cw_lastW = lastW;
                cw_as = as;
                cw_dev = dev;
                cw_blk = blk;
            }
            if (CARRY && ((pm[j] >> lane) & 1u)) {
                // a carried record: history only, decided in an earlier chunk
            } else if (LKO) {  // last-k mode (A37): the scan state goes to k_lastk, which decides
                if (x < n) P.st_out[x] = st_make(lastW, as, dev ? 1u : 0u, blk ? 1u : 0u, 0u);
            } else do {
                CSTAT(0);
                if (kind == IGD_LD && lastW == IGD_NONE32) {  // P2: never written
                    CSTAT(1);
                    break;
                }
                // md: the last writer for a load, the last accessor otherwise.  When
                // md is the previous access of the segment (the common case) the thread / block /
                // warp relations to it are the pair bits balloted above: no lookup, no division.
                const bool prevMd = kind != IGD_LD || lastW == x - 1;
                mdp = prevMd ? x - 1 : lastW;
                const bool isA = kind >= IGD_ATOM && kind <= IGD_EXCH;
                bool same_t, same_b, same_w;
                u32 p = IGD_NONE32;  // md's thread, looked up only when needed
                if (prevMd) {
                    same_t = (tm[j] >> lane) & 1u;
                    same_b = !((dm[j] >> lane) & 1u);
                    same_w = same_b && !((bm[j] >> lane) & 1u);
                } else {
                    p = tk_at(mdp) & 0xFFFFFFu;
                    same_t = p == c;
                    const u32 bp = blk_of(p), bc = blk_of(c);
                    same_b = bp == bc;
                    same_w = same_b && (GEO2 ? (p >> 5) == (c >> 5) : ((p - bp * g.D) >> 5) == ((c - bc * g.D) >> 5));
                }
                // A35 (sticky mode): P3 / P4 need the word never shared across warps or blocks
                const bool unshared = !STK || (!dev && !blk);
                if (same_t && unshared) {  // P3: program order
                    CSTAT(2);
                    break;
                }
                if (as && isA && (same_b || as == IGD_SCOPE_DEVICE)) {  // P6
                    CSTAT(3);
                    break;
                }
                // P4 lockstep clause: md's lane in this instruction's active mask (tk bit 31: full
                // warp; bit 30: own lane only; otherwise the mask itself: in the payload in MV
                // mode, else read from the trace in phase 2 -- and only when no syncwarp separates
                // md and the access, the other half of P4: gathering it up front was a random
                // 32-byte read for 13 % of C5's accesses, 95 % of them then decided by the
                // syncwarp (check counters, r02p))
                if (same_w && unshared && (Z[j] >> 31)) {
                    CSTAT(4);
                    break;
                }
                bool defer_mask = false;
                if (same_w && unshared && !(Z[j] >> 30)) {
                    if (MV) {
                        if (p == IGD_NONE32) p = tk_at(mdp) & 0xFFFFFFu;
                        if ((M[j] >> lane_of(p)) & 1u) break;
                    } else {
                        defer_mask = true;
                    }
                }
                if (!EAGER) sharing(dev, blk);
                fl = (same_w ? QF_SAME_W : 0u) | (same_b ? QF_SAME_B : 0u) | (dev ? QF_DEV : 0u) |
                     (defer_mask ? QF_MASK : 0u) |
                     (blk ? QF_BLK : 0u);
                if (as == IGD_SCOPE_BLOCK) {  // R1 candidate: block-scope atomic, writer elsewhere
                    const bool other =
                        lastW == mdp ? !same_b : blk_of(tk_at(lastW) & 0xFFFFFFu) != blk_of(c);
                    if (other) fl |= QF_R1;
                }
                queue = true;
                CSTAT(6);
            } while (0);
        }
        if (CARRY && P.carry_out && x < n) {
            // streaming mode: after a word's last access of this run, its state goes out as the next
            // chunk's carried pair {head record, last accessor + flags}
            bool last;
            if (x + 1 >= n) last = true;
            else if (lane < 31) last = (kc[j] >> (lane + 1)) & 1u;
            else if (j + 1 < C4_ITEMS) last = kc[(j + 1) % C4_ITEMS] & 1u;
            else last = __ldg(keys + x + 1) != K[j];
            uint4* co = reinterpret_cast<uint4*>(P.carry_out) + 2 * (u64)x;
            if (last) {
                const u32 kd = (Z[j] >> 24) & 0xFu;
                const u32 sX = ((bsm[j] >> lane) & 1u) ? IGD_SCOPE_BLOCK : IGD_SCOPE_DEVICE;
                const u32 lw = kd != IGD_LD ? x : cw_lastW;
                const u32 asA = ((am[j] >> lane) & 1u) ? sX : cw_as;
                const u32 k32 = (u32)K[j];
                if (lw != IGD_NONE32 && lw != x) {
                    const u32 li = (lw - tbase < (u32)C4_TILE) ? s_v[lw - tbase] : acc_at<MV>(P.val, lw).idx;
                    co[0] = make_uint4(k32, li, tk_at(lw), 0u);
                } else {  // no earlier writer to keep: a neutral head (a load, never a writer)
                    co[0] = make_uint4(k32, V[j], (Z[j] & 0xFFFFFFu) | ((u32)IGD_LD << 24), 0u);
                }
                co[1] = make_uint4(k32, V[j], Z[j], (cw_dev ? 1u : 0u) | (cw_blk ? 2u : 0u) | (asA << 2));
            } else {
                co[1] = make_uint4(0u, IGD_NONE32, 0u, 0u);
            }
        }
        const u32 qmask = __ballot_sync(IGD_FULL, queue);
        if (queue) {
            const u32 q = qb + qn + __popc(qmask & lt);
            q_x[q] = x;
            q_md[q] = mdp;
            q_f[q] = (uint8_t)fl;
        }
        qn += __popc(qmask);
        if (hm[j]) cH = j * 32 + hib(hm[j]);
        if (wm[j]) cW = j * 32 + hib(wm[j]);
        if (am[j]) {
            cA = j * 32 + hib(am[j]);
            cAs = ((bsm[j] >> hib(am[j])) & 1u) ? IGD_SCOPE_BLOCK : IGD_SCOPE_DEVICE;
        }
        if (dm[j]) cD = j * 32 + hib(dm[j]);
        if (bm[j]) cB = j * 32 + hib(bm[j]);
    }
    __syncwarp();

    // ---- phase 2: the warp's queued accesses, densely over its lanes ----
    // One entry per lane, its list queries in Table 2's order with early exits.  Issuing all of an
    // entry's queries at once and interleaving two entries per lane were both measured slower
    // (20.9 and 22.2 vs 14.8 ms at C5@1e9, round 1): this phase is bound by the queries' total
    // L2 / issue work, not by the latency of one chain.
    const KeySpace ks = P.ks;
    for (u32 k = lane; k < qn; k += 32) {
        const u32 x = q_x[qb + k], mdp = q_md[qb + k], flags = q_f[qb + k];
        const u32 i = s_v[x - tbase], z = s_z[x - tbase];
        const u32 c = z & 0xFFFFFFu, kind = (z >> 24) & 0xFu;
        u32 mdIdx, mdz;
        if (mdp - tbase < (u32)C4_TILE) {
            mdIdx = s_v[mdp - tbase];
            mdz = s_z[mdp - tbase];
        } else {
            const Acc a = acc_at<MV>(P.val, mdp);
            mdIdx = a.idx;
            mdz = a.tk;
        }
        const u32 p = mdz & 0xFFFFFFu;
        const bool same_w = flags & QF_SAME_W, same_b = flags & QF_SAME_B;
        // A35 (sticky mode): P4 needs neither sharing flag, P5 no DevShared
        const bool p4w = same_w && (!STK || !(flags & (QF_DEV | QF_BLK)));
        const bool p5b = same_b && (!STK || !(flags & QF_DEV));
        u32 type;
        if (WRAP) {
            // reading A33: an ID moved iff the number of its events since md is not a multiple of
            // 2^width (Fig. 4: WarpBarID 6, BlkBarID 8, DevFenceID 6, BlkFenceID 6 bits)
            const u32 gcnt = P.glo != P.ghi ? q_count(P.desc, P.sts, ks.grid, mdIdx, i) : 0u;
            if (p4w && (q_count(P.desc, P.sts, ks.wb + warp_of(c), mdIdx, i) & 63u)) continue;  // P4
            if (p4w && (flags & QF_MASK) && ((mask_of(P, i) >> lane_of(p)) & 1u)) continue;  // P4 lockstep
            if (p5b && ((q_count(P.desc, P.sts, ks.bb + blk_of(c), mdIdx, i) + gcnt) & 255u)) continue;  // P5
            type = (flags & QF_R1) ? IGD_R1 : 0u;
            if (!type) {
                const u32 dfen = q_count(P.desc, P.sts, ks.dev + p, mdIdx, i);  // device fences of md's thread
                const bool noDev = ((dfen + gcnt) & 63u) == 0;
                if (same_b) {
                    if (!(flags & QF_DEV)) {
                        const u32 bfen = q_count(P.desc, P.sts, ks.any + p, mdIdx, i) - dfen;  // block-scope
                        if (noDev && (bfen & 63u) == 0) type = (same_w && !(flags & QF_BLK)) ? IGD_R2 : IGD_R3;
                    }
                } else if (noDev) {
                    type = IGD_R4;
                }
            }
        } else {
        if (p4w && q_between(P.desc, P.sts, ks.wb + warp_of(c), mdIdx, i)) {  // P4: syncwarp
            CSTAT(12);
            continue;
        }
        if (p4w && (flags & QF_MASK)) {  // P4: lockstep, the mask read only now
            CSTAT(5);
            if ((mask_of(P, i) >> lane_of(p)) & 1u) continue;
        }
        const bool grid = q_grid(P, mdIdx, i);
        if (p5b && (grid || q_between(P.desc, P.sts, ks.bb + blk_of(c), mdIdx, i))) {  // P5
            CSTAT(13);
            continue;
        }
        type = (flags & QF_R1) ? IGD_R1 : 0u;
        // R2 (same warp, no sharing) then R3 (same block, no DevShared): md's thread has not fenced
        // (any scope) since md (A1, A30); R4 (other block): no device fence by md's thread.  One
        // query call site for both (divergent lanes would otherwise run two in turn).
        if (!type && !grid && (!same_b || !(flags & QF_DEV))) {
            CSTAT(14);
            if (!q_between(P.desc, P.sts, (same_b ? ks.any : ks.dev) + p, mdIdx, i))
                type = same_b ? ((same_w && !(flags & QF_BLK)) ? IGD_R2 : IGD_R3) : IGD_R4;
        }
        }
        if (!type && P.lv.any) {  // R5: lock sets of the last accessor and of this access
            u32 laIdx, laz;
            if (x - 1 - tbase < (u32)C4_TILE) {
                laIdx = s_v[x - 1 - tbase];
                laz = s_z[x - 1 - tbase];
            } else {
                const Acc a = acc_at<MV>(P.val, x - 1);
                laIdx = a.idx;
                laz = a.tk;
            }
            if (syncx::may_hold(P.lv, c) || syncx::may_hold(P.lv, laz & 0xFFFFFFu)) {
                CSTAT(15);
                u32 L, locks;
                syncx::held_before2(P.lv, c, i, laz & 0xFFFFFFu, laIdx, L, locks);
                if ((locks | L) != 0 && (locks & L) == 0) type = IGD_R5;
            }
        }
        if (type) {
            CSTAT(11);
            const unsigned long long slot = atomicAdd(P.rep_ctr, 1ull);
            if (slot < P.rep_cap) {
                igd_report r;
                // full word from the 32-bit key: the accessed words span < 2^32 from wbase
                if (P.addr_from_ev) r.addr = ev_addr(ld_event(P.ev, i)) & ~3ull;  // tag mode (A36): the key is the entry
                else if (sizeof(KT) == 8) r.addr = (P.wbase + (u64)__ldg(keys + x)) << 2;  // key = word - wbase
                else r.addr = (P.wbase + (u32)((u32)__ldg(keys + x) - (u32)P.wbase)) << 2;
                r.cur = P.first_event + i;
                r.prev = P.first_event + mdIdx;
                r.type = (uint8_t)type;
                r.cur_kind = (uint8_t)kind;
                r.prev_kind = (uint8_t)((mdz >> 24) & 0xFu);
                for (int z2 = 0; z2 < 5; z2++) r.pad[z2] = 0;
                P.rep[slot] = r;
            }
        }
    }
}

}  // namespace check
