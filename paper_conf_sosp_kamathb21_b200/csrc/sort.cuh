// sort.cuh -- a5: stable LSD radix sort of (u32 or u64 key, u32 / u64 / 16-byte value) pairs, one
// kernel per 8-bit digit ("onesweep": upfront digit histograms + per-tile decoupled look-back per
// digit).
//
// Stability: within a tile, each warp owns a contiguous run of 32*ITEMS inputs processed item
// by item in input order; the rank of an input among equal digits is (earlier tiles via
// look-back) + (earlier warps of the tile) + (earlier items / lanes of the warp), i.e. its
// input order.  Sorting accesses that arrive in trace order therefore yields (word, time)
// order, the order the per-word shadow replay needs (SURVEY 8(c) C.3 "equivalent formulation").
//
// Per tile: keys and values arrive in shared memory by one TMA bulk copy each; keys are ranked
// with a warp multisplit (rows ranked alternately by eight ballots and match.any), the tile's
// digit counts are published early and looked back, every input scatters its source position to
// its tile position, and each output slot gathers its key and value from the staged tile and
// writes them in digit runs (the kernel is bound by the shared-memory / MIO pipe: the gather
// needs no reorder buffers and no value registers; 3 CTAs per SM).
#pragma once
#include "common.cuh"

namespace rsort {

#ifndef IGD_SORT_THREADS
#define IGD_SORT_THREADS 256  // a multiple of RADIX: threads >= RADIX own one digit in the per-digit steps
#endif
constexpr int THREADS = IGD_SORT_THREADS;
constexpr int WARPS = THREADS / 32;
#ifndef IGD_SORT_ITEMS
#define IGD_SORT_ITEMS 16
#endif
#ifndef IGD_SORT_EARLY
#define IGD_SORT_EARLY 1  // publish tile digit counts before ranking (C5@1e9: 21.6 -> 21.2 ms over 3 passes)
#endif
#ifndef IGD_SORT_MIX
#define IGD_SORT_MIX 2  // every other row ranked with match.any: C5@1e9 sort 20.4 -> 19.8 ms
#endif
#ifndef IGD_SORT_LB
#define IGD_SORT_LB 4
#endif
constexpr int ITEMS = IGD_SORT_ITEMS;
constexpr int TILE = THREADS * ITEMS;  // 4096
constexpr int RADIX = 256;
static_assert(THREADS % RADIX == 0, "one thread per digit in the per-digit steps");

// Exclusive digit bases for every pass from the 4 x 256 histogram.
__global__ void k_digit_base(const u32* __restrict__ hist, u32* __restrict__ base) {
    __shared__ u32 s[RADIX];
    const int p = blockIdx.x, d = threadIdx.x;
    u32 v = hist[p * RADIX + d];
    s[d] = v;
    __syncthreads();
    // Hillis-Steele inclusive scan (256 elements, once per sort: negligible)
    for (int o = 1; o < RADIX; o <<= 1) {
        u32 t = (d >= o) ? s[d - o] : 0;
        __syncthreads();
        s[d] += t;
        __syncthreads();
    }
    base[p * RADIX + d] = s[d] - v;
}

// 4-digit histogram of a key array (used for report keys; the ingest pass builds its own).
__global__ void k_hist4(const u32* __restrict__ keys, u64 n, u32* __restrict__ hist) {
    __shared__ u32 s[4][RADIX];
    for (int i = threadIdx.x; i < 4 * RADIX; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) {
        u32 k = keys[i];
        atomicAdd(&s[0][k & 255u], 1u);
        atomicAdd(&s[1][(k >> 8) & 255u], 1u);
        atomicAdd(&s[2][(k >> 16) & 255u], 1u);
        atomicAdd(&s[3][k >> 24], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * RADIX; i += blockDim.x) {
        u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

// 8-digit histogram of u64 keys (the wide-key path of a4); digits >= first_digit.
__global__ void k_hist8(const u64* __restrict__ keys, u64 n, u32* __restrict__ hist, int first_digit) {
    __shared__ u32 s[8][RADIX];
    for (int i = threadIdx.x; i < 8 * RADIX; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) {
        const u64 k = keys[i];
        for (int p = first_digit; p < 8; p++) atomicAdd(&s[p][(u32)(k >> (8 * p)) & 255u], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 8 * RADIX; i += blockDim.x) {
        const u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

struct PassParams {
    const void* kin;  // u32 or u64 keys (template KT)
    const void* vin;  // u32, u64 or uint4 values (template VT)
    void* kout;
    void* vout;
    u32 n;
    u32 shift;
    u32 dmask;              // 255, or fewer bits for the top digit of a masked key (tag mode, A36)
    const u32* digit_base;  // [256] exclusive global offsets of this pass's digits
    u64* status;            // [n_tiles * 256] digit statuses (ds_make), tagged with `epoch`
    u32 epoch;              // this pass's tag (1..DS_EPOCH_MAX): no clearing between passes
    u32* tile_ctr;          // zeroed before the pass: tile tickets (the TAIL launch follows the full one)
};

// Mask of the lanes (within vmask) whose 8-bit digit equals this lane's.
template <int MODE>
__device__ __forceinline__ u32 peers_of(u32 d, u32 vmask) {
    if (MODE == 0) {
        return __match_any_sync(IGD_FULL, d) & vmask;
    } else {
        u32 peers = vmask;
#pragma unroll
        for (int b = 0; b < 8; b++) {
            const u32 bit = (d >> b) & 1u;
            const u32 bal = __ballot_sync(IGD_FULL, bit);
            peers &= bit ? bal : ~bal;
        }
        return peers;
    }
}

// Dynamic shared memory of k_onesweep<VT, TAIL, KT>: staged keys, staged values, the u16 source
// position of every output slot.
template <typename VT, typename KT = u32>
constexpr size_t onesweep_smem() {
    return (size_t)TILE * sizeof(KT) + (size_t)TILE * sizeof(VT) + (size_t)TILE * 2;
}

// Decoupled look-back for digit d of `tile`: the sum of the digit's counts over all earlier tiles.
// LB predecessor statuses are requested at once, so a walk back over tiles that have published
// only their aggregate costs one L2 round trip per LB tiles instead of one per tile.
__device__ __forceinline__ u64 lookback_digit(const PassParams& P, u32 tile, u32 d) {
    u64 excl = 0;
    if (tile == 0) return 0;
    long tt = (long)tile - 1;
    bool done = false;
    while (!done) {
        u64 s[IGD_SORT_LB];
#pragma unroll
        for (int q = 0; q < IGD_SORT_LB; q++)
            s[q] = tt - q >= 0 ? ld_relaxed(P.status + (u64)(tt - q) * RADIX + d) : ds_make(ST_INC, P.epoch, 0);
#pragma unroll
        for (int q = 0; q < IGD_SORT_LB; q++) {
            if (!done) {
                s[q] = ds_spin(P.status + (u64)(tt - q) * RADIX + d, s[q], P.epoch);
                excl += s[q] & DS_VAL_MASK;
                done = (s[q] >> 62) == 2;
            }
        }
        tt -= IGD_SORT_LB;
    }
    return excl;
}

// TAIL = false: every tile of the launch is full (no bounds tests on the hot path); TAIL = true:
// the one partial last tile, launched after the full ones (its look-back finds them published).
// KT = u32 (word spans < 2^32 words) or u64 keys (reading a4's wide path: up to 8 digit passes)
template <typename VT, bool TAIL, typename KT = u32>
#ifndef IGD_SORT_MINB
#define IGD_SORT_MINB 3
#endif
__global__ void __launch_bounds__(THREADS, IGD_SORT_MINB) k_onesweep(PassParams P) {
    __shared__ u32 s_whist[WARPS][RADIX];  // per-warp digit counts, then tile position bases
    __shared__ u32 s_gbase[RADIX];
    __shared__ u32 s_tile;
    __shared__ u32 s_wsum[WARPS];
    __shared__ u32 s_cnt[RADIX];  // tile digit counts (IGD_SORT_EARLY)
    __shared__ __align__(8) u64 s_mbar[2];
    extern __shared__ __align__(16) unsigned char s_dyn[];
    KT* s_k = reinterpret_cast<KT*>(s_dyn);                           // keys in, then keys out
    VT* s_v = reinterpret_cast<VT*>(s_dyn + TILE * sizeof(KT));       // values in, then values out
    const VT* vin = reinterpret_cast<const VT*>(P.vin);
    VT* vout = reinterpret_cast<VT*>(P.vout);
    const KT* kin = reinterpret_cast<const KT*>(P.kin);
    KT* kout = reinterpret_cast<KT*>(P.kout);

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) {
        // tile id, then TMA bulk copies of the tile's keys and values into shared memory: the
        // value copy lands while the keys are ranked.  The id is a ticket in CTA start order (the
        // full-tile launch takes 0..full-1, the tail launch after it the last one), so a tile's
        // look-back only waits on running tiles, whatever the dispatch order.
        const u32 tile = atomicAdd(P.tile_ctr, 1u);
        s_tile = tile;
        const u64 base = (u64)tile * TILE;
        if (!TAIL) {
            mbar_init(&s_mbar[0], 1);
            mbar_init(&s_mbar[1], 1);
            mbar_expect_tx(&s_mbar[0], TILE * sizeof(KT));
            bulk_g2s(s_k, kin + base, TILE * sizeof(KT), &s_mbar[0]);
            mbar_expect_tx(&s_mbar[1], TILE * sizeof(VT));
            bulk_g2s(s_v, vin + base, TILE * sizeof(VT), &s_mbar[1]);
        }
    }
    for (int i = t; i < WARPS * RADIX; i += THREADS) (&s_whist[0][0])[i] = 0;
    if (IGD_SORT_EARLY && t < RADIX) s_cnt[t] = 0;
    __syncthreads();
    const u32 tile = s_tile;
    const u32 base = tile * TILE;  // n <= 2^32 - 2^13 (checked by the host)
    const u32 wofs = warp * 32 * ITEMS;
    const u32 wbase = base + wofs;
    const u32 shift = P.shift, dmask = P.dmask;
    constexpr bool full = !TAIL;

    KT key[ITEMS];
    if (full) {
        mbar_wait(&s_mbar[0], 0);
#pragma unroll
        for (int j = 0; j < ITEMS; j++) key[j] = s_k[wofs + j * 32 + lane];
    } else {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u32 i = wbase + j * 32 + lane;
            key[j] = i < P.n ? __ldcs(kin + i) : KT(0);
            s_k[wofs + j * 32 + lane] = key[j];  // the tail tile is staged by plain loads
            s_v[wofs + j * 32 + lane] = i < P.n ? __ldcs(vin + i) : VT{};
        }
    }
    if (IGD_SORT_EARLY) {
        // tile digit counts first, published before ranking (see fused.cuh)
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            if (full || wbase + j * 32 + lane < P.n) atomicAdd(&s_cnt[(u32)(key[j] >> shift) & dmask], 1u);
        __syncthreads();
        if (t < RADIX) st_relaxed(P.status + (u64)tile * RADIX + t, ds_make(tile == 0 ? ST_INC : ST_AGG, P.epoch, s_cnt[t]));
    }
    u32 rank[ITEMS];
    const u32 lt = lanemask_lt();
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const bool valid = full || wbase + j * 32 + lane < P.n;
        const u32 vmask = full ? IGD_FULL : __ballot_sync(IGD_FULL, valid);
        const u32 d = (u32)(key[j] >> shift) & dmask;
        // invalid lanes (last tile) get a unique out-of-range digit; masked out of every peer set.
        // IGD_SORT_MIX = N: one row in N is ranked with match.any (MIO pipe), the others with the
        // 8 ballots (ALU / issue): the two bottleneck on different units
        const u32 peers = (IGD_SORT_MIX && (j % IGD_SORT_MIX) == IGD_SORT_MIX - 1)
                              ? peers_of<0>(valid ? d : (0x100u | lane), vmask)
                              : peers_of<1>(valid ? d : (0x100u | lane), vmask);
        const u32 leader = __ffs(peers) - 1;
        // every lane reads its digit's count (peers read one address: a broadcast), then the
        // leader bumps it -- no shuffle of the leader's value (r02s24: C5 sort 75.7 -> 74.6 ms,
        // fused 38.2 -> 37.8 ms against leader load + store + shuffle or a leader atomicAdd)
        u32 old = 0;
        if (valid) old = s_whist[warp][d];
        __syncwarp();
        if (lane == leader && valid) s_whist[warp][d] = old + __popc(peers);
        rank[j] = old + __popc(peers & lt);
        __syncwarp();
    }
    __syncthreads();
    // per digit (threads < RADIX): tile count, exclusive scan over digits, then every warp's base
    // for the digit (tile exclusive + earlier warps) in place of its count -- one shared load per
    // rank below
    constexpr int DW = RADIX / 32;  // warps that own digits
    u32 cnt = 0, tile_excl = 0, inc = 0;
    u32 c[WARPS];
    const u32 d = t;
    if (t < RADIX) {
#pragma unroll
        for (int w = 0; w < WARPS; w++) {
            c[w] = s_whist[w][d];
            cnt += c[w];
        }
        if (!IGD_SORT_EARLY) st_relaxed(P.status + (u64)tile * RADIX + d, ds_make(tile == 0 ? ST_INC : ST_AGG, P.epoch, cnt));
        inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            u32 x = __shfl_up_sync(IGD_FULL, inc, o);
            if (lane >= (u32)o) inc += x;
        }
        if (lane == 31) s_wsum[warp] = inc;
    }
    __syncthreads();
    if (t < RADIX) {
        u32 wpre = 0;
#pragma unroll
        for (int w = 0; w < DW; w++)
            if ((u32)w < warp) wpre += s_wsum[w];
        tile_excl = wpre + inc - cnt;
        u32 run = tile_excl;
#pragma unroll
        for (int w = 0; w < WARPS; w++) {
            s_whist[w][d] = run;
            run += c[w];
        }
        // Decoupled look-back for this digit: LB predecessor statuses are requested at once, so a
        // walk back over tiles that have published only their aggregate costs one L2 round trip
        // per LB tiles instead of one per tile (C5: 127 -> 118 ms over 4 passes with LB = 4)
        u64 excl = 0;
        if (tile > 0) {
            excl = lookback_digit(P, tile, d);
            st_relaxed(P.status + (u64)tile * RADIX + d, ds_make(ST_INC, P.epoch, excl + cnt));
        }
        // output position of tile position i with digit d = s_gbase[d] + i (u32 arithmetic wraps
        // back into range): one shared load per written element instead of two
        s_gbase[d] = P.digit_base[d] + (u32)excl - tile_excl;
    }
    __syncthreads();
    // Output by gathering: every input scatters only its tile position's source index (u16), and
    // output slot i then reads its key and value from the staged input -- no key / value reorder
    // buffers, no value registers, one barrier; 2 fewer shared-memory round trips per element
    // than reordering keys and values through shared memory (the MIO pipe bounds this kernel)
    {
        u16* s_src = reinterpret_cast<u16*>(s_dyn + TILE * sizeof(KT) + TILE * sizeof(VT));
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u32 d = (u32)(key[j] >> shift) & dmask;
            if (full || wbase + j * 32 + lane < P.n) s_src[rank[j] + s_whist[warp][d]] = (u16)(wofs + j * 32 + lane);
        }
        __syncthreads();
        if (full) mbar_wait(&s_mbar[1], 0);
        const u32 tile_n = full ? (u32)TILE : P.n - base;
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            const u32 i = t + k * THREADS;
            if (full || i < tile_n) {
                const u32 src = s_src[i];
                const KT kk = s_k[src];
                const u32 o = s_gbase[(u32)(kk >> shift) & dmask] + i;
                __stcs(kout + o, kk);
                __stcs(vout + o, s_v[src]);
            }
        }
    }
}

}  // namespace rsort
