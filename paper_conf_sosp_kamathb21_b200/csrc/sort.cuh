// sort.cuh -- a5: stable LSD radix sort of (u32 key, u32 value) pairs, one kernel per 8-bit
// digit ("onesweep": upfront digit histograms + per-tile decoupled look-back per digit).
//
// Stability: within a tile, each warp owns a contiguous run of 32*ITEMS inputs processed item
// by item in input order; the rank of an input among equal digits is (earlier tiles via
// look-back) + (earlier warps of the tile) + (earlier items / lanes of the warp), i.e. its
// input order.  Sorting accesses that arrive in trace order therefore yields (word, time)
// order, the order the per-word shadow replay needs (SURVEY 8(c) C.3 "equivalent formulation").
#pragma once
#include "common.cuh"

namespace rsort {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
constexpr int ITEMS = 16;
constexpr int TILE = THREADS * ITEMS;  // 4096
constexpr int RADIX = 256;

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

struct PassParams {
    const u32* kin;
    const u32* vin;
    u32* kout;
    u32* vout;
    u32 n;
    u32 shift;
    const u32* digit_base;  // [256] exclusive global offsets of this pass's digits
    u64* status;            // [n_tiles * 256], zeroed
    u32* tile_ctr;          // zeroed
};

__global__ void __launch_bounds__(THREADS) k_onesweep(PassParams P) {
    __shared__ u32 s_whist[WARPS][RADIX];
    __shared__ u32 s_tile_excl[RADIX];
    __shared__ u32 s_gbase[RADIX];
    __shared__ u32 s_keys[TILE];
    __shared__ u32 s_vals[TILE];
    __shared__ u32 s_tile;
    __shared__ u32 s_wsum[WARPS];

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) s_tile = atomicAdd(P.tile_ctr, 1u);
    for (int i = t; i < WARPS * RADIX; i += THREADS) (&s_whist[0][0])[i] = 0;
    __syncthreads();
    const u32 tile = s_tile;
    const u64 base = (u64)tile * TILE;
    const u64 wbase = base + (u64)warp * 32 * ITEMS;

    u32 key[ITEMS], val[ITEMS], rank[ITEMS];
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        u64 i = wbase + (u64)j * 32 + lane;
        if (i < P.n) {
            key[j] = __ldcs(P.kin + i);
            val[j] = __ldcs(P.vin + i);
        } else {
            key[j] = 0;
            val[j] = 0;
        }
    }
    const u32 lt = lanemask_lt();
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        u64 i = wbase + (u64)j * 32 + lane;
        bool valid = i < P.n;
        u32 vmask = __ballot_sync(IGD_FULL, valid);
        u32 r = 0;
        if (valid) {
            u32 d = (key[j] >> P.shift) & 255u;
            u32 peers = __match_any_sync(vmask, d);
            u32 leader = __ffs(peers) - 1;
            u32 old = 0;
            if (lane == leader) {
                old = s_whist[warp][d];
                s_whist[warp][d] = old + __popc(peers);
            }
            old = __shfl_sync(peers, old, leader);
            r = old + __popc(peers & lt);
        }
        rank[j] = r;
        __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive over warps, tile count
    u32 cnt;
    {
        const u32 d = t;  // THREADS == RADIX
        u32 sum = 0;
#pragma unroll
        for (int w = 0; w < WARPS; w++) {
            u32 c = s_whist[w][d];
            s_whist[w][d] = sum;
            sum += c;
        }
        cnt = sum;
        u64* st = P.status + (u64)tile * RADIX + d;
        if (tile == 0) {
            st_relaxed(st, ST_INC | cnt);
        } else {
            st_relaxed(st, ST_AGG | cnt);
        }
    }
    // block exclusive scan of cnt over digits
    {
        u32 inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            u32 x = __shfl_up_sync(IGD_FULL, inc, o);
            if (lane >= (u32)o) inc += x;
        }
        if (lane == 31) s_wsum[warp] = inc;
        __syncthreads();
        u32 wpre = 0;
#pragma unroll
        for (int w = 0; w < WARPS; w++)
            if ((u32)w < warp) wpre += s_wsum[w];
        s_tile_excl[t] = wpre + inc - cnt;
    }
    // decoupled look-back for this digit
    {
        const u32 d = t;
        u64 excl = 0;
        if (tile > 0) {
            long tt = (long)tile - 1;
            while (tt >= 0) {
                u64 s;
                do {
                    s = ld_relaxed(P.status + (u64)tt * RADIX + d);
                } while ((s >> 62) == 0);
                excl += s & ST_VAL_MASK;
                if ((s >> 62) == 2) break;
                tt--;
            }
            st_relaxed(P.status + (u64)tile * RADIX + d, ST_INC | (excl + cnt));
        }
        s_gbase[d] = P.digit_base[d] + (u32)excl;
    }
    __syncthreads();
    // local reorder through shared memory
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        u64 i = wbase + (u64)j * 32 + lane;
        if (i < P.n) {
            u32 d = (key[j] >> P.shift) & 255u;
            u32 pos = s_tile_excl[d] + s_whist[warp][d] + rank[j];
            s_keys[pos] = key[j];
            s_vals[pos] = val[j];
        }
    }
    __syncthreads();
    const u32 tile_n = (u32)min((u64)TILE, (u64)P.n - base);
#pragma unroll 4
    for (u32 i = t; i < tile_n; i += THREADS) {
        u32 k = s_keys[i];
        u32 d = (k >> P.shift) & 255u;
        u32 out = s_gbase[d] + (i - s_tile_excl[d]);
        __stcs(P.kout + out, k);
        __stcs(P.vout + out, s_vals[i]);
    }
}

}  // namespace rsort
