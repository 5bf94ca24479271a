// shard.cuh -- multi-GPU partitioning of one rank's trace chunk.
//
// Rank r holds the contiguous global range [first, first + n).  Words are hash-sharded:
// owner(word) = fmix32(low 32 bits of the word) % P.  For the exchange each rank produces
//   * its access records grouped by owner, each group in trace order:
//       uint4 {key = low 32 bits of the word, global index, tk (+ mask summaries), active mask}
//   * its synchronization stream (fences, barriers, grid syncs, CAS/EXCH), in trace order:
//       global index + the raw 16-byte event,
// with a stable count / scan / write structure like the ingest's.  After an all-to-all of the
// records and an all-gather of the sync streams (torch.distributed over NCCL, issued by the
// host binding) every rank rebuilds identical synchronization tables and checks the words it
// owns: the union over ranks is exactly the single-GPU report set (address-shard invariance,
// SURVEY 8(c) C.7 5(b)).
#pragma once
#include "common.cuh"
#include "ingest.cuh"

namespace shard {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
#ifndef IGD_SHARD_ITEMS
#define IGD_SHARD_ITEMS 4  // 4 items, 4 CTAs/SM: sharded C5@1e9 at N=1 108 -> 95 ms per step
#endif
#ifndef IGD_SHARD_MINB
#define IGD_SHARD_MINB 4
#endif
constexpr int ITEMS = IGD_SHARD_ITEMS;
constexpr int TILE = THREADS * ITEMS;
constexpr int MAXP = 16;

__device__ __forceinline__ u32 fmix32(u32 h) {
    h ^= h >> 16;
    h *= 0x85ebca6bu;
    h ^= h >> 13;
    h *= 0xc2b2ae35u;
    h ^= h >> 16;
    return h;
}

struct Params {
    const igd_event* ev;
    u64 n;          // events in this chunk
    u64 first;      // global index of ev[0]
    Geo g;
    KeySpace ks;
    u32 P;          // ranks (owners), <= MAXP
    u32 n_tiles;
    u32* cnt;       // [(P + 1) * (n_tiles + 1)]: row o < P = records for owner o per tile, row P =
                    // sync-stream events per tile; scanned in place per row between the passes
    const u64* obase;  // [P + 1] start of each owner's region in `send`; [P] unused
    uint4* send;
    u32* sync_idx;
    uint4* sync_ev;
    u64* stats;     // [0] min word, [1] max word, [2] first bad global index, [3] grid-changing kernel
                    // boundaries (reading A34; single-context only)
};

template <int PASS>
__global__ void __launch_bounds__(THREADS, IGD_SHARD_MINB) k_shard(Params P) {
    __shared__ u32 s_wc[ITEMS][WARPS][MAXP + 1];  // per (item, warp, destination) counts, then offsets
    const u32 tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const u32 lt = lanemask_lt();
    const Geo g = P.g;
    const u32 NP = P.P;
    u64 wmin = ~0ull, wmax = 0, bad = ~0ull;

    for (u32 tile = blockIdx.x; tile < P.n_tiles; tile += gridDim.x) {
        const u64 base = (u64)tile * TILE;
        uint4 e[ITEMS];
        u32 dst[ITEMS];  // owner for an access record; the sync stream uses bit 31 (both for CAS/EXCH)
        u32 tk[ITEMS], rk[ITEMS], srk[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u64 i = base + (u64)j * THREADS + tid;
            e[j] = (i < P.n) ? ld_event_stream(P.ev, i) : make_uint4(0, 0, 0, 0);
            dst[j] = 0;
            tk[j] = 0;
            if (i < P.n) {
                const u32 t = e[j].z & 0xFFFFFFu, kind = (e[j].z >> 24) & 0xFu;
                const u32 ln = (t - g.block(t) * g.D) & 31u, lanebit = 1u << ln;
                bool grid;
                if (!ingest::rules_ok(e[j], t, ln, g, &grid)) {
                    bad = min(bad, P.first + i);
                } else {
                    // a grid change (A34) is single-context only: counted, the host refuses it
                    if (PASS == 0 && grid) atomicAdd((unsigned long long*)&P.stats[3], 1ull);
                    if (kind <= IGD_EXCH) {
                        const u32 key = (e[j].x >> 2) | (e[j].y << 30);
                        dst[j] = 0x100u | (NP == 1 ? 0u : fmix32(key) % NP);
                        // mask summaries for the check's lockstep clause (as ingest::decode)
                        tk[j] = e[j].z | (e[j].w == IGD_FULL ? (1u << 31) : 0u) | (e[j].w == lanebit ? (1u << 30) : 0u);
                        const u64 word = ev_addr(e[j]) >> 2;
                        wmin = min(wmin, word);
                        wmax = max(wmax, word);
                    }
                    if (kind >= IGD_FENCE || kind == IGD_CAS || kind == IGD_EXCH) dst[j] |= 0x80000000u;
                }
            }
        }
        // per item: warp counts and lane ranks per destination (owners, then the sync stream)
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            for (u32 o = 0; o <= NP; o++) {
                const bool mine = (o < NP) ? ((dst[j] & 0x1FFu) == (0x100u | o)) : (dst[j] >> 31) != 0;
                const u32 bal = __ballot_sync(IGD_FULL, mine);
                if (mine) {
                    if (o < NP) rk[j] = __popc(bal & lt);
                    else srk[j] = __popc(bal & lt);
                }
                if (lane == 0) s_wc[j][warp][o] = __popc(bal);
            }
        }
        __syncthreads();
        if constexpr (PASS == 0) {
            for (u32 o = tid; o <= NP; o += THREADS) {
                u32 s = 0;
                for (int j = 0; j < ITEMS; j++)
                    for (int w = 0; w < WARPS; w++) s += s_wc[j][w][o];
                P.cnt[(u64)o * (P.n_tiles + 1) + tile] = s;
            }
            __syncthreads();
            continue;
        } else {
            // exclusive offsets in (item, warp) order per destination
            for (u32 o = tid; o <= NP; o += THREADS) {
                u32 s = 0;
                for (int j = 0; j < ITEMS; j++)
                    for (int w = 0; w < WARPS; w++) {
                        const u32 c = s_wc[j][w][o];
                        s_wc[j][w][o] = s;
                        s += c;
                    }
            }
            __syncthreads();
#pragma unroll
            for (int j = 0; j < ITEMS; j++) {
                const u64 i = base + (u64)j * THREADS + tid;
                if (i >= P.n) continue;
                const u32 gi = (u32)(P.first + i);
                if (dst[j] & 0x100u) {
                    const u32 o = dst[j] & 0xFFu;
                    const u64 pos = P.obase[o] + P.cnt[(u64)o * (P.n_tiles + 1) + tile] + s_wc[j][warp][o] + rk[j];
                    const u32 key = (e[j].x >> 2) | (e[j].y << 30);
                    P.send[pos] = make_uint4(key, gi, tk[j], e[j].w);
                }
                if (dst[j] >> 31) {
                    const u64 pos = (u64)P.cnt[(u64)NP * (P.n_tiles + 1) + tile] + s_wc[j][warp][NP] + srk[j];
                    P.sync_idx[pos] = gi;
                    P.sync_ev[pos] = e[j];
                }
            }
            __syncthreads();
        }
    }
    if constexpr (PASS == 0) {  // the chunk's word range and first invalid event
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            wmin = min(wmin, __shfl_xor_sync(IGD_FULL, wmin, o));
            wmax = max(wmax, __shfl_xor_sync(IGD_FULL, wmax, o));
            bad = min(bad, __shfl_xor_sync(IGD_FULL, bad, o));
        }
        if (lane == 0) {
            if (wmin != ~0ull) atomicMin((unsigned long long*)&P.stats[0], (unsigned long long)wmin);
            if (wmin != ~0ull) atomicMax((unsigned long long*)&P.stats[1], (unsigned long long)wmax);
            if (bad != ~0ull) atomicMin((unsigned long long*)&P.stats[2], (unsigned long long)bad);
        }
    }
}

// Received records (uint4 {key, idx, tk, mask}) -> the sort keys and their 4 x 8-bit digit
// histograms.  The records themselves are the sort payload (the check reads idx, tk, mask from
// .y .z .w), so no split copy of them is written.
__global__ void __launch_bounds__(256) k_record_keys(const uint4* __restrict__ rec, u32 n, u32* __restrict__ keys,
                                                     u32* __restrict__ hist) {
    __shared__ u32 s[4][256];
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const u32 k = __ldcs(rec + i).x;
        keys[i] = k;
        atomicAdd(&s[0][k & 255u], 1u);
        atomicAdd(&s[1][(k >> 8) & 255u], 1u);
        atomicAdd(&s[2][(k >> 16) & 255u], 1u);
        atomicAdd(&s[3][k >> 24], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) {
        const u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

// Received records -> the sort keys, the single-GPU payload (index | tk << 32) and the keys' 4 x
// 8-bit digit histograms (warp-uniform digits aggregated into one shared atomic).
__global__ void __launch_bounds__(256) k_record_split(const uint4* __restrict__ rec, u32 n, u32* __restrict__ keys,
                                                      u64* __restrict__ vals, u32* __restrict__ hist) {
    __shared__ u32 s[4][256];
    const u32 lane = threadIdx.x & 31u;
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    for (u32 i0 = blockIdx.x * blockDim.x; i0 < n; i0 += gridDim.x * blockDim.x) {
        const u32 i = i0 + threadIdx.x;
        const bool in = i < n;
        const uint4 r = in ? __ldcs(rec + i) : make_uint4(0, 0, 0, 0);
        if (in) {
            keys[i] = r.x;
            vals[i] = (u64)r.y | ((u64)r.z << 32);
        }
#pragma unroll
        for (int p = 0; p < 4; p++) ingest::hist_add(s[p], (r.x >> (8 * p)) & 255u, in, lane);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) {
        const u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

}  // namespace shard
