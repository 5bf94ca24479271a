// ingest.cuh -- a1 + a2 extraction + a4 key build, fused into one streaming pass over the trace.
//
// One read of every 16-byte event:
//   * validates the field rules of include/igd.h (first bad index -> atomicMin),
//   * compacts accesses into (key = low 32 bits of the word, value = event index), in trace
//     order (stable chained-scan compaction with decoupled look-back),
//   * compacts synchronization events into (entity key, timestamp) records (KeySpace), also in
//     trace order, so a stable sort by entity gives per-entity timestamp lists,
//   * builds the 4 x 8-bit digit histograms of both record streams for the radix sorts,
//   * reduces min / max accessed word (the 32-bit key is injective iff max - min < 2^32).
// Persistent CTAs (one per SM slot) pull 4096-event tiles from an atomic counter, so tiles are
// scheduled in order (forward progress for look-back) and histograms are flushed once per CTA.
#pragma once
#include "common.cuh"

namespace ingest {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
constexpr int ITEMS = 16;
constexpr int TILE = THREADS * ITEMS;

struct Params {
    const igd_event* ev;
    u64 n;
    Geo g;
    KeySpace ks;
    u32* acc_key;
    u32* acc_val;
    u32* sync_key;
    u32* sync_val;
    u64 sync_cap;  // records beyond capacity are counted, not written (host re-runs)
    u64* st_acc;   // [n_tiles]
    u64* st_sync;  // [n_tiles]
    u32* tile_ctr;
    u32* hist_acc;   // [4][256]
    u32* hist_sync;  // [4][256]
    u64* stats;      // [0] min word, [1] max word, [2] bad index, [3] n_acc, [4] n_sync, [5] n_lock
    u32 n_tiles;
};

// Field rules (include/igd.h).  Returns the number of access records (0/1) and sync records
// (0..2) this event produces, or -1 if invalid.
struct Decoded {
    u32 ok, acc, nsync;
    u32 key;          // access key
    u32 skey0, skey1; // sync record keys
};

__device__ __forceinline__ Decoded decode(const uint4& e, const Geo& g, const KeySpace& ks) {
    Decoded d;
    d.ok = 1;
    d.acc = 0;
    d.nsync = 0;
    d.key = 0;
    d.skey0 = d.skey1 = 0;
    const u32 tid = ev_tid(e), kind = ev_kind(e), scope = ev_scope(e);
    const u64 addr = ev_addr(e);
    const bool hib = (e.z >> 30) != 0;
    const bool tid_ok = tid < g.T;
    u32 b = 0, w = 0, lanebit = 0;
    if (tid_ok) {
        b = g.block(tid);
        u32 off = tid - b * g.D;
        w = b * g.Wb + (off >> 5);
        lanebit = 1u << (off & 31u);
    }
    const bool inmask = (e.w & lanebit) != 0;
    bool ok = !hib && tid_ok && kind <= IGD_CG_GRID_SYNC;
    if (ok) {
        switch (kind) {
            case IGD_LD:
            case IGD_ST:
                ok = inmask && scope == IGD_SCOPE_NONE;
                break;
            case IGD_ATOM:
            case IGD_CAS:
            case IGD_EXCH:
                ok = inmask && scope != IGD_SCOPE_NONE;
                break;
            case IGD_FENCE:
                ok = addr == 0 && inmask && scope != IGD_SCOPE_NONE;
                break;
            case IGD_SYNCWARP:
            case IGD_CG_TILE_SYNC:
            case IGD_SYNCTHREADS:
            case IGD_CG_BLOCK_SYNC:
                ok = addr == 0 && scope == IGD_SCOPE_NONE;
                break;
            default:  // GRID_SYNC, CG_GRID_SYNC
                ok = addr == 0 && scope == IGD_SCOPE_NONE && tid == 0;
                break;
        }
    }
    if (!ok) {
        d.ok = 0;
        return d;
    }
    if (kind <= IGD_EXCH) {
        d.acc = 1;
        d.key = (u32)(addr >> 2);
        if (kind == IGD_CAS || kind == IGD_EXCH) {
            d.nsync = 1;
            d.skey0 = ks.lock + w;
        }
    } else if (kind == IGD_FENCE) {
        d.skey0 = ks.any + tid;
        d.nsync = 1;
        if (norm_scope(scope) == IGD_SCOPE_DEVICE) {
            d.skey1 = ks.dev + tid;
            d.nsync = 2;
        }
    } else if (kind == IGD_SYNCWARP || kind == IGD_CG_TILE_SYNC) {
        d.skey0 = ks.wb + w;
        d.nsync = 1;
    } else if (kind == IGD_SYNCTHREADS || kind == IGD_CG_BLOCK_SYNC) {
        d.skey0 = ks.bb + b;
        d.nsync = 1;
    } else {
        d.skey0 = ks.grid;
        d.nsync = 1;
    }
    return d;
}

__global__ void __launch_bounds__(THREADS) k_ingest(Params P) {
    __shared__ u32 s_hacc[4][256];
    __shared__ u32 s_hsync[4][256];
    __shared__ u32 s_wtot[ITEMS][WARPS];  // packed (acc | nsync << 16) per (item, warp)
    __shared__ u32 s_woff_acc[ITEMS][WARPS];
    __shared__ u32 s_woff_sync[ITEMS][WARPS];
    __shared__ u64 s_base_acc, s_base_sync;
    __shared__ u32 s_tile;

    const u32 tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    for (int i = tid; i < 4 * 256; i += THREADS) {
        (&s_hacc[0][0])[i] = 0;
        (&s_hsync[0][0])[i] = 0;
    }
    u64 wmin = ~0ull, wmax = 0, bad = ~0ull;
    u64 cnt_acc = 0, cnt_sync = 0, cnt_lock = 0;
    const Geo g = P.g;
    const KeySpace ks = P.ks;

    while (true) {
        __syncthreads();
        if (tid == 0) s_tile = atomicAdd(P.tile_ctr, 1u);
        __syncthreads();
        const u32 tile = s_tile;
        if (tile >= P.n_tiles) break;
        const u64 base = (u64)tile * TILE;

        uint4 e[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            u64 i = base + (u64)j * THREADS + tid;
            e[j] = (i < P.n) ? ld_event_stream(P.ev, i) : make_uint4(0, 0, 0, 0);
        }
        // counts per item, warp-scanned
        u32 excl[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            u64 i = base + (u64)j * THREADS + tid;
            u32 v = 0;
            if (i < P.n) {
                Decoded d = decode(e[j], g, ks);
                if (!d.ok) {
                    bad = min(bad, i);
                } else {
                    v = d.acc | (d.nsync << 16);
                    if (d.acc) {
                        u64 word = ev_addr(e[j]) >> 2;
                        wmin = min(wmin, word);
                        wmax = max(wmax, word);
                        atomicAdd(&s_hacc[0][d.key & 255u], 1u);
                        atomicAdd(&s_hacc[1][(d.key >> 8) & 255u], 1u);
                        atomicAdd(&s_hacc[2][(d.key >> 16) & 255u], 1u);
                        atomicAdd(&s_hacc[3][d.key >> 24], 1u);
                    }
                    if (d.nsync) {
                        atomicAdd(&s_hsync[0][d.skey0 & 255u], 1u);
                        atomicAdd(&s_hsync[1][(d.skey0 >> 8) & 255u], 1u);
                        atomicAdd(&s_hsync[2][(d.skey0 >> 16) & 255u], 1u);
                        atomicAdd(&s_hsync[3][d.skey0 >> 24], 1u);
                    }
                    if (d.nsync == 2) {
                        atomicAdd(&s_hsync[0][d.skey1 & 255u], 1u);
                        atomicAdd(&s_hsync[1][(d.skey1 >> 8) & 255u], 1u);
                        atomicAdd(&s_hsync[2][(d.skey1 >> 16) & 255u], 1u);
                        atomicAdd(&s_hsync[3][d.skey1 >> 24], 1u);
                    }
                    cnt_lock += (d.acc && d.nsync) ? 1 : 0;
                }
            }
            u32 inc = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                u32 t = __shfl_up_sync(IGD_FULL, inc, o);
                if (lane >= (u32)o) inc += t;
            }
            excl[j] = inc - v;
            if (lane == 31) s_wtot[j][warp] = inc;
        }
        __syncthreads();
        // scan the ITEMS x WARPS totals in (item, warp) order; warp 0 does it
        if (warp == 0) {
            constexpr int PER = ITEMS * WARPS / 32;  // 4
            u32 la = 0, ls = 0;
            u32 va[PER], vs[PER];
#pragma unroll
            for (int q = 0; q < PER; q++) {
                int idx = lane * PER + q;
                u32 t = (&s_wtot[0][0])[idx];
                va[q] = t & 0xFFFFu;
                vs[q] = t >> 16;
                la += va[q];
                ls += vs[q];
            }
            u32 ia = la, is = ls;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                u32 ta = __shfl_up_sync(IGD_FULL, ia, o);
                u32 ts = __shfl_up_sync(IGD_FULL, is, o);
                if (lane >= (u32)o) {
                    ia += ta;
                    is += ts;
                }
            }
            u32 ea = ia - la, es = is - ls;
#pragma unroll
            for (int q = 0; q < PER; q++) {
                int idx = lane * PER + q;
                (&s_woff_acc[0][0])[idx] = ea;
                (&s_woff_sync[0][0])[idx] = es;
                ea += va[q];
                es += vs[q];
            }
            const u32 tot_a = __shfl_sync(IGD_FULL, ia, 31);
            const u32 tot_s = __shfl_sync(IGD_FULL, is, 31);
            // publish aggregates, look back
            if (lane == 0) {
                if (tile == 0) {
                    st_relaxed(&P.st_acc[0], ST_INC | tot_a);
                    st_relaxed(&P.st_sync[0], ST_INC | tot_s);
                } else {
                    st_relaxed(&P.st_acc[tile], ST_AGG | tot_a);
                    st_relaxed(&P.st_sync[tile], ST_AGG | tot_s);
                }
            }
            u64 ba = 0, bs = 0;
            if (tile > 0) {
                ba = lookback_sum_warp(P.st_acc, tile);
                bs = lookback_sum_warp(P.st_sync, tile);
                if (lane == 0) {
                    st_relaxed(&P.st_acc[tile], ST_INC | (ba + tot_a));
                    st_relaxed(&P.st_sync[tile], ST_INC | (bs + tot_s));
                }
            }
            if (lane == 0) {
                s_base_acc = ba;
                s_base_sync = bs;
            }
        }
        __syncthreads();
        const u64 ba = s_base_acc, bs = s_base_sync;
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            u64 i = base + (u64)j * THREADS + tid;
            if (i >= P.n) continue;
            Decoded d = decode(e[j], g, ks);
            if (!d.ok) continue;
            u32 ex = excl[j];
            if (d.acc) {
                u64 pos = ba + s_woff_acc[j][warp] + (ex & 0xFFFFu);
                P.acc_key[pos] = d.key;
                P.acc_val[pos] = (u32)i;
            }
            if (d.nsync) {
                u64 pos = bs + s_woff_sync[j][warp] + (ex >> 16);
                if (pos + d.nsync <= P.sync_cap) {
                    P.sync_key[pos] = d.skey0;
                    P.sync_val[pos] = (u32)i;
                }
                if (d.nsync == 2 && pos + 2 <= P.sync_cap) {
                    P.sync_key[pos + 1] = d.skey1;
                    P.sync_val[pos + 1] = (u32)i;
                }
                cnt_sync += d.nsync;
            }
            cnt_acc += d.acc;
        }
    }
    // flush per-CTA results
    for (int i = tid; i < 4 * 256; i += THREADS) {
        u32 a = (&s_hacc[0][0])[i];
        if (a) atomicAdd(&P.hist_acc[i], a);
        u32 s = (&s_hsync[0][0])[i];
        if (s) atomicAdd(&P.hist_sync[i], s);
    }
    // reduce min/max/bad/counts
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        wmin = min(wmin, __shfl_xor_sync(IGD_FULL, wmin, o));
        wmax = max(wmax, __shfl_xor_sync(IGD_FULL, wmax, o));
        bad = min(bad, __shfl_xor_sync(IGD_FULL, bad, o));
        cnt_acc += __shfl_xor_sync(IGD_FULL, cnt_acc, o);
        cnt_sync += __shfl_xor_sync(IGD_FULL, cnt_sync, o);
        cnt_lock += __shfl_xor_sync(IGD_FULL, cnt_lock, o);
    }
    if (lane == 0) {
        if (wmin != ~0ull) atomicMin((unsigned long long*)&P.stats[0], (unsigned long long)wmin);
        if (cnt_acc) atomicMax((unsigned long long*)&P.stats[1], (unsigned long long)wmax);
        if (bad != ~0ull) atomicMin((unsigned long long*)&P.stats[2], (unsigned long long)bad);
        if (cnt_acc) atomicAdd((unsigned long long*)&P.stats[3], (unsigned long long)cnt_acc);
        if (cnt_sync) atomicAdd((unsigned long long*)&P.stats[4], (unsigned long long)cnt_sync);
        if (cnt_lock) atomicAdd((unsigned long long*)&P.stats[5], (unsigned long long)cnt_lock);
    }
}

}  // namespace ingest
