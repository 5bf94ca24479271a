// ingest.cuh -- a1 + a2 extraction + a4 key build: streaming passes over the trace.
//
// Per 16-byte event:
//   * validates the field rules of include/igd.h (first bad index -> atomicMin),
//   * compacts accesses into (key = low 32 bits of the word, value = event index | tk << 32),
//     in trace order (stable compaction: per-tile counts, a scan, then positioned writes),
//   * compacts synchronization events into (entity key, timestamp) records (KeySpace), also in
//     trace order, so a stable sort by entity gives per-entity timestamp lists,
//   * builds the 4 x 8-bit digit histograms of both record streams for the radix sorts
//     (warp-uniform digits -- the common case for the high digits -- cost one shared atomic
//     per warp instead of 32 conflicting ones),
//   * reduces min / max accessed word (the 32-bit key is injective iff max - min < 2^32).
// Persistent CTAs stride over 2048-event tiles; histograms are flushed once per CTA.  Each event
// is decoded into 5 registers; the raw 16 bytes are not kept.
#pragma once
#include "common.cuh"

namespace ingest {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
constexpr int ITEMS = 8;
constexpr int TILE = THREADS * ITEMS;
#ifndef IGD_HIST_MATCH
#define IGD_HIST_MATCH 1  // upper-digit histogram aggregation by match.any (C5@1e9 pass 0: 8.1 -> 7.7 ms)
#endif
#ifndef IGD_HIST_UP_LATE
#define IGD_HIST_UP_LATE 0  // 1: access-key digits 1..3 histogrammed after the fused pass (k_hist_keys; measured +0.8 ms per 1e9 events)
#endif

struct Params {
    const igd_event* ev;
    u64 n;
    Geo g;
    KeySpace ks;
    u32* acc_key;
    u64* acc_val;  // trace index | tk << 32 (the check then needs no event gather)
    u32* sync_key;
    u32* sync_val;
    u64 sync_cap;  // records beyond capacity are counted, not written (host re-runs)
    const u32* gidx;  // sharded mode: global timestamp of each input event (else its position)
    u32* tile_acc;   // [n_tiles + 1] pass 0: access records per tile; scanned to bases
    u32* tile_sync;  // [n_tiles + 1] pass 0: sync records per tile; scanned to bases
    u32* hist_acc;   // [4][256]
    u32* hist_sync;  // [4][256]
    u64* stats;      // [0] min word, [1] max word, [2] bad index, [3] n_acc, [4] n_sync, [5] n_lock,
                     // [6] kernel boundaries that change the grid (reading A34)
    u64* gkb;        // pass 0: indices of those boundaries (first gkb_cap of them, any order)
    u32 gkb_cap;
    u32 n_tiles;
    const u32* skip_bits;  // coalesced mode (A32): bit i = event i is checked by its group's first lane
    int hist0;       // pass 0, fused pipeline: the 4 digit histograms of the access keys (digit 0 for
                     // fused.cuh, 1..3 for the later passes) and no sync-key histograms (k_hist_keys
                     // over the written sync records instead)
};

// Decoded event: flags bit 0 = access, bits 1..2 = number of sync records, bit 3 = CAS/EXCH,
// bit 4 = invalid; key = access key; s0, s1 = sync record keys.
struct Dec {
    u32 flags, key, s0, s1, tk;
};

__device__ __forceinline__ Dec decode(const uint4& e, const Geo& g, const KeySpace& ks) {
    Dec d;
    d.flags = 0;
    d.key = 0;
    d.s0 = d.s1 = 0;
    d.tk = e.z;
    const u32 tid = ev_tid(e), kind = ev_kind(e), scope = ev_scope(e);
    const bool addr0 = (e.x | e.y) == 0;
    const bool tid_ok = tid < g.T;
    u32 b = 0, w = 0, lanebit = 0;
    if (tid_ok) {
        b = g.block(tid);
        const u32 off = tid - b * g.D;
        w = b * g.Wb + (off >> 5);
        lanebit = 1u << (off & 31u);
    }
    const bool inmask = (e.w & lanebit) != 0;
    bool ok = (e.z >> 30) == 0 && tid_ok && kind <= IGD_KERNEL_BOUNDARY;
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
                ok = addr0 && inmask && scope != IGD_SCOPE_NONE;
                break;
            case IGD_SYNCWARP:
            case IGD_CG_TILE_SYNC:
            case IGD_SYNCTHREADS:
            case IGD_CG_BLOCK_SYNC:
                ok = addr0 && scope == IGD_SCOPE_NONE;
                break;
            case IGD_KERNEL_BOUNDARY:  // addr 0, or the next kernel's grid (reading A34)
                ok = scope == IGD_SCOPE_NONE && tid == 0 && (addr0 || geo_code_ok(e.y, e.x));
                break;
            default:  // GRID_SYNC, CG_GRID_SYNC
                ok = addr0 && scope == IGD_SCOPE_NONE && tid == 0;
                break;
        }
    }
    if (!ok) {
        d.flags = 16;
        return d;
    }
    if (kind <= IGD_EXCH) {
        d.key = (e.x >> 2) | (e.y << 30);  // low 32 bits of the word addr >> 2
        d.flags = 1;
        // mask summaries for the check's lockstep clause (tk bits 30..31 are zero in the trace):
        // bit 31 = full warp, bit 30 = only the issuing lane
        d.tk |= (e.w == IGD_FULL ? (1u << 31) : 0u) | (e.w == lanebit ? (1u << 30) : 0u);
        if (kind == IGD_CAS || kind == IGD_EXCH) {
            d.flags |= (1u << 1) | 8u;
            d.s0 = ks.lock + w;
        }
    } else if (kind == IGD_FENCE) {
        d.s0 = ks.any + tid;
        if (norm_scope(scope) == IGD_SCOPE_DEVICE) {
            d.s1 = ks.dev + tid;
            d.flags = 2u << 1;
        } else {
            d.flags = 1u << 1;
        }
    } else if (kind == IGD_SYNCWARP || kind == IGD_CG_TILE_SYNC) {
        d.s0 = ks.wb + w;
        d.flags = 1u << 1;
    } else if (kind == IGD_SYNCTHREADS || kind == IGD_CG_BLOCK_SYNC) {
        d.s0 = ks.bb + b;
        d.flags = 1u << 1;
    } else {
        d.s0 = kind == IGD_KERNEL_BOUNDARY ? ks.kb : ks.grid;
        d.flags = 1u << 1;
        if (kind == IGD_KERNEL_BOUNDARY && !addr0) d.flags |= 32u;  // the grid changes (A34)
    }
    return d;
}

// Histogram update of one 8-bit digit for the lanes in `active`: one shared atomic when all
// active lanes agree on the digit, else one per lane.
__device__ __forceinline__ void hist_add(u32* h, u32 digit, bool on, u32 lane) {
    const u32 active = __ballot_sync(IGD_FULL, on);
    if (!active) return;
    const u32 src = __ffs(active) - 1;
    const u32 first = __shfl_sync(IGD_FULL, digit, src);
    if (__all_sync(IGD_FULL, !on || digit == first)) {
        if (lane == src) atomicAdd(&h[first], __popc(active));
    } else if (on) {
        atomicAdd(&h[digit], 1u);
    }
}

// Pass 0 (count): per tile, the number of access records and sync records; digit histograms,
// min / max word, first invalid event.  Pass 1 (write): the same decode, positions from the
// scanned per-tile counts plus warp scans inside the tile.  Two reads of the trace instead of
// one, but every tile is independent: no look-back chain across 2M tiles (which bounded the
// single-pass variant at ~40 G events/s on B200).
template <int PASS>
#ifndef IGD_INGEST_MINB
#define IGD_INGEST_MINB 4
#endif
__global__ void __launch_bounds__(THREADS, IGD_INGEST_MINB) k_ingest(Params P) {
    __shared__ u32 s_hacc[PASS == 0 ? 4 : 1][256];
    __shared__ u32 s_hsync[PASS == 0 ? 4 : 1][256];
    __shared__ u32 s_hup[PASS == 0 ? 3 : 1][256];  // fused pipeline: access-key digits 1..3
    __shared__ u32 s_wtot[ITEMS][WARPS];  // packed (acc | nsync << 16) per (item, warp)
    __shared__ u32 s_woff[ITEMS][WARPS];  // packed exclusive offsets (acc | sync << 16)

    const u32 tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    if (PASS == 0)
        for (int i = tid; i < 4 * 256; i += THREADS) {
            (&s_hacc[0][0])[i] = 0;
            (&s_hsync[0][0])[i] = 0;
            if (i < 3 * 256) (&s_hup[0][0])[i] = 0;
        }
    u64 wmin = ~0ull, wmax = 0, bad = ~0ull;
    u32 cnt_lock = 0;
    u64 cta_sync = 0;  // thread 0 of pass 0: sync records of this CTA's tiles (64-bit total)
    const Geo g = P.g;
    const KeySpace ks = P.ks;

    for (u32 tile = blockIdx.x; tile < P.n_tiles; tile += gridDim.x) {
        const u64 base = (u64)tile * TILE;
        Dec dv[ITEMS];
        {
            uint4 e[ITEMS];
#pragma unroll
            for (int j = 0; j < ITEMS; j++) {
                const u64 i = base + (u64)j * THREADS + tid;
                e[j] = (i < P.n) ? ld_event_stream(P.ev, i) : make_uint4(0, 0, 0, 0);
            }
#pragma unroll
            for (int j = 0; j < ITEMS; j++) {
                const u64 i = base + (u64)j * THREADS + tid;
                if (i < P.n) {
                    dv[j] = decode(e[j], g, ks);
                    if (P.skip_bits && (dv[j].flags & 1u) && ((__ldg(P.skip_bits + (i >> 5)) >> (i & 31u)) & 1u))
                        dv[j].flags &= ~1u;  // A32: not an access record
                    if (PASS == 0 && (dv[j].flags & 1u)) {
                        const u64 word = ev_addr(e[j]) >> 2;
                        wmin = min(wmin, word);
                        wmax = max(wmax, word);
                    }
                } else {
                    dv[j].flags = 0;
                    dv[j].key = dv[j].s0 = dv[j].s1 = dv[j].tk = 0;
                }
            }
        }
        u32 excl[ITEMS];
        u32 wsum = 0;  // PASS 0: packed warp totals summed over items
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u32 f = dv[j].flags;
            const bool acc = (f & 1u) != 0;
            const u32 ns = (f >> 1) & 3u;
            const u32 v = (acc ? 1u : 0u) | (ns << 16);
            if (PASS == 0) {
                if (f & 16u) bad = min(bad, base + (u64)j * THREADS + tid);
                if (f & 32u) {  // rare: a kernel boundary announcing another grid
                    const unsigned long long slot = atomicAdd((unsigned long long*)&P.stats[6], 1ull);
                    if (slot < P.gkb_cap) P.gkb[slot] = base + (u64)j * THREADS + tid;
                }
                // digit 0 of the access keys for the fused first radix pass (fused.cuh); the other
                // digits: k_hist_keys over its output
                // the low digit is nearly always distinct across lanes: plain shared atomics on
                // four sub-histograms (warp & 3), no warp vote
                if (P.hist0) {
                    const bool acc = (f & 1u) != 0;
                    if (acc) atomicAdd(&s_hacc[warp & 3u][dv[j].key & 255u], 1u);
                    // digits 1..3: one set of atomics per warp when the lanes agree on the upper
                    // 24 bits (lanes of one instruction touch neighbouring words), else per lane
                    const u32 am = IGD_HIST_UP_LATE ? 0u : __ballot_sync(IGD_FULL, acc);
                    if (am) {
                        const u32 hi = dv[j].key >> 8;
                        u32 c;
                        if (IGD_HIST_MATCH) {
                            // one set of atomics per distinct upper-24-bit value among the lanes
                            // (match.any runs on the MIO pipe, off the saturated ALU pipe)
                            const u32 peers = __match_any_sync(IGD_FULL, acc ? hi : (0x1000000u | lane)) & am;
                            c = (acc && lane == (u32)(__ffs(peers) - 1)) ? __popc(peers) : 0u;
                        } else {
                            const u32 src = __ffs(am) - 1;
                            const u32 h0 = __shfl_sync(IGD_FULL, hi, src);
                            const bool uni = __all_sync(IGD_FULL, !acc || hi == h0);
                            c = uni ? (lane == src ? __popc(am) : 0u) : (acc ? 1u : 0u);
                        }
                        if (c) {
                            atomicAdd(&s_hup[0][hi & 255u], c);
                            atomicAdd(&s_hup[1][(hi >> 8) & 255u], c);
                            atomicAdd(&s_hup[2][hi >> 16], c);
                        }
                    }
                }
                if (!P.hist0 && __any_sync(IGD_FULL, ns != 0)) {
#pragma unroll
                    for (int p = 0; p < 4; p++) hist_add(s_hsync[p], (dv[j].s0 >> (8 * p)) & 255u, ns != 0, lane);
#pragma unroll
                    for (int p = 0; p < 4; p++) hist_add(s_hsync[p], (dv[j].s1 >> (8 * p)) & 255u, ns == 2, lane);
                }
                cnt_lock += (f >> 3) & 1u;
                wsum += __reduce_add_sync(IGD_FULL, v);
            } else {
                u32 inc = v;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const u32 t = __shfl_up_sync(IGD_FULL, inc, o);
                    if (lane >= (u32)o) inc += t;
                }
                excl[j] = inc - v;
                if (lane == 31) s_wtot[j][warp] = inc;
            }
        }
        if (PASS == 0) {
            // per-tile totals: one packed word per warp, summed by warp 0
            if (lane == 0) s_wtot[0][warp] = wsum;
            __syncthreads();
            if (warp == 0) {
                const u32 x = lane < WARPS ? s_wtot[0][lane] : 0u;
                const u32 ta = __reduce_add_sync(IGD_FULL, x & 0xFFFFu);
                const u32 ts = __reduce_add_sync(IGD_FULL, x >> 16);
                if (lane == 0) {
                    P.tile_acc[tile] = ta;
                    P.tile_sync[tile] = ts;
                    cta_sync += ts;
                }
            }
            __syncthreads();
            continue;
        }
        __syncthreads();
        // scan the ITEMS x WARPS totals in (item, warp) order; warp 0 does it
        if (warp == 0) {
            constexpr int PER = ITEMS * WARPS / 32;  // 2
            u32 vv[PER];
            u32 la = 0, ls = 0;
#pragma unroll
            for (int q = 0; q < PER; q++) {
                vv[q] = (&s_wtot[0][0])[lane * PER + q];
                la += vv[q] & 0xFFFFu;
                ls += vv[q] >> 16;
            }
            u32 ia = la, is = ls;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const u32 ta = __shfl_up_sync(IGD_FULL, ia, o);
                const u32 ts = __shfl_up_sync(IGD_FULL, is, o);
                if (lane >= (u32)o) {
                    ia += ta;
                    is += ts;
                }
            }
            u32 ea = ia - la, es = is - ls;
#pragma unroll
            for (int q = 0; q < PER; q++) {
                (&s_woff[0][0])[lane * PER + q] = ea | (es << 16);
                ea += vv[q] & 0xFFFFu;
                es += vv[q] >> 16;
            }
        }
        __syncthreads();
        const u64 ba = P.tile_acc[tile], bs = P.tile_sync[tile];  // exclusive tile bases (scanned)
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u32 f = dv[j].flags;
            const u32 wo = s_woff[j][warp];
            const u32 ex = excl[j];
            if ((f & 1u) && P.acc_key) {
                const u64 pos = ba + (wo & 0xFFFFu) + (ex & 0xFFFFu);
                P.acc_key[pos] = dv[j].key;
                P.acc_val[pos] = (base + (u64)j * THREADS + tid) | ((u64)dv[j].tk << 32);
            }
            const u32 ns = (f >> 1) & 3u;
            if (ns) {
                const u64 pos = bs + (wo >> 16) + (ex >> 16);
                const u64 i = base + (u64)j * THREADS + tid;
                const u32 ts = P.gidx ? __ldg(P.gidx + i) : (u32)i;
                if (pos + ns <= P.sync_cap) {
                    P.sync_key[pos] = dv[j].s0;
                    P.sync_val[pos] = ts;
                    if (ns == 2) {
                        P.sync_key[pos + 1] = dv[j].s1;
                        P.sync_val[pos + 1] = ts;
                    }
                }
            }
        }
        __syncthreads();  // s_woff / s_wtot reuse by the next tile
    }
    if (PASS != 0) return;
    // flush per-CTA results
    __syncthreads();
    for (int i = tid; i < 4 * 256; i += THREADS) {
        if (P.hist0) {
            const u32 a = i < 256 ? s_hacc[0][i] + s_hacc[1][i] + s_hacc[2][i] + s_hacc[3][i]
                                  : (&s_hup[0][0])[i - 256];
            if (a) atomicAdd(&P.hist_acc[i], a);
        } else {
            const u32 a = (&s_hacc[0][0])[i];
            if (a) atomicAdd(&P.hist_acc[i], a);
        }
        const u32 s = (&s_hsync[0][0])[i];
        if (s) atomicAdd(&P.hist_sync[i], s);
    }
    u64 cl = cnt_lock;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        wmin = min(wmin, __shfl_xor_sync(IGD_FULL, wmin, o));
        wmax = max(wmax, __shfl_xor_sync(IGD_FULL, wmax, o));
        bad = min(bad, __shfl_xor_sync(IGD_FULL, bad, o));
        cl += __shfl_xor_sync(IGD_FULL, cl, o);
    }
    if (lane == 0) {
        if (wmin != ~0ull) atomicMin((unsigned long long*)&P.stats[0], (unsigned long long)wmin);
        if (wmin != ~0ull) atomicMax((unsigned long long*)&P.stats[1], (unsigned long long)wmax);
        if (bad != ~0ull) atomicMin((unsigned long long*)&P.stats[2], (unsigned long long)bad);
        if (cl) atomicAdd((unsigned long long*)&P.stats[5], (unsigned long long)cl);
    }
    if (tid == 0 && cta_sync) atomicAdd((unsigned long long*)&P.stats[4], (unsigned long long)cta_sync);
}

// ---- pass 0 of the fused single-GPU pipeline (the timed path) ----------------------------------
// The same outputs as k_ingest<0> with hist0 = 1 (field rules -> first invalid index, per-tile
// access / sync-record counts, digit histograms of the access keys, word range, lock events,
// grid-changing kernel boundaries), with a branch-free rule check: one 4-bit rule word per kind
// (lane in mask / scope set or NONE / addr 0 / tid 0) instead of the switch, which was the
// kernel's most divergent line (ncu r02h: 8 % of instructions, 11 % of stall samples), and
// compile-time geometry (GEO2: power-of-two block_dim >= 32) and coalesced-mode (COAL) variants.
//   rule bits: 1 = lane(tid) in mask, 2 = scope != NONE (else == NONE), 4 = addr == 0, 8 = tid == 0
constexpr u64 kRules = 0x1ull | (0x1ull << 4) | (0x3ull << 8) | (0x3ull << 12) | (0x3ull << 16) |
                       (0x7ull << 20) | (0x4ull << 24) | (0x4ull << 28) | (0xCull << 32) | (0x4ull << 36) |
                       (0x4ull << 40) | (0xCull << 44) | (0x8ull << 48);
// sync records per kind (2 bits each): CAS / EXCH 1 (lock list), FENCE 1 (+1 when device scope),
// the barriers, grid syncs and kernel boundaries 1
constexpr u32 kSyncRecs = (1u << 6) | (1u << 8) | (1u << 10) | (1u << 12) | (1u << 14) | (1u << 16) |
                          (1u << 18) | (1u << 20) | (1u << 22) | (1u << 24);

// The rule check folded into tables indexed by the event's top byte (kind | scope << 4 | the two
// reserved bits << 6): kAllowed = the kind exists and its scope rule holds; the remaining rules
// (lane in mask, addr 0, tid 0) are a 3-bit "needed" word per kind tested against the event's
// facts; kNs0 / kNs1 = the number of sync records; kLockIdx = CAS / EXCH.
constexpr u64 p0_allowed() {
    u64 m = 0;
    for (int i = 0; i < 64; i++) {
        const int k = i & 15, sc = i >> 4;
        const bool scoped = (kRules >> (4 * k)) & 2u;
        if (k <= IGD_KERNEL_BOUNDARY && (scoped ? sc != 0 : sc == 0)) m |= 1ull << i;
    }
    return m;
}
constexpr u64 p0_ns(int bit) {
    u64 m = 0;
    for (int i = 0; i < 64; i++) {
        const int k = i & 15, sc = i >> 4;
        const u32 ns = k <= IGD_KERNEL_BOUNDARY ? ((kSyncRecs >> (2 * k)) & 3u) + (k == IGD_FENCE && sc >= 2 ? 1u : 0u) : 0u;
        if ((ns >> bit) & 1u) m |= 1ull << i;
    }
    return m;
}
constexpr u64 p0_need() {
    u64 m = 0;
    for (int k = 0; k < 16; k++) m |= ((kRules >> (4 * k)) & 0xDull) << (4 * k);
    return m;
}
constexpr u64 kAllowed = p0_allowed(), kNs0 = p0_ns(0), kNs1 = p0_ns(1), kNeed = p0_need();

// The field rules of include/igd.h for one event, from the tables above.  lane: the lane of the
// event's tid (only meaningful when tid < T, which the rule also requires).  *grid: a kernel
// boundary that carries the next kernel's grid (reading A34).
__device__ __forceinline__ bool rules_ok(const uint4& e, u32 t, u32 lane, const Geo& g, bool* grid) {
    const u32 top = e.z >> 24, kind = top & 0xFu;
    const bool addr0 = (e.x | e.y) == 0;
    const u32 facts = ((e.w >> lane) & 1u) | (addr0 ? 4u : 0u) | (t == 0u ? 8u : 0u);
    const u32 need = (u32)(kNeed >> (4 * kind)) & 0xDu;
    bool ok = top < 64u && ((kAllowed >> top) & 1u) && t < g.T && (need & ~facts) == 0u;
    *grid = false;
    if (kind == IGD_KERNEL_BOUNDARY && ok && !addr0) {  // rare
        ok = geo_code_ok(e.y, e.x);
        *grid = ok;
    }
    return ok;
}

#ifndef IGD_P0_UNIF
#define IGD_P0_UNIF 0  // 1: upper-digit histogram by a warp-uniform test + per-lane atomics (C5: 19.1 -> 22.6 ms, r02aa)
#endif

template <bool GEO2, bool COAL, bool FULL>
__device__ __forceinline__ void count_tile(const Params& P, const Geo& g, u64 base, u32 tid, u32 lane, u32 warp,
                                           u32 (*s_hacc)[256], u32 (*s_hup)[256], u64& wmin, u64& wmax,
                                           u64& bad, u32& cnt_lock, u32& wsum) {
    uint4 e[ITEMS];
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const u64 i = base + (u64)j * THREADS + tid;
        e[j] = (FULL || i < P.n) ? ld_event_stream(P.ev, i) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const u64 i = base + (u64)j * THREADS + tid;
        const bool in = FULL || i < P.n;
        const u32 t = e[j].z & 0xFFFFFFu, top = e[j].z >> 24, kind = top & 0xFu;
        const u32 ln = GEO2 ? (t & 31u) : ((t - g.block(t) * g.D) & 31u);
        bool grid = false;
        const bool ok = in && rules_ok(e[j], t, ln, g, &grid);
        if (grid) {  // rare: another grid (A34)
            const unsigned long long slot = atomicAdd((unsigned long long*)&P.stats[6], 1ull);
            if (slot < P.gkb_cap) P.gkb[slot] = i;
        }
        if (in && !ok) bad = min(bad, i);
        bool acc = ok && kind <= IGD_EXCH;
        if (COAL && acc && ((__ldg(P.skip_bits + (i >> 5)) >> (i & 31u)) & 1u)) acc = false;  // A32
        const u32 ns = ok ? (u32)((kNs0 >> top) & 1u) | ((u32)((kNs1 >> top) & 1u) << 1) : 0u;
        cnt_lock += (ok && (kind == IGD_CAS || kind == IGD_EXCH)) ? 1u : 0u;
        const u32 key = (e[j].x >> 2) | (e[j].y << 30);
        if (acc) {
            const u64 word = ev_addr(e[j]) >> 2;
            wmin = min(wmin, word);
            wmax = max(wmax, word);
            atomicAdd(&s_hacc[warp & 3u][key & 255u], 1u);
        }
        // digits 1..3 (IGD_HIST_UP_LATE: histogrammed over the fused pass's keys instead)
        const u32 am = IGD_HIST_UP_LATE ? 0u : __ballot_sync(IGD_FULL, acc);
        if (am) {
            const u32 hi = key >> 8;
            if (IGD_P0_UNIF) {
                // one set of atomics when every access of the row shares the upper 24 bits (the
                // common case for warp-contiguous words), else one per lane
                const u32 src = __ffs(am) - 1;
                const u32 h0 = __shfl_sync(IGD_FULL, hi, src);
                const bool uni = __all_sync(IGD_FULL, !acc || hi == h0);
                const u32 c = uni ? (lane == src ? __popc(am) : 0u) : (acc ? 1u : 0u);
                if (c) {
                    atomicAdd(&s_hup[0][hi & 255u], c);
                    atomicAdd(&s_hup[1][(hi >> 8) & 255u], c);
                    atomicAdd(&s_hup[2][hi >> 16], c);
                }
            } else {
                const u32 peers = __match_any_sync(IGD_FULL, acc ? hi : (0x1000000u | lane)) & am;
                const u32 c = (acc && lane == (u32)(__ffs(peers) - 1)) ? __popc(peers) : 0u;
                if (c) {
                    atomicAdd(&s_hup[0][hi & 255u], c);
                    atomicAdd(&s_hup[1][(hi >> 8) & 255u], c);
                    atomicAdd(&s_hup[2][hi >> 16], c);
                }
            }
        }
        wsum += __reduce_add_sync(IGD_FULL, (acc ? 1u : 0u) | (ns << 16));
    }
}

template <bool GEO2, bool COAL>
__global__ void __launch_bounds__(THREADS, IGD_INGEST_MINB) k_count_fused(Params P) {
    __shared__ u32 s_hacc[4][256];
    __shared__ u32 s_hup[3][256];
    __shared__ u32 s_wtot[WARPS];
    const u32 tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    for (int i = tid; i < 4 * 256; i += THREADS) {
        (&s_hacc[0][0])[i] = 0;
        if (i < 3 * 256) (&s_hup[0][0])[i] = 0;
    }
    __syncthreads();
    u64 wmin = ~0ull, wmax = 0, bad = ~0ull;
    u32 cnt_lock = 0;
    u64 cta_sync = 0;
    const Geo g = P.g;
    for (u32 tile = blockIdx.x; tile < P.n_tiles; tile += gridDim.x) {
        const u64 base = (u64)tile * TILE;
        u32 wsum = 0;
        if (base + TILE <= P.n)
            count_tile<GEO2, COAL, true>(P, g, base, tid, lane, warp, s_hacc, s_hup, wmin, wmax, bad, cnt_lock, wsum);
        else
            count_tile<GEO2, COAL, false>(P, g, base, tid, lane, warp, s_hacc, s_hup, wmin, wmax, bad, cnt_lock, wsum);
        if (lane == 0) s_wtot[warp] = wsum;
        __syncthreads();
        if (warp == 0) {
            const u32 x = lane < WARPS ? s_wtot[lane] : 0u;
            const u32 ta = __reduce_add_sync(IGD_FULL, x & 0xFFFFu);
            const u32 ts = __reduce_add_sync(IGD_FULL, x >> 16);
            if (lane == 0) {
                P.tile_acc[tile] = ta;
                P.tile_sync[tile] = ts;
                cta_sync += ts;
            }
        }
        __syncthreads();
    }
    for (int i = tid; i < 4 * 256; i += THREADS) {
        const u32 a = i < 256 ? s_hacc[0][i] + s_hacc[1][i] + s_hacc[2][i] + s_hacc[3][i] : (&s_hup[0][0])[i - 256];
        if (a) atomicAdd(&P.hist_acc[i], a);
    }
    u64 cl = cnt_lock;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        wmin = min(wmin, __shfl_xor_sync(IGD_FULL, wmin, o));
        wmax = max(wmax, __shfl_xor_sync(IGD_FULL, wmax, o));
        bad = min(bad, __shfl_xor_sync(IGD_FULL, bad, o));
        cl += __shfl_xor_sync(IGD_FULL, cl, o);
    }
    if (lane == 0) {
        if (wmin != ~0ull) atomicMin((unsigned long long*)&P.stats[0], (unsigned long long)wmin);
        if (wmin != ~0ull) atomicMax((unsigned long long*)&P.stats[1], (unsigned long long)wmax);
        if (bad != ~0ull) atomicMin((unsigned long long*)&P.stats[2], (unsigned long long)bad);
        if (cl) atomicAdd((unsigned long long*)&P.stats[5], (unsigned long long)cl);
    }
    if (tid == 0 && cta_sync) atomicAdd((unsigned long long*)&P.stats[4], (unsigned long long)cta_sync);
}

// Digit histograms (4 x 8-bit) of the compacted access keys: a light, high-occupancy pass over
// 4 bytes per access, with warp-uniform digits aggregated into one shared atomic.
__global__ void __launch_bounds__(256) k_hist_keys(const u32* __restrict__ keys, u32 n, u32* __restrict__ hist,
                                                   int first_digit, u32 kmask = 0xFFFFFFFFu) {
    __shared__ u32 s[4][256];
    const u32 lane = threadIdx.x & 31u;
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    const u32 n4 = n / 4;
    for (u32 q = blockIdx.x * blockDim.x + threadIdx.x; q - lane < n4; q += gridDim.x * blockDim.x) {
        const bool in = q < n4;
        const uint4 k4 = in ? __ldcs(reinterpret_cast<const uint4*>(keys) + q) : make_uint4(0, 0, 0, 0);
        const u32 kk[4] = {k4.x & kmask, k4.y & kmask, k4.z & kmask, k4.w & kmask};
#pragma unroll
        for (int e = 0; e < 4; e++)
#pragma unroll
            for (int p = 0; p < 4; p++)
                if (p >= first_digit) hist_add(s[p], (kk[e] >> (8 * p)) & 255u, in, lane);
    }
    if (blockIdx.x == 0)  // the n % 4 tail
        for (u32 i = n4 * 4 + threadIdx.x; i < n; i += blockDim.x) {
            const u32 k = keys[i] & kmask;
#pragma unroll
            for (int p = 0; p < 4; p++)
                if (p >= first_digit) atomicAdd(&s[p][(k >> (8 * p)) & 255u], 1u);
        }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) {
        const u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

}  // namespace ingest
