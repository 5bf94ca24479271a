// fused.cuh -- a1/a2/a4 write pass fused with the first a5 radix pass (single GPU).
//
// The unfused pipeline writes the compacted access records (12 B per access) in ingest pass 1
// and the first radix pass reads them back and writes them again sorted by digit 0.  Here one
// onesweep-style kernel reads each 4096-event tile of the trace once (one TMA bulk copy into
// shared memory), decodes it, writes the tile's synchronization records at their trace-order
// positions (bases from ingest pass 0), and ranks the tile's accesses by digit 0 of the word
// key exactly like rsort::k_onesweep -- warp multisplit, per-tile digit counts, decoupled
// look-back -- so the access records leave already sorted by digit 0 (stable: input order is
// trace order).  Saves 24 B per access of HBM traffic and one launch over the accesses.
//
// Shared memory: the 64 KB event tile is dead once decoded, so the digit-sorted key / value
// staging buffers alias it (3 CTAs per SM).
#pragma once
#include "common.cuh"
#include "ingest.cuh"
#include "sort.cuh"

namespace fused {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
#ifndef IGD_FUSED_ITEMS
#define IGD_FUSED_ITEMS 16  // 8 items x 4-5 CTAs/SM measured slower (10.6 -> 10.9 ms at C5@1e9)
#endif
#ifndef IGD_FUSED_MINB
#define IGD_FUSED_MINB 3
#endif
constexpr int ITEMS = IGD_FUSED_ITEMS;
constexpr int TILE = THREADS * ITEMS;  // events per tile: a whole number of ingest pass-0 tiles
constexpr int TPI = TILE / ingest::TILE;  // ingest pass-0 tiles per fused tile
constexpr int RADIX = 256;
#ifndef IGD_FUSED_MIX
#define IGD_FUSED_MIX 0  // N: one row in N ranked with match.any; 0 = ballots only (C5 38.7 -> 38.2 ms, r02s15; N = 2 slower)
#endif
#ifndef IGD_FUSED_EARLY
#define IGD_FUSED_EARLY 1
#endif
static_assert(TILE % ingest::TILE == 0, "sync-record bases come from ingest pass 0 tiles");
static_assert(THREADS == RADIX, "one look-back digit per thread");

struct Params {
    const igd_event* ev;
    u64 n;               // events
    Geo g;
    KeySpace ks;
    const u32* tile_sync;  // exclusive sync-record base of every ingest pass-0 tile
    u32* sync_key;
    u32* sync_val;
    u64 sync_cap;
    const u32* digit_base;  // [256] exclusive global offsets of digit 0 of the access keys
    u64* status;            // [n_tiles * 256] digit statuses tagged with `epoch` (see rsort::PassParams)
    u32 epoch;
    u32* tile_ctr;          // zeroed: tile tickets (CTA start order, see rsort::k_onesweep)
    void* kout;             // access keys (u32 or u64, template KT), sorted by digit 0
    u64 kbase;              // KT = u64: key = word - kbase (kbase's low 8 bits are 0)
    u32 keymask;            // KT = u32: key = low 32 bits of the word & keymask (tag mode, A36:
                            // entry + 10-bit Tag); all ones otherwise
    u64* vout;              // access payload (event index | tk << 32), same order
    const u32* skip_bits;   // coalesced mode (A32): bit i = event i is not an access record
};

// Decode of an event ingest pass 0 has already validated (the same fields as ingest::decode,
// without the rule checks): access key and tk (+ mask summaries), or the sync record keys.
struct FDec {
    u32 key, tk, ns, s0, s1;
    bool acc;
};
// GEO2: block_dim is a power of two >= 32 (block / warp / lane by shifts and masks)
template <bool GEO2>
__device__ __forceinline__ FDec fdecode(const uint4& e, const Geo& g, const KeySpace& ks) {
    FDec d;
    const u32 tid = ev_tid(e), kind = ev_kind(e);
    const u32 b = GEO2 ? tid >> g.dlog : g.block(tid);
    const u32 off = GEO2 ? (tid & (g.D - 1u)) : tid - b * g.D;
    const u32 w = GEO2 ? tid >> 5 : b * g.Wb + (off >> 5);
    d.key = (e.x >> 2) | (e.y << 30);
    d.tk = e.z;
    d.ns = 1;
    d.s1 = 0;
    d.acc = kind <= IGD_EXCH;
    if (d.acc) {
        const u32 lanebit = 1u << (off & 31u);
        d.tk |= (e.w == IGD_FULL ? (1u << 31) : 0u) | (e.w == lanebit ? (1u << 30) : 0u);
        d.ns = kind >= IGD_CAS ? 1u : 0u;
        d.s0 = ks.lock + w;
    } else if (kind == IGD_FENCE) {
        d.s0 = ks.any + tid;
        if (norm_scope(ev_scope(e)) == IGD_SCOPE_DEVICE) {
            d.s1 = ks.dev + tid;
            d.ns = 2;
        }
    } else if (kind == IGD_SYNCWARP || kind == IGD_CG_TILE_SYNC) {
        d.s0 = ks.wb + w;
    } else if (kind == IGD_SYNCTHREADS || kind == IGD_CG_BLOCK_SYNC) {
        d.s0 = ks.bb + b;
    } else {
        d.s0 = kind == IGD_KERNEL_BOUNDARY ? ks.kb : ks.grid;
    }
    return d;
}

// the event tile (16 B per event), or the phase-2 buffers aliasing it if those are larger:
// keys (KT), values (8 B), per-warp digit counts
template <typename KT = u32>
constexpr size_t smem_bytes() {
    return (size_t)TILE * 16 > (size_t)TILE * (sizeof(KT) + 8) + WARPS * RADIX * 4
               ? (size_t)TILE * 16
               : (size_t)TILE * (sizeof(KT) + 8) + WARPS * RADIX * 4;
}

// COAL: warp-coalesced mode (A32) -- a separate instantiation so the default path carries no
// skip-bit test (ncu r02b: 6% of the kernel's instructions)
// KT: u32 keys (low 32 bits of the word; spans < 2^32 words) or u64 keys (word - kbase, the wide
// path of a4)
template <bool COAL, typename KT = u32, bool GEO2 = false>
__global__ void __launch_bounds__(THREADS, IGD_FUSED_MINB) k_ingest_sort0(Params P) {
    __shared__ u32 s_gbase[RADIX];
    __shared__ u32 s_wsum[WARPS];
    __shared__ u32 s_wsync[WARPS];
    __shared__ u32 s_na;
    __shared__ u32 s_cnt[RADIX];  // tile digit counts (early publication)
    __shared__ __align__(8) u64 s_mbar;
    __shared__ u32 s_tile;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    // phase 1: the event tile (64 KB).  Phase 2 (events dead), u32 keys: digit-sorted keys
    // [0, 16K), values [16K, 48K), per-warp digit counts [48K, 56K).
    uint4* s_ev = reinterpret_cast<uint4*>(s_dyn);
    KT* s_k = reinterpret_cast<KT*>(s_dyn);
    u64* s_v = reinterpret_cast<u64*>(s_dyn + TILE * sizeof(KT));
    u32(*s_whist)[RADIX] = reinterpret_cast<u32(*)[RADIX]>(s_dyn + TILE * (sizeof(KT) + 8));
    KT* kout = reinterpret_cast<KT*>(P.kout);

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) {
        // tile ticket in CTA start order (decoupled look-back never waits on an unstarted tile),
        // then one TMA bulk copy of the tile's events
        const u32 tl = atomicAdd(P.tile_ctr, 1u);
        s_tile = tl;
        const u64 b0 = (u64)tl * TILE;
        if (b0 + TILE <= P.n) {
            mbar_init(&s_mbar, 1);
            mbar_expect_tx(&s_mbar, TILE * sizeof(uint4));
            bulk_g2s(s_ev, P.ev + b0, TILE * sizeof(uint4), &s_mbar);
        }
    }
    s_cnt[t] = 0;
    __syncthreads();
    const u32 tile = s_tile;
    const u64 base = (u64)tile * TILE;
    const bool full = base + TILE <= P.n;
    const u32 tile_e = full ? (u32)TILE : (u32)(P.n - base);
    if (!full)
        for (u32 i = t; i < TILE; i += THREADS)
            s_ev[i] = i < tile_e ? ld_event_stream(P.ev, base + i) : make_uint4(0, 0, 0, 0);
    __syncthreads();
    if (full) mbar_wait(&s_mbar, 0);

    // ---- decode: warp w owns events [w * 32 * ITEMS, (w + 1) * 32 * ITEMS) of the tile, item j
    // of lane l being event w * 32 * ITEMS + j * 32 + l (warp-contiguous, item-major = trace order)
    const Geo g = P.g;
    const KeySpace ks = P.ks;
    const u32 wofs = warp * 32 * ITEMS;
    const u32 lt = lanemask_lt();
    KT key[ITEMS];
    u32 tk[ITEMS];
    u32 amask = 0;    // bit j: item j is an access
    u32 nsbits = 0;   // bits 2j..2j+1: sync records of item j (0..2)
    u32 nsync_w = 0;  // sync records of this warp (warp-uniform)
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const u32 p = wofs + j * 32 + lane;
        const uint4 ev = s_ev[p];
        FDec d = fdecode<GEO2>(ev, g, ks);  // valid: ingest pass 0 checked every event
        const bool in = p < tile_e;
        if (COAL && d.acc && in && ((__ldg(P.skip_bits + ((base + p) >> 5)) >> (p & 31u)) & 1u))
            d.acc = false;  // A32: checked by its coalesced group's first lane
        if (sizeof(KT) == 8) key[j] = (KT)((((u64)ev.y << 32) | ev.x) >> 2) - (KT)P.kbase;
        else key[j] = (KT)(d.key & P.keymask);
        tk[j] = d.tk;
        amask |= ((in && d.acc) ? 1u : 0u) << j;
        if (IGD_FUSED_EARLY && in && d.acc) atomicAdd(&s_cnt[(u32)key[j] & 255u], 1u);
        const u32 ns = in ? d.ns : 0u;
        nsbits |= ns << (2 * j);
        // the event's own slot now holds its sync record keys (read back by this thread only)
        if (ns) *reinterpret_cast<uint2*>(&s_ev[p]) = make_uint2(d.s0, d.s1);
        nsync_w += __reduce_add_sync(IGD_FULL, ns);
    }
    if (lane == 0) s_wsync[warp] = nsync_w;
    __syncthreads();
    // The tile's digit counts are known before any ranking: publish them now, so successors
    // looking back rarely find this tile not ready (their spin was most of this kernel's issue
    // slots when the aggregate was published after ranking, ncu r01 v5)
    if (IGD_FUSED_EARLY) st_relaxed(P.status + (u64)tile * RADIX + t, ds_make(tile == 0 ? ST_INC : ST_AGG, P.epoch, s_cnt[t]));

    // ---- synchronization records, in trace order: base of this tile (ingest pass 0) + earlier
    // warps + earlier (item, lane) of this warp; keys from the event slots
    if (nsync_w) {
        u32 wpre = 0;
#pragma unroll
        for (int w = 0; w < WARPS; w++)
            if ((u32)w < warp) wpre += s_wsync[w];
        u64 pos = (u64)P.tile_sync[TPI * tile] + wpre;
#pragma unroll 1
        for (int j = 0; j < ITEMS; j++) {
            const u32 p = wofs + j * 32 + lane;
            const u32 ns = (nsbits >> (2 * j)) & 3u;
            const u32 b1 = __ballot_sync(IGD_FULL, ns >= 1), b2 = __ballot_sync(IGD_FULL, ns == 2);
            if (!(b1 | b2)) continue;
            const u64 my = pos + __popc(b1 & lt) + __popc(b2 & lt);
            if (ns && my + ns <= P.sync_cap) {
                const uint2 sk = *reinterpret_cast<const uint2*>(&s_ev[p]);
                const u32 ts = (u32)(base + p);
                P.sync_key[my] = sk.x;
                P.sync_val[my] = ts;
                if (ns == 2) {
                    P.sync_key[my + 1] = sk.y;
                    P.sync_val[my + 1] = ts;
                }
            }
            pos += __popc(b1) + __popc(b2);
        }
    }
    __syncthreads();  // the event tile is dead
    for (int i = t; i < WARPS * RADIX; i += THREADS) (&s_whist[0][0])[i] = 0;
    __syncthreads();

    // ---- rank the accesses by digit 0 (warp multisplit, as rsort::k_onesweep)
    u32 rank2[ITEMS / 2];  // ranks (< TILE <= 2^16) packed in pairs: register budget of 3 CTAs/SM
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const bool valid = (amask >> j) & 1u;
        const u32 vmask = __ballot_sync(IGD_FULL, valid);
        const u32 d = (u32)key[j] & 255u;
        const u32 peers = (IGD_FUSED_MIX > 0 && (j % (IGD_FUSED_MIX > 0 ? IGD_FUSED_MIX : 1)) == IGD_FUSED_MIX - 1)
                              ? rsort::peers_of<0>(valid ? d : (0x100u | lane), vmask)
                                                    : rsort::peers_of<1>(valid ? d : (0x100u | lane), vmask);
        const u32 leader = __ffs(peers) - 1;
        // every lane reads its digit's count (peers read one address: a broadcast), then the
        // leader bumps it -- no shuffle of the leader's value (r02s24: C5 sort 75.7 -> 74.6 ms,
        // fused 38.2 -> 37.8 ms against leader load + store + shuffle or a leader atomicAdd)
        u32 old = 0;
        if (valid) old = s_whist[warp][d];
        __syncwarp();
        if (lane == leader && valid) s_whist[warp][d] = old + __popc(peers);
        const u32 r = old + __popc(peers & lt);
        if (j & 1) rank2[j / 2] |= r << 16;
        else rank2[j / 2] = r;
        __syncwarp();
    }
    __syncthreads();

    // ---- per digit: tile count, exclusive scan over digits, every warp's tile position base
    u32 cnt, tile_excl;
    {
        const u32 d = t;
        u32 c[WARPS];
        cnt = 0;
#pragma unroll
        for (int w = 0; w < WARPS; w++) {
            c[w] = s_whist[w][d];
            cnt += c[w];
        }
        if (!IGD_FUSED_EARLY) st_relaxed(P.status + (u64)tile * RADIX + d, ds_make(tile == 0 ? ST_INC : ST_AGG, P.epoch, cnt));
        u32 inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const u32 x = __shfl_up_sync(IGD_FULL, inc, o);
            if (lane >= (u32)o) inc += x;
        }
        if (lane == 31) s_wsum[warp] = inc;
        __syncthreads();
        u32 wpre = 0;
#pragma unroll
        for (int w = 0; w < WARPS; w++)
            if ((u32)w < warp) wpre += s_wsum[w];
        tile_excl = wpre + inc - cnt;
        if (t == RADIX - 1) s_na = wpre + inc;  // accesses in this tile
        u32 run = tile_excl;
#pragma unroll
        for (int w = 0; w < WARPS; w++) {
            s_whist[w][d] = run;
            run += c[w];
        }
    }
    // ---- look-back for digit t (LB statuses per round trip, as rsort::k_onesweep)
    {
        const u32 dg = t;
        u64 excl = 0;
        if (tile > 0) {
            long tt = (long)tile - 1;
            bool done = false;
            while (!done) {
                u64 s[IGD_SORT_LB];
#pragma unroll
                for (int q = 0; q < IGD_SORT_LB; q++)
                    s[q] = tt - q >= 0 ? ld_relaxed(P.status + (u64)(tt - q) * RADIX + dg) : ds_make(ST_INC, P.epoch, 0);
#pragma unroll
                for (int q = 0; q < IGD_SORT_LB; q++) {
                    if (!done) {
                        s[q] = ds_spin(P.status + (u64)(tt - q) * RADIX + dg, s[q], P.epoch);
                        excl += s[q] & DS_VAL_MASK;
                        done = (s[q] >> 62) == 2;
                    }
                }
                tt -= IGD_SORT_LB;
            }
            st_relaxed(P.status + (u64)tile * RADIX + dg, ds_make(ST_INC, P.epoch, excl + cnt));
        }
        s_gbase[dg] = P.digit_base[dg] + (u32)excl - tile_excl;  // position = s_gbase[d] + i
    }
    __syncthreads();
    // ---- records to their tile positions: key, payload (event index | tk << 32), digit
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        if ((amask >> j) & 1u) {
            const u32 d = (u32)key[j] & 255u;
            const u32 r = ((rank2[j / 2] >> (16 * (j & 1))) & 0xFFFFu) + s_whist[warp][d];
            s_k[r] = key[j];
            s_v[r] = (base + wofs + j * 32 + lane) | ((u64)tk[j] << 32);
        }
    }
    __syncthreads();
    // ---- out in digit runs
    const u32 na = s_na;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const u32 i = t + k * THREADS;
        if (i < na) {
            const KT kk = s_k[i];
            const u32 o = s_gbase[(u32)kk & 255u] + i;
            __stcs(kout + o, kk);
            __stcs(P.vout + o, s_v[i]);
        }
    }
}

}  // namespace fused
