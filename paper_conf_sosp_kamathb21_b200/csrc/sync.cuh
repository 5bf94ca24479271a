// sync.cuh -- a2 epoch tables and a3 lock inference.
//
// a2: after the stable sort of synchronization records by entity key, offsets[e] is the first
//     record of entity e (CSR).  The per-entity timestamp lists replace the paper's bounded
//     per-thread / per-warp / per-block counters (Fig. 4, Fig. 5) by exact
//     "was there a sync of this entity in (a, b)?" queries (reading A16).
// a3: per-warp lock-table state machine of §6.3: atomicCAS inserts an 18-bit
//     address hash (Valid, not Active), a fence of matching-or-wider scope activates entries,
//     atomicExch invalidates the entry with the same hash and scope, a CAS executed by more
//     than one lane switches the warp to per-thread tables for good, a grid sync
//     is a device fence by every thread (reading A15), a kernel boundary resets every table and
//     the isThread bit (reading A31).  One CUDA warp replays one traced warp, lane l
//     owning thread l's per-thread table; each lane emits change points (ts, bloom) of its
//     thread's effective held-lock Bloom summary (the warp table's while isThread is
//     unset, its own table after) so the check asks "locks of thread c just before event i" with
//     one binary search on one list.
#pragma once
#include "common.cuh"

namespace syncx {

// offsets[e] = lower_bound(keys, e) for e in [0, E]
__global__ void k_csr_offsets(const u32* __restrict__ keys, u32 n, u32 E, u32* __restrict__ off) {
    for (u64 e = (u64)blockIdx.x * blockDim.x + threadIdx.x; e <= E; e += (u64)gridDim.x * blockDim.x) {
        u32 lo = 0, hi = n;
        while (lo < hi) {
            u32 mid = (lo + hi) >> 1;
            if (__ldg(keys + mid) < (u32)e) lo = mid + 1;
            else hi = mid;
        }
        off[e] = lo;
    }
}

// ---------------------------------------------------------------------------------------------
// Lock tables.  An entry is packed in a u32: bit 31 valid, bit 30 active, bits 28..29 scope,
// bits 0..17 the 18-bit hash.
__device__ __forceinline__ u32 le_valid(u32 e) { return e >> 31; }
__device__ __forceinline__ u32 le_active(u32 e) { return (e >> 30) & 1u; }
__device__ __forceinline__ u32 le_scope(u32 e) { return (e >> 28) & 3u; }
__device__ __forceinline__ u32 le_hash(u32 e) { return e & 0x3FFFFu; }

struct Table {
    u32 e[3];
    __device__ __forceinline__ void clear() { e[0] = e[1] = e[2] = 0; }
    // "sets the Active bit ... for all entries with matching or narrower scope"
    __device__ __forceinline__ void activate(u32 s) {
#pragma unroll
        for (int k = 0; k < 3; k++)
            if (le_valid(e[k]) && le_scope(e[k]) <= s) e[k] |= (1u << 30);
    }
    // insert on atomicCAS (readings A9): dedup (hash, scope), lowest free slot,
    // dropped when full
    __device__ __forceinline__ void insert(u32 h, u32 s) {
#pragma unroll
        for (int k = 0; k < 3; k++)
            if (le_valid(e[k]) && le_hash(e[k]) == h && le_scope(e[k]) == s) return;
#pragma unroll
        for (int k = 0; k < 3; k++)
            if (!le_valid(e[k])) {
                e[k] = (1u << 31) | (s << 28) | h;
                return;
            }
    }
    // remove on atomicExch: "Valid bit of any entry matching the address hash and scope is unset"
    __device__ __forceinline__ void remove(u32 h, u32 s) {
#pragma unroll
        for (int k = 0; k < 3; k++)
            if (le_valid(e[k]) && le_hash(e[k]) == h && le_scope(e[k]) == s) e[k] = 0;
    }
    // an entry a fence could still activate (valid, not active)
    __device__ __forceinline__ bool pending() const {
        bool p = false;
#pragma unroll
        for (int k = 0; k < 3; k++) p |= le_valid(e[k]) && !le_active(e[k]);
        return p;
    }
    __device__ __forceinline__ u32 held() const {
        u32 b = 0;
#pragma unroll
        for (int k = 0; k < 3; k++)
            if (le_valid(e[k]) && le_active(e[k])) b |= lock_bloom(le_hash(e[k]));
        return b;
    }
};

struct LockParams {
    const igd_event* ev;
    Geo g;
    KeySpace ks;
    const u32* off;       // CSR offsets of sync records
    const u32* sts;       // sorted sync timestamps
    u32* tcnt;            // [T+1] thread change-point counts (pass 0) -> offsets after the scan
    const u32* toff;      // [T+1] (pass 1)
    u64* tpts;            // thread change points (ts << 16 | bloom)
    const u32* gidx;      // sharded mode: global timestamps of the events in `ev` (sorted), else NULL
    u32 gn;
    const uint8_t* fdev;  // per sorted sync record of an AnyF list: 1 = a device-scope fence
};

// Scope of every fence in the AnyF lists (1 = device or system): a merge of thread t's AnyF and
// DevF lists (a device fence is on both, A12).  Lets the lock replay read a fence's scope from a
// byte next to its timestamp instead of the trace or a second list cursor.
__global__ void k_fence_scopes(const u32* __restrict__ off, const u32* __restrict__ sts, KeySpace ks, u32 T,
                               uint8_t* __restrict__ fdev) {
    const u32 t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= T) return;
    u32 f = off[ks.any + t];
    const u32 f_hi = off[ks.any + t + 1];
    u32 d = off[ks.dev + t];
    const u32 d_hi = off[ks.dev + t + 1];
    u32 dts = d < d_hi ? sts[d] : IGD_NONE32;
    for (; f < f_hi; f++) {
        const u32 ts = sts[f];
        const bool dev = dts == ts;
        fdev[f] = dev ? 1 : 0;
        if (dev) dts = ++d < d_hi ? sts[d] : IGD_NONE32;
    }
}

// The event with timestamp ts: ev[ts] on one GPU; in sharded mode `ev` is the all-gathered
// synchronization stream and its position is found by binary search on the timestamps.
__device__ __forceinline__ uint4 event_at(const LockParams& P, u32 ts) {
    if (ts == IGD_NONE32) return make_uint4(0, 0, 0, 0);
    if (!P.gidx) return ld_event(P.ev, ts);
    u32 lo = 0, hi = P.gn;
    while (lo < hi) {
        const u32 mid = (lo + hi) >> 1;
        if (__ldg(P.gidx + mid) < ts) lo = mid + 1;
        else hi = mid;
    }
    return ld_event(P.ev, lo);
}

// One warp per traced warp.  WRITE = false: count change points; true: write them.
// The replay is a serial chain per traced warp (one iteration per lock / fence / grid event), so
// every load it depends on is issued ahead: each lane keeps its next two fence timestamps with
// their scopes (k_fence_scopes: no event load), and the warp holds a window of its next 32 lock
// events, loaded in parallel and read by shuffles; fences that cannot activate anything are
// skipped (sync-heavy C5: chained per-event loads and no-op fences made this kernel 43 ms).
template <bool WRITE>
__global__ void __launch_bounds__(256) k_lock_infer(LockParams P) {
    const u32 lane = threadIdx.x & 31u;
    const u32 w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (w >= P.g.W) return;
    const KeySpace ks = P.ks;
    const u32 b = w / P.g.Wb, wi = w - b * P.g.Wb;
    const u32 my_off = wi * 32 + lane;
    const bool has_thread = my_off < P.g.D;
    const u32 my_t = b * P.g.D + my_off;
    u32 lk_lo = P.off[ks.lock + w];
    const u32 lk_hi = P.off[ks.lock + w + 1];
    if (lk_lo == lk_hi) {  // never a CAS / EXCH: no lock state
        if (!WRITE && has_thread) P.tcnt[my_t] = 0;
        return;
    }
    u32 f_lo = 0, f_hi = 0;
    if (has_thread) {
        f_lo = P.off[ks.any + my_t];
        f_hi = P.off[ks.any + my_t + 1];
    }
    u32 g_lo = P.off[ks.grid], g_hi = P.off[ks.grid + 1];
    u32 k_lo = P.off[ks.kb], k_hi = P.off[ks.kb + 1];

    Table wt, tt;
    wt.clear();
    tt.clear();
    bool isThread = false;
    u32 held = 0;  // this lane's effective held-lock Bloom
    u32 nt = 0;
    u32 tout = (WRITE && has_thread) ? P.toff[my_t] : 0;

    auto ts_at = [&](u32 pos, u32 hi) -> u32 { return pos < hi ? __ldg(P.sts + pos) : IGD_NONE32; };
    auto dev_at = [&](u32 pos, u32 hi) -> u32 { return pos < hi ? P.fdev[pos] : 0u; };
    u32 fA = ts_at(f_lo, f_hi), fB = ts_at(f_lo + 1, f_hi);  // this lane's next two fences
    u32 sA = dev_at(f_lo, f_hi), sB = dev_at(f_lo + 1, f_hi);  // ... and their scopes (1 = device)
    // the warp's lock events come in bursts (a lock section's CAS / EXCH of every locked lane):
    // a window of the next 32, lane i holding event lk_lo + i, loaded in parallel
    u32 win = lk_lo;  // lock index held by lane 0
    u32 w_ts = ts_at(win + lane, lk_hi);
    uint4 w_ev = event_at(P, w_ts);
    u32 lA = __shfl_sync(IGD_FULL, w_ts, 0);
    u32 g_next = ts_at(g_lo, g_hi);
    u32 k_next = ts_at(k_lo, k_hi);
    auto lower = [&](u32 lo, u32 hi, u32 v) -> u32 {  // first position in [lo, hi) with ts >= v
        while (lo < hi) {
            const u32 mid = (lo + hi) >> 1;
            if (__ldg(P.sts + mid) < v) lo = mid + 1;
            else hi = mid;
        }
        return lo;
    };
    // first position >= lo with ts >= v, given ts[lo] < v: exponential probes, then a binary search
    // (the target is usually a few entries ahead)
    auto gallop = [&](u32 lo, u32 hi, u32 v) -> u32 {
        u32 prev = lo, step = 1;
        while (true) {
            const u32 q = prev + step;
            if (q >= hi || __ldg(P.sts + q) >= v) return lower(prev + 1, q < hi ? q : hi, v);
            prev = q;
            step <<= 1;
        }
    };
    while (true) {
        // A fence can only change the lock state by activating a valid, inactive entry of the
        // fencing thread's table (the warp's until isThread).  Without one, this lane's fences up
        // to the next lock event / grid sync / kernel boundary are no-ops: jump over them (a lock
        // section's later fences and release fences are the bulk of a lock-heavy warp's stream).
        const u32 next_rel = min(min(lA, g_next), k_next);
        if (fA < next_rel && !(isThread ? tt.pending() : wt.pending())) {
            if (fB >= next_rel) {  // one fence to skip: the next one is in registers already
                f_lo++;
                fA = fB;
                sA = sB;
            } else {
                f_lo = gallop(f_lo + 1, f_hi, next_rel);
                fA = ts_at(f_lo, f_hi);
                sA = dev_at(f_lo, f_hi);
            }
            fB = ts_at(f_lo + 1, f_hi);
            sB = dev_at(f_lo + 1, f_hi);
        }
        const u32 f_min = __reduce_min_sync(IGD_FULL, fA);
        const u32 ts = min(min(f_min, k_next), min(lA, g_next));
        if (ts == IGD_NONE32) break;
        if (ts == k_next) {
            // kernel boundary: the next kernel's locking protocol is inferred afresh (A31)
            wt.clear();
            tt.clear();
            isThread = false;
            k_lo++;
            k_next = ts_at(k_lo, k_hi);
        } else if (ts == g_next) {
            // grid sync: every thread fences at device scope (A15)
            wt.activate(IGD_SCOPE_DEVICE);
            tt.activate(IGD_SCOPE_DEVICE);
            g_lo++;
            g_next = ts_at(g_lo, g_hi);
        } else if (ts == lA) {
            const u32 q = lk_lo - win;
            uint4 e;
            e.x = __shfl_sync(IGD_FULL, w_ev.x, q);
            e.y = __shfl_sync(IGD_FULL, w_ev.y, q);
            e.z = __shfl_sync(IGD_FULL, w_ev.z, q);
            e.w = __shfl_sync(IGD_FULL, w_ev.w, q);
            lk_lo++;
            if (lk_lo - win == 32u) {  // window consumed: the next 32
                win = lk_lo;
                w_ts = ts_at(win + lane, lk_hi);
                w_ev = event_at(P, w_ts);
            }
            lA = lk_lo < lk_hi ? __shfl_sync(IGD_FULL, w_ts, lk_lo - win) : IGD_NONE32;
            const u32 kind = ev_kind(e), s = norm_scope(ev_scope(e));
            const u32 h = lock_h18(ev_addr(e) >> 2);
            const u32 el = P.g.lane(ev_tid(e));
            if (kind == IGD_CAS) {
                if (!isThread && __popc(e.w) > 1) isThread = true;
                if (isThread) {
                    if (lane == el) tt.insert(h, s);
                } else {
                    wt.insert(h, s);
                }
            } else {  // EXCH
                if (isThread) {
                    if (lane == el) tt.remove(h, s);
                } else {
                    wt.remove(h, s);
                }
            }
        } else {
            // a fence by the lane whose next fence is ts (its scope from the fdev byte)
            const u32 owner = __ffs(__ballot_sync(IGD_FULL, fA == ts)) - 1;
            u32 s = 0;
            if (lane == owner) {
                s = sA ? IGD_SCOPE_DEVICE : IGD_SCOPE_BLOCK;
                f_lo++;
                fA = fB;
                sA = sB;
                fB = ts_at(f_lo + 1, f_hi);
                sB = dev_at(f_lo + 1, f_hi);
            }
            s = __shfl_sync(IGD_FULL, s, owner);
            if (isThread) {
                if (lane == owner) tt.activate(s);
            } else {
                wt.activate(s);
            }
        }
        // change point of this lane's thread: effective table = per-warp until isThread is set
        const u32 h = isThread ? tt.held() : wt.held();
        if (h != held && has_thread) {
            if (WRITE) P.tpts[tout + nt] = ((u64)ts << 16) | h;
            nt++;
            held = h;
        }
    }
    if (!WRITE && has_thread) P.tcnt[my_t] = nt;
}

// held-lock Bloom of thread c just before event i (the check's L(c, i)): the last change point
// of c with ts < i
struct LockView {
    const u32* toff;  // [T+1] per-thread change-point offsets
    const u64* tpts;  // change points (ts << 16 | bloom)
    const u32* tbits; // [ceil(T/32)] bit t: thread t ever holds a lock (has change points)
    u32 any;          // 0 when the trace has no CAS/EXCH at all
};
// A thread that never holds a lock has an empty Bloom at every time: R5 needs one of the two
// threads to have change points (a 1-bit-per-thread table, L1-resident, in front of the searches)
__device__ __forceinline__ bool may_hold(const LockView& V, u32 t) { return (__ldg(V.tbits + (t >> 5)) >> (t & 31u)) & 1u; }

__global__ void k_lock_bits(const u32* __restrict__ toff, u32 T, u32* __restrict__ bits) {
    const u32 w = blockIdx.x * blockDim.x + threadIdx.x;
    if (w * 32 >= T) return;
    u32 b = 0;
    for (u32 k = 0; k < 32 && w * 32 + k < T; k++) b |= (toff[w * 32 + k + 1] > toff[w * 32 + k] ? 1u : 0u) << k;
    bits[w] = b;
}

// Lock sets of two (thread, time) pairs at once -- R5's L(c, i) and the last accessor's -- with
// the two searches interleaved (independent L2 chains).  Short lists (<= 4 change points, most
// threads) are scanned from independent loads instead of a dependent binary search.
__device__ __forceinline__ u32 held_short(const u64* __restrict__ tpts, u32 lo, u32 hi, u32 i) {
    u32 L = 0;
#pragma unroll
    for (u32 k = 0; k < 4; k++) {
        if (lo + k < hi) {
            const u64 v = __ldg(tpts + lo + k);
            if ((u32)(v >> 16) < i) L = (u32)(v & 0xFFFFu);
        }
    }
    return L;
}
__device__ __forceinline__ void held_before2(const LockView& V, u32 c0, u32 i0, u32 c1, u32 i1, u32& L0, u32& L1) {
    u32 lo0 = __ldg(V.toff + c0), hi0 = __ldg(V.toff + c0 + 1);
    u32 lo1 = __ldg(V.toff + c1), hi1 = __ldg(V.toff + c1 + 1);
    const bool s0 = hi0 - lo0 <= 4u, s1 = hi1 - lo1 <= 4u;
    if (s0 && s1) {
        L0 = held_short(V.tpts, lo0, hi0, i0);
        L1 = held_short(V.tpts, lo1, hi1, i1);
        return;
    }
    const u32 b0 = lo0, b1 = lo1;
    while (lo0 < hi0 || lo1 < hi1) {
        const u32 m0 = (lo0 + hi0) >> 1, m1 = (lo1 + hi1) >> 1;
        const bool a0 = lo0 < hi0, a1 = lo1 < hi1;
        const u64 v0 = a0 ? __ldg(V.tpts + m0) : 0ull, v1 = a1 ? __ldg(V.tpts + m1) : 0ull;
        if (a0) {
            if ((u32)(v0 >> 16) < i0) lo0 = m0 + 1;
            else hi0 = m0;
        }
        if (a1) {
            if ((u32)(v1 >> 16) < i1) lo1 = m1 + 1;
            else hi1 = m1;
        }
    }
    L0 = lo0 > b0 ? (u32)(__ldg(V.tpts + lo0 - 1) & 0xFFFFu) : 0u;
    L1 = lo1 > b1 ? (u32)(__ldg(V.tpts + lo1 - 1) & 0xFFFFu) : 0u;
}

// ---------------------------------------------------------------------------------------------
// Exclusive scan of u32 counts (in place allowed), chained look-back. n includes the sentinel.
constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 8;
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_excl(const u32* in, u32* out, u32 n, u64* status,
                                                          u32* tile_ctr) {
    __shared__ u32 s_tile;
    __shared__ u32 s_wsum[SCAN_THREADS / 32];
    __shared__ u64 s_base;
    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) s_tile = atomicAdd(tile_ctr, 1u);
    __syncthreads();
    const u32 tile = s_tile;
    const u64 base = (u64)tile * SCAN_THREADS * SCAN_ITEMS + (u64)t * SCAN_ITEMS;
    u32 v[SCAN_ITEMS];
    u32 sum = 0;
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; j++) {
        v[j] = (base + j < n) ? in[base + j] : 0;
        sum += v[j];
    }
    u32 inc = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        u32 x = __shfl_up_sync(IGD_FULL, inc, o);
        if (lane >= (u32)o) inc += x;
    }
    if (lane == 31) s_wsum[warp] = inc;
    __syncthreads();
    u32 wpre = 0, total = 0;
#pragma unroll
    for (int w = 0; w < SCAN_THREADS / 32; w++) {
        if ((u32)w < warp) wpre += s_wsum[w];
        total += s_wsum[w];
    }
    if (warp == 0) {
        if (lane == 0) st_relaxed(&status[tile], (tile == 0 ? ST_INC : ST_AGG) | total);
        u64 b = 0;
        if (tile > 0) {
            b = lookback_sum_warp(status, tile);
            if (lane == 0) st_relaxed(&status[tile], ST_INC | (b + total));
        }
        if (lane == 0) s_base = b;
    }
    __syncthreads();
    u32 run = (u32)s_base + wpre + inc - sum;
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; j++) {
        if (base + j < n) out[base + j] = run;
        run += v[j];
    }
}

}  // namespace syncx
