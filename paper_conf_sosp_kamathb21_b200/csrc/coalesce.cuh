// coalesce.cuh -- warp-coalesced check mode (§6.5; reading A32): marks the events
// that a coalesced group's first lane checks on behalf of.
//
// A group is a run of popcount(mask) >= 2 consecutive events of one warp instruction: same
// warp, kind (LD or ATOM), scope, mask and word, lanes strictly ascending from the mask's lowest
// lane.  With link(i) = "events i-1 and i agree on (warp, kind, scope, mask, word) and lane(i-1)
// < lane(i)", event i of such an instruction (rank r among the mask's lanes, cnt = popc(mask))
// is a skipped member iff r > 0 and link(k) holds for every k in (i - r, i - r + cnt - 1]:
// cnt strictly ascending lanes drawn from the mask's cnt lanes are exactly the mask's lanes.
//
// One warp walks a run of 32-event rows with a three-row window (previous, current, next) in
// registers: the link bits of the window are three ballots, a group (at most 32 events) lies
// inside the window, and the skipped members of the current row leave as one 32-bit word of the
// output bitmap (bit i & 31 of word i >> 5).  The trace is read once (plus one halo row per run).
#pragma once
#include "common.cuh"

namespace coal {

constexpr int THREADS = 256;
constexpr int ROWS = 16;  // rows per warp run

struct Ev {
    u32 w, kind, scope, mask, lane;
    u64 word;
};

__device__ __forceinline__ Ev load_ev(const igd_event* ev, u64 n, u64 i, const Geo& g) {
    Ev e;
    if (i < n) {
        const uint4 r = ld_event_stream(ev, i);
        const u32 tid = ev_tid(r);
        e.kind = ev_kind(r);
        e.scope = ev_scope(r);
        e.mask = r.w;
        e.word = ev_addr(r) >> 2;
        e.w = g.warp(tid);
        e.lane = g.lane(tid);
    } else {
        e.kind = 0xFu;  // no link to or from positions past the end
        e.scope = e.mask = e.lane = e.w = 0;
        e.word = 0;
    }
    return e;
}

// link of event (this lane's `cur`) with its predecessor `prv`
__device__ __forceinline__ bool linked(const Ev& prv, const Ev& cur) {
    const bool groupable = cur.kind == IGD_LD || cur.kind == IGD_ATOM;
    return groupable && prv.kind == cur.kind && prv.scope == cur.scope && prv.mask == cur.mask && prv.w == cur.w &&
           prv.word == cur.word && prv.lane < cur.lane;
}

// bits [lo, hi] of a 96-bit mask (m0 = bits 0..31, m1 = 32..63, m2 = 64..95) all set?
__device__ __forceinline__ bool all_set(u32 m0, u32 m1, u32 m2, int lo, int hi) {
    if (lo > hi) return true;
    bool ok = true;
#pragma unroll
    for (int q = 0; q < 3; q++) {
        const int a = max(lo, 32 * q), b = min(hi, 32 * q + 31);
        if (a <= b) {
            const u32 width = (u32)(b - a + 1);
            const u32 want = (width == 32 ? 0xFFFFFFFFu : ((1u << width) - 1u)) << (a - 32 * q);
            const u32 m = q == 0 ? m0 : q == 1 ? m1 : m2;
            ok = ok && (m & want) == want;
        }
    }
    return ok;
}

__global__ void __launch_bounds__(THREADS) k_coalesce_marks(const igd_event* __restrict__ ev, u64 n, Geo g,
                                                           u32* __restrict__ skip_bits) {
    const u32 lane = threadIdx.x & 31u;
    const u64 rows = (n + 31) / 32;
    const u64 warp_id = ((u64)blockIdx.x * THREADS + threadIdx.x) >> 5;
    const u64 r0 = warp_id * ROWS;
    if (r0 >= rows) return;
    // window: previous row (p), current (c), next (x); links of each (lane 0 of a row links to
    // lane 31 of the row before)
    Ev p = load_ev(ev, n, r0 > 0 ? (r0 - 1) * 32 + lane : ~0ull, g);
    Ev c = load_ev(ev, n, r0 * 32 + lane, g);
    Ev pp_last;  // lane 31 of the row before p (for p's lane-0 link)
    {
        const Ev t = load_ev(ev, n, r0 > 1 ? (r0 - 2) * 32 + 31 : ~0ull, g);
        pp_last = t;
    }
    auto row_links = [&](const Ev& prev_row_any, const Ev& row) -> u32 {
        // predecessor of this lane's event: lane-1 of the same row, or lane 31 of prev_row_any
        Ev q;
        q.kind = __shfl_sync(IGD_FULL, row.kind, (lane + 31) & 31);
        q.scope = __shfl_sync(IGD_FULL, row.scope, (lane + 31) & 31);
        q.mask = __shfl_sync(IGD_FULL, row.mask, (lane + 31) & 31);
        q.w = __shfl_sync(IGD_FULL, row.w, (lane + 31) & 31);
        q.lane = __shfl_sync(IGD_FULL, row.lane, (lane + 31) & 31);
        q.word = __shfl_sync(IGD_FULL, row.word, (lane + 31) & 31);
        if (lane == 0) q = prev_row_any;
        return __ballot_sync(IGD_FULL, linked(q, row));
    };
    auto last_of = [&](const Ev& row) -> Ev {  // lane 31's event, broadcast
        Ev q;
        q.kind = __shfl_sync(IGD_FULL, row.kind, 31);
        q.scope = __shfl_sync(IGD_FULL, row.scope, 31);
        q.mask = __shfl_sync(IGD_FULL, row.mask, 31);
        q.w = __shfl_sync(IGD_FULL, row.w, 31);
        q.lane = __shfl_sync(IGD_FULL, row.lane, 31);
        q.word = __shfl_sync(IGD_FULL, row.word, 31);
        return q;
    };
    u32 Lp = row_links(pp_last, p);
    Ev p_last = last_of(p);
    u32 Lc = row_links(p_last, c);
    for (int k = 0; k < ROWS && r0 + k < rows; k++) {
        const u64 r = r0 + k;
        const Ev x = load_ev(ev, n, (r + 1) * 32 + lane, g);
        const Ev c_last = last_of(c);
        const u32 Lx = row_links(c_last, x);
        // this lane's event: position 32 + lane of the window
        const u32 cnt = __popc(c.mask);
        const u32 rank = __popc(c.mask & ((1u << c.lane) - 1u));
        const bool groupable = (c.kind == IGD_LD || c.kind == IGD_ATOM) && cnt >= 2 && ((c.mask >> c.lane) & 1u);
        const int s = 32 + (int)lane - (int)rank, e = s + (int)cnt - 1;
        const bool member = groupable && rank > 0 && all_set(Lp, Lc, Lx, s + 1, e);
        const u32 bits = __ballot_sync(IGD_FULL, member);
        if (lane == 0 && r * 32 < n) skip_bits[r] = bits;
        Lp = Lc;
        Lc = Lx;
        c = x;
    }
}

}  // namespace coal
