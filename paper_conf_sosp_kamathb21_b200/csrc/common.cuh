// common.cuh -- device helpers shared by the libigd kernels (sm_100a).
// Nothing here is shared with oracle/: the oracle has its own reader and constants.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/igd.h"
#include "../../include/igd_debug.h"

typedef uint32_t u32;
typedef uint64_t u64;
typedef uint16_t u16;

#define IGD_FULL 0xFFFFFFFFu
#define IGD_NONE32 0xFFFFFFFFu

// ---- fast unsigned division by a runtime-invariant divisor (Granlund-Montgomery) ----------
struct FastDiv {
    u32 d, m, s;
    __host__ void init(u32 div) {
        d = div;
        u32 l = 0;
        while ((1ull << l) < div) l++;
        s = l;
        m = (u32)((((1ull << 32) * ((1ull << l) - div)) / div) + 1);
    }
    __device__ __forceinline__ u32 div(u32 n) const {
        u32 hi = __umulhi(m, n);
        return (u32)(((u64)hi + n) >> s);
    }
};

// ---- grid geometry of the traced kernel --------------------------
struct Geo {
    u32 D;   // block_dim
    u32 Wb;  // warps per block = ceil(D/32)
    u32 T;   // threads
    u32 W;   // warps
    u32 B;   // blocks
    FastDiv fd;
    u32 dlog;  // log2(D) when D is a power of two, else 32
    u32 a32;   // D % 32 == 0: warps never straddle blocks, so warp(t) = t / 32 and lane(t) = t % 32
    __host__ void init(u32 nb, u32 bd) {
        D = bd;
        Wb = (bd + 31) / 32;
        B = nb;
        T = nb * bd;
        W = nb * Wb;
        fd.init(bd);
        dlog = 32;
        for (u32 l = 0; l < 32; l++)
            if ((1u << l) == bd) dlog = l;
        a32 = bd % 32 == 0 ? 1u : 0u;
    }
#ifndef IGD_GEO_FAST
#define IGD_GEO_FAST 0
#endif
    __device__ __forceinline__ u32 block(u32 t) const {
        if (IGD_GEO_FAST) return dlog < 32 ? t >> dlog : fd.div(t);
        return fd.div(t);
    }
    __device__ __forceinline__ u32 warp(u32 t) const {
        if (IGD_GEO_FAST && a32) return t >> 5;
        u32 b = fd.div(t);
        return b * Wb + ((t - b * D) >> 5);
    }
    __device__ __forceinline__ u32 lane(u32 t) const {
        if (IGD_GEO_FAST && a32) return t & 31u;
        u32 b = fd.div(t);
        return (t - b * D) & 31u;
    }
};

// ---- synchronization-entity key space (CSR of timestamps) ------------------
//   [0,T) fences of thread t (any scope)         "AnyF"
//   [T,2T) device/system fences of thread t       "DevF"
//   [2T,2T+W) syncwarps of warp w                 "WBar"
//   [2T+W,2T+W+B) syncthreads of block b          "BBar"
//   2T+W+B  grid syncs                            "Grid"
//   [2T+W+B+1, 2T+2W+B+1) CAS/EXCH of warp w      "Lock"
//   2T+2W+B+1 kernel boundaries                   "Kb" (multi-kernel traces, reading A31)
struct KeySpace {
    u32 any, dev, wb, bb, grid, lock, kb, E;
    __host__ void init(const Geo& g) {
        any = 0;
        dev = g.T;
        wb = 2 * g.T;
        bb = 2 * g.T + g.W;
        grid = bb + g.B;
        lock = grid + 1;
        kb = lock + g.W;
        E = kb + 1;
    }
};

// ---- decoupled look-back status words --------------------------------------------------------
// bits 63..62: 0 = not ready, 1 = aggregate, 2 = inclusive prefix; bits 61..0: value.
#define ST_AGG (1ull << 62)
#define ST_INC (2ull << 62)
#define ST_VAL_MASK ((1ull << 62) - 1)

__device__ __forceinline__ void st_relaxed(u64* p, u64 v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ u64 ld_relaxed(const u64* p) {
    u64 v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Digit statuses of the radix passes (rsort, fused) also carry the pass's epoch in bits 61..40,
// values in bits 39..0: a status of an earlier pass reads as "not ready", so the per-(tile, digit)
// buffer is never cleared between passes (it was ~2 GB of memset per pass at C5).
#define DS_VAL_MASK ((1ull << 40) - 1)
#define DS_EPOCH_MAX 0x3FFFFFu
__device__ __forceinline__ u64 ds_make(u64 state, u32 epoch, u64 v) { return state | ((u64)epoch << 40) | v; }
__device__ __forceinline__ bool ds_ready(u64 s, u32 epoch) {
    return (s >> 62) != 0 && ((u32)(s >> 40) & DS_EPOCH_MAX) == epoch;
}
__device__ __forceinline__ u64 ds_spin(const u64* p, u64 s, u32 epoch) {
    while (!ds_ready(s, epoch)) s = ld_relaxed(p);
    return s;
}

// Wait until a look-back status word is published (non-zero state).  The back-off frees issue
// slots for the other CTAs of the SM while a predecessor tile is still working.
#ifndef IGD_SPIN_NS
#define IGD_SPIN_NS 0
#endif
__device__ __forceinline__ u64 spin_status(const u64* p, u64 s) {
    while ((s >> 62) == 0) {
        if (IGD_SPIN_NS) __nanosleep(IGD_SPIN_NS);
        s = ld_relaxed(p);
    }
    return s;
}

// Exclusive prefix of a u64 sum over tiles [0, tile): single thread walks back.
__device__ __forceinline__ u64 lookback_sum(u64* status, u32 tile) {
    u64 excl = 0;
    long t = (long)tile - 1;
    while (t >= 0) {
        u64 s;
        do {
            s = ld_relaxed(&status[t]);
        } while ((s >> 62) == 0);
        excl += s & ST_VAL_MASK;
        if ((s >> 62) == 2) break;
        t--;
    }
    return excl;
}

// Warp-cooperative variant: lanes probe 32 predecessors at a time. Returns the exclusive
// prefix in every lane.  Must be called by a full warp.
__device__ __forceinline__ u64 lookback_sum_warp(u64* status, u32 tile) {
    const u32 lane = threadIdx.x & 31u;
    u64 excl = 0;
    long top = (long)tile - 1;  // highest tile not yet consumed
    while (top >= 0) {
        long t = top - (long)lane;
        u64 s = ST_INC;  // tiles < 0 behave as inclusive zero
        if (t >= 0) {
            do {
                s = ld_relaxed(&status[t]);
            } while ((s >> 62) == 0);
        }
        u32 inc_mask = __ballot_sync(IGD_FULL, (s >> 62) == 2);
        // consume lanes 0..k where k = first inclusive lane (or all 32)
        u32 k = inc_mask ? (__ffs(inc_mask) - 1) : 31;
        u64 v = (lane <= k) ? (s & ST_VAL_MASK) : 0;
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(IGD_FULL, v, o);
        excl += v;
        if (inc_mask) break;
        top -= 32;
    }
    return excl;
}

// ---- TMA bulk copies (cp.async.bulk, global -> shared, completion on an mbarrier) ----------
__device__ __forceinline__ u32 smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(u64* mbar, u32 count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u64* mbar, u32 bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes)
                 : "memory");
}
// bytes: multiple of 16; src, dst: 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, u32 bytes, u64* mbar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(mbar))
        : "memory");
}
__device__ __forceinline__ void mbar_arrive(u64* mbar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(mbar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* mbar, u32 phase) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(mbar)),
        "r"(phase)
        : "memory");
}

__device__ __forceinline__ u32 lanemask_lt() {
    u32 m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Load one 16-byte event as uint4 (x,y = addr lo/hi, z = tk, w = mask), streaming.
__device__ __forceinline__ uint4 ld_event(const igd_event* ev, u64 i) {
    return __ldg(reinterpret_cast<const uint4*>(ev) + i);
}
__device__ __forceinline__ uint4 ld_event_stream(const igd_event* ev, u64 i) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(reinterpret_cast<const uint4*>(ev) + i));
    return r;
}

__device__ __forceinline__ u32 ev_tid(const uint4& e) { return e.z & 0xFFFFFFu; }
__device__ __forceinline__ u32 ev_kind(const uint4& e) { return (e.z >> 24) & 0xFu; }
__device__ __forceinline__ u32 ev_scope(const uint4& e) { return (e.z >> 28) & 0x3u; }
__device__ __forceinline__ u64 ev_addr(const uint4& e) { return (u64)e.x | ((u64)e.y << 32); }

// Reading A34 (per-kernel geometry): a KERNEL_BOUNDARY's nonzero addr = (n_blocks << 32) |
// block_dim of the next kernel; valid when both are >= 1 and the grid has <= 2^24 threads
__host__ __device__ __forceinline__ bool geo_code_ok(u32 nb, u32 bd) {
    return nb >= 1 && bd >= 1 && (u64)nb * bd <= (1ull << 24);
}

// normalised scope: SYSTEM == DEVICE (reading A12)
__device__ __forceinline__ u32 norm_scope(u32 s) { return s == IGD_SCOPE_SYSTEM ? IGD_SCOPE_DEVICE : s; }

// Reading A8: 18-bit address hash and 2-way 16-bit Bloom summary of a lock.
__device__ __forceinline__ u32 lock_h18(u64 word) { return ((u32)word * 0x9E3779B1u) >> 14; }
__device__ __forceinline__ u32 lock_bloom(u32 h) { return (1u << (h & 15u)) | (1u << ((h >> 4) & 15u)); }

// first x > a in ts[lo,hi) exists and x < b   (between(list, a, b))
__device__ __forceinline__ bool between(const u32* __restrict__ ts, u32 lo, u32 hi, u32 a, u32 b) {
    u32 end = hi;
    while (lo < hi) {
        u32 mid = (lo + hi) >> 1;
        if (__ldg(ts + mid) <= a) lo = mid + 1;
        else hi = mid;
    }
    return lo < end && __ldg(ts + lo) < b;
}
