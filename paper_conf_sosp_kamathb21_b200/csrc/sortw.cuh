// sortw.cuh -- a5 with wide digits: the access sort's passes after the fused digit-0 pass as
// passes of up to 11 bits, so a 30-bit word key takes 8 + 11 + 11 bits -- two passes over the
// 12-byte records after the fused pass instead of three 8-bit ones (24 B per access per pass).
//
// Same contract as rsort::k_onesweep (stable LSD pass: (earlier chunks) + (earlier sub-tiles of
// the chunk) + (earlier warps of the sub-tile) + (earlier items / lanes of the warp) = input
// order), restructured for 2048 digits:
//   * a CTA owns a CHUNK of SUBS consecutive 4096-key sub-tiles (a ticket in CTA start order);
//   * phase A counts the chunk's digits (keys read once, kept in L2 with an evict_last policy)
//     and publishes the chunk's 2048 counts at once;
//   * phase B looks back per digit over earlier chunks (one look-back per CHUNK keys, not per
//     4096: the per-(tile, digit) status traffic of an 11-bit onesweep would be a third of the
//     data traffic);
//   * phase C ranks each sub-tile with a warp multisplit into per-warp u16 digit counts, turns
//     them into tile positions, reorders keys and values through shared memory and writes them
//     at running per-digit output offsets.
#pragma once
#include "common.cuh"

namespace rsortw {

constexpr int THREADS = 256;
constexpr int WARPS = THREADS / 32;
constexpr int ITEMS = 16;
constexpr int SUB = THREADS * ITEMS;  // keys per sub-tile
#ifndef IGD_SORTW_SUBS
#define IGD_SORTW_SUBS 8
#endif
constexpr int SUBS = IGD_SORTW_SUBS;
constexpr u32 CHUNK = (u32)SUB * SUBS;  // keys per CTA
constexpr int RBITS = 11;                // widest digit
constexpr int RADIX = 1 << RBITS;
constexpr int DPT = RADIX / THREADS;     // consecutive digits owned by a thread in the per-digit steps
static_assert(DPT == 8, "per-digit steps move 8 u16 counts as one uint4");
#ifndef IGD_SORTW_MIX
#define IGD_SORTW_MIX 2  // one row in N ranked with match.any, the others with ballots
#endif

struct Params {
    const u32* kin;
    const u64* vin;
    u32* kout;
    u64* vout;
    u32 n;
    u32 shift;              // digit = (key >> shift) & dmask
    u32 dmask;              // <= RADIX - 1
    const u32* digit_base;  // [RADIX] exclusive global offsets of this pass's digits
    u64* status;            // [n_chunks * RADIX] digit statuses (ds_make), tagged with `epoch`
    u32 epoch;
    u32* tile_ctr;  // zeroed: chunk tickets
};

// dynamic shared memory: per-warp u16 counts, reordered keys, reordered values, running offsets,
// per-sub-tile output bases (phase A: the chunk's digit counts)
constexpr size_t OFF_WH = 0;
constexpr size_t OFF_K = OFF_WH + (size_t)WARPS * RADIX * 2;
constexpr size_t OFF_V = OFF_K + (size_t)SUB * 4;
constexpr size_t OFF_RUN = OFF_V + (size_t)SUB * 8;
constexpr size_t OFF_GB = OFF_RUN + (size_t)RADIX * 4;
constexpr size_t SMEM = OFF_GB + (size_t)RADIX * 4;  // 96 KB: 2 CTAs per SM

__device__ __forceinline__ uint4 ld_keep_v4(const uint4* p, u64 pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ u32 ld_keep(const u32* p, u64 pol) {
    u32 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ u64 policy_evict_last() {
    u64 pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void st_relaxed_v2(u64* p, u64 a, u64 b) {
    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_relaxed_v2(const u64* p, u64& a, u64& b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

// Exclusive digit bases of `npass` wide histograms ([npass][RADIX]), one CTA of RADIX/2 threads each.
__global__ void __launch_bounds__(RADIX / 2) k_digit_base_w(const u32* __restrict__ hist, u32* __restrict__ base) {
    __shared__ u32 s_w[RADIX / 64];
    const u32 p = blockIdx.x, t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    const u32 v0 = hist[p * RADIX + 2 * t], v1 = hist[p * RADIX + 2 * t + 1];
    u32 inc = v0 + v1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const u32 x = __shfl_up_sync(IGD_FULL, inc, o);
        if (lane >= (u32)o) inc += x;
    }
    if (lane == 31) s_w[warp] = inc;
    __syncthreads();
    u32 wpre = 0;
    for (u32 w = 0; w < warp; w++) wpre += s_w[w];
    const u32 ex = wpre + inc - v0 - v1;
    base[p * RADIX + 2 * t] = ex;
    base[p * RADIX + 2 * t + 1] = ex + v0;
}

// Histograms of two wide digits of u32 keys (persistent grid, shared-memory counts flushed once
// per CTA): digit p = (key >> sh[p]) & m[p].
__global__ void __launch_bounds__(256) k_hist_w(const u32* __restrict__ keys, u32 n, u32 sh0, u32 m0, u32 sh1, u32 m1,
                                                u32* __restrict__ hist) {
    __shared__ u32 s[2][RADIX];
    for (int i = threadIdx.x; i < 2 * RADIX; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    const u32 n4 = n / 4;
    for (u32 q = blockIdx.x * blockDim.x + threadIdx.x; q < n4; q += gridDim.x * blockDim.x) {
        const uint4 k4 = __ldcs(reinterpret_cast<const uint4*>(keys) + q);
        const u32 kk[4] = {k4.x, k4.y, k4.z, k4.w};
#pragma unroll
        for (int e = 0; e < 4; e++) {
            atomicAdd(&s[0][(kk[e] >> sh0) & m0], 1u);
            atomicAdd(&s[1][(kk[e] >> sh1) & m1], 1u);
        }
    }
    if (blockIdx.x == 0)
        for (u32 i = n4 * 4 + threadIdx.x; i < n; i += blockDim.x) {
            const u32 k = keys[i];
            atomicAdd(&s[0][(k >> sh0) & m0], 1u);
            atomicAdd(&s[1][(k >> sh1) & m1], 1u);
        }
    __syncthreads();
    for (int i = threadIdx.x; i < 2 * RADIX; i += blockDim.x) {
        const u32 v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

// Mask of the lanes (within vmask) whose digit (< RADIX) equals d.
template <int MODE>
__device__ __forceinline__ u32 peers_w(u32 d, u32 vmask) {
    if (MODE == 0) return __match_any_sync(IGD_FULL, d) & vmask;
    u32 peers = vmask;
#pragma unroll
    for (int b = 0; b < RBITS; b++) {
        const u32 bit = (d >> b) & 1u;
        const u32 bal = __ballot_sync(IGD_FULL, bit);
        peers &= bit ? bal : ~bal;
    }
    return peers;
}

__global__ void __launch_bounds__(THREADS, 2) k_sweep_w(Params P) {
    __shared__ u32 s_wsum[WARPS];
    __shared__ u32 s_tile;
    __shared__ __align__(8) u64 s_mbar;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    u16* s_wh = reinterpret_cast<u16*>(s_dyn + OFF_WH);
    u32* s_k = reinterpret_cast<u32*>(s_dyn + OFF_K);
    u64* s_v = reinterpret_cast<u64*>(s_dyn + OFF_V);
    u32* s_run = reinterpret_cast<u32*>(s_dyn + OFF_RUN);
    u32* s_gb = reinterpret_cast<u32*>(s_dyn + OFF_GB);
    u32* s_cnt = s_gb;  // phase A

    const u32 t = threadIdx.x, lane = t & 31u, warp = t >> 5;
    if (t == 0) {
        s_tile = atomicAdd(P.tile_ctr, 1u);
        mbar_init(&s_mbar, 1);
    }
    for (int i = t; i < RADIX; i += THREADS) s_cnt[i] = 0;
    __syncthreads();
    const u32 chunk = s_tile;
    const u32 cbase = chunk * CHUNK;  // n <= 2^32 - 2^17 (host)
    const u32 cn = min(CHUNK, P.n - cbase);
    const u32 shift = P.shift, dmask = P.dmask;
    const u64 pol = policy_evict_last();

    // ---- phase A: the chunk's digit counts (keys stay in L2 for phase C)
    if (cn == CHUNK) {
        const uint4* k4 = reinterpret_cast<const uint4*>(P.kin + cbase);
#pragma unroll 4
        for (u32 q = t; q < CHUNK / 4; q += THREADS) {
            const uint4 v = ld_keep_v4(k4 + q, pol);
            atomicAdd(&s_cnt[(v.x >> shift) & dmask], 1u);
            atomicAdd(&s_cnt[(v.y >> shift) & dmask], 1u);
            atomicAdd(&s_cnt[(v.z >> shift) & dmask], 1u);
            atomicAdd(&s_cnt[(v.w >> shift) & dmask], 1u);
        }
    } else {
        for (u32 i = t; i < cn; i += THREADS) atomicAdd(&s_cnt[(ld_keep(P.kin + cbase + i, pol) >> shift) & dmask], 1u);
    }
    __syncthreads();

    // ---- phase B: publish the chunk's counts, look back per digit (thread t owns digits
    // t*DPT .. t*DPT+7: vector status accesses), running output offsets
    {
        const u32 d0 = t * DPT;
        u32 cnt[DPT];
        {
            const uint4 a = *reinterpret_cast<const uint4*>(s_cnt + d0);
            const uint4 b = *reinterpret_cast<const uint4*>(s_cnt + d0 + 4);
            cnt[0] = a.x, cnt[1] = a.y, cnt[2] = a.z, cnt[3] = a.w;
            cnt[4] = b.x, cnt[5] = b.y, cnt[6] = b.z, cnt[7] = b.w;
        }
        u64* my = P.status + (u64)chunk * RADIX + d0;
        const u64 st0 = chunk == 0 ? ST_INC : ST_AGG;
#pragma unroll
        for (int k = 0; k < DPT; k += 2)
            st_relaxed_v2(my + k, ds_make(st0, P.epoch, cnt[k]), ds_make(st0, P.epoch, cnt[k + 1]));
        u64 excl[DPT];
#pragma unroll
        for (int k = 0; k < DPT; k++) excl[k] = 0;
        if (chunk > 0) {
            u32 pending = (1u << DPT) - 1u;
            long tt = (long)chunk - 1;
            while (pending) {
                const u64* ps = P.status + (u64)tt * RADIX + d0;
                u64 s[DPT];
#pragma unroll
                for (int k = 0; k < DPT; k += 2) ld_relaxed_v2(ps + k, s[k], s[k + 1]);
#pragma unroll
                for (int k = 0; k < DPT; k++) {
                    if ((pending >> k) & 1u) {
                        s[k] = ds_spin(ps + k, s[k], P.epoch);
                        excl[k] += s[k] & DS_VAL_MASK;
                        if ((s[k] >> 62) == 2) pending &= ~(1u << k);
                    }
                }
                tt--;
            }
#pragma unroll
            for (int k = 0; k < DPT; k += 2)
                st_relaxed_v2(my + k, ds_make(ST_INC, P.epoch, excl[k] + cnt[k]),
                              ds_make(ST_INC, P.epoch, excl[k + 1] + cnt[k + 1]));
        }
        const uint4 b0 = *reinterpret_cast<const uint4*>(P.digit_base + d0);
        const uint4 b1 = *reinterpret_cast<const uint4*>(P.digit_base + d0 + 4);
        *reinterpret_cast<uint4*>(s_run + d0) =
            make_uint4(b0.x + (u32)excl[0], b0.y + (u32)excl[1], b0.z + (u32)excl[2], b0.w + (u32)excl[3]);
        *reinterpret_cast<uint4*>(s_run + d0 + 4) =
            make_uint4(b1.x + (u32)excl[4], b1.y + (u32)excl[5], b1.z + (u32)excl[6], b1.w + (u32)excl[7]);
    }

    // ---- phase C: sub-tiles in order
    const u32 wofs = warp * 32 * ITEMS;
    const u32 lt = lanemask_lt();
    for (u32 sb = 0; sb < cn; sb += SUB) {
        const u32 base = cbase + sb;
        const u32 sn = min((u32)SUB, cn - sb);
        const bool full = sn == (u32)SUB;
        __syncthreads();  // the previous sub-tile's readers of s_wh / s_k / s_v / s_gb are done
        {
            uint4* w4 = reinterpret_cast<uint4*>(s_wh);
#pragma unroll
            for (int i = 0; i < WARPS * RADIX * 2 / 16 / THREADS; i++) w4[t + i * THREADS] = make_uint4(0, 0, 0, 0);
        }
        // full sub-tiles: the values arrive in s_v by one TMA bulk copy while the keys are ranked
        const u32 phase = (sb / SUB) & 1u;
        if (full && t == 0) {
            mbar_expect_tx(&s_mbar, SUB * sizeof(u64));
            bulk_g2s(s_v, P.vin + base, SUB * sizeof(u64), &s_mbar);
        }
        u32 key[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const u32 i = wofs + j * 32 + lane;
            key[j] = (full || i < sn) ? __ldcs(P.kin + base + i) : 0u;
        }
        __syncthreads();
        u32 rank2[ITEMS / 2];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const bool valid = full || wofs + j * 32 + lane < sn;
            const u32 vmask = full ? IGD_FULL : __ballot_sync(IGD_FULL, valid);
            const u32 d = (key[j] >> shift) & dmask;
            // invalid lanes (partial sub-tile) are masked out of every peer set and never write
            const u32 peers = (IGD_SORTW_MIX && (j % IGD_SORTW_MIX) == IGD_SORTW_MIX - 1) ? peers_w<0>(d, vmask)
                                                                                          : peers_w<1>(d, vmask);
            const u32 leader = __ffs(peers) - 1;
            u32 old = 0;
            if (lane == leader && valid) {
                old = s_wh[warp * RADIX + d];
                s_wh[warp * RADIX + d] = (u16)(old + __popc(peers));
            }
            old = __shfl_sync(IGD_FULL, old, leader & 31u);
            const u32 r = old + __popc(peers & lt);
            if (j & 1) rank2[j / 2] |= r << 16;
            else rank2[j / 2] = r;
            __syncwarp();
        }
        __syncthreads();
        // per digit: sub-tile counts, exclusive scan over the 2048 digits, every warp's tile
        // position base for its digits (u16, < 4096) in place of its counts
        {
            const u32 d0 = t * DPT;
            u32 cnt[DPT];
            {
                u32 cp[DPT / 2] = {0, 0, 0, 0};  // u16 pairs: a digit's count is <= 4096
#pragma unroll
                for (int w = 0; w < WARPS; w++) {
                    const uint4 q = *reinterpret_cast<const uint4*>(s_wh + w * RADIX + d0);
                    cp[0] += q.x, cp[1] += q.y, cp[2] += q.z, cp[3] += q.w;
                }
#pragma unroll
                for (int k = 0; k < DPT; k++) cnt[k] = (cp[k / 2] >> (16 * (k & 1))) & 0xFFFFu;
            }
            u32 loc[DPT], tot = 0;
#pragma unroll
            for (int k = 0; k < DPT; k++) {
                loc[k] = tot;
                tot += cnt[k];
            }
            u32 inc = tot;
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
            const u32 texcl = wpre + inc - tot;  // sub-tile position of digit d0's first key
            u32 run[DPT];
#pragma unroll
            for (int k = 0; k < DPT; k++) run[k] = texcl + loc[k];
            // s_gb[d] = s_run[d] - (tile position of d's first key); s_run[d] += count
            {
                uint4 r0 = *reinterpret_cast<const uint4*>(s_run + d0);
                uint4 r1 = *reinterpret_cast<const uint4*>(s_run + d0 + 4);
                *reinterpret_cast<uint4*>(s_gb + d0) =
                    make_uint4(r0.x - run[0], r0.y - run[1], r0.z - run[2], r0.w - run[3]);
                *reinterpret_cast<uint4*>(s_gb + d0 + 4) =
                    make_uint4(r1.x - run[4], r1.y - run[5], r1.z - run[6], r1.w - run[7]);
                *reinterpret_cast<uint4*>(s_run + d0) =
                    make_uint4(r0.x + cnt[0], r0.y + cnt[1], r0.z + cnt[2], r0.w + cnt[3]);
                *reinterpret_cast<uint4*>(s_run + d0 + 4) =
                    make_uint4(r1.x + cnt[4], r1.y + cnt[5], r1.z + cnt[6], r1.w + cnt[7]);
            }
            // per-warp bases as u16 pairs (< 4096: no carry between the halves)
            u32 rp[DPT / 2];
#pragma unroll
            for (int k = 0; k < DPT; k += 2) rp[k / 2] = run[k] | (run[k + 1] << 16);
#pragma unroll
            for (int w = 0; w < WARPS; w++) {
                uint4* q = reinterpret_cast<uint4*>(s_wh + w * RADIX + d0);
                const uint4 c = *q;
                *q = make_uint4(rp[0], rp[1], rp[2], rp[3]);
                rp[0] += c.x, rp[1] += c.y, rp[2] += c.z, rp[3] += c.w;
            }
        }
        __syncthreads();
        u64 val[ITEMS];
        if (full) {
            mbar_wait(&s_mbar, phase);
#pragma unroll
            for (int j = 0; j < ITEMS; j++) val[j] = s_v[wofs + j * 32 + lane];
        } else {
#pragma unroll
            for (int j = 0; j < ITEMS; j++) {
                const u32 i = wofs + j * 32 + lane;
                val[j] = i < sn ? __ldcs(P.vin + base + i) : 0ull;
            }
        }
        // keys and values to their sub-tile positions
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            if (full || wofs + j * 32 + lane < sn) {
                const u32 d = (key[j] >> shift) & dmask;
                const u32 pos = ((rank2[j / 2] >> (16 * (j & 1))) & 0xFFFFu) + s_wh[warp * RADIX + d];
                rank2[j / 2] = (j & 1) ? (rank2[j / 2] & 0xFFFFu) | (pos << 16) : (rank2[j / 2] & 0xFFFF0000u) | pos;
                s_k[pos] = key[j];
            }
        }
        __syncthreads();  // every staged value is in registers
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            if (full || wofs + j * 32 + lane < sn) s_v[(rank2[j / 2] >> (16 * (j & 1))) & 0xFFFFu] = val[j];
        __syncthreads();
        // out in digit runs
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            const u32 i = t + k * THREADS;
            if (full || i < sn) {
                const u32 kk = s_k[i];
                const u32 o = s_gb[(kk >> shift) & dmask] + i;
                __stcs(P.kout + o, kk);
                __stcs(P.vout + o, s_v[i]);
            }
        }
        // the next sub-tile's TMA copy overwrites s_v: order this thread's generic accesses
        // before it (async proxy)
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
}

}  // namespace rsortw
