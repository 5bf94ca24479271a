// lastk.cuh -- paper-fidelity mode A37: last-k accessor histories.
//
// §6.7: "tracking the last 2, 4, and 8 accessors to a memory location in the
// metadata instead of only the last accessor".  Reading A37: the candidates md_1..md_k are the
// last k writers (loads) or the last k accessors (stores, atomics) of the word, newest first;
// each is checked against the current access with Table 2 (P3-P6, then R1-R5), the word-level
// state (Valid, Modified, Atomic / Scope, DevShared / BlkShared, Locks) being the word's as in
// the default check, and the first racy candidate is reported (one report per access, A21).
//
// The ballot scan of k_check4 runs first in "state out" mode and leaves, per sorted access, the
// packed segment state before it (last-writer position, scope of the last atomic, the sticky
// sharing flags; a mark for segment heads).  One thread per access then walks its candidates in
// the sorted array: stores / atomics the previous k accesses of the same segment, loads the
// chain of last writers (the state of the last writer holds the writer before it).  This mode is
// a fidelity instrument, not the timed path: it favours a direct restatement over speed.
#pragma once
#include "check.cuh"
#include "check4.cuh"

namespace lastk {

struct Params {
    check::Params C;
    const u64* st;  // per sorted access: the packed segment state (check.cuh st_make) or ST_HEAD_MARK
    u32 k;          // history depth, 2..8
};

template <bool MV>
__device__ __forceinline__ check::Acc at(const check::Params& P, u32 pos) {
    return check::acc_at<MV>(P.val, pos);
}

// WRAP: Fig. 4-width IDs (A33); STK: sticky sharing flags in P3-P5 (A35); KT: key type.
template <bool WRAP, bool STK, typename KT>
__global__ void __launch_bounds__(256) k_lastk(Params L) {
    const check::Params& P = L.C;
    const u32 x = blockIdx.x * blockDim.x + threadIdx.x;
    if (x >= P.n) return;
    const u64 s = __ldg(L.st + x);
    if (check::st_head(s)) return;  // P1: first access of the word (this kernel)
    const KT* keys = reinterpret_cast<const KT*>(P.key);
    const Geo g = P.g;
    const KeySpace ks = P.ks;
    const check::Acc cur = at<false>(P, x);
    const u32 i = cur.idx, c = cur.tk & 0xFFFFFFu, kind = (cur.tk >> 24) & 0xFu;
    const u32 lastW = check::st_lastW(s), as = check::st_as(s);
    const bool dev = check::st_dev(s), blk = check::st_blk(s);
    if (kind == IGD_LD && lastW == IGD_NONE32) return;  // P2: never written
    const bool isA = kind >= IGD_ATOM && kind <= IGD_EXCH;
    const KT myKey = keys[x];
    // R1's last writer and R5's last accessor are the word's, whatever the candidate
    const u32 bc = g.block(c), wc = g.warp(c);
    const bool r1 = as == IGD_SCOPE_BLOCK && lastW != IGD_NONE32 && g.block(at<false>(P, lastW).tk & 0xFFFFFFu) != bc;
    u32 Lc = 0, locks = 0;
    if (P.lv.any) {
        const check::Acc la = at<false>(P, x - 1);
        if (syncx::may_hold(P.lv, c) || syncx::may_hold(P.lv, la.tk & 0xFFFFFFu))
            syncx::held_before2(P.lv, c, i, la.tk & 0xFFFFFFu, la.idx, Lc, locks);
    }
    u32 mask = 0;
    bool have_mask = false;
    u32 mp = kind == IGD_LD ? lastW : x - 1;
    for (u32 q = 0; q < L.k; q++) {
        if (q > 0) {  // the next older candidate
            if (kind == IGD_LD) {
                const u64 sm = __ldg(L.st + mp);
                mp = check::st_head(sm) ? IGD_NONE32 : check::st_lastW(sm);
            } else {
                mp = mp == 0 ? IGD_NONE32 : mp - 1;
                if (mp != IGD_NONE32 && keys[mp] != myKey) mp = IGD_NONE32;
            }
        }
        if (mp == IGD_NONE32) break;
        const check::Acc md = at<false>(P, mp);
        // a kernel boundary between the candidate and the access ends the word's history (A31)
        if (P.has_kb && check::q_between_inl(P.desc, P.sts, ks.kb, md.idx, i)) break;
        const u32 p = md.tk & 0xFFFFFFu;
        const u32 bp = g.block(p), wp = g.warp(p);
        const bool same_b = bp == bc, same_w = wp == wc;
        const bool unshared = !STK || (!dev && !blk);
        if (p == c && unshared) continue;                                   // P3
        if (as && isA && (same_b || as == IGD_SCOPE_DEVICE)) continue;      // P6
        if (same_w && unshared) {                                           // P4
            bool lockstep;
            if (cur.tk >> 31) lockstep = true;
            else if ((cur.tk >> 30) & 1u) lockstep = false;  // only the issuing lane (p != c)
            else {
                if (!have_mask) {
                    mask = ld_event(P.ev, i).w;
                    have_mask = true;
                }
                lockstep = (mask >> g.lane(p)) & 1u;
            }
            if (lockstep) continue;
        }
        u32 type = 0;
        if (WRAP) {
            const u32 gcnt = P.glo != P.ghi ? check::q_count(P.desc, P.sts, ks.grid, md.idx, i) : 0u;
            if (same_w && unshared && (check::q_count(P.desc, P.sts, ks.wb + wc, md.idx, i) & 63u)) continue;
            if (same_b && (!STK || !dev) && ((check::q_count(P.desc, P.sts, ks.bb + bc, md.idx, i) + gcnt) & 255u))
                continue;
            const u32 dfen = check::q_count(P.desc, P.sts, ks.dev + p, md.idx, i);
            const bool noDev = ((dfen + gcnt) & 63u) == 0;
            const u32 bfen = check::q_count(P.desc, P.sts, ks.any + p, md.idx, i) - dfen;
            const bool noAny = noDev && (bfen & 63u) == 0;
            if (r1) type = IGD_R1;
            else if (same_w && noAny && !dev && !blk) type = IGD_R2;
            else if (same_b && noAny && !dev) type = IGD_R3;
            else if (!same_b && noDev) type = IGD_R4;
        } else {
            if (same_w && unshared && check::q_between(P.desc, P.sts, ks.wb + wc, md.idx, i)) continue;
            const bool grid = check::q_grid(P, md.idx, i);
            if (same_b && (!STK || !dev) && (grid || check::q_between(P.desc, P.sts, ks.bb + bc, md.idx, i))) continue;
            const bool noAny = !grid && !check::q_between(P.desc, P.sts, ks.any + p, md.idx, i);
            const bool noDev = !grid && !check::q_between(P.desc, P.sts, ks.dev + p, md.idx, i);
            if (r1) type = IGD_R1;
            else if (same_w && noAny && !dev && !blk) type = IGD_R2;
            else if (same_b && noAny && !dev) type = IGD_R3;
            else if (!same_b && noDev) type = IGD_R4;
        }
        if (!type && (locks | Lc) != 0 && (locks & Lc) == 0) type = IGD_R5;
        if (type) {
            const unsigned long long slot = atomicAdd(P.rep_ctr, 1ull);
            if (slot < P.rep_cap) {
                igd_report r;
                if (P.addr_from_ev) r.addr = ev_addr(ld_event(P.ev, i)) & ~3ull;
                else if (sizeof(KT) == 8) r.addr = (P.wbase + (u64)myKey) << 2;
                else r.addr = (P.wbase + (u32)((u32)myKey - (u32)P.wbase)) << 2;
                r.cur = P.first_event + i;
                r.prev = P.first_event + md.idx;
                r.type = (uint8_t)type;
                r.cur_kind = (uint8_t)kind;
                r.prev_kind = (uint8_t)((md.tk >> 24) & 0xFu);
                for (int z2 = 0; z2 < 5; z2++) r.pad[z2] = 0;
                P.rep[slot] = r;
            }
            return;
        }
    }
}

}  // namespace lastk
