/*
 * igd_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded CPU oracle of iGUARD's race check (Kamath & Basu,
 * SOSP'21, /root/reference/PAPER.md, cited as P:<line>), restated as a sequential
 * shadow-memory replay of a fixed-order trace (readings A1-A30
 * listed in DESIGN.md "Readings").
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this library.  It shares no code, header, constant or helper with the
 * CUDA path (paper_conf_sosp_kamathb21_b200/csrc): it has its own trace reader, its own
 * kind/scope codes, its own hash constants.
 *
 * Algorithm, in the paper's order (Fig. 6):
 *   synchronization events update the synchronization metadata (Fig. 5),
 *   atomicCAS / atomicExch / fences drive lock inference (§6.3),
 *   every load / store / atomic reads the word's memory metadata, runs the two-tier
 *   check of Table 2 (P1..P6 then R1..R5, §6.4) and writes
 *   the metadata back.
 *
 * Counters are exact u64 (reading A16) instead of the 6/8-bit fields of Fig. 4.
 * Per-word state is exact (no tag aliasing, A18).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- trace encoding, read with the oracle's own reader ---------------- */
enum { O_LD = 0, O_ST = 1, O_ATOM = 2, O_CAS = 3, O_EXCH = 4, O_FENCE = 5, O_SYNCWARP = 6,
       O_SYNCTHREADS = 7, O_GRID = 8, O_CG_TILE = 9, O_CG_BLOCK = 10, O_CG_GRID = 11,
       O_KERNEL = 12 /* kernel boundary (reading A31) */ };
enum { S_NONE = 0, S_BLOCK = 1, S_DEVICE = 2, S_SYSTEM = 3 };
enum { R_NONE = 0, R1 = 1, R2 = 2, R3 = 3, R4 = 4, R5 = 5 };

typedef struct {
    uint64_t addr;
    uint32_t tid, kind, scope, mask;
} o_event;

/* little-endian decode of one 16-byte record: addr u64 | tk u32 | mask u32 */
static int o_read_event(const uint8_t* p, o_event* e) {
    uint64_t addr = 0;
    uint32_t tk = 0, mask = 0;
    for (int b = 0; b < 8; b++) addr |= (uint64_t)p[b] << (8 * b);
    for (int b = 0; b < 4; b++) tk |= (uint32_t)p[8 + b] << (8 * b);
    for (int b = 0; b < 4; b++) mask |= (uint32_t)p[12 + b] << (8 * b);
    e->addr = addr;
    e->tid = tk & 0xFFFFFFu;
    e->kind = (tk >> 24) & 0xFu;
    e->scope = (tk >> 28) & 0x3u;
    e->mask = mask;
    return (tk >> 30) == 0; /* bits 30-31 must be zero */
}

typedef struct {
    uint64_t addr, cur, prev;
    uint8_t type, cur_kind, prev_kind, pad[5];
} o_report; /* 32 bytes, same field meaning as igd_report */

/* ---- thread geometry (C.1) ---------------------------------- */
typedef struct { uint32_t D, Wb, threads, blocks, warps; } o_geom;
static uint32_t g_block(const o_geom* g, uint32_t t) { return t / g->D; }
static uint32_t g_warp(const o_geom* g, uint32_t t) { return (t / g->D) * g->Wb + (t % g->D) / 32; }
static uint32_t g_lane(const o_geom* g, uint32_t t) { return (t % g->D) % 32; }

/* ---- lock tables (Fig. 7; §6.3) ------------------------------ */
typedef struct { uint8_t valid, active, scope; uint32_t h18; } o_lock;
typedef struct { o_lock e[3]; } o_table; /* "up to 3 separate locks" P:1083-1085 */

/* reading A8: 18-bit address hash and the 2-way 16-bit Bloom summary */
static uint32_t o_h18(uint64_t word) { return ((uint32_t)word * 0x9E3779B1u) >> 14; }
static uint16_t o_bloom(uint32_t h) { return (uint16_t)((1u << (h & 15u)) | (1u << ((h >> 4) & 15u))); }

/* activate: "sets the Active bit ... for all entries with matching or narrower scope" P:1076-1077 */
static void o_activate(o_table* T, uint32_t s) {
    for (int k = 0; k < 3; k++)
        if (T->e[k].valid && T->e[k].scope <= s) T->e[k].active = 1;
}
/* held(t): OR of the Bloom bits of valid+active entries */
static uint16_t o_held_of(const o_table* T) {
    uint16_t b = 0;
    for (int k = 0; k < 3; k++)
        if (T->e[k].valid && T->e[k].active) b |= o_bloom(T->e[k].h18);
    return b;
}

/* ---- shadow memory: one exact entry per 4-byte word (Fig. 4) ------------- */
typedef struct {
    uint64_t idx;                 /* trace index of the access */
    uint32_t tid;                 /* full thread id (A19) */
    uint32_t kind;
    uint64_t sDEV, sANY, sWB, sBB; /* counters snapshotted at the access */
} o_rec;

typedef struct {
    uint64_t word;
    uint64_t kernel;              /* kernel (boundaries before it) the entry was written in (A31) */
    uint8_t used;                 /* hash slot occupied */
    uint8_t valid, modified, atomic, ascope, devShared, blkShared;
    uint16_t locks;               /* Bloom of the last accessor's held locks (A7) */
    uint32_t tag;                 /* tag-aliasing mode (A36): the 10-bit Tag of the entry's word */
    o_rec LA, LW;                 /* last accessor, last writer */
    o_rec* hist;                  /* last-k mode (A37): [0,8) accessors, [8,16) writers, newest first */
    uint8_t nla, nlw;             /*   how many of each are held */
} o_shadow;

typedef struct {
    o_shadow* slot;
    uint64_t cap, count;
} o_map;

static uint64_t o_mix(uint64_t x) { /* slot spreading only; not semantic */
    x ^= x >> 33; x *= 0xff51afd7ed558ccdULL; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ULL; x ^= x >> 33;
    return x;
}
static int o_map_grow(o_map* m);
static o_shadow* o_map_get(o_map* m, uint64_t word) {
    if ((m->count + 1) * 4 > m->cap * 3)
        if (!o_map_grow(m)) return NULL;
    uint64_t i = o_mix(word) & (m->cap - 1);
    while (m->slot[i].used && m->slot[i].word != word) i = (i + 1) & (m->cap - 1);
    if (!m->slot[i].used) {
        memset(&m->slot[i], 0, sizeof(o_shadow));
        m->slot[i].used = 1;
        m->slot[i].word = word;
        m->count++;
    }
    return &m->slot[i];
}
static int o_map_grow(o_map* m) {
    uint64_t ncap = m->cap ? m->cap * 2 : 1024;
    o_shadow* ns = (o_shadow*)calloc(ncap, sizeof(o_shadow));
    if (!ns) return 0;
    for (uint64_t i = 0; i < m->cap; i++) {
        if (!m->slot[i].used) continue;
        uint64_t j = o_mix(m->slot[i].word) & (ncap - 1);
        while (ns[j].used) j = (j + 1) & (ncap - 1);
        ns[j] = m->slot[i];
    }
    free(m->slot);
    m->slot = ns;
    m->cap = ncap;
    return 1;
}

/* address shard used by --addr-shard (C.7 5(b)); the hash is not semantic */
static uint32_t o_fmix32(uint32_t h) {
    h ^= h >> 16; h *= 0x85ebca6bu; h ^= h >> 13; h *= 0xc2b2ae35u; h ^= h >> 16;
    return h;
}

/* return codes (same numeric meaning as include/igd.h, restated) */
#define O_OK 0
#define O_EINVAL (-1)
#define O_ETRACE (-2)
#define O_ENOMEM (-4)

/* Reading A34 (per-kernel geometry, "the number of warps per threadblock remains
   constant for a kernel but can vary across kernels"): a KERNEL_BOUNDARY whose addr is
   nonzero carries the next kernel's grid as (n_blocks << 32) | block_dim. */
static int o_geom_code_ok(uint64_t code) {
    uint64_t nb = code >> 32, bd = code & 0xFFFFFFFFu;
    return nb >= 1 && bd >= 1 && nb * bd <= (1u << 24);
}
static void o_geom_set(o_geom* g, uint32_t n_blocks, uint32_t block_dim) {
    g->D = block_dim;
    g->Wb = (block_dim + 31) / 32;
    g->blocks = n_blocks;
    g->threads = n_blocks * block_dim;
    g->warps = n_blocks * g->Wb;
}

/* Field rules per kind. Returns 1 when the event is well-formed. */
static int o_valid(const o_event* e, const o_geom* g) {
    if (e->kind > O_KERNEL) return 0;
    if (e->tid >= g->threads) return 0;
    uint32_t lanebit = 1u << g_lane(g, e->tid);
    switch (e->kind) {
    case O_LD: case O_ST:
        return (e->mask & lanebit) && e->scope == S_NONE;
    case O_ATOM: case O_CAS: case O_EXCH:
        return (e->mask & lanebit) && e->scope != S_NONE;
    case O_FENCE:
        return e->addr == 0 && (e->mask & lanebit) && e->scope != S_NONE;
    case O_SYNCWARP: case O_CG_TILE: case O_SYNCTHREADS: case O_CG_BLOCK:
        return e->addr == 0 && e->scope == S_NONE;
    case O_GRID: case O_CG_GRID:
        return e->addr == 0 && e->scope == S_NONE && e->tid == 0;
    case O_KERNEL: /* addr: 0, or the next kernel's geometry (reading A34) */
        return e->scope == S_NONE && e->tid == 0 && (e->addr == 0 || o_geom_code_ok(e->addr));
    }
    return 0;
}

/*
 * Warp-coalesced check mode (reading A32, §6.5): "if the active threads within a
 * warp are accessing the same location using load or atomic instructions ... only a single
 * thread checks for races ... on behalf of all active threads".  A coalesced group is a run of
 * popcount(mask) >= 2 consecutive events of one warp instruction -- same warp, kind (LD or ATOM;
 * CAS / EXCH are lock operations, and stay per lane), scope, mask and word, lanes
 * strictly ascending -- starting at the mask's lowest lane.  Every member but the first is
 * neither checked nor recorded in the word's shadow entry (Step 3).
 */
static void o_mark_coalesced(const uint8_t* events, uint64_t n, const o_geom* g, uint8_t* skip) {
    for (uint64_t i = 0; i < n; i++) {
        o_event e;
        o_read_event(events + 16 * i, &e);
        if (e.kind != O_LD && e.kind != O_ATOM) continue;
        uint32_t cnt = (uint32_t)__builtin_popcount(e.mask);
        if (cnt < 2 || g_lane(g, e.tid) != (uint32_t)__builtin_ctz(e.mask) || i + cnt > n) continue;
        int ok = 1;
        uint32_t prev_lane = g_lane(g, e.tid);
        for (uint32_t q = 1; q < cnt && ok; q++) {
            o_event f;
            o_read_event(events + 16 * (i + q), &f);
            ok = f.kind == e.kind && f.scope == e.scope && f.mask == e.mask &&
                 g_warp(g, f.tid) == g_warp(g, e.tid) && (f.addr >> 2) == (e.addr >> 2) &&
                 g_lane(g, f.tid) > prev_lane;
            prev_lane = g_lane(g, f.tid);
        }
        if (ok)
            for (uint32_t q = 1; q < cnt; q++) skip[i + q] = 1;
    }
}

/*
 * igdo_run: replay events[0..n) (16-byte records) of one kernel with grid geometry
 * (n_blocks, block_dim).  Only words w with shard(w) == shard_k (of shard_K; K=1 means
 * all) are shadow-checked; all synchronization and lock events are replayed regardless
 * (C.7 5(b)).  Reports are written in ascending `cur` order (A21) to out[0..cap); the
 * total is returned in *n_reports.  On an ill-formed event returns O_ETRACE and its index
 * in *bad_index.
 */
int igdo_run_ex3(const uint8_t* events, uint64_t n, uint32_t n_blocks, uint32_t block_dim,
                 uint32_t shard_k, uint32_t shard_K, uint32_t flags, uint32_t tag_log2, uint32_t hist_k,
                 o_report* out, uint64_t cap, uint64_t* n_reports, uint64_t* bad_index) {
    *n_reports = 0;
    *bad_index = 0;
    if (n_blocks == 0 || block_dim == 0) return O_EINVAL;
    if ((uint64_t)n_blocks * block_dim > (1u << 24)) return O_EINVAL;
    if (shard_K == 0 || shard_k >= shard_K) return O_EINVAL;
    if (tag_log2 != 0 && (tag_log2 < 8 || tag_log2 > 22)) return O_EINVAL;
    if (hist_k != 1 && hist_k != 2 && hist_k != 4 && hist_k != 8) return O_EINVAL;
    const int sticky = (flags & 4u) != 0; /* A35: literal sticky sharing flags in P3-P5 */

    o_geom g;
    o_geom_set(&g, n_blocks, block_dim);

    /* validate everything first (the oracle applies the 8(b) rules independently), each event
       against the geometry of its own kernel (A34) */
    for (uint64_t i = 0; i < n; i++) {
        o_event e;
        int ok = o_read_event(events + 16 * i, &e);
        if (!ok || !o_valid(&e, &g)) { *bad_index = i; return O_ETRACE; }
        if (e.kind == O_KERNEL && e.addr != 0) o_geom_set(&g, (uint32_t)(e.addr >> 32), (uint32_t)e.addr);
    }
    o_geom_set(&g, n_blocks, block_dim);

    /* C.2 synchronization state: exact, unbounded counters.  Sized for the largest grid of the
       trace (A34: a kernel boundary may change the geometry) */
    uint64_t maxT = g.threads, maxW = g.warps, maxB = g.blocks;
    for (uint64_t i = 0; i < n; i++) {
        o_event e;
        o_read_event(events + 16 * i, &e);
        if (e.kind == O_KERNEL && e.addr != 0) {
            o_geom h;
            o_geom_set(&h, (uint32_t)(e.addr >> 32), (uint32_t)e.addr);
            if (h.threads > maxT) maxT = h.threads;
            if (h.warps > maxW) maxW = h.warps;
            if (h.blocks > maxB) maxB = h.blocks;
        }
    }
    uint64_t* devF = (uint64_t*)calloc(maxT, sizeof(uint64_t));
    uint64_t* anyF = (uint64_t*)calloc(maxT, sizeof(uint64_t));
    uint64_t* wbar = (uint64_t*)calloc(maxW, sizeof(uint64_t));
    uint64_t* bbar = (uint64_t*)calloc(maxB, sizeof(uint64_t));
    uint64_t G = 0;
    uint64_t kernel = 0; /* kernel boundaries so far (A31) */
    o_table* wt = (o_table*)calloc(maxW, sizeof(o_table));
    o_table* tt = (o_table*)calloc(maxT, sizeof(o_table));
    uint8_t* isThread = (uint8_t*)calloc(maxW, 1);
    uint8_t* touched = (uint8_t*)calloc(maxW, 1); /* warps whose tables were ever filled */
    uint32_t* touched_list = (uint32_t*)calloc(maxW, sizeof(uint32_t));
    uint32_t n_touched = 0;
    o_map map = {0, 0, 0};
    uint8_t* skip = (flags & 1u) ? (uint8_t*)calloc(n ? n : 1, 1) : NULL; /* A32 coalesced members */
    const int wrap = (flags & 2u) != 0; /* A33: paper-width synchronization IDs */
    int rc = O_OK;
    if (!devF || !anyF || !wbar || !bbar || !wt || !tt || !isThread || !touched || !touched_list ||
        ((flags & 1u) && !skip)) {
        rc = O_ENOMEM;
        goto done;
    }
    if (skip) o_mark_coalesced(events, n, &g, skip);

#define DEV(t) (devF[t] + G)
#define ANY(t) (anyF[t] + G)
#define WB(w) (wbar[w])
#define BB(b) (bbar[b] + G)
#define TABLE(t) (isThread[g_warp(&g, t)] ? &tt[t] : &wt[g_warp(&g, t)])

    for (uint64_t i = 0; i < n; i++) {
        o_event e;
        o_read_event(events + 16 * i, &e);
        uint32_t k = e.kind, c = e.tid;
        uint32_t s = (e.scope == S_SYSTEM) ? S_DEVICE : e.scope; /* A12: SYSTEM == DEVICE */
        /* CG syncs are their constituents (A15) */
        if (k == O_CG_TILE) k = O_SYNCWARP;
        if (k == O_CG_BLOCK) k = O_SYNCTHREADS;
        if (k == O_CG_GRID) k = O_GRID;

        /* ---- Step 1: synchronization metadata (Fig. 5) ---- */
        if (k == O_FENCE) {
            if (s >= S_DEVICE) devF[c]++;  /* DevFenceId (Fig. 5b) */
            anyF[c]++;                     /* any fence changes DevFenceID or BlkFenceID */
            o_activate(TABLE(c), s);       /* activateLocks(scope) P:1076-1077 */
            continue;
        }
        if (k == O_SYNCWARP) { wbar[g_warp(&g, c)]++; continue; } /* A14: mask ignored */
        if (k == O_SYNCTHREADS) { bbar[g_block(&g, c)]++; continue; } /* Fig. 5a; A13 */
        if (k == O_GRID) {
            /* A15: a device fence by every thread (incl. lock activation) + a barrier for
               every block; implemented through the G term of DEV/ANY/BB */
            G++;
            for (uint32_t q = 0; q < n_touched; q++) {
                uint32_t w = touched_list[q];
                o_activate(&wt[w], S_DEVICE);
                uint32_t b = w / g.Wb, wi = w % g.Wb;
                for (uint32_t l = 0; l < 32; l++) {
                    uint32_t off = wi * 32 + l;
                    if (off >= g.D) break;
                    o_activate(&tt[b * g.D + off], S_DEVICE);
                }
            }
            continue;
        }

        if (k == O_KERNEL) {
            /* A31: the kernel ends.  Its implicit all-thread barrier orders
               every access before it before every access after it: every word's shadow entry
               is discarded (lazily, by kernel number), and the next kernel's locking protocol
               is inferred afresh: lock tables and isThread bits reset. */
            kernel++;
            for (uint32_t q = 0; q < n_touched; q++) {
                uint32_t w = touched_list[q];
                memset(&wt[w], 0, sizeof(o_table));
                isThread[w] = 0;
                touched[w] = 0;
                uint32_t b = w / g.Wb, wi = w % g.Wb;
                for (uint32_t l = 0; l < 32; l++) {
                    uint32_t off = wi * 32 + l;
                    if (off >= g.D) break;
                    memset(&tt[b * g.D + off], 0, sizeof(o_table));
                }
            }
            n_touched = 0;
            if (e.addr != 0) {
                /* A34: the next kernel runs on another grid.  Every shadow entry is discarded
                   (above, by kernel number) and no counter snapshot survives the boundary, so
                   the synchronization counters restart with the new thread / warp / block ids */
                o_geom_set(&g, (uint32_t)(e.addr >> 32), (uint32_t)e.addr);
                memset(devF, 0, maxT * sizeof(uint64_t));
                memset(anyF, 0, maxT * sizeof(uint64_t));
                memset(wbar, 0, maxW * sizeof(uint64_t));
                memset(bbar, 0, maxB * sizeof(uint64_t));
                G = 0;
            }
            continue;
        }

        /* ---- Step 3: an access (LD/ST/ATOM/CAS/EXCH) ---- */
        int isWrite = (k != O_LD);                                /* atomics are stores */
        int isAtomic = (k == O_ATOM || k == O_CAS || k == O_EXCH);
        uint64_t word = e.addr >> 2;                              /* 4-byte granularity */
        uint32_t w_c = g_warp(&g, c), b_c = g_block(&g, c);
        uint16_t L = o_held_of(TABLE(c));                        /* 3.1: before own update (A11) */

        /* A36 tag aliasing: the metadata entry of `word` is word mod 2^tag_log2, and the entry's
           10-bit Tag (Fig. 4) is the next 10 bits of the word */
        uint64_t mkey = tag_log2 ? (word & ((1ull << tag_log2) - 1)) : word;
        uint32_t tag = tag_log2 ? (uint32_t)((word >> tag_log2) & 1023u) : 0;
        int owned = (shard_K == 1) || ((o_fmix32((uint32_t)mkey ^ (uint32_t)(mkey >> 32)) % shard_K) == shard_k);
        if (skip && skip[i]) owned = 0; /* A32: checked by its group's first lane */
        if (owned) {
            o_shadow* S = o_map_get(&map, mkey);
            if (!S) { rc = O_ENOMEM; goto done; }
            if (S->valid && (S->kernel != kernel || S->tag != tag)) {
                /* A31: from an earlier kernel; A36: the entry belongs to another word (Tag
                   mismatch) -- the access claims it as a fresh entry */
                uint64_t wd = S->word;
                o_rec* hh = S->hist;
                memset(S, 0, sizeof(*S));
                S->used = 1;
                S->word = wd;
                S->hist = hh;
            }
            if (hist_k > 1 && !S->hist) {
                S->hist = (o_rec*)calloc(16, sizeof(o_rec));
                if (!S->hist) { rc = O_ENOMEM; goto done; }
            }
            if (!S->valid) goto writeback;                        /* P1: first access (this kernel) */

            /* sharing flags vs the last accessor, sticky (A5) */
            {
                uint32_t la = S->LA.tid;
                if (g_block(&g, la) != b_c) S->devShared = 1;
                else if (g_warp(&g, la) != w_c) S->blkShared = 1;
            }
            if (k == O_LD && !S->modified) goto writeback;        /* P2: no write (A25) */

            /* A37 last-k histories (§6.7): the candidates md_1..md_K are the last K
               writers (loads) or accessors (stores, atomics), newest first; each is checked in
               turn and the first racy one is reported.  K = 1 is Table 2 as written. */
            const o_rec* cands[8];
            int ncand = 1;
            cands[0] = (k == O_LD) ? &S->LW : &S->LA; /* Table 2 definitions */
            if (hist_k > 1) {
                int have = (k == O_LD) ? S->nlw : S->nla;
                ncand = have < (int)hist_k ? have : (int)hist_k;
                for (int q = 0; q < ncand; q++) cands[q] = &S->hist[(k == O_LD ? 8 : 0) + q];
            }
            for (int cq = 0; cq < ncand; cq++) {
                const o_rec* md = cands[cq];
                uint32_t p = md->tid;
                uint32_t w_p = g_warp(&g, p), b_p = g_block(&g, p);
                /* preliminary checks (reading A4: md.* = relation between md and curr) */
                int P3 = (p == c);
                int P4, P5, noAny, noDev;
                if (!wrap) {
                    P4 = (w_p == w_c) && (WB(w_c) != md->sWB || (e.mask >> g_lane(&g, p)) & 1u);
                    P5 = (b_p == b_c) && (BB(b_c) != md->sBB);
                    noAny = (ANY(p) == md->sANY); /* A1: md's thread has not fenced since */
                    noDev = (DEV(p) == md->sDEV);
                } else {
                    /* A33: the IDs have Fig. 4's widths -- WarpBarID 6, BlkBarID 8, DevFenceID 6,
                       BlkFenceID 6 bits -- so "unchanged" means a multiple of 2^width events */
                    uint64_t dWB = WB(w_c) - md->sWB, dBB = BB(b_c) - md->sBB;
                    uint64_t dDev = DEV(p) - md->sDEV;
                    uint64_t dBlk = (ANY(p) - DEV(p)) - (md->sANY - md->sDEV); /* block-scope fences */
                    P4 = (w_p == w_c) && ((dWB & 63u) != 0 || (e.mask >> g_lane(&g, p)) & 1u);
                    P5 = (b_p == b_c) && ((dBB & 255u) != 0);
                    noDev = (dDev & 63u) == 0;
                    noAny = noDev && (dBlk & 63u) == 0;
                }
                if (sticky) {
                    /* A35 literal reading: Table 2 gates P3 and P4 on !DevShared AND !BlkShared
                       and P5 on !DevShared, taken as the word's sticky flags */
                    if (S->devShared || S->blkShared) { P3 = 0; P4 = 0; }
                    if (S->devShared) P5 = 0;
                }
                int P6 = S->atomic && isAtomic && (b_p == b_c || S->ascope == S_DEVICE);
                if (P3 || P4 || P5 || P6) continue;

                /* race checks in order; first true is reported */
                int type = R_NONE;
                if (S->atomic && S->ascope == S_BLOCK && g_block(&g, S->LW.tid) != b_c) type = R1;
                else if (w_p == w_c && noAny && !S->devShared && !S->blkShared) type = R2;
                else if (b_p == b_c && noAny && !S->devShared) type = R3;
                else if (b_p != b_c && noDev) type = R4;
                else if ((S->locks | L) != 0 && (S->locks & L) == 0) type = R5; /* A3, A7 */
                if (type != R_NONE) {
                    if (*n_reports < cap) {
                        o_report* r = &out[*n_reports];
                        memset(r, 0, sizeof(*r));
                        r->addr = word << 2;
                        r->cur = i;
                        r->prev = md->idx;
                        r->type = (uint8_t)type;
                        r->cur_kind = (uint8_t)e.kind;
                        r->prev_kind = (uint8_t)md->kind;
                    }
                    (*n_reports)++;
                    break; /* at most one report per access (A21) */
                }
            }
        writeback: /* Fig. 6 "Race -> Writeback": always done (A11) */
            {
                o_rec r;
                r.idx = i; r.tid = c; r.kind = e.kind;
                r.sDEV = DEV(c); r.sANY = ANY(c); r.sWB = WB(w_c); r.sBB = BB(b_c);
                S->valid = 1;
                S->kernel = kernel;
                S->tag = tag;
                S->LA = r;
                S->locks = L;
                if (isWrite) { S->modified = 1; S->LW = r; }
                if (S->hist) { /* A37: push the record onto the histories */
                    memmove(&S->hist[1], &S->hist[0], 7 * sizeof(o_rec));
                    S->hist[0] = r;
                    if (S->nla < 8) S->nla++;
                    if (isWrite) {
                        memmove(&S->hist[9], &S->hist[8], 7 * sizeof(o_rec));
                        S->hist[8] = r;
                        if (S->nlw < 8) S->nlw++;
                    }
                }
                if (isAtomic) { S->atomic = 1; S->ascope = (uint8_t)s; }
            }
        }

        /* ---- Step 4: lock-table update for CAS / EXCH, after the check (A9-A11) ---- */
        if (k == O_CAS || k == O_EXCH) {
            uint32_t h = o_h18(word);
            if (k == O_CAS) {
                /* isThread: more than one lane executes the CAS together */
                if (!isThread[w_c] && __builtin_popcount(e.mask) > 1) isThread[w_c] = 1;
                if (!touched[w_c]) { touched[w_c] = 1; touched_list[n_touched++] = w_c; }
                o_table* T = TABLE(c);
                /* "up to 3 separate locks": a CAS on a lock already in the table
                   (same hash and scope, e.g. the retries of a spin loop) adds nothing (A9) */
                int present = 0;
                for (int q = 0; q < 3; q++)
                    if (T->e[q].valid && T->e[q].h18 == h && T->e[q].scope == s) present = 1;
                int slot = -1; /* the lowest free slot */
                for (int q = 2; q >= 0; q--)
                    if (!T->e[q].valid) slot = q;
                if (slot < 0) present = 1; /* full table: the insert is dropped (A9) */
                if (!present) {
                    T->e[slot].valid = 1; T->e[slot].active = 0;
                    T->e[slot].scope = (uint8_t)s; T->e[slot].h18 = h;
                }
            } else {
                /* atomicExch unsets Valid of entries matching hash and scope */
                o_table* T = TABLE(c);
                for (int q = 0; q < 3; q++)
                    if (T->e[q].valid && T->e[q].h18 == h && T->e[q].scope == s) {
                        T->e[q].valid = 0; T->e[q].active = 0;
                    }
            }
        }
    }

done:
    for (uint64_t q = 0; q < map.cap; q++)
        if (map.slot[q].used) free(map.slot[q].hist);
    free(devF); free(anyF); free(wbar); free(bbar); free(wt); free(tt);
    free(isThread); free(touched); free(touched_list); free(map.slot); free(skip);
    return rc;
}

int igdo_run_ex(const uint8_t* events, uint64_t n, uint32_t n_blocks, uint32_t block_dim,
                uint32_t shard_k, uint32_t shard_K, uint32_t flags, o_report* out, uint64_t cap,
                uint64_t* n_reports, uint64_t* bad_index) {
    return igdo_run_ex3(events, n, n_blocks, block_dim, shard_k, shard_K, flags, 0, 1, out, cap, n_reports,
                        bad_index);
}

int igdo_run(const uint8_t* events, uint64_t n, uint32_t n_blocks, uint32_t block_dim,
             uint32_t shard_k, uint32_t shard_K, o_report* out, uint64_t cap,
             uint64_t* n_reports, uint64_t* bad_index) {
    return igdo_run_ex(events, n, n_blocks, block_dim, shard_k, shard_K, 0, out, cap, n_reports, bad_index);
}

/* Test hook (reading A8): the 18-bit lock hash of a word and its 16-bit Bloom summary, so
   tests can pin what the paper fixes -- an 18-bit hash and a 16-bit summary with two
   hash functions, "2-way bloom filter". */
void igdo_lock_hash(uint64_t word, uint32_t* h18, uint32_t* bloom) {
    *h18 = o_h18(word);
    *bloom = o_bloom(*h18);
}

/* Exported constants so the Python side can check it loaded this library. */
int igdo_version(void) { return 2; }
