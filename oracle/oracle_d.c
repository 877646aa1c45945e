/*
 * ORACLE-D: a plain, slow, single-threaded CPU implementation of the data-race DEFINITION.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py (its
 * cpu_baseline leg and `--impl reference`) may load or call this file.  It shares no code,
 * header, table or constant generator with the CUDA path (paper_conf_sc_jacobsonbg24_b200/):
 * it does NOT run the HiRace state machine; it evaluates the happens-before race definition
 * directly, so it can judge the state machine.
 *
 * What it computes:
 *   C1.1  events e = (key, tid, kind, g, b, w); block = tid / blockDim,
 *         warp = (tid mod blockDim) / warpSize                         PAPER.md L164 (T_bwt), L259
 *         key: global -> word index; shared -> 1<<63 | block<<32 | word (shared memory is per
 *         block); 8/16-byte accesses cover 2/4 words, sub-word accesses their
 *         containing word (per-element shadow; reading R8).  With
 *         element size 1 << gran_log2 < 4 (oracle_races_gran) "word" reads "element".
 *   C1.2  Concurrent(e1,e2) <=> tid1 != tid2 and g1 == g2 and
 *         [block1 != block2 or (b1 == b2 and (warp1 != warp2 or w1 == w2))]
 *         (barrier semantics PAPER.md L122, L211-213; grid epoch PAPER.md L221, reading R4)
 *   C1.3  Conflict: R-R never; atomic-atomic only if not both grid-scope and the two threads
 *         are in different blocks; every other pair (incl. plain read vs atomic) conflicts
 *         ("at least one of the accesses is a write", L223-229; readings R2, R3)
 *         policy 1 (RELAXED_READ_ATOMIC, reading R2b): a pair
 *         conflicts iff one is a write, or both are atomics of different blocks and not both
 *         grid-scope (a plain read never conflicts with an atomic)
 *   C1.4  racing pair = Concurrent and Conflict; level GRID / BLOCK / WARP
 *   C1.5  a key is flagged iff it has a racing pair
 *   C1.6  class: g* = smallest g with a racing pair; GRID if a racing pair of g* is GRID-level;
 *         otherwise b* = smallest b with a racing pair in g*, BLOCK if a racing pair in
 *         (g*, b*) is BLOCK-level, else WARP                                 (reading R6)
 *
 * Algorithm (C2): expand words, qsort by (key, g, block, b, warp, w, tid), then for every
 * (key, g) test the three levels with per-group kind masks.  A level has a racing pair iff
 * two DISTINCT groups (blocks / warps of one (block,b) / threads of one (block,b,warp,w))
 * hold a conflicting pair of kinds: concurrency at each level is exactly "different group
 * inside the same enclosing epoch" (C1.2), and conflict depends only on the two kinds and
 * on whether the blocks are equal (C1.3).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint64_t addr;
    uint32_t tid;
    uint32_t meta;
} oracle_event; /* the 16-byte trace record produced by tracegen */

typedef struct {
    uint64_t key;
    uint32_t g, block, b, warp, w, tid, kind;
} access_t;

enum { K_READ = 0, K_WRITE = 1, K_ATOMIC_BLOCK = 2, K_ATOMIC_GRID = 3 };
enum { CLS_NONE = 0, CLS_WARP = 1, CLS_BLOCK = 2, CLS_GRID = 3 };

static const uint64_t SHARED = 1ull << 63;

static int is_atomic(uint32_t k) { return k == K_ATOMIC_BLOCK || k == K_ATOMIC_GRID; }

/* C1.3 */
static int conflict(uint32_t k1, uint32_t k2, int same_block, int policy)
{
    if (policy == 1 && (k1 == K_READ || k2 == K_READ) && k1 != K_WRITE && k2 != K_WRITE)
        return 0; /* read vs read or read vs atomic */
    if (k1 == K_READ && k2 == K_READ)
        return 0;
    if (is_atomic(k1) && is_atomic(k2)) {
        if (k1 == K_ATOMIC_GRID && k2 == K_ATOMIC_GRID)
            return 0;
        if (same_block)
            return 0;
        return 1;
    }
    return 1;
}

/* exists i != j with kind k1 in masks[i], kind k2 in masks[j], conflict(k1,k2) */
static int distinct_conflict(const uint8_t *masks, size_t n, int same_block, int policy)
{
    for (uint32_t k1 = 0; k1 < 4; k1++) {
        for (uint32_t k2 = 0; k2 < 4; k2++) {
            if (!conflict(k1, k2, same_block, policy))
                continue;
            size_t c1 = 0, c2 = 0, f1 = 0, f2 = 0;
            for (size_t i = 0; i < n; i++) {
                if ((masks[i] >> k1) & 1) {
                    if (c1 == 0)
                        f1 = i;
                    c1++;
                }
                if ((masks[i] >> k2) & 1) {
                    if (c2 == 0)
                        f2 = i;
                    c2++;
                }
            }
            if (c1 >= 1 && c2 >= 1 && !(c1 == 1 && c2 == 1 && f1 == f2))
                return 1;
        }
    }
    return 0;
}

static int cmp_access(const void *pa, const void *pb)
{
    const access_t *a = (const access_t *)pa, *b = (const access_t *)pb;
#define CMP(f)                  \
    if (a->f != b->f)           \
        return a->f < b->f ? -1 : 1;
    CMP(key) CMP(g) CMP(block) CMP(b) CMP(warp) CMP(w) CMP(tid)
#undef CMP
    return 0;
}

/* Growable scratch array of group masks. */
typedef struct {
    uint8_t *m;
    size_t n, cap;
} masks_t;

static int masks_push(masks_t *s, uint8_t v)
{
    if (s->n == s->cap) {
        size_t nc = s->cap ? 2 * s->cap : 64;
        uint8_t *p = (uint8_t *)realloc(s->m, nc);
        if (!p)
            return -1;
        s->m = p;
        s->cap = nc;
    }
    s->m[s->n++] = v;
    return 0;
}

/*
 * Returns the number of flagged keys (>= 0; only the first `cap` are written, in increasing
 * key order), or a negative error: -1 bad argument / out of memory, -2 the definition's
 * C1.6 premise failed (no GRID pair although >= 2 blocks touched the key in g*; cannot happen
 * by C1.2/C1.3 and is reported so a test can pin it).
 * out_g receives g* (the grid epoch of the first racing pair).
 */
/*
 * ---------------------------------------------------------------------------------------------
 * Partial-mask warp synchronisation ("masked warp
 * synchronization primitives may be used to implement non-hierarchical barrier points";
 * DESIGN.md reading R20).
 *
 *   C1.1''  Inside one block epoch (g, b) a warp's synchronisations -- full-mask __syncwarp /
 *           votes and partial __syncwarp(mask) -- are numbered 1, 2, ... in a linear order that
 *           respects every lane's program order.  An access's w is the number of the last sync
 *           its lane passed (0 = none).  The log lists the partial syncs (warp = block *
 *           warps_per_block + warp, mask over lanes, g, b, w); unlisted numbers are full-mask.
 *   C1.2''  Two accesses of different lanes of one warp in one (g, b), w1 <= w2:
 *           e1 happens before e2  <=>  w1 < w2 and a chain of syncs s_1 < ... < s_m exists with
 *           w1 < s_1, s_m <= w2, lane1 in M(s_1), lane2 in M(s_m), and consecutive syncs of the
 *           chain sharing a lane (M(s_k) & M(s_k+1) != 0) -- the transitive closure of program
 *           order and sync rendezvous.  Concurrent <=> not ordered.  Evaluated literally: the set
 *           of lanes that know of e1 starts as {lane1} and absorbs M(s) for every s in
 *           (w1, w2] whose mask meets it.  With only full masks this is "w1 == w2" (C1.2).
 *   Everything else (other warps, blocks, epochs, conflict, class) is C1.2-C1.6 unchanged.
 * ---------------------------------------------------------------------------------------------
 */
typedef struct {
    uint32_t warp, mask, meta, pad;
} oracle_sync; /* tracegen.SYNC_DTYPE; meta = w:9 << 5 | b:10 << 14 | g:8 << 24 */

static uint64_t sync_key(uint32_t g, uint32_t b, uint32_t warp)
{
    return ((uint64_t)g << 50) | ((uint64_t)b << 40) | warp;
}
static uint64_t sync_key_of(const oracle_sync *s)
{
    return sync_key((s->meta >> 24) & 255, (s->meta >> 14) & 1023, s->warp);
}

/* the log entries of warp `warp` in (g, b): [*lo, *hi) of the sorted log */
static void sync_family(const oracle_sync *sy, uint64_t nsync, uint32_t g, uint32_t b, uint32_t warp, uint64_t *lo,
                        uint64_t *hi)
{
    const uint64_t k = sync_key(g, b, warp);
    uint64_t a = 0, z = nsync;
    while (a < z) {
        uint64_t m = (a + z) / 2;
        if (sync_key_of(&sy[m]) < k)
            a = m + 1;
        else
            z = m;
    }
    *lo = a;
    while (a < nsync && sync_key_of(&sy[a]) == k)
        a++;
    *hi = a;
}

/* M(s): the listed mask of sync number s, or all lanes (unlisted = full-mask sync) */
static uint32_t sync_mask(const oracle_sync *f, uint64_t nf, uint32_t s, int *listed)
{
    for (uint64_t i = 0; i < nf; i++)
        if (((f[i].meta >> 5) & 511) == s) {
            *listed = 1;
            return f[i].mask;
        }
    *listed = 0;
    return 0xffffffffu;
}

/* C1.2'': does the access of lane i after sync w1 happen before the access of lane j after
 * sync w2 (w1 < w2)? */
static int masked_ordered(const oracle_sync *f, uint64_t nf, uint32_t i, uint32_t w1, uint32_t j, uint32_t w2)
{
    uint32_t know = 1u << i;
    for (uint32_t s = w1 + 1; s <= w2; s++) {
        int listed;
        const uint32_t m = sync_mask(f, nf, s, &listed);
        if (m & know)
            know |= m;
    }
    return (know >> j) & 1u;
}

/* WARP level of one (key, g, block, b, warp) group with a partial-sync log: a conflicting
 * concurrent pair of accesses of different threads?  acc[0..m) sorted by (w, tid).  Returns 1 /
 * 0, or -4 when an access claims a partial sync its lane is not in. */
static int masked_warp_race(const access_t *acc, uint64_t m, const oracle_sync *f, uint64_t nf, uint32_t block_threads,
                            uint32_t warp_size, int policy)
{
    for (uint64_t x = 0; x < m; x++) {
        const uint32_t lx = (acc[x].tid % block_threads) % warp_size;
        int listed;
        const uint32_t mx = acc[x].w ? sync_mask(f, nf, acc[x].w, &listed) : 0xffffffffu;
        if (!((mx >> lx) & 1u))
            return -4;
    }
    for (uint64_t x = 0; x < m; x++)
        for (uint64_t y = x + 1; y < m; y++) {
            if (acc[x].tid == acc[y].tid || !conflict(acc[x].kind, acc[y].kind, 1, policy))
                continue;
            const uint32_t lx = (acc[x].tid % block_threads) % warp_size;
            const uint32_t ly = (acc[y].tid % block_threads) % warp_size;
            if (acc[x].w == acc[y].w || !masked_ordered(f, nf, lx, acc[x].w, ly, acc[y].w))
                return 1;
        }
    return 0;
}

static int64_t races_core(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                          uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap, int policy,
                          uint32_t gran_log2, const oracle_sync *sy, uint64_t nsync)
{
    if (policy != 0 && policy != 1)
        return -1;
    if (block_threads == 0 || warp_size == 0 || (n && !ev) || gran_log2 > 2 || (nsync && !sy))
        return -1;
    if (nsync && (warp_size > 32 || gran_log2 != 2))
        return -1;
    for (uint64_t i = 0; i < nsync; i++) { /* C1.1'': a sorted log of real partial syncs */
        const uint32_t w = (sy[i].meta >> 5) & 511;
        if (w == 0 || sy[i].mask == 0 || (warp_size < 32 && (sy[i].mask >> warp_size)) || (sy[i].meta & 31))
            return -4;
        if (i && !(sync_key_of(&sy[i - 1]) < sync_key_of(&sy[i]) ||
                   (sync_key_of(&sy[i - 1]) == sync_key_of(&sy[i]) && ((sy[i - 1].meta >> 5) & 511) < w)))
            return -4;
    }
    const uint32_t wpb = (block_threads + warp_size - 1) / warp_size;
    /* C1.1: expand to element-level accesses; an element ("granule") is 1 << gran_log2 bytes
     * (per-element shadow; reading R8: 4-byte words by default, bytes
     * or half-words for arrays of such elements) */
    const uint32_t granule = 1u << gran_log2;
    uint64_t nacc = 0;
    for (uint64_t i = 0; i < n; i++) {
        uint32_t sz = 1u << ((ev[i].meta >> 2) & 7);
        nacc += sz <= granule ? 1 : sz / granule;
    }
    access_t *acc = (access_t *)malloc((nacc ? nacc : 1) * sizeof(access_t));
    if (!acc)
        return -1;
    uint64_t j = 0;
    for (uint64_t i = 0; i < n; i++) {
        uint32_t meta = ev[i].meta;
        uint32_t kind = meta & 3, sz = 1u << ((meta >> 2) & 7);
        uint32_t w = (meta >> 5) & 511, b = (meta >> 14) & 1023, g = (meta >> 24) & 255;
        uint32_t tid = ev[i].tid;
        uint32_t block = tid / block_threads;
        uint32_t warp = (tid % block_threads) / warp_size;
        int shared = (ev[i].addr & SHARED) != 0;
        uint64_t word0 = (ev[i].addr & ~SHARED) >> gran_log2;
        uint32_t nw = sz <= granule ? 1 : sz / granule;
        for (uint32_t k = 0; k < nw; k++) {
            access_t *a = &acc[j++];
            uint64_t word = word0 + k;
            a->key = shared ? (SHARED | ((uint64_t)block << 32) | (word & 0xffffffffull)) : word;
            a->g = g;
            a->block = block;
            a->b = b;
            a->warp = warp;
            a->w = w;
            a->tid = tid;
            a->kind = kind;
        }
    }
    /* C2.2 */
    qsort(acc, nacc, sizeof(access_t), cmp_access);

    masks_t blocks = {0}, warps = {0}, threads = {0};
    int64_t nflag = 0;
    int err = 0;
    uint64_t i = 0;
    while (i < nacc && !err) {
        uint64_t key = acc[i].key, kend = i;
        while (kend < nacc && acc[kend].key == key)
            kend++;
        int cls = CLS_NONE;
        uint32_t gstar = 0;
        /* C2.3: each grid epoch of this key, in increasing g */
        for (uint64_t gs = i; gs < kend && cls == CLS_NONE;) {
            uint32_t g = acc[gs].g;
            uint64_t ge = gs;
            while (ge < kend && acc[ge].g == g)
                ge++;
            /* GRID level: groups = blocks */
            blocks.n = 0;
            int has_block_race_at_min_b = 0, have_min_b = 0;
            uint32_t min_b = 0;
            for (uint64_t bs = gs; bs < ge;) {
                uint32_t blk = acc[bs].block;
                uint64_t be = bs;
                uint8_t bmask = 0;
                while (be < ge && acc[be].block == blk)
                    bmask |= (uint8_t)(1u << acc[be].kind), be++;
                if (masks_push(&blocks, bmask))
                    err = -1;
                /* per block epoch b of this block */
                for (uint64_t es = bs; es < be;) {
                    uint32_t b = acc[es].b;
                    uint64_t ee = es;
                    while (ee < be && acc[ee].b == b)
                        ee++;
                    /* BLOCK level: groups = warps of (block, b) */
                    warps.n = 0;
                    int warp_race = 0;
                    for (uint64_t ws = es; ws < ee;) {
                        uint32_t wp = acc[ws].warp;
                        uint64_t we = ws;
                        uint8_t wmask = 0;
                        while (we < ee && acc[we].warp == wp)
                            wmask |= (uint8_t)(1u << acc[we].kind), we++;
                        if (masks_push(&warps, wmask))
                            err = -1;
                        /* WARP level: groups = threads of (block, b, warp, w); with partial
                         * syncs in this (g, b) of this warp, the pairs of C1.2'' */
                        uint64_t flo = 0, fhi = 0;
                        if (nsync)
                            sync_family(sy, nsync, g, b, blk * wpb + wp, &flo, &fhi);
                        if (fhi > flo) {
                            const int r = masked_warp_race(acc + ws, we - ws, sy + flo, fhi - flo, block_threads,
                                                           warp_size, policy);
                            if (r < 0)
                                err = r;
                            else if (r)
                                warp_race = 1;
                        }
                        for (uint64_t xs = ws; fhi == flo && xs < we;) {
                            uint32_t w = acc[xs].w;
                            uint64_t xe = xs;
                            while (xe < we && acc[xe].w == w)
                                xe++;
                            threads.n = 0;
                            for (uint64_t ts = xs; ts < xe;) {
                                uint32_t t = acc[ts].tid;
                                uint8_t tmask = 0;
                                while (ts < xe && acc[ts].tid == t)
                                    tmask |= (uint8_t)(1u << acc[ts].kind), ts++;
                                if (masks_push(&threads, tmask))
                                    err = -1;
                            }
                            if (distinct_conflict(threads.m, threads.n, 1, policy))
                                warp_race = 1;
                            xs = xe;
                        }
                        ws = we;
                    }
                    int block_race = distinct_conflict(warps.m, warps.n, 1, policy);
                    if ((block_race || warp_race) && (!have_min_b || b < min_b)) {
                        have_min_b = 1;
                        min_b = b;
                        has_block_race_at_min_b = block_race;
                    } else if ((block_race || warp_race) && have_min_b && b == min_b && block_race) {
                        has_block_race_at_min_b = 1;
                    }
                    es = ee;
                }
                bs = be;
            }
            int grid_race = distinct_conflict(blocks.m, blocks.n, 0, policy);
            if (grid_race) {
                cls = CLS_GRID;
            } else if (have_min_b) {
                if (blocks.n >= 2)
                    err = -2; /* C1.6 premise: only one block can touch the key in g* */
                cls = has_block_race_at_min_b ? CLS_BLOCK : CLS_WARP;
            }
            gstar = g;
            gs = ge;
        }
        if (cls != CLS_NONE) {
            if ((uint64_t)nflag < cap) {
                if (out_key)
                    out_key[nflag] = key;
                if (out_cls)
                    out_cls[nflag] = (uint8_t)cls;
                if (out_g)
                    out_g[nflag] = (uint8_t)gstar;
            }
            nflag++;
        }
        i = kend;
    }
    free(blocks.m);
    free(warps.m);
    free(threads.m);
    free(acc);
    return err ? err : nflag;
}

int64_t oracle_races_gran(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                          uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap, int policy,
                          uint32_t gran_log2)
{
    return races_core(ev, n, block_threads, warp_size, out_key, out_cls, out_g, cap, policy, gran_log2, NULL, 0);
}

/* C1 with the partial-mask warp syncs of C1.1''/C1.2'' (4-byte words).  Returns as
 * oracle_races_gran, plus -4: malformed log, or an access after a partial sync its lane is not
 * in. */
int64_t oracle_races_masked(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                            const oracle_sync *syncs, uint64_t nsync, uint64_t *out_key, uint8_t *out_cls,
                            uint8_t *out_g, uint64_t cap, int policy)
{
    return races_core(ev, n, block_threads, warp_size, out_key, out_cls, out_g, cap, policy, 2, syncs, nsync);
}

int64_t oracle_races_policy(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                            uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap, int policy)
{
    return oracle_races_gran(ev, n, block_threads, warp_size, out_key, out_cls, out_g, cap, policy, 2);
}

int64_t oracle_races(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                     uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap)
{
    return oracle_races_policy(ev, n, block_threads, warp_size, out_key, out_cls, out_g, cap, 0);
}

/*
 * ---------------------------------------------------------------------------------------------
 * Cluster level (reading R16): thread < warp < block < CLUSTER < grid.
 * PAPER.md L134 ("easily extended to ... deeper hierarchies"), L431, L490; the thread-block
 * cluster is the level sm_90+/sm_100 adds between the block and the grid.
 *
 *   C1.1'  cluster(e) = block(e) / cluster_blocks (consecutive block ids form a cluster);
 *          epochs g > c > b > w are nested: c = cluster barriers (barrier.cluster arrive+wait)
 *          passed since the last g, b = __syncthreads passed since the last c (a cluster barrier
 *          is also a rendezvous of every block of the cluster), w as before.
 *          Event encoding (tracegen.pack_cluster_addr): addr bits 56..62 = c; for shared
 *          accesses addr bits 48..55 = DSMEM target (0 = own block, r+1 = the block of cluster
 *          rank r); bits 0..47 = byte offset.  Shared key = 1<<63 | target_block<<32 | word.
 *   C1.2'  Concurrent <=> tid1 != tid2 and g1 == g2 and [cluster1 != cluster2 or (c1 == c2 and
 *          (block1 != block2 or (b1 == b2 and (warp1 != warp2 or w1 == w2))))]
 *   C1.3   Conflict as above (strict policy only), same_block = the ACCESSING threads' blocks.
 *   C1.4'  level GRID (clusters differ) / CLUSTER (blocks differ) / BLOCK (warps differ) / WARP
 *   C1.6'  class: g* = smallest racing g; GRID if a racing pair of g* is GRID-level; else c* =
 *          smallest c with a racing pair in g*, CLUSTER if a racing pair in (g*, c*) is
 *          CLUSTER-level; else b*, BLOCK / WARP as in C1.6 inside (g*, c*).
 * Class codes: WARP 1, BLOCK 2, GRID 3, CLUSTER 4 (coarseness WARP < BLOCK < CLUSTER < GRID).
 * ---------------------------------------------------------------------------------------------
 */
enum { CLS_CLUSTER = 4 };

typedef struct {
    uint64_t key;
    uint32_t g, cl, c, block, b, warp, w, tid, kind;
} caccess_t;

static int cmp_caccess(const void *pa, const void *pb)
{
    const caccess_t *a = (const caccess_t *)pa, *b = (const caccess_t *)pb;
#define CMP(f)                  \
    if (a->f != b->f)           \
        return a->f < b->f ? -1 : 1;
    CMP(key) CMP(g) CMP(cl) CMP(c) CMP(block) CMP(b) CMP(warp) CMP(w) CMP(tid)
#undef CMP
    return 0;
}

/* Returns the flagged-key count (first `cap` written in key order), -1 bad argument / out of
 * memory, -2 a C1.6' premise failed, -3 a DSMEM target outside the cluster. */
int64_t oracle_races_cluster(const oracle_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                             uint32_t cluster_blocks, uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g,
                             uint64_t cap)
{
    if (block_threads == 0 || warp_size == 0 || cluster_blocks == 0 || cluster_blocks > 255 || (n && !ev))
        return -1;
    const uint64_t OFF_MASK = (1ull << 48) - 1;
    uint64_t nacc = 0;
    for (uint64_t i = 0; i < n; i++) {
        uint32_t sz = 1u << ((ev[i].meta >> 2) & 7);
        nacc += sz <= 4 ? 1 : sz / 4;
    }
    caccess_t *acc = (caccess_t *)malloc((nacc ? nacc : 1) * sizeof(caccess_t));
    if (!acc)
        return -1;
    uint64_t j = 0;
    for (uint64_t i = 0; i < n; i++) {
        uint32_t meta = ev[i].meta;
        uint32_t kind = meta & 3, sz = 1u << ((meta >> 2) & 7);
        uint32_t w = (meta >> 5) & 511, b = (meta >> 14) & 1023, g = (meta >> 24) & 255;
        uint64_t addr = ev[i].addr;
        uint32_t c = (uint32_t)((addr >> 56) & 127);
        uint32_t tid = ev[i].tid;
        uint32_t block = tid / block_threads;
        uint32_t warp = (tid % block_threads) / warp_size;
        uint32_t cl = block / cluster_blocks;
        int shared = (addr & SHARED) != 0;
        uint32_t target = block;
        if (shared) {
            uint32_t t = (uint32_t)((addr >> 48) & 255);
            if (t) {
                if (t - 1 >= cluster_blocks) {
                    free(acc);
                    return -3;
                }
                target = cl * cluster_blocks + (t - 1);
            }
        } else if ((addr >> 48) & 255) {
            free(acc);
            return -1; /* DSMEM target on a global access */
        }
        uint64_t word0 = (addr & OFF_MASK) >> 2;
        uint32_t nw = sz <= 4 ? 1 : sz / 4;
        for (uint32_t k = 0; k < nw; k++) {
            caccess_t *a = &acc[j++];
            uint64_t word = word0 + k;
            a->key = shared ? (SHARED | ((uint64_t)target << 32) | (word & 0xffffffffull)) : word;
            a->g = g;
            a->cl = cl;
            a->c = c;
            a->block = block;
            a->b = b;
            a->warp = warp;
            a->w = w;
            a->tid = tid;
            a->kind = kind;
        }
    }
    qsort(acc, nacc, sizeof(caccess_t), cmp_caccess);

    masks_t clusters = {0}, blocks = {0}, warps = {0}, threads = {0};
    int64_t nflag = 0;
    int err = 0;
    uint64_t i = 0;
    while (i < nacc && !err) {
        uint64_t key = acc[i].key, kend = i;
        while (kend < nacc && acc[kend].key == key)
            kend++;
        int cls = CLS_NONE;
        uint32_t gstar = 0;
        for (uint64_t gs = i; gs < kend && cls == CLS_NONE;) {
            uint32_t g = acc[gs].g;
            uint64_t ge = gs;
            while (ge < kend && acc[ge].g == g)
                ge++;
            /* GRID level: groups = clusters of g */
            clusters.n = 0;
            int have_c = 0, cl_race_at_c = 0, have_b = 0, blk_race_at_b = 0;
            uint32_t min_c = 0;
            uint32_t nclusters_touching = 0;
            for (uint64_t ks = gs; ks < ge;) {
                uint32_t cl = acc[ks].cl;
                uint64_t ke = ks;
                uint8_t kmask = 0;
                while (ke < ge && acc[ke].cl == cl)
                    kmask |= (uint8_t)(1u << acc[ke].kind), ke++;
                if (masks_push(&clusters, kmask))
                    err = -1;
                nclusters_touching++;
                /* per cluster epoch c */
                for (uint64_t cs = ks; cs < ke;) {
                    uint32_t c = acc[cs].c;
                    uint64_t ce = cs;
                    while (ce < ke && acc[ce].c == c)
                        ce++;
                    /* CLUSTER level: groups = blocks of (cluster, c) */
                    blocks.n = 0;
                    int lower_race = 0, c_have_b = 0, c_blk_race_at_b = 0;
                    uint32_t c_min_b = 0;
                    for (uint64_t bs = cs; bs < ce;) {
                        uint32_t blk = acc[bs].block;
                        uint64_t be = bs;
                        uint8_t bmask = 0;
                        while (be < ce && acc[be].block == blk)
                            bmask |= (uint8_t)(1u << acc[be].kind), be++;
                        if (masks_push(&blocks, bmask))
                            err = -1;
                        for (uint64_t es = bs; es < be;) {
                            uint32_t b = acc[es].b;
                            uint64_t ee = es;
                            while (ee < be && acc[ee].b == b)
                                ee++;
                            /* BLOCK level: groups = warps of (block, b) */
                            warps.n = 0;
                            int warp_race = 0;
                            for (uint64_t ws = es; ws < ee;) {
                                uint32_t wp = acc[ws].warp;
                                uint64_t we = ws;
                                uint8_t wmask = 0;
                                while (we < ee && acc[we].warp == wp)
                                    wmask |= (uint8_t)(1u << acc[we].kind), we++;
                                if (masks_push(&warps, wmask))
                                    err = -1;
                                /* WARP level: groups = threads of (block, b, warp, w) */
                                for (uint64_t xs = ws; xs < we;) {
                                    uint32_t w = acc[xs].w;
                                    uint64_t xe = xs;
                                    while (xe < we && acc[xe].w == w)
                                        xe++;
                                    threads.n = 0;
                                    for (uint64_t ts = xs; ts < xe;) {
                                        uint32_t t = acc[ts].tid;
                                        uint8_t tmask = 0;
                                        while (ts < xe && acc[ts].tid == t)
                                            tmask |= (uint8_t)(1u << acc[ts].kind), ts++;
                                        if (masks_push(&threads, tmask))
                                            err = -1;
                                    }
                                    if (distinct_conflict(threads.m, threads.n, 1, 0))
                                        warp_race = 1;
                                    xs = xe;
                                }
                                ws = we;
                            }
                            int block_race = distinct_conflict(warps.m, warps.n, 1, 0);
                            if (block_race || warp_race) {
                                lower_race = 1;
                                if (!c_have_b || b < c_min_b) {
                                    c_have_b = 1;
                                    c_min_b = b;
                                    c_blk_race_at_b = block_race;
                                } else if (b == c_min_b && block_race) {
                                    c_blk_race_at_b = 1;
                                }
                            }
                            es = ee;
                        }
                        bs = be;
                    }
                    int cluster_race = distinct_conflict(blocks.m, blocks.n, 0, 0);
                    if (cluster_race || lower_race) {
                        if (!have_c || c < min_c) { /* c ascends inside a cluster; a second
                                                       * racing cluster fails the premise below */
                            have_c = 1;
                            min_c = c;
                            cl_race_at_c = cluster_race;
                            if (!cluster_race && blocks.n >= 2)
                                err = -2; /* only one block may touch the key in (g*, c*) */
                            have_b = c_have_b;
                            blk_race_at_b = c_blk_race_at_b;
                        }
                    }
                    cs = ce;
                }
                ks = ke;
            }
            int grid_race = distinct_conflict(clusters.m, clusters.n, 0, 0);
            if (grid_race) {
                cls = CLS_GRID;
            } else if (have_c) {
                if (nclusters_touching >= 2)
                    err = -2; /* C1.6' premise: only one cluster can touch the key in g* */
                if (cl_race_at_c)
                    cls = CLS_CLUSTER;
                else if (have_b)
                    cls = blk_race_at_b ? CLS_BLOCK : CLS_WARP;
                else
                    err = -2;
            }
            gstar = g;
            gs = ge;
        }
        if (cls != CLS_NONE) {
            if ((uint64_t)nflag < cap) {
                if (out_key)
                    out_key[nflag] = key;
                if (out_cls)
                    out_cls[nflag] = (uint8_t)cls;
                if (out_g)
                    out_g[nflag] = (uint8_t)gstar;
            }
            nflag++;
        }
        i = kend;
    }
    free(clusters.m);
    free(blocks.m);
    free(warps.m);
    free(threads.m);
    free(acc);
    return err ? err : nflag;
}
