/*
 * ORACLE-D, all-core driver: address-sharded parallel evaluation of the race definition.
 *
 * TEST INFRASTRUCTURE ONLY (same rules as oracle_d.c: only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load it; it shares nothing with the CUDA
 * path).
 *
 * Why this is still the definition: a key's verdict (C1.5) and class (C1.6) depend only on the
 * accesses to that key (PAPER.md L101 defines a race per memory location).
 * So the element-level accesses can be split by key into disjoint shards, each shard evaluated
 * by the pinned single-thread function oracle_races_gran (oracle_d.c, unchanged), and the
 * flagged keys of all shards concatenated and sorted.  This is SURVEY §8(c) C2's "multi-threaded
 * over address shards" and §8(d)'s "std::thread::hardware_concurrency() threads over address
 * shards".
 *
 * Steps (no blocking or reordering beyond the split):
 *   1. each of T threads takes a contiguous slice of the events and counts its element-level
 *      accesses per shard (shard = mix64(key) mod S; the key is C1.1's: global element index, or
 *      1<<63 | block<<32 | element for shared memory);
 *   2. shard-major offsets (exclusive scan over (shard, thread));
 *   3. each thread writes its accesses as single-element events into their shards: the address
 *      becomes the element's aligned address, the size field the element size, everything else
 *      (tid, kind, g, b, w) is copied, so oracle_races_gran recomputes the same key and
 *      coordinates (C1.1);
 *   4. the T threads take shards from a shared counter and run oracle_races_gran on each;
 *   5. the flagged (key, class, g*) triples of all shards are sorted by key.
 * The result equals oracle_races_gran on the whole trace (pinned by tests/test_oracle_par.py on
 * random, multi-element, shared-memory, policy and granularity traces and on configs 1, 2, 4).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint64_t addr;
    uint32_t tid;
    uint32_t meta;
} par_event; /* the 16-byte trace record (same layout as oracle_d.c's oracle_event) */

int64_t oracle_races_gran(const par_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                          uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap, int policy,
                          uint32_t gran_log2);

static const uint64_t SHARED = 1ull << 63;

static uint64_t mix64(uint64_t x)
{
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    x *= 0xc4ceb9fe1a85ec53ull;
    x ^= x >> 33;
    return x;
}

typedef struct {
    uint64_t key;
    uint8_t cls, g;
} flagged_t;

typedef struct job job_t;

typedef struct {
    job_t *J;
    int t;
} arg_t;

struct job {
    const par_event *ev;
    uint64_t n;
    uint32_t block_threads, warp_size, gran_log2;
    int policy, T, S;
    uint64_t *counts;  /* [T][S] */
    uint64_t *offsets; /* [S][T] start of (shard, thread) */
    uint64_t *shard_off;
    par_event *part;
    flagged_t **res;
    int64_t *res_n;
    int next_shard;
    pthread_mutex_t mu;
    int err;
};

/* C1.1: element k of event e -> (key, single-element event) */
static void slice(const job_t *J, int t, uint64_t *lo, uint64_t *hi)
{
    *lo = J->n * (uint64_t)t / (uint64_t)J->T;
    *hi = J->n * (uint64_t)(t + 1) / (uint64_t)J->T;
}

static void *count_main(void *p)
{
    arg_t *a = (arg_t *)p;
    job_t *J = a->J;
    uint64_t lo, hi;
    slice(J, a->t, &lo, &hi);
    uint64_t *cnt = J->counts + (uint64_t)a->t * J->S;
    const uint32_t granule = 1u << J->gran_log2;
    for (uint64_t i = lo; i < hi; i++) {
        const par_event *e = &J->ev[i];
        const uint32_t sz = 1u << ((e->meta >> 2) & 7);
        const uint32_t nw = sz <= granule ? 1 : sz / granule;
        const int shared = (e->addr & SHARED) != 0;
        const uint64_t word0 = (e->addr & ~SHARED) >> J->gran_log2;
        const uint32_t block = e->tid / J->block_threads;
        for (uint32_t k = 0; k < nw; k++) {
            const uint64_t word = word0 + k;
            const uint64_t key = shared ? (SHARED | ((uint64_t)block << 32) | (word & 0xffffffffull)) : word;
            cnt[mix64(key) % (uint64_t)J->S]++;
        }
    }
    return NULL;
}

static void *fill_main(void *p)
{
    arg_t *a = (arg_t *)p;
    job_t *J = a->J;
    uint64_t lo, hi;
    slice(J, a->t, &lo, &hi);
    uint64_t *pos = (uint64_t *)malloc((size_t)J->S * sizeof(uint64_t));
    if (!pos) {
        J->err = -1;
        return NULL;
    }
    for (int s = 0; s < J->S; s++)
        pos[s] = J->offsets[(uint64_t)s * J->T + a->t];
    const uint32_t granule = 1u << J->gran_log2;
    for (uint64_t i = lo; i < hi; i++) {
        const par_event *e = &J->ev[i];
        const uint32_t sz = 1u << ((e->meta >> 2) & 7);
        const uint32_t nw = sz <= granule ? 1 : sz / granule;
        const int shared = (e->addr & SHARED) != 0;
        const uint64_t word0 = (e->addr & ~SHARED) >> J->gran_log2;
        const uint32_t block = e->tid / J->block_threads;
        for (uint32_t k = 0; k < nw; k++) {
            const uint64_t word = word0 + k;
            const uint64_t key = shared ? (SHARED | ((uint64_t)block << 32) | (word & 0xffffffffull)) : word;
            par_event *o = &J->part[pos[mix64(key) % (uint64_t)J->S]++];
            o->addr = (shared ? SHARED : 0) | (word << J->gran_log2);
            o->tid = e->tid;
            o->meta = (e->meta & ~(7u << 2)) | (J->gran_log2 << 2); /* one element */
        }
    }
    free(pos);
    return NULL;
}

static void *shard_main(void *p)
{
    arg_t *a = (arg_t *)p;
    job_t *J = a->J;
    for (;;) {
        pthread_mutex_lock(&J->mu);
        const int s = J->next_shard++;
        pthread_mutex_unlock(&J->mu);
        if (s >= J->S || J->err)
            return NULL;
        const uint64_t o = J->shard_off[s], m = J->shard_off[s + 1] - o;
        uint64_t cap = m ? m : 1; /* a shard flags at most one key per access: one call */
        for (;;) {
            uint64_t *k = (uint64_t *)malloc(cap * sizeof(uint64_t));
            uint8_t *c = (uint8_t *)malloc(cap), *g = (uint8_t *)malloc(cap);
            if (!k || !c || !g) {
                free(k), free(c), free(g);
                J->err = -1;
                return NULL;
            }
            const int64_t r = oracle_races_gran(J->part + o, m, J->block_threads, J->warp_size, k, c, g, cap,
                                                J->policy, J->gran_log2);
            if (r < 0) {
                free(k), free(c), free(g);
                J->err = (int)r;
                return NULL;
            }
            if ((uint64_t)r > cap) {
                free(k), free(c), free(g);
                cap = (uint64_t)r;
                continue;
            }
            flagged_t *f = (flagged_t *)malloc((r ? (size_t)r : 1) * sizeof(flagged_t));
            if (!f) {
                free(k), free(c), free(g);
                J->err = -1;
                return NULL;
            }
            for (int64_t i = 0; i < r; i++) {
                f[i].key = k[i];
                f[i].cls = c[i];
                f[i].g = g[i];
            }
            free(k), free(c), free(g);
            J->res[s] = f;
            J->res_n[s] = r;
            break;
        }
    }
}

static int cmp_flagged(const void *pa, const void *pb)
{
    const flagged_t *a = (const flagged_t *)pa, *b = (const flagged_t *)pb;
    return a->key < b->key ? -1 : a->key > b->key ? 1 : 0;
}

static int run_threads(job_t *J, void *(*fn)(void *))
{
    pthread_t *th = (pthread_t *)malloc((size_t)J->T * sizeof(pthread_t));
    arg_t *args = (arg_t *)malloc((size_t)J->T * sizeof(arg_t));
    if (!th || !args) {
        free(th), free(args);
        return -1;
    }
    int started = 0;
    for (int t = 0; t < J->T; t++) {
        args[t].J = J;
        args[t].t = t;
        if (pthread_create(&th[t], NULL, fn, &args[t]) != 0) {
            J->err = -1;
            break;
        }
        started++;
    }
    for (int t = 0; t < started; t++)
        pthread_join(th[t], NULL);
    free(th), free(args);
    return J->err;
}

/*
 * Same contract as oracle_races_gran (oracle_d.c): returns the number of flagged keys (only the
 * first `cap` are written, sorted by key) or a negative error.  nthreads >= 1 worker threads,
 * nshards >= 1 key shards (more shards = less memory per shard).
 */
int64_t oracle_races_par(const par_event *ev, uint64_t n, uint32_t block_threads, uint32_t warp_size,
                         uint64_t *out_key, uint8_t *out_cls, uint8_t *out_g, uint64_t cap, int policy,
                         uint32_t gran_log2, int nthreads, int nshards)
{
    if (nthreads < 1 || nshards < 1 || block_threads == 0 || warp_size == 0 || (n && !ev) || gran_log2 > 2 ||
        (policy != 0 && policy != 1))
        return -1;
    job_t J;
    memset(&J, 0, sizeof(J));
    J.ev = ev;
    J.n = n;
    J.block_threads = block_threads;
    J.warp_size = warp_size;
    J.gran_log2 = gran_log2;
    J.policy = policy;
    J.T = nthreads;
    J.S = nshards;
    pthread_mutex_init(&J.mu, NULL);
    int64_t ret = -1;
    J.counts = (uint64_t *)calloc((size_t)J.T * J.S, sizeof(uint64_t));
    J.offsets = (uint64_t *)malloc((size_t)J.T * J.S * sizeof(uint64_t));
    J.shard_off = (uint64_t *)malloc(((size_t)J.S + 1) * sizeof(uint64_t));
    J.res = (flagged_t **)calloc((size_t)J.S, sizeof(flagged_t *));
    J.res_n = (int64_t *)calloc((size_t)J.S, sizeof(int64_t));
    if (!J.counts || !J.offsets || !J.shard_off || !J.res || !J.res_n)
        goto done;
    /* 1 */
    if (run_threads(&J, count_main))
        goto done;
    /* 2 */
    uint64_t acc = 0;
    for (int s = 0; s < J.S; s++) {
        J.shard_off[s] = acc;
        for (int t = 0; t < J.T; t++) {
            J.offsets[(uint64_t)s * J.T + t] = acc;
            acc += J.counts[(uint64_t)t * J.S + s];
        }
    }
    J.shard_off[J.S] = acc;
    /* 3 */
    J.part = (par_event *)malloc((acc ? acc : 1) * sizeof(par_event));
    if (!J.part)
        goto done;
    if (run_threads(&J, fill_main))
        goto done;
    /* 4 */
    if (run_threads(&J, shard_main)) {
        ret = J.err;
        goto done;
    }
    free(J.part);
    J.part = NULL;
    /* 5 */
    int64_t total = 0;
    for (int s = 0; s < J.S; s++)
        total += J.res_n[s];
    flagged_t *all = (flagged_t *)malloc((total ? (size_t)total : 1) * sizeof(flagged_t));
    if (!all)
        goto done;
    int64_t k = 0;
    for (int s = 0; s < J.S; s++) {
        if (J.res_n[s])
            memcpy(all + k, J.res[s], (size_t)J.res_n[s] * sizeof(flagged_t));
        k += J.res_n[s];
    }
    qsort(all, (size_t)total, sizeof(flagged_t), cmp_flagged);
    for (int64_t i = 0; i < total && (uint64_t)i < cap; i++) {
        if (out_key)
            out_key[i] = all[i].key;
        if (out_cls)
            out_cls[i] = all[i].cls;
        if (out_g)
            out_g[i] = all[i].g;
    }
    free(all);
    ret = total;
done:
    if (J.res)
        for (int s = 0; s < J.S; s++)
            free(J.res[s]);
    free(J.res), free(J.res_n), free(J.part), free(J.counts), free(J.offsets), free(J.shard_off);
    pthread_mutex_destroy(&J.mu);
    return ret;
}
