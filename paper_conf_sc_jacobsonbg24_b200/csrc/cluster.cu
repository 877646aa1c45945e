/*
 * cluster.cu — replay with a thread-block-cluster level (DESIGN.md reading
 * R16; "easily extended to ... deeper hierarchies", L431).
 *
 * The hierarchy is thread < warp < block < cluster (cluster_blocks consecutive blocks) < grid.
 * Events carry the cluster epoch c in addr bits 56..62 and, for shared accesses, a DSMEM target
 * in addr bits 48..55 (0 = own block, r+1 = cluster rank r); see include/hirace.h.  Records are
 * the 8-byte cluster layout state:6 | g:8 | c:7 | b:8 | w:8 | tid:27 and the transition is the
 * derived 34-state table (fsm_table.cpp clus::rules) through hirace::cluster::step — the same
 * inline function the CPU bisimulation test runs.
 *
 * k_cluster_replay is one persistent cooperative kernel: every warp finds the end of the
 * current (g,c,b,w) batch by a 32-ary search over the batch-sorted events, the grid covers the
 * batch in a grid-stride loop (kU = 4 events per thread per iteration, loads issued together;
 * Algorithm 1's load / step / CAS loop per event,
 * PAPER.md L249-279, with no store when the record is unchanged), and a grid barrier separates batches (all events of a
 * batch are pairwise concurrent or program-ordered in one thread: PAPER.md L177).
 * Collection is an ordered compaction of the RACE records in shadow (= key) order written here
 * (k_cluster_count per 4096-record tile, host prefix over the tiles, k_cluster_emit at each
 * tile's offset); no library kernel on this path.
 */
#include <cooperative_groups.h>
#include <vector>

#include <stdlib.h>
#include <string.h>

#include "hirace.h"
#include "hirace_device.cuh"
#include "internal.h"

namespace cg = cooperative_groups;
using namespace hirace::cluster;

struct hirace_cluster_ctx {
    hirace_config cfg;
    uint32_t cluster_blocks;
    uint64_t global_words, smem_words, shadow_words;
    unsigned long long *shadow;
    unsigned char *table;       /* 16 KB transition table            */
    unsigned char *race_class;  /* 64 entries: state -> class (0..4) */
    unsigned int *err;          /* sticky device error flags          */
    unsigned long long *stats;  /* [0] checked word accesses, [1] CAS retries */
    int grid;
    int sm_count;
    hirace_status sticky;
    uint64_t *coll_tiles;       /* collect scratch: per-tile counts / offsets */
    uint64_t coll_tiles_cap;
    hirace_race *coll_rows;     /* collect scratch: output rows              */
    uint64_t coll_rows_cap;
};

namespace {

enum : unsigned int { ERR_BAD_TRACE = 1u, ERR_RANGE = 2u };
constexpr int kThreads = 256;

/* (g, c, b, w) in lexicographic order: g:8 | c:7 | b:10 | w:9 */
__device__ __forceinline__ uint64_t batch_key(const hirace_event &e)
{
    const uint64_t c = (e.addr >> 56) & 127u;
    return ((uint64_t)(e.meta >> 24) << 26) | (c << 19) | ((e.meta >> 5) & ((1u << 19) - 1u));
}

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

/* 16-byte event, streaming: read once, so no L1 allocation (the records are what should stay
 * cached) */
__device__ __forceinline__ hirace_event ld_event_stream(const hirace_event *p)
{
    uint32_t x, y, z, w;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(x), "=r"(y), "=r"(z), "=r"(w)
                 : "l"(p));
    hirace_event e;
    e.addr = (uint64_t)x | ((uint64_t)y << 32);
    e.tid = z;
    e.meta = w;
    return e;
}

struct Geo {
    uint32_t block_threads, warp_size, cluster_blocks, grid_blocks;
    uint64_t global_words, smem_words;
    uint32_t bt_log2, ws_log2, cb_log2; /* valid when all three sizes are powers of two (P2) */
};

/* Decode one event: range checks, DSMEM owner, first shadow index and word count.  Returns
 * false (and sets ERR_RANGE) for an out-of-range event. */
template <bool P2>
__device__ __forceinline__ bool decode_event(const hirace_event &e, const Geo &G, unsigned int *err, uint64_t &idx0,
                                             uint32_t &nw)
{
    const uint32_t meta = e.meta, tid = e.tid;
    const uint32_t size = 1u << ((meta >> 2) & 7u);
    const uint32_t w = (meta >> 5) & 511u, b = (meta >> 14) & 1023u;
    const uint32_t tgt = (uint32_t)(e.addr >> 48) & 255u;
    const bool shared = (e.addr >> 63) != 0;
    const uint64_t off = e.addr & ((1ull << 48) - 1);
    const uint32_t block = P2 ? tid >> G.bt_log2 : tid / G.block_threads;
    if (b > MAX_B || w > MAX_W || tid > MAX_TID || block >= G.grid_blocks || size > 16u ||
        (!shared && tgt != 0) || (tgt != 0 && tgt - 1u >= G.cluster_blocks)) {
        atomicOr(err, ERR_RANGE);
        return false;
    }
    const uint32_t cl = P2 ? block >> G.cb_log2 : block / G.cluster_blocks;
    const uint32_t owner = tgt ? cl * G.cluster_blocks + (tgt - 1u) : block;
    const uint64_t word0 = off >> 2;
    nw = size <= 4u ? 1u : size >> 2;
    const uint64_t limit = shared ? G.smem_words : G.global_words;
    if (owner >= G.grid_blocks || word0 + nw > limit) {
        atomicOr(err, ERR_RANGE);
        return false;
    }
    idx0 = shared ? G.global_words + (uint64_t)owner * G.smem_words + word0 : word0;
    return true;
}

/* Algorithm 1's load / step / CAS loop on one record whose value o was
 * already loaded; no store when the record is unchanged (linearised at the coherent load).
 * P2: power-of-two geometry, label by shifts (label_p2); else the generic step(). */
template <bool P2>
__device__ __forceinline__ void commit(const hirace_event &e, unsigned long long *p, unsigned long long o,
                                       const unsigned char *table, const Geo &G, unsigned long long &retries)
{
    const uint32_t meta = e.meta;
    const uint32_t kind = meta & 3u, w = (meta >> 5) & 511u, b = (meta >> 14) & 1023u, g = meta >> 24;
    const uint32_t c = (uint32_t)(e.addr >> 56) & 127u;
    for (;;) {
        uint32_t rep;
        const unsigned long long nv =
            P2 ? step_labelled(o, label_p2(o, e.tid, kind, g, c, b, w, G.bt_log2, G.ws_log2, G.cb_log2), e.tid, g,
                               c, b, w, table)
               : step(o, e.tid, kind, g, c, b, w, table, G.block_threads, G.warp_size, G.cluster_blocks, &rep);
        if (nv == o)
            break;
        const unsigned long long prev = atomicCAS(p, o, nv);
        if (prev == o)
            break;
        o = prev;
        retries++;
    }
}

/* kU events per thread per iteration of the grid-stride loop: their event loads, then their
 * record loads, are issued back to back so kU L2/HBM round trips overlap (the chain event ->
 * record -> CAS is latency-bound with one event in flight). */
constexpr int kU = 4;

template <bool P2>
__global__ void __launch_bounds__(kThreads, 4) k_cluster_replay(const hirace_event *__restrict__ ev, uint32_t n,
                                                             unsigned long long *shadow, const unsigned char *gtable,
                                                             Geo G, unsigned int *err, unsigned long long *stats)
{
    __shared__ unsigned char table[TABLE_BYTES];
    for (uint32_t i = threadIdx.x; i < TABLE_BYTES / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(table)[i] = reinterpret_cast<const uint4 *>(gtable)[i];
    __syncthreads();
    cg::grid_group grid = cg::this_grid();
    const uint64_t gsize = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t gtid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long checked = 0, retries = 0;
    uint32_t start = 0;
    while (start < n) {
        const uint64_t key0 = batch_key(ev[start]);
        /* end = first index > start whose batch key differs (upper bound; sorted input), by a
         * 32-ary search: each lane probes one of 32 evenly spaced events, the ballot's prefix of
         * "key <= key0" lanes narrows the range 32x per round (5 dependent loads for 16M events
         * instead of 24 for a binary search).  The loop is grid-uniform, so all lanes are here. */
        const uint32_t lane = threadIdx.x & 31u;
        uint32_t lo = start + 1, hi = n;
        while (lo < hi) {
            const uint32_t stride = (uint32_t)(((uint64_t)(hi - lo) + 31u) / 32u);
            const uint64_t q = (uint64_t)lo + (uint64_t)lane * stride;
            const bool le = q < hi && batch_key(ev[q]) <= key0;
            const uint32_t t = __popc(__ballot_sync(0xffffffffu, le));
            if (t == 0) {
                hi = lo;
            } else {
                const uint64_t nhi = (uint64_t)lo + (uint64_t)t * stride;
                lo = lo + (t - 1u) * stride + 1u;
                hi = nhi < hi ? (uint32_t)nhi : hi;
            }
        }
        const uint32_t end = lo;
        /* grid-stride over the batch: consecutive warps take consecutive 32-event chunks, each
         * thread kU of them per iteration (i, i + gsize, ...).  Contiguous per-warp or per-CTA
         * shares (the three-level replay's layout) were measured slower on the halo workloads
         * (profiles/r1_cluster_ab.txt).  Events of one batch are pairwise concurrent or
         * program-ordered in one thread, so the order in which a thread commits
         * its kU events does not change the flagged set. */
        for (uint64_t i = start + gtid; i < end; i += kU * gsize) {
            hirace_event e[kU];
            bool v[kU];
#pragma unroll
            for (int k = 0; k < kU; k++) {
                v[k] = i + k * gsize < end;
                if (v[k])
                    e[k] = ld_event_stream(ev + i + k * gsize);
            }
            uint64_t idx[kU];
            uint32_t nw[kU];
#pragma unroll
            for (int k = 0; k < kU; k++) {
                if (v[k] && batch_key(e[k]) != key0) {
                    atomicOr(err, ERR_BAD_TRACE); /* not batch-sorted */
                    v[k] = false;
                }
                if (v[k])
                    v[k] = decode_event<P2>(e[k], G, err, idx[k], nw[k]);
            }
            unsigned long long o[kU];
#pragma unroll
            for (int k = 0; k < kU; k++)
                if (v[k])
                    o[k] = ld_relaxed(shadow + idx[k]);
#pragma unroll
            for (int k = 0; k < kU; k++) {
                if (!v[k])
                    continue;
                commit<P2>(e[k], shadow + idx[k], o[k], table, G, retries);
                for (uint32_t j = 1; j < nw[k]; j++) /* wide access: one record per word */
                    commit<P2>(e[k], shadow + idx[k] + j, ld_relaxed(shadow + idx[k] + j), table, G, retries);
                checked += nw[k];
            }
        }
        grid.sync();
        start = end;
    }
    if (checked)
        atomicAdd(&stats[0], checked);
    if (retries)
        atomicAdd(&stats[1], retries);
}

/* Collection: an ordered compaction of the RACE records in shadow (= key) order, two passes
 * over 4096-record tiles (count, then emit at the tile's offset with a block scan). */
constexpr uint32_t kCollTile = 4096, kCollThreads = 256, kCollPer = kCollTile / kCollThreads;

__device__ __forceinline__ uint32_t coll_block_scan(uint32_t mine, uint32_t *s_w, uint32_t *total)
{
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    uint32_t incl = mine;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if ((int)lane >= d)
            incl += y;
    }
    if (lane == 31)
        s_w[wid] = incl;
    __syncthreads();
    uint32_t before = 0, all = 0;
    for (uint32_t w = 0; w < nw; w++) {
        const uint32_t x = s_w[w];
        before += w < wid ? x : 0u;
        all += x;
    }
    *total = all;
    return before + incl - mine;
}

__global__ void __launch_bounds__(kCollThreads) k_cluster_count(const unsigned long long *__restrict__ shadow,
                                                                uint64_t nw, const unsigned char *__restrict__ cls,
                                                                uint32_t *tile_cnt)
{
    __shared__ uint32_t s_w[32];
    const uint64_t w0 = (uint64_t)blockIdx.x * kCollTile + (uint64_t)threadIdx.x * kCollPer;
    uint32_t n = 0;
    for (uint32_t k = 0; k < kCollPer; k++)
        n += (w0 + k < nw && cls[__ldcs(shadow + w0 + k) & 63u] != 0) ? 1u : 0u;
    uint32_t tot;
    coll_block_scan(n, s_w, &tot);
    if (threadIdx.x == 0)
        tile_cnt[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kCollThreads) k_cluster_emit(const unsigned long long *__restrict__ shadow,
                                                               uint64_t nw, const unsigned char *__restrict__ cls,
                                                               const uint64_t *tile_off, uint64_t cap,
                                                               uint64_t global_words, uint64_t smem_words,
                                                               hirace_race *out)
{
    __shared__ uint32_t s_w[32];
    const uint64_t w0 = (uint64_t)blockIdx.x * kCollTile + (uint64_t)threadIdx.x * kCollPer;
    uint32_t n = 0;
    for (uint32_t k = 0; k < kCollPer; k++)
        n += (w0 + k < nw && cls[shadow[w0 + k] & 63u] != 0) ? 1u : 0u;
    uint32_t tot;
    uint64_t pos = tile_off[blockIdx.x] + coll_block_scan(n, s_w, &tot);
    for (uint32_t k = 0; k < kCollPer && n; k++) {
        const uint64_t idx = w0 + k;
        if (idx >= nw)
            break;
        const unsigned long long r = shadow[idx];
        if (cls[r & 63u] == 0)
            continue;
        if (pos < cap) {
            uint64_t key = idx;
            if (idx >= global_words) {
                const uint64_t s = idx - global_words;
                key = HIRACE_SHARED_BIT | ((s / smem_words) << 32) | (s % smem_words);
            }
            out[pos].key = key;
            out[pos].cls_and_epoch = (uint32_t)cls[r & 63u] | (uint32_t)((r >> SH_G) & 255u) << 8;
            out[pos].detect_tid = (uint32_t)(r >> SH_TID);
        }
        pos++;
    }
}

__global__ void k_cluster_fill(unsigned long long *p, uint64_t n)
{
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = 0ull;
}

hirace_status cuda_status(cudaError_t e) { return e == cudaSuccess ? HIRACE_OK : HIRACE_E_CUDA; }

hirace_status sync_errors(hirace_cluster_ctx *ctx)
{
    unsigned int h = 0;
    if (cudaMemcpy(&h, ctx->err, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess)
        return HIRACE_E_CUDA;
    if (h && ctx->sticky == HIRACE_OK)
        ctx->sticky = HIRACE_E_BAD_TRACE;
    return ctx->sticky;
}

} // namespace

extern "C" {

hirace_status hirace_cluster_alloc(const hirace_config *cfg, uint32_t cluster_blocks, hirace_cluster_ctx **out)
{
    if (!cfg || !out || !cfg->grid_blocks || !cfg->block_threads || !cfg->warp_size || !cluster_blocks ||
        cluster_blocks > 255 || cfg->grid_blocks % cluster_blocks != 0 || cfg->granularity_log2 != 2 ||
        (cfg->global_bytes & 3) || (cfg->smem_bytes_per_block & 3) || /* as hirace_shadow_alloc */
        (uint64_t)cfg->grid_blocks * cfg->block_threads > (uint64_t)MAX_TID + 1)
        return HIRACE_E_INVAL;
    *out = nullptr;
    if (cudaSetDevice(cfg->device) != cudaSuccess)
        return HIRACE_E_CUDA;
    hirace_cluster_ctx *c = (hirace_cluster_ctx *)calloc(1, sizeof(hirace_cluster_ctx));
    if (!c)
        return HIRACE_E_NOMEM;
    c->cfg = *cfg;
    c->cluster_blocks = cluster_blocks;
    c->global_words = cfg->global_bytes / 4;
    c->smem_words = cfg->smem_bytes_per_block / 4u;
    c->shadow_words = c->global_words + (uint64_t)cfg->grid_blocks * c->smem_words;
    unsigned char table[TABLE_BYTES], cls[64] = {0};
    uint32_t nst = 0;
    if (hirace_fsm_table_cluster(table, &nst) != HIRACE_OK) {
        free(c);
        return HIRACE_E_INVAL;
    }
    for (uint32_t s = 0; s < nst; s++)
        cls[s] = (unsigned char)hirace_fsm_cluster_class(s);
    cudaError_t e = cudaMalloc(&c->shadow, (c->shadow_words ? c->shadow_words : 1) * 8);
    if (e == cudaSuccess)
        e = cudaMalloc(&c->table, TABLE_BYTES);
    if (e == cudaSuccess)
        e = cudaMalloc(&c->race_class, 64);
    if (e == cudaSuccess)
        e = cudaMalloc(&c->err, sizeof(unsigned int));
    if (e == cudaSuccess)
        e = cudaMalloc(&c->stats, 2 * sizeof(unsigned long long));
    if (e == cudaSuccess)
        e = cudaMemcpy(c->table, table, TABLE_BYTES, cudaMemcpyHostToDevice);
    if (e == cudaSuccess)
        e = cudaMemcpy(c->race_class, cls, 64, cudaMemcpyHostToDevice);
    int per_sm = 0;
    if (e == cudaSuccess)
        e = cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, cfg->device);
    if (e == cudaSuccess) { /* both instantiations may launch: the smaller occupancy bounds the grid */
        int per_sm2 = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_cluster_replay<false>, kThreads, 0);
        if (e == cudaSuccess)
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm2, k_cluster_replay<true>, kThreads, 0);
        per_sm = per_sm2 < per_sm ? per_sm2 : per_sm;
    }
    if (e != cudaSuccess || per_sm < 1) {
        hirace_cluster_free(c);
        return e == cudaErrorMemoryAllocation ? HIRACE_E_NOMEM : HIRACE_E_CUDA;
    }
    c->grid = c->sm_count * (per_sm < 4 ? per_sm : 4);
    hirace_status st = hirace_cluster_reset(c, nullptr);
    if (st == HIRACE_OK)
        st = cuda_status(cudaDeviceSynchronize());
    if (st != HIRACE_OK) {
        hirace_cluster_free(c);
        return st;
    }
    *out = c;
    return HIRACE_OK;
}

hirace_status hirace_cluster_free(hirace_cluster_ctx *c)
{
    if (!c)
        return HIRACE_E_INVAL;
    cudaFree(c->shadow);
    cudaFree(c->table);
    cudaFree(c->race_class);
    cudaFree(c->err);
    cudaFree(c->stats);
    cudaFree(c->coll_tiles);
    cudaFree(c->coll_rows);
    free(c);
    return HIRACE_OK;
}

hirace_status hirace_cluster_reset(hirace_cluster_ctx *c, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    hirace_impl::note_launches(1);
    k_cluster_fill<<<c->sm_count * 4, 256, 0, st>>>(c->shadow, c->shadow_words);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess)
        e = cudaMemsetAsync(c->err, 0, sizeof(unsigned int), st);
    if (e == cudaSuccess)
        e = cudaMemsetAsync(c->stats, 0, 2 * sizeof(unsigned long long), st);
    c->sticky = HIRACE_OK;
    return cuda_status(e);
}

hirace_status hirace_cluster_replay(hirace_cluster_ctx *c, const hirace_event *d_events, uint64_t n, void *stream)
{
    if (!c || (n && !d_events) || n >= (1ull << 32))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (!n)
        return HIRACE_OK;
    Geo G{c->cfg.block_threads, c->cfg.warp_size, c->cluster_blocks, c->cfg.grid_blocks, c->global_words,
          c->smem_words, 0, 0, 0};
    const auto pow2 = [](uint32_t x) { return x && !(x & (x - 1)); };
    const bool p2 = pow2(G.block_threads) && pow2(G.warp_size) && pow2(G.cluster_blocks);
    if (p2) {
        G.bt_log2 = __builtin_ctz(G.block_threads);
        G.ws_log2 = __builtin_ctz(G.warp_size);
        G.cb_log2 = __builtin_ctz(G.cluster_blocks);
    }
    uint32_t nn = (uint32_t)n;
    const hirace_event *ev = d_events;
    unsigned long long *shadow = c->shadow;
    const unsigned char *table = c->table;
    void *args[] = {(void *)&ev, (void *)&nn, (void *)&shadow, (void *)&table, (void *)&G, (void *)&c->err,
                    (void *)&c->stats};
    hirace_impl::note_launches(1);
    return cuda_status(cudaLaunchCooperativeKernel(p2 ? (const void *)k_cluster_replay<true> : (const void *)k_cluster_replay<false>, dim3(c->grid), dim3(kThreads),
                                                   args, 0, (cudaStream_t)stream));
}

hirace_status hirace_cluster_collect(hirace_cluster_ctx *c, hirace_race *h_out, uint64_t cap, uint64_t *n_total)
{
    if (!c || !n_total || (cap && !h_out))
        return HIRACE_E_INVAL;
    if (cudaDeviceSynchronize() != cudaSuccess)
        return HIRACE_E_CUDA;
    hirace_status st = sync_errors(c);
    if (st != HIRACE_OK)
        return st;
    const uint64_t nw = c->shadow_words;
    const uint64_t ntiles = (nw + kCollTile - 1) / kCollTile;
    if (ntiles == 0) {
        *n_total = 0;
        return HIRACE_OK;
    }
    /* scratch: tile counts / offsets (shadow / 4096 entries), rows of at most cap records;
     * context-owned, grown on demand */
    cudaError_t e = cudaSuccess;
    if (ntiles > c->coll_tiles_cap) {
        cudaFree(c->coll_tiles);
        c->coll_tiles = nullptr;
        c->coll_tiles_cap = 0;
        if ((e = cudaMalloc(&c->coll_tiles, ntiles * sizeof(uint64_t))) != cudaSuccess)
            return HIRACE_E_NOMEM;
        c->coll_tiles_cap = ntiles;
    }
    uint32_t *cnt = reinterpret_cast<uint32_t *>(c->coll_tiles);
    hirace_impl::note_launches(1);
    k_cluster_count<<<(unsigned)ntiles, kCollThreads>>>(c->shadow, nw, c->race_class, cnt);
    std::vector<uint32_t> h_cnt(ntiles);
    if ((e = cudaMemcpy(h_cnt.data(), cnt, ntiles * sizeof(uint32_t), cudaMemcpyDeviceToHost)) != cudaSuccess)
        return HIRACE_E_CUDA;
    std::vector<uint64_t> h_off(ntiles);
    uint64_t total = 0;
    for (uint64_t t = 0; t < ntiles; t++) {
        h_off[t] = total;
        total += h_cnt[t];
    }
    const uint64_t m = total < cap ? total : cap;
    if (m) {
        if (m > c->coll_rows_cap) {
            cudaFree(c->coll_rows);
            c->coll_rows = nullptr;
            c->coll_rows_cap = 0;
            if ((e = cudaMalloc(&c->coll_rows, m * sizeof(hirace_race))) != cudaSuccess)
                return HIRACE_E_NOMEM;
            c->coll_rows_cap = m;
        }
        if ((e = cudaMemcpy(c->coll_tiles, h_off.data(), ntiles * sizeof(uint64_t), cudaMemcpyHostToDevice)) !=
            cudaSuccess)
            return HIRACE_E_CUDA;
        hirace_impl::note_launches(1);
        k_cluster_emit<<<(unsigned)ntiles, kCollThreads>>>(c->shadow, nw, c->race_class, c->coll_tiles, m,
                                                           c->global_words, c->smem_words ? c->smem_words : 1,
                                                           c->coll_rows);
        if ((e = cudaGetLastError()) == cudaSuccess)
            e = cudaMemcpy(h_out, c->coll_rows, m * sizeof(hirace_race), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess)
            return HIRACE_E_CUDA;
    }
    *n_total = total;
    return HIRACE_OK;
}

hirace_status hirace_cluster_get_stats(hirace_cluster_ctx *c, uint64_t *checked, uint64_t *cas_retries)
{
    if (!c)
        return HIRACE_E_INVAL;
    unsigned long long h[2] = {0, 0};
    if (cudaMemcpy(h, c->stats, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess)
        return HIRACE_E_CUDA;
    if (checked)
        *checked = h[0];
    if (cas_retries)
        *cas_retries = h[1];
    return HIRACE_OK;
}

hirace_status hirace_cluster_get_dev_ctx(hirace_cluster_ctx *c, const void *global_base, hirace_cluster_dev_ctx *out)
{
    if (!c || !out)
        return HIRACE_E_INVAL;
    out->shadow = c->shadow;
    out->table = c->table;
    out->error_flags = c->err;
    out->stats = c->stats;
    out->global_base = global_base;
    out->global_words = c->global_words;
    out->smem_words = (unsigned int)c->smem_words;
    out->grid_blocks = c->cfg.grid_blocks;
    out->block_threads = c->cfg.block_threads;
    out->warp_size = c->cfg.warp_size;
    out->cluster_blocks = c->cluster_blocks;
    out->g = 0;
    return HIRACE_OK;
}

} /* extern "C" */
