/*
 * hirace_kernels.cu — sm_100a kernels of the HiRace hot path.
 *
 *   k_batches                         a9  batch discovery + validation (replay input sorted by
 *                                         (g,b,w)), one CTA
 *   (k_replay, the a1-a9 hot kernel, lives in replay.cu)
 *   k_collect                         a7  order-preserving compaction of RACE records (collect.cuh)
 *   k_rebase                          a8  grid-epoch wrap sweep
 *   k_bucket_*                        a10 owner bucketing for the address-sharded mode
 */
#include <atomic>
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
#include "collect.cuh"
#include "kernel_common.cuh"

namespace hirace_impl {

using namespace hirace;

/* ---------------------------------------------------------------------------------------- */
/* a9: batch discovery.  Boundaries = {p : key(p) != key(p-1)}.  A chunk [lo,hi) can hold a  */
/* boundary only if key(max(lo,1)-1) != key(hi-1) (true for sorted input); dirty chunks are   */
/* split 32-way by one warp until single positions are tested.  Unsorted input may hide     */
/* boundaries; the replay kernel then sees an event whose key differs from its batch key and */
/* flags HIRACE_E_BAD_TRACE, so validation is complete without a second full read.          */
/* ---------------------------------------------------------------------------------------- */

constexpr int kFindThreads = 1024;
constexpr int kFindWarps = kFindThreads / 32;
constexpr int kFindStack = 160;

__device__ __forceinline__ bool chunk_dirty(const hirace_event *ev, uint32_t lo, uint32_t hi)
{
    uint32_t q = lo > 1 ? lo : 1;
    if (q >= hi)
        return false;
    return batch_key_at(ev, q - 1) != batch_key_at(ev, hi - 1);
}

struct FindSmem {
    uint32_t list[32768];                 /* boundary positions; list[0] = 0 */
    uint32_t lo[kFindWarps][kFindStack];  /* per-warp refinement stacks */
    uint32_t len[kFindWarps][kFindStack];
    uint32_t count;
};

/* One CTA: (1) each lane probes one 32768-event chunk (2 loads), (2) the warp refines each
 * dirty chunk 32-way down to single positions, (3) bitonic sort of the boundaries, emit
 * batch_off[0..nb], zero the per-batch claim counters, check keys strictly increase. */
__global__ void __launch_bounds__(kFindThreads) k_batches(const hirace_event *__restrict__ ev, uint32_t n,
                                                          uint32_t *off, uint32_t *nbatches, uint32_t *batch_ctr,
                                                          unsigned int *err, unsigned int *grid_bar)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    FindSmem &S = *reinterpret_cast<FindSmem *>(smem_raw);
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (threadIdx.x == 0)
        *grid_bar = 0; /* the replay kernel's grid-barrier counter (stream-ordered before it) */
    if (threadIdx.x == 0) {
        S.count = 1;
        S.list[0] = 0;
    }
    __syncthreads();
    if (n == 0) {
        if (threadIdx.x == 0) {
            *nbatches = 0;
            off[0] = 0;
        }
        return;
    }
    const uint64_t nchunks = (n + kFindChunk - 1) / kFindChunk;
    for (uint64_t t0 = (uint64_t)wid * 32; t0 < nchunks; t0 += (uint64_t)kFindWarps * 32) {
        const uint64_t t = t0 + lane;
        const uint32_t lo = (uint32_t)(t * kFindChunk);
        const bool d = t < nchunks && chunk_dirty(ev, lo, (uint32_t)min((uint64_t)lo + kFindChunk, (uint64_t)n));
        for (uint32_t dm = __ballot_sync(0xffffffffu, d); dm; dm &= dm - 1) {
            const uint32_t clo0 = (uint32_t)((t0 + __ffs(dm) - 1) * kFindChunk);
            int sp = 1;
            if (lane == 0) {
                S.lo[wid][0] = clo0;
                S.len[wid][0] = (uint32_t)min((uint64_t)kFindChunk, (uint64_t)n - clo0);
            }
            __syncwarp();
            while (sp > 0) {
                sp--;
                const uint32_t clo = S.lo[wid][sp], clen = S.len[wid][sp];
                __syncwarp();
                if (clen <= 32) {
                    const uint32_t p = clo + lane;
                    if (lane < clen && p >= 1 && batch_key_at(ev, p) != batch_key_at(ev, p - 1)) {
                        const uint32_t k = atomicAdd(&S.count, 1u);
                        if (k < 32768u)
                            S.list[k] = p;
                    }
                } else {
                    const uint32_t sub = (clen + 31) / 32;
                    const uint32_t slo = clo + lane * sub;
                    const uint32_t shi = min(slo + sub, clo + clen);
                    const bool dd = slo < clo + clen && chunk_dirty(ev, slo, shi);
                    const uint32_t mask = __ballot_sync(0xffffffffu, dd);
                    const uint32_t rank = __popc(mask & ((1u << lane) - 1));
                    if (dd && sp + rank < kFindStack) {
                        S.lo[wid][sp + rank] = slo;
                        S.len[wid][sp + rank] = shi - slo;
                    }
                    sp = min(sp + __popc(mask), kFindStack);
                    __syncwarp();
                }
            }
        }
    }
    __syncthreads();
    const uint32_t nb = S.count;
    if (nb > HIRACE_MAX_BATCHES) {
        if (threadIdx.x == 0) {
            *nbatches = 0;
            atomicOr(err, ERR_BATCHES | ERR_BAD_TRACE);
        }
        return;
    }
    uint32_t P = 1;
    while (P < nb)
        P <<= 1;
    for (uint32_t i = nb + threadIdx.x; i < P; i += blockDim.x)
        S.list[i] = 0xffffffffu;
    __syncthreads();
    for (uint32_t k = 2; k <= P; k <<= 1) {
        for (uint32_t j = k >> 1; j > 0; j >>= 1) {
            for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) {
                const uint32_t ixj = i ^ j;
                if (ixj > i) {
                    const uint32_t x = S.list[i], y = S.list[ixj];
                    if ((x > y) == ((i & k) == 0)) {
                        S.list[i] = y;
                        S.list[ixj] = x;
                    }
                }
            }
            __syncthreads();
        }
    }
    for (uint32_t i = threadIdx.x; i < nb; i += blockDim.x) {
        off[i] = S.list[i];
        batch_ctr[i] = 0;
        if (i > 0 && !(batch_key_at(ev, S.list[i]) > batch_key_at(ev, S.list[i - 1])))
            atomicOr(err, ERR_BAD_TRACE);
    }
    if (threadIdx.x == 0) {
        off[nb] = n;
        *nbatches = nb;
    }
}

cudaError_t launch_find_batches(const hirace_event *ev, uint32_t n, const Scratch &s, unsigned int *err,
                                int sm_count, cudaStream_t st)
{
    (void)sm_count;
    note_launches(1);
    k_batches<<<1, kFindThreads, sizeof(FindSmem), st>>>(ev, n, s.batch_off, s.nbatches, s.batch_ctr, err,
                                                         s.grid_bar);
    return cudaGetLastError();
}

/* ---------------------------------------------------------------------------------------- */
/* a7: collect = order-preserving compaction of RACE records (keys come out sorted: global   */
/* words first, then shared words block-major)                                               */
/* ---------------------------------------------------------------------------------------- */

/* the standalone collect kernel (k_collect<R>) and its launcher live in replay.cu, next to
 * the fused collect, instantiated per record layout */

/* ---------------------------------------------------------------------------------------- */
/* a8: grid-epoch wrap — every access before a grid barrier happens-before every later one,  */
/* so non-RACE records can restart at INIT; RACE records keep their class and get the        */
/* reserved epoch 255 so no later epoch compares equal (no spurious upgrades).               */
/* ---------------------------------------------------------------------------------------- */

__global__ void k_rebase(unsigned long long *shadow, uint64_t nwords)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nwords; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t o = shadow[i];
        if (st_of(o) >= ST_RACE_W)
            shadow[i] = (o & ~((uint64_t)255 << SH_G)) | ((uint64_t)255 << SH_G);
        else if (o)
            shadow[i] = 0;
    }
}

cudaError_t launch_rebase(const hirace_dev_ctx &c, uint64_t shadow_words, cudaStream_t st)
{
    note_launches(1);
    k_rebase<<<148 * 8, 256, 0, st>>>(c.shadow, shadow_words);
    return cudaGetLastError();
}

/* ---------------------------------------------------------------------------------------- */
/* a10: owner bucketing (stable counting sort by owner rank)                                 */
/* ---------------------------------------------------------------------------------------- */

constexpr int kBucketThreads = 256;
constexpr int kBucketTile = 4096;
constexpr int kMaxRanks = 32;

constexpr uint32_t kShardChunkLog2 = 14; /* owner granularity: 2^14 words = 64 KiB */

/* owner rank of an access: global words by 64 KiB chunk, shared words by block (block mod
 * nranks), so all of a block's shared accesses meet on one rank whichever rank traced them */
__device__ __forceinline__ uint32_t owner_of(const hirace_event &e, int nranks, uint32_t block_threads)
{
    if (e.addr & HIRACE_SHARED_BIT)
        return (uint32_t)((e.tid / block_threads) % (uint32_t)nranks);
    return (uint32_t)((((e.addr & ~HIRACE_SHARED_BIT) >> 2) >> kShardChunkLog2) % (uint64_t)nranks);
}

/* global byte address -> the owner's shard-local byte address (chunk c of the owner becomes
 * local chunk c / nranks); shared addresses are unchanged */
__device__ __forceinline__ uint64_t shard_local_addr(uint64_t addr, int nranks)
{
    if (addr & HIRACE_SHARED_BIT)
        return addr;
    const uint64_t word = addr >> 2;
    const uint64_t chunk = word >> kShardChunkLog2;
    const uint64_t local = ((chunk / (uint64_t)nranks) << kShardChunkLog2) | (word & ((1u << kShardChunkLog2) - 1));
    return (local << 2) | (addr & 3u);
}

__global__ void __launch_bounds__(kBucketThreads) k_bucket_hist(const hirace_event *__restrict__ in, uint32_t n,
                                                                int nranks, uint32_t block_threads, uint32_t *tile_hist,
                                                                unsigned int *err)
{
    __shared__ uint32_t s_h[kMaxRanks];
    if (threadIdx.x < kMaxRanks)
        s_h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * kBucketTile;
    for (int it = 0; it < kBucketTile / kBucketThreads; it++) {
        uint64_t i = base + (uint64_t)it * kBucketThreads + threadIdx.x;
        if (i < n) {
            const hirace_event e = in[i];
            atomicAdd(&s_h[owner_of(e, nranks, block_threads)], 1u);
            /* a 16-byte event cannot be split: a global access straddling two owner chunks
             * needs the wire format (hirace_bucket_wire) */
            const uint32_t szl = (e.meta >> 2) & 7u;
            if (nranks > 1 && !(e.addr & HIRACE_SHARED_BIT) && szl > 2) {
                const uint64_t w0 = e.addr >> 2, w1 = w0 + (szl <= 4 ? (1u << (szl - 2)) : 1u) - 1;
                if ((w0 >> kShardChunkLog2) != (w1 >> kShardChunkLog2))
                    atomicOr(err, hirace::ERR_BAD_TRACE);
            }
        }
    }
    __syncthreads();
    if (threadIdx.x < (unsigned)nranks)
        tile_hist[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x] = s_h[threadIdx.x];
}

/* exclusive scan over tile_hist laid out owner-major [owner][tile]; counts per owner */
__global__ void __launch_bounds__(1024) k_bucket_scan(uint32_t *tile_hist, uint32_t ntiles, int nranks,
                                                      unsigned long long *d_counts)
{
    __shared__ unsigned long long s_w[32];
    __shared__ unsigned long long s_carry;
    const uint64_t total = (uint64_t)ntiles * nranks;
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (threadIdx.x == 0)
        s_carry = 0;
    __syncthreads();
    for (uint64_t b0 = 0; b0 < total; b0 += 1024) {
        uint64_t i = b0 + threadIdx.x;
        unsigned long long v = i < total ? tile_hist[i] : 0, x = v;
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
            if ((int)lane >= o)
                x += y;
        }
        if (lane == 31)
            s_w[wid] = x;
        __syncthreads();
        if (wid == 0) {
            unsigned long long t = s_w[lane];
            for (int o = 1; o < 32; o <<= 1) {
                unsigned long long y = __shfl_up_sync(0xffffffffu, t, o);
                if ((int)lane >= o)
                    t += y;
            }
            s_w[lane] = t;
        }
        __syncthreads();
        if (i < total)
            tile_hist[i] = (uint32_t)(s_carry + (wid ? s_w[wid - 1] : 0) + x - v);
        __syncthreads();
        if (threadIdx.x == 0)
            s_carry += s_w[31];
        __syncthreads();
    }
    /* per-owner counts = difference of consecutive owner starts */
    if (threadIdx.x < (unsigned)nranks) {
        uint64_t start = tile_hist[(uint64_t)threadIdx.x * ntiles];
        uint64_t next = threadIdx.x + 1 < (unsigned)nranks ? tile_hist[(uint64_t)(threadIdx.x + 1) * ntiles] : s_carry;
        d_counts[threadIdx.x] = next - start;
    }
}

__global__ void __launch_bounds__(kBucketThreads) k_bucket_scatter(const hirace_event *__restrict__ in, uint32_t n,
                                                                   int nranks, uint32_t block_threads,
                                                                   const uint32_t *__restrict__ tile_off,
                                                                   hirace_event *out)
{
    __shared__ uint32_t s_run[kMaxRanks];
    __shared__ uint32_t s_wc[kBucketThreads / 32][kMaxRanks];
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (threadIdx.x < kMaxRanks)
        s_run[threadIdx.x] = threadIdx.x < (unsigned)nranks ? tile_off[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x] : 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * kBucketTile;
    for (int it = 0; it < kBucketTile / kBucketThreads; it++) {
        const uint64_t i = base + (uint64_t)it * kBucketThreads + threadIdx.x;
        hirace_event e{0, 0, 0};
        uint32_t own = 0xffffffffu;
        if (i < n) {
            e = in[i];
            own = owner_of(e, nranks, block_threads);
        }
        const uint32_t peers = __match_any_sync(0xffffffffu, own);
        const uint32_t rank_in_warp = __popc(peers & ((1u << lane) - 1));
        if (threadIdx.x < kBucketThreads)
            for (int r = lane; r < kMaxRanks; r += 32)
                s_wc[wid][r] = 0;
        __syncwarp();
        if (own != 0xffffffffu && rank_in_warp == 0)
            s_wc[wid][own] = __popc(peers);
        __syncthreads();
        if (own != 0xffffffffu) {
            uint32_t before = s_run[own];
            for (uint32_t w = 0; w < wid; w++)
                before += s_wc[w][own];
            e.addr = shard_local_addr(e.addr, nranks);
            out[before + rank_in_warp] = e;
        }
        __syncthreads();
        if (threadIdx.x < (unsigned)nranks) {
            uint32_t t = 0;
            for (int w = 0; w < kBucketThreads / 32; w++)
                t += s_wc[w][threadIdx.x];
            s_run[threadIdx.x] += t;
        }
        __syncthreads();
    }
}

cudaError_t launch_bucket(const hirace_dev_ctx &c, const hirace_event *in, uint32_t n, int nranks, int my_rank,
                          hirace_event *out, unsigned long long *d_counts, uint32_t *d_tile_hist, uint32_t ntiles,
                          cudaStream_t st)
{
    note_launches(3);
    (void)my_rank; /* shared words go to their block's owner (owner_of) */
    k_bucket_hist<<<ntiles, kBucketThreads, 0, st>>>(in, n, nranks, c.block_threads, d_tile_hist, c.error_flags);
    k_bucket_scan<<<1, 1024, 0, st>>>(d_tile_hist, ntiles, nranks, d_counts);
    k_bucket_scatter<<<ntiles, kBucketThreads, 0, st>>>(in, n, nranks, c.block_threads, d_tile_hist, out);
    return cudaGetLastError();
}

/* ---------------------------------------------------------------------------------------- */
/* a10: wire bucketing — one batch at a time, owner-grouped 8-byte wire records               */
/* ---------------------------------------------------------------------------------------- */

/* words covered by an event of size 1 << szl (sub-word accesses map to their word) */
__device__ __forceinline__ uint32_t words_of(uint32_t szl) { return szl <= 2 ? 1u : (szl <= 4 ? 1u << (szl - 2) : 0u); }

/* wire record of word k of event e, and its owner (include/hirace.h) */
__device__ __forceinline__ uint64_t wire_of(const hirace_event &e, uint32_t k, int nranks, uint32_t block_threads,
                                            uint32_t &owner)
{
    const bool sh = (e.addr & HIRACE_SHARED_BIT) != 0;
    const uint64_t word = ((e.addr & ~HIRACE_SHARED_BIT) >> 2) + k;
    uint64_t w;
    if (sh) {
        owner = (e.tid / block_threads) % (uint32_t)nranks;
        w = word;
    } else {
        const uint64_t chunk = word >> kShardChunkLog2;
        owner = (uint32_t)(chunk % (uint64_t)nranks);
        w = ((chunk / (uint64_t)nranks) << kShardChunkLog2) | (word & ((1u << kShardChunkLog2) - 1));
    }
    if (w >= (1ull << 31) || e.tid >= (1u << 30)) { /* beyond the wire format: bad input */
        owner = 0xffffffffu;
        return 0;
    }
    return w | (sh ? 0x80000000ull : 0ull) | ((uint64_t)e.tid << 32) | ((uint64_t)(e.meta & 3u) << 62);
}

__global__ void __launch_bounds__(kBucketThreads) k_wire_hist(const hirace_event *__restrict__ in, uint32_t lo,
                                                              uint32_t hi, int nranks, uint32_t block_threads,
                                                              uint32_t *tile_hist, unsigned int *err)
{
    __shared__ uint32_t s_h[kMaxRanks];
    if (threadIdx.x < kMaxRanks)
        s_h[threadIdx.x] = 0;
    __syncthreads();
    const uint32_t base = lo + blockIdx.x * kBucketTile;
    for (uint32_t it = 0; it < kBucketTile / kBucketThreads; it++) {
        const uint32_t i = base + it * kBucketThreads + threadIdx.x;
        if (i < hi) {
            const hirace_event e = in[i];
            const uint32_t nw = words_of((e.meta >> 2) & 7u);
            if (nw == 0)
                atomicOr(err, hirace::ERR_BAD_TRACE);
            for (uint32_t k = 0; k < nw; k++) {
                uint32_t own;
                (void)wire_of(e, k, nranks, block_threads, own);
                if (own < (uint32_t)nranks)
                    atomicAdd(&s_h[own], 1u);
                else
                    atomicOr(err, hirace::ERR_BAD_TRACE);
            }
        }
    }
    __syncthreads();
    if (threadIdx.x < (unsigned)nranks)
        tile_hist[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x] = s_h[threadIdx.x];
}

/* exclusive scan of this batch's [owner][tile] histogram, offset by the records of earlier
 * batches (*running, updated); the batch's per-owner counts go to counts_row[nranks] */
__global__ void __launch_bounds__(1024) k_wire_scan(uint32_t *tile_hist, uint32_t ntiles, int nranks,
                                                    unsigned long long *running, unsigned long long *counts_row,
                                                    unsigned long long *tile_off)
{
    __shared__ unsigned long long s_w[32];
    __shared__ unsigned long long s_carry;
    const uint64_t total = (uint64_t)ntiles * nranks;
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const unsigned long long base = *running;
    if (threadIdx.x == 0)
        s_carry = 0;
    __syncthreads();
    for (uint64_t b0 = 0; b0 < total; b0 += 1024) {
        const uint64_t i = b0 + threadIdx.x;
        const unsigned long long v = i < total ? tile_hist[i] : 0;
        unsigned long long x = v;
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
            if ((int)lane >= o)
                x += y;
        }
        if (lane == 31)
            s_w[wid] = x;
        __syncthreads();
        if (wid == 0) {
            unsigned long long t = s_w[lane];
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long y = __shfl_up_sync(0xffffffffu, t, o);
                if ((int)lane >= o)
                    t += y;
            }
            s_w[lane] = t;
        }
        __syncthreads();
        if (i < total)
            tile_off[i] = base + s_carry + (wid ? s_w[wid - 1] : 0) + x - v;
        __syncthreads();
        if (threadIdx.x == 0)
            s_carry += s_w[31];
        __syncthreads();
    }
    if (threadIdx.x < (unsigned)nranks) {
        const unsigned long long start = tile_off[(uint64_t)threadIdx.x * ntiles];
        const unsigned long long next =
            threadIdx.x + 1 < (unsigned)nranks ? tile_off[(uint64_t)(threadIdx.x + 1) * ntiles] : base + s_carry;
        counts_row[threadIdx.x] = next - start;
    }
    __syncthreads();
    if (threadIdx.x == 0)
        *running = base + s_carry;
}

/* scatter: each word gets a slot in its (owner) segment; order inside a batch is free
 * (PAPER.md L177), so slots are taken with warp-aggregated shared-memory counters */
/* peer != nullptr (peer dispatch, hirace_dispatch_wire): the record goes straight to its
 * owner's receive buffer peer[owner] (its own memory, or a peer GPU's / another process's
 * buffer mapped through CUDA IPC, stores travelling over NVLink), at the slot given by the
 * per-owner offsets in tile_off; no capacity check (the offsets come from exchanged counts) */
__global__ void __launch_bounds__(kBucketThreads) k_wire_scatter(const hirace_event *__restrict__ in, uint32_t lo,
                                                                 uint32_t hi, int nranks, uint32_t block_threads,
                                                                 const unsigned long long *__restrict__ tile_off,
                                                                 unsigned long long *out, uint64_t cap,
                                                                 unsigned int *err,
                                                                 unsigned long long *const *__restrict__ peer)
{
    __shared__ unsigned long long s_run[kMaxRanks];
    const uint32_t lane = threadIdx.x & 31;
    if (threadIdx.x < (unsigned)nranks)
        s_run[threadIdx.x] = tile_off[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x];
    __syncthreads();
    const uint32_t base = lo + blockIdx.x * kBucketTile;
    for (uint32_t it = 0; it < kBucketTile / kBucketThreads; it++) {
        const uint32_t i = base + it * kBucketThreads + threadIdx.x;
        hirace_event e{0, 0, 0};
        uint32_t nw = 0;
        if (i < hi) {
            e = in[i];
            nw = words_of((e.meta >> 2) & 7u);
        }
        const uint32_t maxw = __reduce_max_sync(0xffffffffu, nw);
        for (uint32_t k = 0; k < maxw; k++) {
            uint32_t own = 0xffffffffu;
            uint64_t w = 0;
            if (k < nw)
                w = wire_of(e, k, nranks, block_threads, own); /* own = ~0: invalid, skipped (hist flagged it) */
            const uint32_t peers = __match_any_sync(0xffffffffu, own);
            const int leader = __ffs(peers) - 1;
            unsigned long long slot = 0;
            if (own != 0xffffffffu && (int)lane == leader)
                slot = atomicAdd(&s_run[own], (unsigned long long)__popc(peers));
            slot = __shfl_sync(0xffffffffu, slot, leader) + __popc(peers & ((1u << lane) - 1));
            if (own != 0xffffffffu) {
                if (peer)
                    __stcs(peer[own] + slot, (unsigned long long)w); /* streaming store to the owner */
                else if (slot < cap)
                    out[slot] = w;
                else
                    atomicOr(err, 8u); /* capacity exceeded: reported by the host call */
            }
        }
    }
}

cudaError_t launch_bucket_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, uint32_t block_threads,
                               unsigned long long *out, uint64_t cap, uint32_t *d_tile_hist,
                               unsigned long long *d_tile_off, unsigned long long *d_running,
                               unsigned long long *d_counts_row, unsigned int *err, cudaStream_t st)
{
    const uint32_t ntiles = (hi - lo + kBucketTile - 1) / kBucketTile;
    if (ntiles == 0)
        return cudaMemsetAsync(d_counts_row, 0, nranks * sizeof(unsigned long long), st);
    note_launches(3);
    k_wire_hist<<<ntiles, kBucketThreads, 0, st>>>(in, lo, hi, nranks, block_threads, d_tile_hist, err);
    k_wire_scan<<<1, 1024, 0, st>>>(d_tile_hist, ntiles, nranks, d_running, d_counts_row, d_tile_off);
    if (out)
        k_wire_scatter<<<ntiles, kBucketThreads, 0, st>>>(in, lo, hi, nranks, block_threads, d_tile_off, out, cap, err,
                                                          nullptr);
    return cudaGetLastError();
}

/* per-owner exclusive scan of one batch's [owner][tile] histogram, each owner's slots starting
 * at owner_base[owner] (its segment in that owner's receive buffer) */
__global__ void __launch_bounds__(1024) k_wire_scan_peer(const uint32_t *tile_hist, uint32_t ntiles, int nranks,
                                                         const unsigned long long *owner_base,
                                                         unsigned long long *tile_off)
{
    __shared__ unsigned long long s_w[32];
    __shared__ unsigned long long s_carry;
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int r = 0; r < nranks; r++) {
        if (threadIdx.x == 0)
            s_carry = owner_base[r];
        __syncthreads();
        for (uint32_t t0 = 0; t0 < ntiles; t0 += 1024) {
            const uint32_t t = t0 + threadIdx.x;
            const unsigned long long v = t < ntiles ? tile_hist[(uint64_t)r * ntiles + t] : 0;
            unsigned long long x = v;
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
                if ((int)lane >= o)
                    x += y;
            }
            if (lane == 31)
                s_w[wid] = x;
            __syncthreads();
            if (wid == 0) {
                unsigned long long q = s_w[lane];
                for (int o = 1; o < 32; o <<= 1) {
                    const unsigned long long y = __shfl_up_sync(0xffffffffu, q, o);
                    if ((int)lane >= o)
                        q += y;
                }
                s_w[lane] = q;
            }
            __syncthreads();
            if (t < ntiles)
                tile_off[(uint64_t)r * ntiles + t] = s_carry + (wid ? s_w[wid - 1] : 0) + x - v;
            __syncthreads();
            if (threadIdx.x == 0)
                s_carry += s_w[31];
            __syncthreads();
        }
    }
}

cudaError_t launch_dispatch_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, uint32_t block_threads,
                                 unsigned long long *const *d_peer, const unsigned long long *d_owner_base,
                                 uint32_t *d_tile_hist, unsigned long long *d_tile_off, unsigned int *err,
                                 cudaStream_t st)
{
    const uint32_t ntiles = (hi - lo + kBucketTile - 1) / kBucketTile;
    if (ntiles == 0)
        return cudaSuccess;
    note_launches(3);
    k_wire_hist<<<ntiles, kBucketThreads, 0, st>>>(in, lo, hi, nranks, block_threads, d_tile_hist, err);
    k_wire_scan_peer<<<1, 1024, 0, st>>>(d_tile_hist, ntiles, nranks, d_owner_base, d_tile_off);
    k_wire_scatter<<<ntiles, kBucketThreads, 0, st>>>(in, lo, hi, nranks, block_threads, d_tile_off, nullptr, 0, err,
                                                      d_peer);
    return cudaGetLastError();
}

/* a11 + counters: the whole context reset as ONE launch (shadow := INIT, reports, stats and
 * error flags := 0) instead of four memsets */
__global__ void __launch_bounds__(256) k_reset(uint4 *shadow, uint64_t n16, unsigned long long *report_count,
                                               unsigned long long *stats, unsigned int *err)
{
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n16; i += stride)
        __stcs(shadow + i, make_uint4(0, 0, 0, 0));
    if (blockIdx.x == 0 && threadIdx.x < 4)
        stats[threadIdx.x] = 0;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *report_count = 0;
        *err = 0;
    }
}

cudaError_t launch_reset(void *shadow, uint64_t bytes, unsigned long long *report_count, unsigned long long *stats,
                         unsigned int *err, int sm_count, cudaStream_t st)
{
    const uint64_t n16 = bytes / 16;
    uint64_t blocks = (n16 + 255) / 256;
    const uint64_t cap = (uint64_t)(sm_count > 0 ? sm_count : 148) * 8;
    blocks = blocks < 1 ? 1 : (blocks > cap ? cap : blocks);
    note_launches(1);
    k_reset<<<(unsigned)blocks, 256, 0, st>>>(reinterpret_cast<uint4 *>(shadow), n16, report_count, stats, err);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess && (bytes & 15)) /* shadow sizes are multiples of 4: a ragged 4/8/12-byte tail */
        e = cudaMemsetAsync(static_cast<char *>(shadow) + n16 * 16, 0, bytes & 15, st);
    return e;
}

/* ---- epoch reset (include/hirace.h hirace_set_reset_mode EPOCH; reading R19) -----
 * gep[0] = gbase (offset the replay adds to the trace's g), gep[1] = gnext (first epoch no
 * record of this check uses).  A reset clears the RACE records listed in the report buffer
 * (every RACE record was reported when it entered RACE) and moves gbase to gnext; when the
 * buffer overflowed it sweeps the whole shadow and starts over at 0. */
__global__ void __launch_bounds__(256) k_epoch_reset(hirace_dev_ctx c, uint64_t shadow_words)
{
    const unsigned long long nrep = *c.report_count;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t i0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (nrep <= c.report_capacity) {
        for (uint64_t i = i0; i < nrep; i += stride) {
            const uint64_t key = c.reports[i].key;
            uint64_t idx = key;
            if (key & HIRACE_SHARED_BIT)
                idx = c.global_words + ((key >> 32) & 0x7fffffffull) * c.smem_words + (key & 0xffffffffull);
            if (idx < shadow_words)
                c.shadow[idx] = 0ull;
        }
    } else {
        for (uint64_t i = i0; i < shadow_words; i += stride)
            __stcs(c.shadow + i, 0ull);
    }
}

__global__ void k_epoch_reset_fin(hirace_dev_ctx c, unsigned int *gep)
{
    if (threadIdx.x < 4)
        c.stats[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
        const bool covered = *c.report_count <= c.report_capacity;
        gep[0] = covered ? gep[1] : 0u;
        gep[1] = gep[0];
        *c.report_count = 0;
        *c.error_flags = 0;
    }
}

/* raw g of the last batch (batches are sorted by key, g in the top bits) */
__device__ __forceinline__ uint32_t last_batch_g(const hirace_event *ev, const uint32_t *off, const uint32_t *nbp)
{
    if (!ev || !nbp)
        return 0u;
    const uint32_t nb = *nbp;
    return nb ? (__ldg(&ev[off[nb - 1]].meta) >> 24) : 0u;
}

/* Before a replay: when gbase + the trace's largest g would pass 254 (or force), rebase: records
 * of this check (g >= gbase) keep their epochs minus gbase, older ones become INIT. */
__global__ void __launch_bounds__(256) k_epoch_prep(hirace_dev_ctx c, uint64_t shadow_words, const unsigned int *gep,
                                                    const hirace_event *ev, const uint32_t *off, const uint32_t *nbp,
                                                    int force)
{
    const uint32_t gbase = gep[0], gmax = last_batch_g(ev, off, nbp);
    if (!force && gbase + gmax <= 254u)
        return;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < shadow_words; i += stride) {
        const unsigned long long r = c.shadow[i];
        if (r == 0ull)
            continue;
        const uint32_t g = (uint32_t)(r >> SH_G) & 255u;
        const unsigned long long n =
            g >= gbase ? ((r & ~(255ull << SH_G)) | ((unsigned long long)(g - gbase) << SH_G)) : 0ull;
        if (n != r)
            c.shadow[i] = n;
    }
}

__global__ void k_epoch_prep_fin(unsigned int *gep, const hirace_event *ev, const uint32_t *off, const uint32_t *nbp,
                                 int force)
{
    if (threadIdx.x != 0)
        return;
    const uint32_t gmax = last_batch_g(ev, off, nbp);
    if (force || gep[0] + gmax > 254u) {
        gep[1] = gep[1] > gep[0] ? gep[1] - gep[0] : 0u;
        gep[0] = 0;
    }
    const uint32_t need = gep[0] + gmax + 1u;
    if (need > gep[1])
        gep[1] = need;
}

cudaError_t launch_epoch_reset(const hirace_dev_ctx &c, uint64_t shadow_words, unsigned int *gep, int sm_count,
                               cudaStream_t st)
{
    note_launches(2);
    k_epoch_reset<<<sm_count * 8, 256, 0, st>>>(c, shadow_words);
    k_epoch_reset_fin<<<1, 32, 0, st>>>(c, gep);
    return cudaGetLastError();
}

cudaError_t launch_epoch_prep(const hirace_dev_ctx &c, uint64_t shadow_words, unsigned int *gep,
                              const hirace_event *ev, const uint32_t *off, const uint32_t *nbp, int force,
                              int sm_count, cudaStream_t st)
{
    note_launches(2);
    k_epoch_prep<<<sm_count * 8, 256, 0, st>>>(c, shadow_words, gep, ev, off, nbp, force);
    k_epoch_prep_fin<<<1, 32, 0, st>>>(gep, ev, off, nbp, force);
    return cudaGetLastError();
}

/* ---- per-batch completion flags of the peer dispatch -------------------------
 * A sender releases global batch j to every owner after its dispatch kernels for j (stream
 * order): a system-scope release fence, then one red.add on each owner's flag j (peer memory).
 * An owner's stream waits (acquire loads) until its flag j reached target = (runs so far that
 * used j) x nranks, then replays batch j: replay of j overlaps the senders' later batches. */
__global__ void k_peer_release(unsigned int *const *flags, int nranks, uint32_t j0, uint32_t j1)
{
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    for (uint32_t q = threadIdx.x; q < (uint32_t)nranks * (j1 - j0 + 1u); q += blockDim.x) {
        unsigned int *f = flags[q % (uint32_t)nranks] + j0 + q / (uint32_t)nranks;
        asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(f) : "memory");
    }
}

__global__ void k_peer_wait(const unsigned int *flags, uint32_t j, uint32_t target)
{
    if (threadIdx.x == 0) {
        unsigned int v;
        for (;;) {
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + j) : "memory");
            if (v >= target)
                break;
            __nanosleep(256);
        }
    }
}

cudaError_t launch_peer_release(unsigned int *const *d_flags, int nranks, uint32_t j0, uint32_t j1, cudaStream_t st)
{
    note_launches(1);
    k_peer_release<<<1, 128, 0, st>>>(d_flags, nranks, j0, j1);
    return cudaGetLastError();
}

cudaError_t launch_peer_wait(const unsigned int *flags, uint32_t j, uint32_t target, cudaStream_t st)
{
    note_launches(1);
    k_peer_wait<<<1, 32, 0, st>>>(flags, j, target);
    return cudaGetLastError();
}

static std::atomic<unsigned long long> g_launches{0};

void note_launches(unsigned k)
{
    g_launches.fetch_add(k, std::memory_order_relaxed);
}

unsigned long long launch_count()
{
    return g_launches.load(std::memory_order_relaxed);
}

cudaError_t kernels_init(int device)
{
    (void)device;
    cudaError_t e = cudaFuncSetAttribute(k_batches, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(FindSmem));
    if (e != cudaSuccess)
        return e;
    if ((e = replay_init()) != cudaSuccess)
        return e;
    return window_init();
}

} // namespace hirace_impl
