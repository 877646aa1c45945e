/*
 * hirace_kernels.cu — sm_100a kernels of the HiRace hot path.
 *
 *   k_find_batches / k_sort_batches  a9  batch discovery + validation (replay input sorted by
 *                                         (g,b,w))
 *   (k_replay, the a1-a9 hot kernel, lives in replay.cu)
 *   k_collect_*                       a7  order-preserving compaction of RACE records
 *   k_rebase                          a8  grid-epoch wrap sweep
 *   k_bucket_*                        a10 owner bucketing for the address-sharded mode
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
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

constexpr int kFindWarps = 8;
constexpr int kFindStack = 160;

__device__ __forceinline__ bool chunk_dirty(const hirace_event *ev, uint32_t lo, uint32_t hi)
{
    uint32_t q = lo > 1 ? lo : 1;
    if (q >= hi)
        return false;
    return batch_key_at(ev, q - 1) != batch_key_at(ev, hi - 1);
}

__global__ void __launch_bounds__(kFindWarps * 32) k_find_batches(const hirace_event *__restrict__ ev, uint32_t n,
                                                                  uint32_t *pos, uint32_t *count, uint32_t cap)
{
    __shared__ uint32_t s_lo[kFindWarps][kFindStack];
    __shared__ uint32_t s_len[kFindWarps][kFindStack];
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint32_t wg = blockIdx.x * kFindWarps + wid, nwarps = gridDim.x * kFindWarps;
    for (uint64_t t = wg; t * kFindChunk < n; t += nwarps) {
        uint32_t lo = (uint32_t)(t * kFindChunk);
        uint32_t len = min(kFindChunk, n - lo);
        int sp = 0;
        bool d = lane == 0 && chunk_dirty(ev, lo, lo + len);
        if (__shfl_sync(0xffffffffu, d ? 1 : 0, 0)) {
            if (lane == 0) {
                s_lo[wid][0] = lo;
                s_len[wid][0] = len;
            }
            sp = 1;
        }
        __syncwarp();
        while (sp > 0) {
            sp--;
            uint32_t clo = s_lo[wid][sp], clen = s_len[wid][sp];
            __syncwarp();
            if (clen <= 32) {
                uint32_t p = clo + lane;
                bool b = lane < clen && p >= 1 && batch_key_at(ev, p) != batch_key_at(ev, p - 1);
                if (b) {
                    uint32_t i = atomicAdd(count, 1u);
                    if (i < cap)
                        pos[i] = p;
                }
            } else {
                uint32_t sub = (clen + 31) / 32;
                uint32_t slo = clo + lane * sub;
                uint32_t shi = min(slo + sub, clo + clen);
                bool dd = slo < clo + clen && chunk_dirty(ev, slo, shi);
                uint32_t mask = __ballot_sync(0xffffffffu, dd);
                uint32_t rank = __popc(mask & ((1u << lane) - 1));
                if (dd && sp + rank < kFindStack) {
                    s_lo[wid][sp + rank] = slo;
                    s_len[wid][sp + rank] = shi - slo;
                }
                sp = min(sp + __popc(mask), kFindStack);
                __syncwarp();
            }
        }
    }
}

/* single CTA: sort boundary positions (bitonic in shared memory), emit batch_off[0..nb] and  */
/* check that batch keys strictly increase                                                   */
__global__ void __launch_bounds__(1024) k_sort_batches(const hirace_event *__restrict__ ev, uint32_t n,
                                                       const uint32_t *raw, const uint32_t *raw_count,
                                                       uint32_t *off, uint32_t *nbatches, uint32_t *batch_ctr,
                                                       unsigned int *err)
{
    extern __shared__ uint32_t s[];
    const uint32_t found = *raw_count;
    if (n == 0) {
        if (threadIdx.x == 0) {
            *nbatches = 0;
            off[0] = 0;
        }
        return;
    }
    if (found + 1 > HIRACE_MAX_BATCHES) {
        if (threadIdx.x == 0) {
            *nbatches = 0;
            atomicOr(err, ERR_BATCHES | ERR_BAD_TRACE);
        }
        return;
    }
    const uint32_t nb = found + 1;
    uint32_t P = 1;
    while (P < nb)
        P <<= 1;
    for (uint32_t i = threadIdx.x; i < P; i += blockDim.x)
        s[i] = i == 0 ? 0u : (i < nb ? raw[i - 1] : 0xffffffffu);
    __syncthreads();
    for (uint32_t k = 2; k <= P; k <<= 1) {
        for (uint32_t j = k >> 1; j > 0; j >>= 1) {
            for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) {
                uint32_t ixj = i ^ j;
                if (ixj > i) {
                    uint32_t a = s[i], b = s[ixj];
                    bool up = (i & k) == 0;
                    if ((a > b) == up) {
                        s[i] = b;
                        s[ixj] = a;
                    }
                }
            }
            __syncthreads();
        }
    }
    for (uint32_t i = threadIdx.x; i < nb; i += blockDim.x) {
        off[i] = s[i];
        batch_ctr[i] = 0; /* tile-claim counters of the replay kernel */
        if (i > 0 && !(batch_key_at(ev, s[i]) > batch_key_at(ev, s[i - 1])))
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
    cudaError_t e = cudaMemsetAsync(s.raw_count, 0, sizeof(uint32_t), st);
    if (e != cudaSuccess)
        return e;
    if (n > 1) {
        uint64_t chunks = (n + kFindChunk - 1) / kFindChunk;
        uint64_t ctas = (chunks + kFindWarps - 1) / kFindWarps;
        int grid = (int)(ctas < (uint64_t)sm_count * 4 ? ctas : (uint64_t)sm_count * 4);
        k_find_batches<<<grid, kFindWarps * 32, 0, st>>>(ev, n, s.raw_pos, s.raw_count, HIRACE_MAX_BATCHES - 1);
    }
    /* dynamic smem sized for the worst case; the kernel uses next_pow2(nb) of it */
    k_sort_batches<<<1, 1024, 32768 * sizeof(uint32_t), st>>>(ev, n, s.raw_pos, s.raw_count, s.batch_off,
                                                              s.nbatches, s.batch_ctr, err);
    return cudaGetLastError();
}

/* ---------------------------------------------------------------------------------------- */
/* a7: collect = order-preserving compaction of RACE records (keys come out sorted: global   */
/* words first, then shared words block-major)                                               */
/* ---------------------------------------------------------------------------------------- */

__global__ void __launch_bounds__(kCollectThreads) k_collect_count(const unsigned long long *__restrict__ shadow,
                                                                   uint64_t nwords, uint32_t *tile_counts)
{
    __shared__ uint32_t s_w[kCollectThreads / 32];
    const uint64_t base = (uint64_t)blockIdx.x * kCollectTile;
    uint32_t cnt = 0;
    for (int it = 0; it < kCollectTile / kCollectThreads / 2; it++) {
        uint64_t wi = base + ((uint64_t)it * kCollectThreads + threadIdx.x) * 2;
        if (wi + 1 < nwords) {
            ulonglong2 v = __ldcs(reinterpret_cast<const ulonglong2 *>(shadow + wi));
            cnt += (st_of(v.x) >= ST_RACE_W) + (st_of(v.y) >= ST_RACE_W);
        } else if (wi < nwords) {
            cnt += st_of(shadow[wi]) >= ST_RACE_W;
        }
    }
    cnt = __reduce_add_sync(0xffffffffu, cnt);
    if ((threadIdx.x & 31) == 0)
        s_w[threadIdx.x >> 5] = cnt;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t t = 0;
        for (int i = 0; i < kCollectThreads / 32; i++)
            t += s_w[i];
        tile_counts[blockIdx.x] = t;
    }
}

/* single CTA exclusive scan of tile counts; total -> *d_total */
__global__ void __launch_bounds__(1024) k_collect_scan(uint32_t *tile_counts, uint64_t ntiles,
                                                       unsigned long long *d_total)
{
    __shared__ unsigned long long s_w[32];
    __shared__ unsigned long long s_carry;
    if (threadIdx.x == 0)
        s_carry = 0;
    __syncthreads();
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (uint64_t b0 = 0; b0 < ntiles; b0 += 1024) {
        uint64_t i = b0 + threadIdx.x;
        unsigned long long v = i < ntiles ? tile_counts[i] : 0;
        unsigned long long x = v;
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
        unsigned long long excl = s_carry + (wid ? s_w[wid - 1] : 0) + x - v;
        if (i < ntiles)
            tile_counts[i] = (uint32_t)excl; /* offsets fit: at most shadow words < 2^37; see cap */
        __syncthreads();
        if (threadIdx.x == 0)
            s_carry += s_w[31];
        __syncthreads();
    }
    if (threadIdx.x == 0)
        *d_total = s_carry;
}

__global__ void __launch_bounds__(kCollectThreads) k_collect_write(const unsigned long long *__restrict__ shadow,
                                                                   uint64_t nwords, uint64_t global_words,
                                                                   uint32_t smem_words,
                                                                   const uint32_t *__restrict__ tile_off,
                                                                   hirace_race *out, uint64_t cap)
{
    __shared__ uint32_t s_w[kCollectThreads / 32];
    __shared__ uint32_t s_run;
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint64_t base = (uint64_t)blockIdx.x * kCollectTile;
    if (threadIdx.x == 0)
        s_run = 0;
    __syncthreads();
    const uint64_t toff = tile_off[blockIdx.x];
    for (int it = 0; it < kCollectTile / kCollectThreads; it++) {
        const uint64_t wi = base + (uint64_t)it * kCollectThreads + threadIdx.x;
        uint64_t o = wi < nwords ? shadow[wi] : 0;
        const bool f = st_of(o) >= ST_RACE_W;
        const uint32_t m = __ballot_sync(0xffffffffu, f);
        if (lane == 0)
            s_w[wid] = __popc(m);
        __syncthreads();
        uint32_t before = s_run;
        for (uint32_t w = 0; w < wid; w++)
            before += s_w[w];
        if (f) {
            const uint64_t posn = toff + before + __popc(m & ((1u << lane) - 1));
            if (posn < cap) {
                hirace_race r;
                if (wi < global_words) {
                    r.key = wi;
                } else {
                    const uint64_t sidx = wi - global_words;
                    const uint64_t blk = sidx / smem_words;
                    r.key = HIRACE_SHARED_BIT | (blk << 32) | (sidx - blk * smem_words);
                }
                r.cls_and_epoch = race_class(st_of(o)) | (g_of(o) << 8);
                r.detect_tid = tid_of(o);
                out[posn] = r;
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t t = 0;
            for (int w = 0; w < kCollectThreads / 32; w++)
                t += s_w[w];
            s_run += t;
        }
        __syncthreads();
    }
}

cudaError_t launch_collect(const hirace_dev_ctx &c, uint64_t shadow_words, const Scratch &s, hirace_race *out,
                           uint64_t cap, unsigned long long *d_total, cudaStream_t st)
{
    const uint64_t ntiles = s.ntiles;
    k_collect_count<<<(unsigned)ntiles, kCollectThreads, 0, st>>>(c.shadow, shadow_words, s.tile_counts);
    k_collect_scan<<<1, 1024, 0, st>>>(s.tile_counts, ntiles, d_total);
    k_collect_write<<<(unsigned)ntiles, kCollectThreads, 0, st>>>(c.shadow, shadow_words, c.global_words,
                                                                  c.smem_words ? c.smem_words : 1, s.tile_counts,
                                                                  out, cap);
    return cudaGetLastError();
}

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
    k_rebase<<<148 * 8, 256, 0, st>>>(c.shadow, shadow_words);
    return cudaGetLastError();
}

/* ---------------------------------------------------------------------------------------- */
/* a10: owner bucketing (stable counting sort by owner rank)                                 */
/* ---------------------------------------------------------------------------------------- */

constexpr int kBucketThreads = 256;
constexpr int kBucketTile = 4096;
constexpr int kMaxRanks = 32;

__device__ __forceinline__ uint32_t owner_of(const hirace_event &e, int nranks, int my_rank)
{
    if (e.addr & HIRACE_SHARED_BIT)
        return (uint32_t)my_rank;
    return (uint32_t)((((e.addr & ~HIRACE_SHARED_BIT) >> 2) >> 14) % (uint64_t)nranks);
}

__global__ void __launch_bounds__(kBucketThreads) k_bucket_hist(const hirace_event *__restrict__ in, uint32_t n,
                                                                int nranks, int my_rank, uint32_t *tile_hist)
{
    __shared__ uint32_t s_h[kMaxRanks];
    if (threadIdx.x < kMaxRanks)
        s_h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * kBucketTile;
    for (int it = 0; it < kBucketTile / kBucketThreads; it++) {
        uint64_t i = base + (uint64_t)it * kBucketThreads + threadIdx.x;
        if (i < n)
            atomicAdd(&s_h[owner_of(in[i], nranks, my_rank)], 1u);
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
                                                                   int nranks, int my_rank,
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
            own = owner_of(e, nranks, my_rank);
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
    (void)c;
    k_bucket_hist<<<ntiles, kBucketThreads, 0, st>>>(in, n, nranks, my_rank, d_tile_hist);
    k_bucket_scan<<<1, 1024, 0, st>>>(d_tile_hist, ntiles, nranks, d_counts);
    k_bucket_scatter<<<ntiles, kBucketThreads, 0, st>>>(in, n, nranks, my_rank, d_tile_hist, out);
    return cudaGetLastError();
}

cudaError_t kernels_init(int device)
{
    (void)device;
    return cudaFuncSetAttribute(k_sort_batches, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                32768 * (int)sizeof(uint32_t));
}

} // namespace hirace_impl
