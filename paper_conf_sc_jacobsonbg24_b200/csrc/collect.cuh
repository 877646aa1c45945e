/* collect.cuh — a7 collection as a grid-wide phase of a cooperative kernel.
 *
 * The flagged words are exactly the shadow records in a RACE state (RACE is sticky, one
 * record per word), so an order-preserving compaction of the shadow yields the unique,
 * key-sorted race set (global words first, then shared words block-major).  Each CTA owns a
 * contiguous range of 4096-word tiles: pass 1 counts its flagged words, one grid barrier
 * publishes the per-CTA counts, each CTA sums the counts before it, and pass 2 re-reads its
 * range (now L2-hot) and writes the records in order. */
#ifndef HIRACE_COLLECT_CUH
#define HIRACE_COLLECT_CUH

#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"

namespace hirace_impl {

constexpr int kCollectPerThread = 16; /* consecutive words per thread per tile */
static_assert(kCollectTile == 256 * kCollectPerThread, "collect tile = 256 threads x 16 words");

/* flagged-word count of the 16 words of this thread in tile t; words kept in v */
__device__ __forceinline__ uint32_t collect_load(const unsigned long long *shadow, uint64_t nwords, uint64_t w0,
                                                 ulonglong2 (&v)[kCollectPerThread / 2])
{
    uint32_t n = 0;
#pragma unroll
    for (int k = 0; k < kCollectPerThread / 2; k++) {
        const uint64_t wi = w0 + 2 * k;
        v[k] = wi + 1 < nwords ? reinterpret_cast<const ulonglong2 *>(shadow + w0)[k]
                               : make_ulonglong2(wi < nwords ? shadow[wi] : 0ull, 0ull);
        n += (hirace::st_of(v[k].x) >= hirace::ST_RACE_W) + (hirace::st_of(v[k].y) >= hirace::ST_RACE_W);
    }
    return n;
}

/* block-wide exclusive scan of `mine` over blockDim.x threads (multiple of 32, <= 1024);
 * returns the exclusive prefix and the block total in *total.  s_w: 32 words of smem. */
__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t mine, uint32_t *s_w, uint32_t *total)
{
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    uint32_t incl = mine;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if ((int)lane >= d)
            incl += y;
    }
    __syncthreads();
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

/* grid-wide collect; every thread of every CTA of a cooperative launch must call it.
 * cta_cnt: gridDim.x words of scratch.  Writes min(cap, total) records and *d_total. */
__device__ __forceinline__ void collect_phase(const hirace_dev_ctx &c, uint64_t nwords, hirace_race *out,
                                              uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt,
                                              unsigned int *bar, unsigned int &bar_epoch)
{
    __shared__ uint32_t s_w[32];
    __shared__ unsigned long long s_base;
    const uint64_t ntiles = (nwords + kCollectTile - 1) / kCollectTile;
    const uint64_t t0 = ntiles * blockIdx.x / gridDim.x, t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
    const uint32_t tpb = blockDim.x; /* threads cover a tile in kCollectTile / tpb rounds */
    ulonglong2 v[kCollectPerThread / 2];
    /* pass 1: count */
    uint32_t mine = 0;
    for (uint64_t t = t0; t < t1; t++)
        for (uint32_t r = threadIdx.x; r < kCollectTile / kCollectPerThread; r += tpb)
            mine += collect_load(c.shadow, nwords, t * kCollectTile + (uint64_t)r * kCollectPerThread, v);
    uint32_t cta_total;
    block_exclusive_scan(mine, s_w, &cta_total);
    if (threadIdx.x == 0)
        cta_cnt[blockIdx.x] = cta_total;
    grid_sync(bar, gridDim.x, bar_epoch);
    /* prefix of the CTAs before this one */
    unsigned long long part = 0;
    for (uint32_t k = threadIdx.x; k < blockIdx.x; k += tpb)
        part += __ldcg(&cta_cnt[k]);
#pragma unroll
    for (int d = 16; d > 0; d >>= 1)
        part += __shfl_xor_sync(0xffffffffu, part, d);
    __syncthreads();
    if (threadIdx.x == 0)
        s_base = 0;
    __syncthreads();
    if ((threadIdx.x & 31) == 0 && part)
        atomicAdd(&s_base, part);
    __syncthreads();
    unsigned long long base = s_base;
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
        *d_total = base + cta_total;
    /* pass 2: ordered write (skipped by CTAs without flagged words) */
    const uint64_t global_words = c.global_words;
    const uint64_t smem_words = c.smem_words ? c.smem_words : 1;
    for (uint64_t t = cta_total ? t0 : t1; t < t1; t++) {
        for (uint32_t r0 = 0; r0 < kCollectTile / kCollectPerThread; r0 += tpb) {
            const uint32_t r = r0 + threadIdx.x;
            const uint64_t w0 = t * kCollectTile + (uint64_t)r * kCollectPerThread;
            const uint32_t n = r < kCollectTile / kCollectPerThread ? collect_load(c.shadow, nwords, w0, v) : 0u;
            uint32_t round_total;
            const uint32_t excl = block_exclusive_scan(n, s_w, &round_total);
            uint64_t pos = base + excl;
            if (n) {
#pragma unroll
                for (int k = 0; k < kCollectPerThread; k++) {
                    const uint64_t o = (k & 1) ? v[k / 2].y : v[k / 2].x;
                    if (hirace::st_of(o) >= hirace::ST_RACE_W) {
                        if (pos < cap) {
                            const uint64_t wi = w0 + k;
                            hirace_race rr;
                            if (wi < global_words) {
                                rr.key = wi;
                            } else {
                                const uint64_t sidx = wi - global_words;
                                const uint64_t blk = sidx / smem_words;
                                rr.key = HIRACE_SHARED_BIT | (blk << 32) | (sidx - blk * smem_words);
                            }
                            rr.cls_and_epoch = hirace::race_class(hirace::st_of(o)) | (hirace::g_of(o) << 8);
                            rr.detect_tid = hirace::tid_of(o);
                            out[pos] = rr;
                        }
                        pos++;
                    }
                }
            }
            base += round_total;
        }
    }
}

} // namespace hirace_impl

#endif
