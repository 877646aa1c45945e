/* collect.cuh — a7 collection as a grid-wide phase of a cooperative kernel.
 *
 * The flagged words are exactly the shadow records in a RACE state (RACE is sticky, one
 * record per word), so an order-preserving compaction of the shadow yields the unique,
 * key-sorted race set (global words first, then shared words block-major).  Instantiated per
 * record layout (record.cuh).  Each CTA owns a
 * contiguous range of 4096-word tiles: pass 1 counts its flagged words, one grid barrier
 * publishes the per-CTA counts, each CTA sums the counts before it, and pass 2 re-reads its
 * range (now L2-hot) and writes the records in order. */
#ifndef HIRACE_COLLECT_CUH
#define HIRACE_COLLECT_CUH

#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"
#include "record.cuh"

namespace hirace_impl {

constexpr int kCollectPerThread = 16; /* consecutive words per thread per tile */

/* epoch reset: records hold g + offset; collected rows carry the trace's g */
__device__ __forceinline__ uint32_t gsub(const hirace_dev_ctx &c) { return c.g_base ? *c.g_base : 0u; }
static_assert(kCollectTile == 256 * kCollectPerThread, "collect tile = 256 threads x 16 words");

/* flagged-word count of the 16 words of this thread in tile t; words kept in v (16-byte
 * vector loads: 2 records of 8 bytes or 4 compact records each) */
template <typename R>
__device__ __forceinline__ uint32_t collect_load(const R *shadow, uint64_t nwords, uint64_t w0,
                                                 R (&v)[kCollectPerThread])
{
    constexpr int per = 16 / sizeof(R);
    uint32_t n = 0;
#pragma unroll
    for (int k = 0; k < kCollectPerThread / per; k++) {
        const uint64_t wi = w0 + (uint64_t)per * k;
        if (wi + per <= nwords) {
            const uint4 q = reinterpret_cast<const uint4 *>(shadow + w0)[k];
            if (sizeof(R) == 8) {
                v[per * k] = (R)(((unsigned long long)q.y << 32) | q.x);
                v[per * k + 1] = (R)(((unsigned long long)q.w << 32) | q.z);
            } else {
                v[per * k] = (R)q.x;
                v[per * k + 1] = (R)q.y;
                v[per * k + 2] = (R)q.z;
                v[per * k + 3] = (R)q.w;
            }
        } else {
#pragma unroll
            for (int j = 0; j < per; j++)
                v[per * k + j] = wi + j < nwords ? shadow[wi + j] : (R)0;
        }
    }
#pragma unroll
    for (int k = 0; k < kCollectPerThread; k++)
        n += hirace::st_of(v[k]) >= hirace::ST_RACE_W;
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
template <typename R>
__device__ __forceinline__ void collect_phase(const hirace_dev_ctx &c, uint64_t nwords, hirace_race *out,
                                              uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt,
                                              unsigned int *bar, unsigned int &bar_epoch)
{
    __shared__ uint32_t s_w[32];
    __shared__ unsigned long long s_base;
    const uint64_t ntiles = (nwords + kCollectTile - 1) / kCollectTile;
    const uint64_t t0 = ntiles * blockIdx.x / gridDim.x, t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
    const uint32_t tpb = blockDim.x; /* threads cover a tile in kCollectTile / tpb rounds */
    R v[kCollectPerThread];
    const R *const shadow = shadow_as<R>(c);
    const Rec<R> rec(c);
    /* pass 1: count — a streaming read of the CTA's range: each warp takes 4 KB blocks, lane l
     * loading 16-byte vectors l, l+32, ... (every load instruction fully coalesced, 8 in flight
     * per lane); the order of the words does not matter for a count */
    uint32_t mine = 0;
    {
        constexpr uint32_t kVec = 16 / sizeof(R);            /* records per 16-byte vector    */
        constexpr uint32_t kBlockWords = 32 * 8 * kVec;      /* words per warp block (4 KB)   */
        const uint64_t wb = t0 * (uint64_t)kCollectTile;
        const uint64_t we = min(t1 * (uint64_t)kCollectTile, nwords);
        const uint32_t lane = threadIdx.x & 31, nwarp = blockDim.x >> 5;
        for (uint64_t b0 = wb + (uint64_t)(threadIdx.x >> 5) * kBlockWords; b0 < we;
             b0 += (uint64_t)nwarp * kBlockWords) {
            uint4 q[8];
            const uint4 *src = reinterpret_cast<const uint4 *>(shadow + b0);
            if (b0 + kBlockWords <= we) {
#pragma unroll
                for (int k = 0; k < 8; k++)
                    q[k] = __ldcs(src + k * 32 + lane);
            } else {
#pragma unroll
                for (int k = 0; k < 8; k++) {
                    const uint64_t w = b0 + (uint64_t)(k * 32 + lane) * kVec;
                    q[k] = w + kVec <= we ? __ldcs(src + k * 32 + lane) : make_uint4(0, 0, 0, 0);
                    if (w < we && w + kVec > we) { /* ragged tail: scalar records */
                        __align__(16) R t[kVec];
#pragma unroll
                        for (uint32_t j = 0; j < kVec; j++)
                            t[j] = w + j < we ? shadow[w + j] : (R)0;
                        q[k] = *reinterpret_cast<const uint4 *>(t);
                    }
                }
            }
#pragma unroll
            for (int k = 0; k < 8; k++) {
                const uint32_t xs[4] = {q[k].x, q[k].y, q[k].z, q[k].w};
#pragma unroll
                for (int j = 0; j < 4; j++) /* the state is in the low 5 bits of each record's
                                             * low word (u64: words 0 and 2; u32: every word) */
                    if (sizeof(R) == 4 || (j & 1) == 0)
                        mine += (xs[j] & 31u) >= hirace::ST_RACE_W;
            }
        }
    }
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
            const uint32_t n = r < kCollectTile / kCollectPerThread ? collect_load<R>(shadow, nwords, w0, v) : 0u;
            uint32_t round_total;
            const uint32_t excl = block_exclusive_scan(n, s_w, &round_total);
            uint64_t pos = base + excl;
            if (n) {
#pragma unroll
                for (int k = 0; k < kCollectPerThread; k++) {
                    const R o = v[k];
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
                            rr.cls_and_epoch = hirace::race_class(hirace::st_of(o)) | (((rec.g(o) - gsub(c)) & 255u) << 8);
                            rr.detect_tid = rec.tid(o);
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

/* Single-load variant of collect_phase for small shadows (every warp's share of its CTA's word
 * range is at most kRowsMax rows of 32 words): each warp reads its rows once, coalesced, keeps
 * them in registers with their ballot masks across the grid barrier, and writes its flagged
 * records in order after the CTA prefix — one shadow read and no block-wide scans.  Same
 * output as collect_phase.  Returns false (nothing done) when the shadow is too large. */
constexpr uint32_t kRowsMax = 8;

template <typename R>
__device__ __forceinline__ bool collect_phase_small(const hirace_dev_ctx &c, uint64_t nwords, hirace_race *out,
                                                    uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt,
                                                    unsigned int *bar, unsigned int &bar_epoch)
{
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    const uint64_t w0 = nwords * blockIdx.x / gridDim.x, w1 = nwords * (blockIdx.x + 1) / gridDim.x;
    const uint64_t rows = (w1 - w0 + 31) / 32;
    /* uniform across the grid (both paths must agree on every CTA's range): the largest CTA
     * range, in rows of 32 words, must fit kRowsMax rows per warp */
    const uint64_t max_rows = ((nwords + gridDim.x - 1) / gridDim.x + 31) / 32;
    if (max_rows > (uint64_t)kRowsMax * nwarp)
        return false;
    __shared__ uint32_t s_wc[32];
    __shared__ unsigned long long s_base;
    const R *const shadow = shadow_as<R>(c);
    const Rec<R> rec(c);
    const uint32_t r0 = (uint32_t)(rows * wid / nwarp), r1 = (uint32_t)(rows * (wid + 1) / nwarp);
    R v[kRowsMax];
    uint32_t m[kRowsMax];
    uint32_t mine = 0;
#pragma unroll
    for (uint32_t k = 0; k < kRowsMax; k++) {
        const uint64_t idx = w0 + (uint64_t)(r0 + k) * 32 + lane;
        v[k] = (r0 + k < r1 && idx < w1) ? __ldcg(shadow + idx) : (R)0;
    }
#pragma unroll
    for (uint32_t k = 0; k < kRowsMax; k++) {
        m[k] = __ballot_sync(0xffffffffu, hirace::st_of(v[k]) >= hirace::ST_RACE_W);
        mine += __popc(m[k]);
    }
    if (lane == 0)
        s_wc[wid] = mine;
    __syncthreads();
    uint32_t before = 0, total = 0;
    for (uint32_t w = 0; w < nwarp; w++) {
        const uint32_t x = s_wc[w];
        before += w < wid ? x : 0u;
        total += x;
    }
    if (threadIdx.x == 0)
        cta_cnt[blockIdx.x] = total;
    grid_sync(bar, gridDim.x, bar_epoch);
    /* prefix of the CTAs before this one */
    unsigned long long part = 0;
    for (uint32_t k = threadIdx.x; k < blockIdx.x; k += blockDim.x)
        part += __ldcg(&cta_cnt[k]);
#pragma unroll
    for (int d = 16; d > 0; d >>= 1)
        part += __shfl_xor_sync(0xffffffffu, part, d);
    if (threadIdx.x == 0)
        s_base = 0;
    __syncthreads();
    if (lane == 0 && part)
        atomicAdd(&s_base, part);
    __syncthreads();
    const unsigned long long base = s_base;
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
        *d_total = base + total;
    if (!total)
        return true;
    uint64_t pos = base + before;
    const uint64_t global_words = c.global_words;
    const uint64_t smem_words = c.smem_words ? c.smem_words : 1;
#pragma unroll
    for (uint32_t k = 0; k < kRowsMax; k++) {
        if ((m[k] >> lane) & 1u) {
            const uint64_t at = pos + __popc(m[k] & ((1u << lane) - 1u));
            if (at < cap) {
                const uint64_t wi = w0 + (uint64_t)(r0 + k) * 32 + lane;
                hirace_race rr;
                if (wi < global_words) {
                    rr.key = wi;
                } else {
                    const uint64_t sidx = wi - global_words;
                    const uint64_t blk = sidx / smem_words;
                    rr.key = HIRACE_SHARED_BIT | (blk << 32) | (sidx - blk * smem_words);
                }
                rr.cls_and_epoch = hirace::race_class(hirace::st_of(v[k])) | (((rec.g(v[k]) - gsub(c)) & 255u) << 8);
                rr.detect_tid = rec.tid(v[k]);
                out[at] = rr;
            }
        }
        pos += __popc(m[k]);
    }
    return true;
}

/* ---- report-buffer collection ("Collect = device sort + unique(key, max
 * class); fallback = shadow scan") -------------------------------------------------------
 * Every word that reaches RACE appends a report when its CAS enters RACE or upgrades the class
 * (replay.cu append_reports, hirace_device.cuh report_one), so while the buffer has not
 * overflowed the reported keys are exactly the flagged words.  For a large shadow with few
 * races this replaces the full shadow scan (config 5: 32 GiB) by a sort of the reports: one
 * CTA sorts the keys in shared memory, drops duplicates, and reads each word's final record
 * (class, g*, detecting thread) from the shadow.  Output = the scan's output (unique keys in
 * key order, which is shadow order). */
constexpr uint32_t kReportSortCap = 16384; /* keys sorted in shared memory (128 KB) */
constexpr int kReportThreads = 1024;

/* the report path applies: report mode on, and every report fits the buffer and the sort */
__device__ __forceinline__ bool reports_cover(const hirace_dev_ctx &c)
{
    const unsigned long long n = __ldcg(c.report_count);
    return n <= kReportSortCap && n <= c.report_capacity;
}

template <typename R>
__device__ __forceinline__ void collect_reports_cta(const hirace_dev_ctx &c, hirace_race *out, uint64_t cap,
                                                    unsigned long long *d_total, unsigned long long *s_keys)
{
    __shared__ uint32_t s_w[32];
    const unsigned long long n = __ldcg(c.report_count);
    if (n > kReportSortCap || n > c.report_capacity)
        return; /* the shadow scan collects */
    uint32_t P = 1;
    while (P < (uint32_t)n)
        P <<= 1;
    for (uint32_t i = threadIdx.x; i < P; i += blockDim.x)
        s_keys[i] = i < n ? __ldcg(&c.reports[i].key) : ~0ull;
    __syncthreads();
    for (uint32_t k = 2; k <= P; k <<= 1) { /* bitonic sort, ascending */
        for (uint32_t j = k >> 1; j > 0; j >>= 1) {
            for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) {
                const uint32_t ixj = i ^ j;
                if (ixj > i) {
                    const unsigned long long x = s_keys[i], y = s_keys[ixj];
                    if ((x > y) == ((i & k) == 0)) {
                        s_keys[i] = y;
                        s_keys[ixj] = x;
                    }
                }
            }
            __syncthreads();
        }
    }
    /* each thread: a contiguous run of sorted keys; keep first occurrences whose record is RACE */
    const uint32_t per = (P + blockDim.x - 1) / blockDim.x;
    const uint32_t lo = threadIdx.x * per, hi = min(lo + per, (uint32_t)n);
    const R *const shadow = shadow_as<R>(c);
    const Rec<R> rec(c);
    const uint64_t smem_words = c.smem_words ? c.smem_words : 1;
    uint32_t mine = 0;
    for (uint32_t i = lo; i < hi; i++)
        mine += (i == 0 || s_keys[i] != s_keys[i - 1]) ? 1u : 0u;
    uint32_t total;
    uint64_t pos = block_exclusive_scan(mine, s_w, &total);
    for (uint32_t i = lo; i < hi; i++) {
        const unsigned long long key = s_keys[i];
        if (i != 0 && key == s_keys[i - 1])
            continue;
        const uint64_t idx = (key & HIRACE_SHARED_BIT)
                                 ? c.global_words + ((key >> 32) & 0x7fffffffull) * smem_words + (key & 0xffffffffull)
                                 : key;
        const R o = (R)__ldcg(shadow + idx);
        if (pos < cap) {
            hirace_race rr;
            rr.key = key;
            rr.cls_and_epoch = hirace::race_class(hirace::st_of(o)) | (((rec.g(o) - gsub(c)) & 255u) << 8);
            rr.detect_tid = rec.tid(o);
            out[pos] = rr;
        }
        pos++;
    }
    if (threadIdx.x == 0)
        *d_total = total;
}

} // namespace hirace_impl

#endif
