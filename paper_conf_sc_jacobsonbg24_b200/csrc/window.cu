/*
 * window.cu — window-major replay: the per-access shadow-state update (§8(a) a1-a7) for
 * shadows far larger than L2 (config 5: 2^32 words, 32 GiB of records).
 *
 * Why.  The batch-major kernel (replay.cu) walks a batch's events in trace order.  On config 5
 * most shadow accesses are then first touches of random 32-byte sectors of a 32 GiB array: DRAM
 * row activations, not bytes, bound it (1.7e10 load+CAS pairs/s; profiles/r2/mb_patterns.json).
 * The same pairs in address order run at 9.8e10/s.  The trace fixes only the order of the batches
 * (g,b,w) for each word; inside a batch any order is a linear extension of happens-before
 * (PAPER.md L177), and different words never interact (the record is per element, PAPER.md
 * L162).  So the accesses can be regrouped by shadow window as long as every window keeps its
 * batches in order.
 *
 * Pipeline (one check; all kernels read sizes from device memory, so the step is one CUDA graph):
 *   k_w_prep       pass-1 items: each batch cut into parts of p1 events, in batch order
 *   k_w_hist1      per item, element accesses per digit d0 = low d0b bits of the window id
 *   k_w_scan       exclusive scan of the digit x item matrix (digit-major): output offsets
 *   k_w_scatter1   8-byte records into digit order; within an item (one batch) order is free
 *   [d1b > 0: a second counting sort on the high digit d1, over chunks of the pass-1 output
 *    cut into pieces at (d0, batch) segment boundaries, so batch order survives:
 *    k_w_hist2, k_w_scan, k_w_scatter2]
 *   k_w_scan       window starts from the per-window counts
 *   k_w_classify   heavy windows (more records than one SM should replay) / light windows
 *   k_w_hseg       batch starts inside every heavy window (binary search)
 *   k_w_heavy      heavy windows, all CTAs, global-shadow CAS path (replay_core.cuh), one grid
 *                  barrier per batch
 *   k_w_light      one CTA per light window: TMA bulk copy of the window's records into shared
 *                  memory (or zero fill when the window is stale: lazy reset), the records'
 *                  transitions with shared-memory CAS, __syncthreads where the batch changes,
 *                  TMA bulk copy back
 *   collect        report buffer (k_collect_reports), else stale windows := INIT and the scan
 * Record (8 bytes): lo = word-in-window:14 | kind:2 | f:16 (pass 1 of two: d1; final: batch
 * index), hi = tid.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "collect.cuh"
#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"
#include "record.cuh"
#include "replay_core.cuh"

namespace hirace_impl {

namespace {

constexpr int kPassThreads = 512;
constexpr int kLightThreads = 256;
constexpr uint32_t kRing = 1024; /* records per ring buffer (8 KB) */
constexpr uint32_t kMaxD0 = 1024, kMaxD1 = 4096;
using u64 = unsigned long long;

__device__ __forceinline__ u64 wrec(uint32_t word, uint32_t kind, uint32_t f, uint32_t tid)
{
    return ((u64)tid << 32) | (u64)(word | (kind << 14) | (f << 16));
}

__device__ __forceinline__ u64 ld_rec(const u64 *p)
{
    u64 v;
    asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

/* ---- a2 for the partition: the element accesses of one event --------------------------- */
struct Elems {
    uint64_t idx0; /* shadow index of the first element                          */
    uint32_t ne;   /* elements (0: skipped: filtered out, or invalid -> bad)     */
    uint32_t tid, kind;
};

/* Same validity rules as the batch-major decode (replay.cu): batch key, access size, thread
 * id, extent, filter; invalid events raise BAD_TRACE and are not checked. */
__device__ __forceinline__ Elems elems_of(const uint4 &e, uint32_t key, const hirace_dev_ctx &c, const geom &G,
                                          uint32_t tid_max, uint32_t &bad)
{
    Elems E;
    E.tid = e.z;
    E.kind = e.w & 3u;
    E.ne = 0;
    E.idx0 = 0;
    const uint32_t meta = e.w, szl = (meta >> 2) & 7u, gran = c.gran_log2;
    const bool sh = (int)e.y < 0;
    const uint64_t word = ((((uint64_t)(e.y & 0x7fffffffu)) << 32) | e.x) >> gran;
    const uint32_t ne = szl <= gran ? 1u : (1u << (szl - gran));
    bool sel = true;
    if (c.f_active)
        sel = (E.tid & c.f_tid_mask) == c.f_tid_match &&
              (sh ? (c.f_spaces & 2u) != 0 : ((c.f_spaces & 1u) != 0 && word >= c.f_glo && word < c.f_ghi));
    if (!sel)
        return E;
    const bool ok = (meta >> 5) == key && szl <= 4u && E.tid <= tid_max && (key >> 19) != 255u &&
                    (sh ? word + ne <= c.smem_words : word + ne <= c.global_words);
    if (!ok) {
        bad = 1;
        return E;
    }
    E.ne = ne;
    E.idx0 = sh ? c.global_words + (uint64_t)block_of(E.tid, G) * c.smem_words + word : word;
    return E;
}

/* ---- device-sized exclusive scan: three plain launches (reduce, scan of the partials, apply).
 * a[0 .. rows * (*cols) + extra) in place (cols null: extra elements); *total_out = the sum;
 * optional *ceil_out = ceil(sum / ceil_div); a check_total above cap raises ERR_CAPACITY and
 * sets *abort (every later window kernel then stands down).  G = the grid of the reduce and
 * apply launches (a kernel argument, so every launch splits the array the same way). */
__device__ __forceinline__ uint64_t scan_n(uint32_t rows, const uint32_t *cols, uint32_t extra)
{
    return (cols ? (uint64_t)rows * *cols : 0ull) + extra;
}

__global__ void __launch_bounds__(1024) k_w_scan_reduce(const uint32_t *a, uint32_t rows, const uint32_t *cols,
                                                        uint32_t extra, uint32_t G, uint32_t *partials,
                                                        const unsigned long long *check_total, uint64_t cap,
                                                        uint32_t *abort, unsigned int *err)
{
    __shared__ uint32_t s_w[32];
    if (*abort)
        return;
    if (check_total && *check_total > cap) { /* the records would not fit rec1 / rec2 */
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            atomicOr(err, ERR_CAPACITY);
            atomicExch(abort, 1u);
        }
        return;
    }
    const uint64_t n = scan_n(rows, cols, extra), chunk = (n + G - 1) / G;
    const uint64_t lo = min(n, chunk * blockIdx.x), hi = min(n, lo + chunk);
    uint32_t sum = 0;
    for (uint64_t i = lo + threadIdx.x; i < hi; i += blockDim.x)
        sum += a[i];
    uint32_t tot;
    block_exclusive_scan(sum, s_w, &tot);
    if (threadIdx.x == 0)
        partials[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(1024) k_w_scan_partials(uint32_t *partials, uint32_t G, uint32_t *total_out,
                                                          uint32_t *ceil_out, uint32_t ceil_div, const uint32_t *abort)
{
    __shared__ uint32_t s_w[32];
    if (*abort)
        return;
    const uint32_t v = threadIdx.x < G ? partials[threadIdx.x] : 0u;
    uint32_t tot;
    const uint32_t ex = block_exclusive_scan(v, s_w, &tot);
    if (threadIdx.x < G)
        partials[threadIdx.x] = ex;
    if (threadIdx.x == 0) {
        if (total_out)
            *total_out = tot;
        if (ceil_out)
            *ceil_out = (uint32_t)(((uint64_t)tot + ceil_div - 1) / ceil_div);
    }
}

__global__ void __launch_bounds__(1024) k_w_scan_apply(uint32_t *a, uint32_t rows, const uint32_t *cols, uint32_t extra,
                                                       uint32_t G, const uint32_t *partials, const uint32_t *abort)
{
    __shared__ uint32_t s_w[32];
    if (*abort)
        return;
    const uint64_t n = scan_n(rows, cols, extra), chunk = (n + G - 1) / G;
    const uint64_t lo = min(n, chunk * blockIdx.x), hi = min(n, lo + chunk);
    uint32_t run = partials[blockIdx.x];
    constexpr int PER = 4;
    for (uint64_t base = lo; base < hi; base += (uint64_t)blockDim.x * PER) {
        uint32_t v[PER], mine = 0;
        const uint64_t i0 = base + (uint64_t)threadIdx.x * PER;
#pragma unroll
        for (int k = 0; k < PER; k++) {
            v[k] = i0 + k < hi ? a[i0 + k] : 0u;
            mine += v[k];
        }
        uint32_t tile;
        uint32_t ex = block_exclusive_scan(mine, s_w, &tile) + run;
#pragma unroll
        for (int k = 0; k < PER; k++) {
            if (i0 + k < hi)
                a[i0 + k] = ex;
            ex += v[k];
        }
        run += tile;
        __syncthreads(); /* s_w reuse */
    }
}

/* ---- pass-1 items (one CTA): each batch cut into parts of p1 events --------------------- */
__global__ void __launch_bounds__(1024) k_w_prep(const hirace_event *ev, const uint32_t *off, const uint32_t *nbp,
                                                 WinDev W, unsigned int *err)
{
    __shared__ uint32_t s_w[32];
    const uint32_t nb = *nbp;
    uint32_t run = 0;
    for (uint32_t b0 = 0; b0 < nb; b0 += blockDim.x) {
        const uint32_t b = b0 + threadIdx.x;
        uint32_t parts = 0;
        if (b < nb) {
            const uint32_t len = off[b + 1] - off[b];
            parts = (len + W.p1 - 1) / W.p1;
            W.batch_key[b] = __ldg(&ev[off[b]].meta) >> 5;
        }
        uint32_t tot;
        const uint32_t ex = block_exclusive_scan(parts, s_w, &tot) + run;
        if (b < nb) {
            W.item1_first[b] = ex;
            if (ex + parts <= W.items1_cap)
                for (uint32_t p = 0; p < parts; p++) {
                    const uint32_t s0 = off[b] + p * W.p1;
                    const uint32_t s1 = min(off[b + 1], s0 + W.p1);
                    W.items1[ex + p] = make_uint4(s0, s1, b, 0);
                }
        }
        run += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        W.item1_first[nb] = run;
        W.aux[kAuxItems1] = run;
        if (run > W.items1_cap) {
            atomicOr(err, ERR_CAPACITY);
            W.aux[kAuxAbort] = 1;
        }
    }
}

/* pass 1: per item, element accesses per digit d0 (count) or their records (scatter) */
template <bool SCATTER>
__global__ void __launch_bounds__(kPassThreads) k_w_pass1(hirace_dev_ctx c, const uint4 *__restrict__ ev, WinDev W)
{
    __shared__ uint32_t s_cnt[kMaxD0];
    __shared__ uint32_t s_items;
    if (W.aux[kAuxAbort])
        return;
    geom G = make_geom(c);
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t tid_max = total_threads > 0xffffffffull ? 0xffffffffu : (uint32_t)(total_threads - 1);
    const uint32_t ni = W.aux[kAuxItems1], R0 = 1u << W.d0b, wmask = (1u << W.wl) - 1u;
    const bool two = W.d1b != 0;
    uint32_t bad = 0;
    for (uint32_t item = blockIdx.x; item < ni; item += gridDim.x) {
        const uint4 it = W.items1[item];
        for (uint32_t d = threadIdx.x; d < R0; d += blockDim.x)
            s_cnt[d] = SCATTER ? W.count1[(uint64_t)d * ni + item] : 0u;
        if (threadIdx.x == 0)
            s_items = 0;
        __syncthreads();
        const uint32_t key = W.batch_key[it.z];
        uint32_t mine = 0;
        for (uint32_t i = it.x + threadIdx.x; i < it.y; i += blockDim.x) {
            const uint4 e = ld_event(ev + i);
            const Elems E = elems_of(e, key, c, G, tid_max, bad);
            mine += E.ne;
            for (uint32_t k = 0; k < E.ne; k++) {
                const uint64_t idx = E.idx0 + k;
                const uint32_t win = (uint32_t)(idx >> W.wl), d0 = win & (R0 - 1u);
                const uint32_t pos = atomicAdd(&s_cnt[d0], 1u);
                if (SCATTER)
                    W.rec1[pos] = wrec((uint32_t)idx & wmask, E.kind, two ? (win >> W.d0b) : it.z, E.tid);
            }
        }
        if (!SCATTER) {
            mine = __reduce_add_sync(0xffffffffu, mine);
            if ((threadIdx.x & 31) == 0 && mine)
                atomicAdd(&s_items, mine);
        }
        __syncthreads();
        if (!SCATTER && threadIdx.x == 0 && s_items)
            atomicAdd(W.elems, (unsigned long long)s_items);
        if (!SCATTER)
            for (uint32_t d = threadIdx.x; d < R0; d += blockDim.x) {
                const uint32_t v = s_cnt[d];
                W.count1[(uint64_t)d * ni + item] = v;
                if (!two && v)
                    atomicAdd(&W.win_cnt[d], v);
            }
        __syncthreads();
    }
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
}

/* start of pass-1 segment j = (d0 = j / nb, batch = j % nb) in rec1; j = R0 * nb: the end */
__device__ __forceinline__ uint32_t seg1(const WinDev &W, uint32_t j, uint32_t nb, uint32_t ni, uint32_t R0,
                                         uint32_t total1)
{
    if (j >= R0 * nb)
        return total1;
    return W.count1[(uint64_t)(j / nb) * ni + W.item1_first[j % nb]];
}

/* pass 2: chunks of the pass-1 output, cut into pieces at (d0, batch) segment boundaries;
 * count per d1 (+ per-window counts) or scatter into the final records */
template <bool SCATTER>
__global__ void __launch_bounds__(kPassThreads) k_w_pass2(WinDev W, const uint32_t *nbp)
{
    __shared__ uint32_t s_cnt[kMaxD1];
    __shared__ uint32_t s_win[kMaxD1];
    if (W.aux[kAuxAbort])
        return;
    const uint32_t nb = *nbp, ni = W.aux[kAuxItems1], R0 = 1u << W.d0b, R1 = 1u << W.d1b;
    const uint32_t total1 = W.aux[kAuxTotal1], nc = W.aux[kAuxChunks2];
    const uint32_t nseg = R0 * nb;
    for (uint32_t ch = blockIdx.x; ch < nc; ch += gridDim.x) {
        const uint32_t a = ch * W.p2, b = min(total1, a + W.p2);
        for (uint32_t d = threadIdx.x; d < R1; d += blockDim.x) {
            s_cnt[d] = SCATTER ? W.count2[(uint64_t)d * nc + ch] : 0u;
            s_win[d] = 0;
        }
        /* last segment j with seg1(j) <= a */
        uint32_t lo = 0, hi = nseg; /* seg1(lo) <= a < seg1(hi) */
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (seg1(W, mid, nb, ni, R0, total1) <= a)
                lo = mid;
            else
                hi = mid;
        }
        __syncthreads();
        for (uint32_t j = lo; j < nseg; j++) {
            const uint32_t s0 = max(a, seg1(W, j, nb, ni, R0, total1));
            if (s0 >= b)
                break;
            const uint32_t s1 = min(b, seg1(W, j + 1, nb, ni, R0, total1));
            if (s1 <= s0)
                continue;
            const uint32_t d0 = j / nb, batch = j % nb;
            for (uint32_t i = s0 + threadIdx.x; i < s1; i += blockDim.x) {
                const u64 r = ld_rec(W.rec1 + i);
                const uint32_t lo32 = (uint32_t)r, d1 = (lo32 >> 16) & (R1 - 1u);
                const uint32_t pos = atomicAdd(&s_cnt[d1], 1u);
                if (SCATTER)
                    W.rec2[pos] = ((r >> 32) << 32) | (u64)((lo32 & 0xffffu) | (batch << 16));
                else
                    atomicAdd(&s_win[d1], 1u);
            }
            __syncthreads(); /* the next piece (next batch of this d0) lands after this one */
            if (!SCATTER) {
                for (uint32_t d = threadIdx.x; d < R1; d += blockDim.x)
                    if (s_win[d]) {
                        atomicAdd(&W.win_cnt[(d << W.d0b) | d0], s_win[d]);
                        s_win[d] = 0;
                    }
                __syncthreads();
            }
        }
        if (!SCATTER)
            for (uint32_t d = threadIdx.x; d < R1; d += blockDim.x)
                W.count2[(uint64_t)d * nc + ch] = s_cnt[d];
        __syncthreads();
    }
}


/* ---- scatter with per-digit sector buffers ------------------------------------------------
 * Records go to their digit's output run through an 8-record shared-memory buffer; a flush
 * writes only whole 32-byte sectors (4 records) of the run, so DRAM never sees a partial-sector
 * write (which ECC turns into a read-modify-write) except at the two ends of each run of an
 * item.  A digit that receives more than 8 records between flushes writes the excess straight
 * to its final position (hot digits; still exact). */
constexpr uint32_t kMaxBufDigits = 1024;
template <uint32_t BUF, uint32_t RMAX> struct ScatterSmem {
    u64 buf[RMAX * BUF];
    uint32_t cnt[RMAX], done[RMAX], base[RMAX];
};

template <uint32_t BUF, uint32_t RMAX>
__device__ __forceinline__ void sc_put(ScatterSmem<BUF, RMAX> &S, u64 *out, uint32_t d, u64 rec)
{
    const uint32_t slot = atomicAdd(&S.cnt[d], 1u);
    if (slot - S.done[d] < BUF)
        S.buf[d * BUF + (slot & (BUF - 1))] = rec;
    else
        out[S.base[d] + slot] = rec;
}

/* thread per digit: write the buffered records up to the last whole sector (all if final);
 * 16-byte stores where the destination is 16-byte aligned */
template <uint32_t BUF, uint32_t RMAX>
__device__ __forceinline__ void sc_flush(ScatterSmem<BUF, RMAX> &S, u64 *out, uint32_t R, bool final)
{
    for (uint32_t d = threadIdx.x; d < R; d += blockDim.x) {
        const uint32_t c = S.cnt[d], dn = S.done[d], base = S.base[d];
        uint32_t e, nd;
        if (c - dn > BUF) { /* overflowed: [dn + BUF, c) went straight out */
            e = dn + BUF;
            nd = c;
        } else if (final) {
            e = nd = c;
        } else {
            const uint32_t al = (base + c) & ~3u; /* last sector boundary of the run so far */
            e = nd = al > base + dn ? al - base : dn;
        }
        const u64 *b = S.buf + d * BUF;
        uint32_t k = dn;
        if (k < e && ((base + k) & 1u)) {
            out[base + k] = b[k & (BUF - 1)];
            k++;
        }
        for (; k + 1 < e; k += 2) {
            const u64 x = b[k & (BUF - 1)], y = b[(k + 1) & (BUF - 1)];
            *reinterpret_cast<ulonglong2 *>(out + base + k) = make_ulonglong2(x, y);
        }
        if (k < e)
            out[base + k] = b[k & (BUF - 1)];
        S.done[d] = nd;
    }
}

/* pass 1 scatter: per item (one batch), records into digit d0 order; EV events per thread per
 * sub-tile between flushes */
template <uint32_t BUF, uint32_t RMAX, int EV>
__global__ void __launch_bounds__(kPassThreads) k_w_scatter1(hirace_dev_ctx c, const uint4 *__restrict__ ev, WinDev W)
{
    extern __shared__ __align__(128) unsigned char s_dyn[];
    ScatterSmem<BUF, RMAX> &S = *reinterpret_cast<ScatterSmem<BUF, RMAX> *>(s_dyn);
    if (W.aux[kAuxAbort])
        return;
    geom G = make_geom(c);
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t tid_max = total_threads > 0xffffffffull ? 0xffffffffu : (uint32_t)(total_threads - 1);
    const uint32_t ni = W.aux[kAuxItems1], R0 = 1u << W.d0b, wmask = (1u << W.wl) - 1u;
    const bool two = W.d1b != 0;
    const uint32_t T = blockDim.x;
    uint32_t bad = 0;
    for (uint32_t item = blockIdx.x; item < ni; item += gridDim.x) {
        const uint4 it = W.items1[item];
        for (uint32_t d = threadIdx.x; d < R0; d += T) {
            S.cnt[d] = 0;
            S.done[d] = 0;
            S.base[d] = W.count1[(uint64_t)d * ni + item];
        }
        __syncthreads();
        const uint32_t key = W.batch_key[it.z];
        uint4 nx[EV]; /* the next sub-tile's events are in flight while this one is scattered */
#pragma unroll
        for (int k = 0; k < EV; k++) {
            const uint32_t i = it.x + k * T + threadIdx.x;
            nx[k] = i < it.y ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
        }
        for (uint32_t i0 = it.x; i0 < it.y; i0 += T * EV) {
            uint4 e[EV];
#pragma unroll
            for (int k = 0; k < EV; k++) {
                e[k] = nx[k];
                const uint32_t i = i0 + T * EV + k * T + threadIdx.x;
                if (i < it.y)
                    nx[k] = ld_event(ev + i);
            }
#pragma unroll
            for (int k = 0; k < EV; k++) {
                if (i0 + k * T + threadIdx.x < it.y) {
                    const Elems E = elems_of(e[k], key, c, G, tid_max, bad);
                    for (uint32_t q = 0; q < E.ne; q++) {
                        const uint64_t idx = E.idx0 + q;
                        const uint32_t win = (uint32_t)(idx >> W.wl);
                        sc_put(S, W.rec1, win & (R0 - 1u),
                               wrec((uint32_t)idx & wmask, E.kind, two ? (win >> W.d0b) : it.z, E.tid));
                    }
                }
            }
            __syncthreads();
            sc_flush(S, W.rec1, R0, false);
            __syncthreads();
        }
        sc_flush(S, W.rec1, R0, true);
        __syncthreads();
    }
    (void)bad; /* reported by the count pass */
}

/* pass 2 scatter: per chunk of the pass-1 output, piece by piece ((d0, batch) segments in
 * order), records into digit d1 order; the record's f field becomes the batch index */
template <uint32_t BUF, uint32_t RMAX, int EV>
__global__ void __launch_bounds__(kPassThreads) k_w_scatter2(WinDev W, const uint32_t *nbp)
{
    extern __shared__ __align__(128) unsigned char s_dyn[];
    ScatterSmem<BUF, RMAX> &S = *reinterpret_cast<ScatterSmem<BUF, RMAX> *>(s_dyn);
    if (W.aux[kAuxAbort])
        return;
    const uint32_t nb = *nbp, ni = W.aux[kAuxItems1], R0 = 1u << W.d0b, R1 = 1u << W.d1b;
    const uint32_t total1 = W.aux[kAuxTotal1], nc = W.aux[kAuxChunks2];
    const uint32_t nseg = R0 * nb, T = blockDim.x;
    for (uint32_t ch = blockIdx.x; ch < nc; ch += gridDim.x) {
        const uint32_t a = ch * W.p2, b = min(total1, a + W.p2);
        for (uint32_t d = threadIdx.x; d < R1; d += T) {
            S.cnt[d] = 0;
            S.done[d] = 0;
            S.base[d] = W.count2[(uint64_t)d * nc + ch];
        }
        uint32_t lo = 0, hi = nseg; /* last segment j with seg1(j) <= a */
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (seg1(W, mid, nb, ni, R0, total1) <= a)
                lo = mid;
            else
                hi = mid;
        }
        __syncthreads();
        for (uint32_t j = lo; j < nseg; j++) {
            const uint32_t s0 = max(a, seg1(W, j, nb, ni, R0, total1));
            if (s0 >= b)
                break;
            const uint32_t s1 = min(b, seg1(W, j + 1, nb, ni, R0, total1));
            if (s1 <= s0)
                continue;
            const uint32_t batch = j % nb;
            u64 nx[EV]; /* next sub-tile in flight */
#pragma unroll
            for (int k = 0; k < EV; k++) {
                const uint32_t i = s0 + k * T + threadIdx.x;
                nx[k] = i < s1 ? ld_rec(W.rec1 + i) : 0ull;
            }
            for (uint32_t i0 = s0; i0 < s1; i0 += T * EV) {
                u64 r[EV];
#pragma unroll
                for (int k = 0; k < EV; k++) {
                    r[k] = nx[k];
                    const uint32_t i = i0 + T * EV + k * T + threadIdx.x;
                    if (i < s1)
                        nx[k] = ld_rec(W.rec1 + i);
                }
#pragma unroll
                for (int k = 0; k < EV; k++)
                    if (i0 + k * T + threadIdx.x < s1) {
                        const uint32_t lo32 = (uint32_t)r[k];
                        sc_put(S, W.rec2, (lo32 >> 16) & (R1 - 1u),
                               ((r[k] >> 32) << 32) | (u64)((lo32 & 0xffffu) | (batch << 16)));
                    }
                __syncthreads(); /* also: the next piece (next batch of this d0) lands after this one */
                sc_flush(S, W.rec2, R1, false);
                __syncthreads();
            }
        }
        sc_flush(S, W.rec2, R1, true);
        __syncthreads();
    }
}

/* heavy (more records than H) and light (non-empty) window lists */
__global__ void __launch_bounds__(256) k_w_classify(WinDev W)
{
    if (W.aux[kAuxAbort])
        return;
    const uint32_t total = W.win_cnt[W.nw];
    const uint32_t H = W.heavy_force ? W.heavy_force : max(1u << 18, total / (2u * W.light_ctas));
    for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < W.nw; w += gridDim.x * blockDim.x) {
        const uint32_t cnt = W.win_cnt[w + 1] - W.win_cnt[w];
        bool heavy = cnt > H;
        if (heavy) {
            const uint32_t k = atomicAdd(&W.aux[kAuxNHeavy], 1u);
            if (k < W.heavy_cap)
                W.heavy[k] = w;
            else
                heavy = false; /* list full: replayed as a light window (slower, still exact) */
        }
        if (!heavy && cnt) {
            const uint32_t k = atomicAdd(&W.aux[kAuxNLight], 1u);
            W.light[k] = w;
        }
    }
}

/* batch starts inside the heavy windows: hseg[i][b] = first record of window heavy[i] whose
 * batch is >= b (records are batch-sorted inside a window); one thread per (i, b) */
__global__ void __launch_bounds__(256) k_w_hseg(WinDev W, const uint32_t *nbp)
{
    if (W.aux[kAuxAbort])
        return;
    const uint32_t nb = *nbp, nh = min(W.aux[kAuxNHeavy], W.heavy_cap);
    for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < nh * (nb + 1); q += gridDim.x * blockDim.x) {
        const uint32_t i = q / (nb + 1), b = q % (nb + 1), w = W.heavy[i];
        uint32_t lo = W.win_cnt[w], hi = W.win_cnt[w + 1];
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (((uint32_t)W.rec2[mid] >> 16) < b)
                lo = mid + 1;
            else
                hi = mid;
        }
        W.hseg[i * (nb + 1) + b] = lo;
    }
}

/* heavy windows through the global shadow: all CTAs, grid barrier per batch (the batch-major
 * hot path of replay_core.cuh on the regrouped records) */
__global__ void __launch_bounds__(kReplayThreads, 2) k_w_heavy(hirace_dev_ctx c, WinDev W, const uint32_t *nbp)
{
    __shared__ __align__(16) unsigned char s_table[2048 + RAW_TABLE_BYTES];
    __shared__ unsigned long long s_stats[4];
    __shared__ uint32_t s_pre[kWinHeavyCap + 1];
    if (W.aux[kAuxAbort])
        return;
    const uint32_t nh = min(W.aux[kAuxNHeavy], W.heavy_cap);
    if (nh == 0)
        return;
    for (int i = threadIdx.x; i < (2048 + RAW_TABLE_BYTES) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(s_table)[i] = __ldg(reinterpret_cast<const uint4 *>(c.table) + i);
    if (threadIdx.x < 4)
        s_stats[threadIdx.x] = 0;
    const uint32_t nb = *nbp, cur = *W.cur_gen, wsz = 1u << W.wl;
    unsigned int epoch = 0;
    /* stale heavy windows := INIT (lazy reset) */
    {
        const uint64_t per = (uint64_t)wsz / 2; /* uint4 per window */
        const uint64_t nq = per * nh;
        for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < nq; q += (uint64_t)gridDim.x * blockDim.x) {
            const uint32_t w = W.heavy[q / per];
            if (W.gen[w] != cur)
                reinterpret_cast<uint4 *>(c.shadow)[(uint64_t)w * per + q % per] = make_uint4(0, 0, 0, 0);
        }
        grid_sync(W.bar + 1, gridDim.x, epoch);
        if (blockIdx.x == 0)
            for (uint32_t i = threadIdx.x; i < nh; i += blockDim.x)
                W.gen[W.heavy[i]] = cur;
    }
    geom G = make_geom(c);
    const Rec<u64> rec(c);
    const unsigned char *const raw = s_table + 2048;
    const uint32_t lane = threadIdx.x & 31, below = (1u << lane) - 1;
    const uint32_t tab_s = smem_u32(s_table);
    const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t wmask = wsz - 1u;
    Counters cnt{0, 0, 0, 0};
    for (uint32_t b = 0; b < nb; b++) {
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t run = 0;
            for (uint32_t i = 0; i < nh; i++) {
                s_pre[i] = run;
                run += W.hseg[i * (nb + 1) + b + 1] - W.hseg[i * (nb + 1) + b];
            }
            s_pre[nh] = run;
        }
        __syncthreads();
        const uint32_t tot = s_pre[nh];
        if (tot == 0)
            continue; /* uniform: no records of this batch in any heavy window */
        const Batch B = make_batch<u64>(W.batch_key[b], rec);
        uint32_t i, iend;
        warp_share(0, tot, warp_global, nwarps, lane, i, iend);
        for (; i - lane < iend; i += 32) {
            Lane L;
            L.ok = i < iend;
            L.idx = NONE;
            L.tid = 0;
            L.kind = 0;
            if (L.ok) {
                uint32_t k = 0;
                while (k + 1 < nh && s_pre[k + 1] <= i)
                    k++;
                const u64 r = ld_rec(W.rec2 + W.hseg[k * (nb + 1) + b] + (i - s_pre[k]));
                L.tid = (uint32_t)(r >> 32);
                L.kind = ((uint32_t)r >> 14) & 3u;
                L.idx = ((uint64_t)W.heavy[k] << W.wl) | ((uint32_t)r & wmask);
            }
            process_decoded<u64>(L, B, c, G, rec, raw, tab_s, cnt, lane, below);
        }
        grid_sync(W.bar + 1, gridDim.x, epoch);
    }
    flush_stats(c, cnt, s_stats, lane);
}

/* ---- light windows: one CTA per window, the window's records in shared memory ------------ */

__device__ __forceinline__ u64 lds64(const u64 *p)
{
    u64 v;
    asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(smem_u32(p)) : "memory");
    return v;
}
__device__ __forceinline__ u64 cas_shared(u64 *p, u64 cmp, u64 val)
{
    u64 v;
    asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(v) : "r"(smem_u32(p)), "l"(cmp), "l"(val) : "memory");
    return v;
}

/* one record per lane (ok lanes), record in shared memory: load, transition, CAS if changed;
 * lanes whose CAS lost are grouped per word and their leader folds them (warp-collective) */
__device__ __forceinline__ void light_step(u64 *sh, bool ok, uint32_t word, uint32_t tid, uint32_t kind,
                                           const Batch &B, uint32_t wbase_hi, uint64_t wbase, const hirace_dev_ctx &c,
                                           const geom &G, const Rec<u64> &rec, const unsigned char *raw,
                                           Counters &cnt, uint32_t lane, uint32_t below)
{
    (void)wbase_hi;
    u64 *p = sh + word;
    const u64 o = ok ? lds64(p) : 0ull;
    cnt.checked += ok;
    const uint32_t ent = raw[((uint32_t)(o & 31u) << 7) | rec.label(o, tid, kind, B.ep, G)];
    const u64 n = rec.next(o, ent, tid, B.ep);
    const bool do_cas = ok && n != o;
    cnt.cas += do_cas;
    const u64 prev = do_cas ? cas_shared(p, o, n) : o;
    const bool failed = do_cas && prev != o;
    const bool rep = (ent & E_REPORT) && do_cas && !failed;
    if (!__any_sync(0xffffffffu, failed || rep))
        return;
    uint32_t cls = 0, rtid = tid;
    if (rep) {
        const uint32_t cn = race_class(st_of(n)), co = race_class(st_of(o));
        cls = cn > co ? cn : 0u;
    }
    if (__any_sync(0xffffffffu, failed)) {
        const uint32_t peers = __match_any_sync(0xffffffffu, failed ? word : 0xffffffffu);
        const bool lead = failed && (peers & below) == 0;
        cls |= commit_groups<u64>(p, prev, lead ? peers : 0u, tid, kind, G, raw, B, rec, cnt, rtid, false);
    }
    if (__any_sync(0xffffffffu, cls != 0)) {
        Lane L;
        L.idx = wbase + word;
        L.tid = tid;
        L.kind = kind;
        L.ok = true;
        append_reports(c, cls, key_of_idx(L, c, G), B.graw, rtid, lane);
    }
}

/* Light-window replay.  Dynamic shared memory = [window records: 2^wl x 8 B][record ring:
 * 2 x kRing x 8 B].  Per window: the window comes in by TMA bulk copy (or is zero-filled when
 * stale), the window's access records stream through the two-buffer ring by TMA bulk copies
 * (chunk k+2 is requested as soon as chunk k is consumed), each tile of blockDim records is
 * processed by the whole CTA, with a __syncthreads where the batch changes, and the window goes
 * back by TMA bulk copy while the next window starts. */
__global__ void __launch_bounds__(kLightThreads, 4) k_w_light(hirace_dev_ctx c, WinDev W)
{
    extern __shared__ __align__(128) unsigned char s_dyn[];
    __shared__ __align__(16) unsigned char s_raw[RAW_TABLE_BYTES];
    __shared__ unsigned long long s_stats[4];
    __shared__ __align__(8) uint64_t s_mbar[3]; /* shadow, ring 0, ring 1 */
    __shared__ uint32_t s_w;
    if (W.aux[kAuxAbort])
        return;
    const uint32_t wsz = 1u << W.wl, wbytes = wsz * 8u, wmask = wsz - 1u;
    u64 *const sh = reinterpret_cast<u64 *>(s_dyn);
    u64 *const ring = sh + wsz;

    for (int i = threadIdx.x; i < RAW_TABLE_BYTES / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(s_raw)[i] = __ldg(reinterpret_cast<const uint4 *>(c.table + 2048) + i);
    if (threadIdx.x < 4)
        s_stats[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
        for (int k = 0; k < 3; k++)
            mbar_init(&s_mbar[k], 1);
        fence_mbar_init();
    }
    __syncthreads();
    geom G = make_geom(c);
    const Rec<u64> rec(c);
    const uint32_t lane = threadIdx.x & 31, below = (1u << lane) - 1;
    const uint32_t nl = W.aux[kAuxNLight], cur = *W.cur_gen;
    Counters cnt{0, 0, 0, 0};
    uint32_t ph_sh = 0, ph_ring = 0; /* mbarrier parities (bit k: ring buffer k) */
    for (;;) {
        if (threadIdx.x == 0)
            s_w = atomicAdd(&W.aux[kAuxQueue], 1u);
        __syncthreads();
        const uint32_t qi = s_w;
        if (qi >= nl)
            break;
        const uint32_t w = W.light[qi];
        const uint32_t beg = W.win_cnt[w], end = W.win_cnt[w + 1];
        u64 *const gw = reinterpret_cast<u64 *>(c.shadow) + ((uint64_t)w << W.wl);
        const bool fresh = W.gen[w] != cur;
        const uint32_t a0 = beg & ~1u, aend = (end + 1u) & ~1u; /* 16-byte aligned record range */
        const uint32_t nch = (aend - a0 + kRing - 1) / kRing;
        if (threadIdx.x == 0) {
            /* the previous window's bulk store must have read shared memory before reuse */
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            for (uint32_t k = 0; k < 2 && k < nch; k++) {
                const uint32_t s0 = a0 + k * kRing, m = min(kRing, aend - s0);
                mbar_arrive_expect_tx(&s_mbar[1 + k], m * 8u);
                bulk_g2s(ring + k * kRing, W.rec2 + s0, m * 8u, &s_mbar[1 + k]);
            }
            if (!fresh) {
                mbar_arrive_expect_tx(&s_mbar[0], wbytes);
                for (uint32_t o = 0; o < wbytes; o += 32768u)
                    bulk_g2s(s_dyn + o, reinterpret_cast<const unsigned char *>(gw) + o, min(32768u, wbytes - o),
                             &s_mbar[0]);
            }
        }
        __syncthreads();
        if (fresh) { /* lazy reset: a stale window is all INIT */
            for (uint32_t q = threadIdx.x; q < wsz / 2; q += blockDim.x)
                reinterpret_cast<uint4 *>(sh)[q] = make_uint4(0, 0, 0, 0);
        } else {
            mbar_wait(&s_mbar[0], ph_sh);
            ph_sh ^= 1u;
        }
        uint32_t cur_b = 0xffffffffu;
        for (uint32_t k = 0; k < nch; k++) {
            const uint32_t bi = k & 1u;
            mbar_wait(&s_mbar[1 + bi], (ph_ring >> bi) & 1u);
            ph_ring ^= 1u << bi;
            __syncthreads(); /* zero fill (first chunk) / previous chunk done */
            const uint32_t c0 = a0 + k * kRing;
            const u64 *const rb = ring + bi * kRing;
            const uint32_t lo = max(beg, c0), hi = min(end, c0 + kRing);
            if (cur_b == 0xffffffffu)
                cur_b = (uint32_t)rb[lo - c0] >> 16;
            for (uint32_t base = lo; base < hi; base += blockDim.x) {
                const uint32_t i = base + threadIdx.x;
                const bool valid = i < hi;
                const u64 rr = valid ? rb[i - c0] : 0ull;
                const uint32_t lo32 = (uint32_t)rr, my_b = valid ? lo32 >> 16 : 0xffffffffu;
                const uint32_t tid = (uint32_t)(rr >> 32), kind = (lo32 >> 14) & 3u, word = lo32 & wmask;
                const uint32_t hi_b = (uint32_t)rb[min(hi, base + blockDim.x) - 1u - c0] >> 16;
                const uint32_t lo_b = (uint32_t)rb[base - c0] >> 16;
                if (lo_b == hi_b) { /* one batch: concurrent; after the previous tile if the batch moved on */
                    if (lo_b != cur_b)
                        __syncthreads();
                    if (__any_sync(0xffffffffu, valid)) {
                        const Batch B = make_batch<u64>(W.batch_key[lo_b], rec);
                        light_step(sh, valid, word, tid, kind, B, 0, (uint64_t)w << W.wl, c, G, rec, s_raw, cnt, lane,
                                   below);
                    }
                    cur_b = hi_b;
                    continue;
                }
                /* several batches: batch steps, a barrier where the batch changes */
                const bool act = valid;
                uint32_t b = cur_b;
                for (;;) {
                    if (__any_sync(0xffffffffu, act && my_b == b)) { /* warp-uniform: records are batch-sorted */
                        const Batch B = make_batch<u64>(W.batch_key[b], rec);
                        light_step(sh, act && my_b == b, word, tid, kind, B, 0, (uint64_t)w << W.wl, c, G, rec,
                                   s_raw, cnt, lane, below);
                    }
                    if (b == hi_b)
                        break;
                    /* every access of batch b in this window is done before a later batch starts
                     * (the barrier), and the tile is batch-sorted, so the next batch is the one of
                     * the first record past the le records of batches <= b */
                    const uint32_t le = (uint32_t)__syncthreads_count(valid && my_b <= b);
                    b = (uint32_t)rb[base + le - c0] >> 16;
                }
                cur_b = hi_b;
            }
            __syncthreads(); /* this ring buffer is consumed */
            if (threadIdx.x == 0 && k + 2 < nch) {
                const uint32_t s0 = a0 + (k + 2) * kRing, m = min(kRing, aend - s0);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_arrive_expect_tx(&s_mbar[1 + bi], m * 8u);
                bulk_g2s(ring + bi * kRing, W.rec2 + s0, m * 8u, &s_mbar[1 + bi]);
            }
        }
        __syncthreads();
        /* write the window back (the async proxy reads what the generic proxy wrote) */
        if (threadIdx.x == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            for (uint32_t o = 0; o < wbytes; o += 32768u)
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(
                                 reinterpret_cast<unsigned char *>(gw) + o),
                             "r"(smem_u32(s_dyn + o)), "r"(min(32768u, wbytes - o))
                             : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            W.gen[w] = cur;
        }
    }
    if (threadIdx.x == 0)
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    flush_stats(c, cnt, s_stats, lane);
}

/* diagnostics (HIRACE_WIN_VALIDATE): records of every window batch-sorted, per-window counts
 * consistent; violations counted into aux[kAuxViolations] */
__global__ void k_w_validate(WinDev W)
{
    if (W.aux[kAuxAbort])
        return;
    for (uint32_t w = blockIdx.x; w < W.nw; w += gridDim.x) {
        const uint32_t b0 = W.win_cnt[w], b1 = W.win_cnt[w + 1];
        if (b1 < b0 && threadIdx.x == 0)
            atomicAdd(&W.aux[kAuxViolations], 1000000u);
        for (uint32_t i = b0 + 1 + threadIdx.x; i < b1; i += blockDim.x)
            if (((uint32_t)W.rec2[i] >> 16) < ((uint32_t)W.rec2[i - 1] >> 16))
                atomicAdd(&W.aux[kAuxViolations], 1u);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0 && W.win_cnt[W.nw] != W.aux[kAuxTotal1])
        atomicAdd(&W.aux[kAuxViolations], 1u << 30);
}

/* lazy reset: the generation moves on, so every window reads as INIT until replayed */
__global__ void k_w_lazy_reset(uint32_t *cur_gen, unsigned long long *report_count, unsigned long long *stats,
                               unsigned int *err)
{
    if (threadIdx.x == 0) {
        *cur_gen += 1u;
        *report_count = 0;
        *err = 0;
    }
    if (threadIdx.x < 4)
        stats[threadIdx.x] = 0;
}

/* stale windows := INIT, gen := current (before any path that reads the shadow directly) */
__global__ void __launch_bounds__(256) k_w_materialize(hirace_dev_ctx c, WinDev W, int only_if_scan)
{
    if (only_if_scan && reports_cover(c))
        return;
    const uint32_t cur = *W.cur_gen, per = (1u << W.wl) / 2;
    for (uint32_t w = blockIdx.x; w < W.nw; w += gridDim.x) {
        if (W.gen[w] == cur)
            continue;
        uint4 *p = reinterpret_cast<uint4 *>(c.shadow) + (uint64_t)w * per;
        for (uint32_t q = threadIdx.x; q < per; q += blockDim.x)
            p[q] = make_uint4(0, 0, 0, 0);
        __syncthreads();
        if (threadIdx.x == 0)
            W.gen[w] = cur;
    }
}

size_t light_smem_of(uint32_t wl)
{
    /* window records | record ring */
    return ((size_t)8u << wl) + 2u * kRing * 8u;
}
size_t light_smem(const WinDev &W) { return light_smem_of(W.wl); }

} // namespace

const void *window_light_kernel() { return (const void *)k_w_light; }
int window_light_threads() { return kLightThreads; }
size_t window_light_smem(uint32_t wl) { return light_smem_of(wl); }

cudaError_t window_init()
{
    cudaError_t e0;
#define W_SMEM(fn, bytes)                                                                                            \
    if ((e0 = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(bytes))) != cudaSuccess)  \
        return e0;
    W_SMEM((k_w_scatter1<16, 512, 4>), sizeof(ScatterSmem<16, 512>));
    W_SMEM((k_w_scatter1<8, 1024, 2>), sizeof(ScatterSmem<8, 1024>));
    W_SMEM((k_w_scatter2<16, 512, 4>), sizeof(ScatterSmem<16, 512>));
    W_SMEM((k_w_scatter2<8, 1024, 2>), sizeof(ScatterSmem<8, 1024>));
#undef W_SMEM
    return cudaFuncSetAttribute(k_w_light, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)window_light_smem(14));
}

namespace {
cudaError_t coop_scan(const hirace_dev_ctx &c, const WinDev &W, uint32_t *a, uint32_t rows, const uint32_t *cols,
                      uint32_t extra, uint32_t *total_out, uint32_t *ceil_out, uint32_t ceil_div,
                      const unsigned long long *check_total, uint64_t cap, int sm_count, cudaStream_t st)
{
    const uint32_t G = (uint32_t)(sm_count < kScanMaxCtas ? sm_count : kScanMaxCtas);
    uint32_t *abort = W.aux + kAuxAbort;
    note_launches(3);
    k_w_scan_reduce<<<G, 1024, 0, st>>>(a, rows, cols, extra, G, W.partials, check_total, cap, abort,
                                        c.error_flags);
    k_w_scan_partials<<<1, 1024, 0, st>>>(W.partials, G, total_out, ceil_out, ceil_div ? ceil_div : 1u, abort);
    k_w_scan_apply<<<G, 1024, 0, st>>>(a, rows, cols, extra, G, W.partials, abort);
    return cudaGetLastError();
}
} // namespace

cudaError_t launch_lazy_reset(const hirace_dev_ctx &c, const WinDev &W, cudaStream_t st)
{
    note_launches(1);
    k_w_lazy_reset<<<1, 32, 0, st>>>(W.cur_gen, c.report_count, c.stats, c.error_flags);
    return cudaGetLastError();
}

cudaError_t launch_materialize(const hirace_dev_ctx &c, const WinDev &W, int only_if_scan, int sm_count,
                               cudaStream_t st)
{
    note_launches(1);
    k_w_materialize<<<sm_count * 8, 256, 0, st>>>(c, W, only_if_scan);
    return cudaGetLastError();
}

cudaError_t launch_window_check(const hirace_dev_ctx &c, const WinDev &W, const Scratch &s, const hirace_event *ev,
                                uint32_t n, int sm_count, int replay_grid, cudaStream_t st, uint64_t shadow_words,
                                hirace_race *out, uint64_t cap, unsigned long long *d_total)
{
    (void)n;
    cudaError_t e;
#define W_TRY(x)                                                                                                      \
    do {                                                                                                              \
        if ((e = (x)) != cudaSuccess)                                                                                 \
            return e;                                                                                                 \
    } while (0)
    const bool two = W.d1b != 0;
    const int pgrid = sm_count * 4;
    /* per-check scratch state: counters, window counts, lists */
    W_TRY(cudaMemsetAsync(W.aux, 0, kAuxCount * sizeof(uint32_t), st));
    W_TRY(cudaMemsetAsync(W.elems, 0, sizeof(unsigned long long), st));
    W_TRY(cudaMemsetAsync(W.win_cnt, 0, ((size_t)W.nw + 1) * sizeof(uint32_t), st));
    note_launches(5);
    k_w_prep<<<1, 1024, 0, st>>>(ev, s.batch_off, s.nbatches, W, c.error_flags);
    k_w_pass1<false><<<pgrid, kPassThreads, 0, st>>>(c, reinterpret_cast<const uint4 *>(ev), W);
    W_TRY(cudaGetLastError());
    W_TRY(coop_scan(c, W, W.count1, 1u << W.d0b, W.aux + kAuxItems1, 0, W.aux + kAuxTotal1, W.aux + kAuxChunks2, W.p2,
                    W.elems, W.elem_cap, sm_count, st));
    if ((1u << W.d0b) <= 512)
        k_w_scatter1<16, 512, 4><<<pgrid, kPassThreads, sizeof(ScatterSmem<16, 512>), st>>>(
            c, reinterpret_cast<const uint4 *>(ev), W);
    else if ((1u << W.d0b) <= kMaxBufDigits)
        k_w_scatter1<8, 1024, 2><<<pgrid, kPassThreads, sizeof(ScatterSmem<8, 1024>), st>>>(
            c, reinterpret_cast<const uint4 *>(ev), W);
    else
        k_w_pass1<true><<<pgrid, kPassThreads, 0, st>>>(c, reinterpret_cast<const uint4 *>(ev), W);
    W_TRY(cudaGetLastError());
    if (two) {
        note_launches(2);
        k_w_pass2<false><<<pgrid, kPassThreads, 0, st>>>(W, s.nbatches);
        W_TRY(cudaGetLastError());
        W_TRY(coop_scan(c, W, W.count2, 1u << W.d1b, W.aux + kAuxChunks2, 0, W.aux + kAuxTotal2, nullptr, 1,
                        nullptr, 0, sm_count, st));
        if ((1u << W.d1b) <= 512)
            k_w_scatter2<16, 512, 4><<<pgrid, kPassThreads, sizeof(ScatterSmem<16, 512>), st>>>(W, s.nbatches);
        else if ((1u << W.d1b) <= kMaxBufDigits)
            k_w_scatter2<8, 1024, 2><<<pgrid, kPassThreads, sizeof(ScatterSmem<8, 1024>), st>>>(W, s.nbatches);
        else
            k_w_pass2<true><<<pgrid, kPassThreads, 0, st>>>(W, s.nbatches);
        W_TRY(cudaGetLastError());
    }
    W_TRY(coop_scan(c, W, W.win_cnt, 1, nullptr, W.nw + 1, nullptr, nullptr, 1, nullptr, 0, sm_count, st));
    if (getenv("HIRACE_WIN_VALIDATE"))
        k_w_validate<<<sm_count * 4, 256, 0, st>>>(W);
    note_launches(2);
    k_w_classify<<<sm_count * 4, 256, 0, st>>>(W);
    k_w_hseg<<<sm_count, 256, 0, st>>>(W, s.nbatches);
    W_TRY(cudaGetLastError());
    {
        W_TRY(cudaMemsetAsync(W.bar + 1, 0, sizeof(unsigned int), st));
        hirace_dev_ctx cc = c;
        WinDev ww = W;
        const uint32_t *nbp = s.nbatches;
        void *args[] = {&cc, &ww, &nbp};
        note_launches(1);
        W_TRY(cudaLaunchCooperativeKernel((const void *)k_w_heavy, dim3(replay_grid), dim3(kReplayThreads), args, 0,
                                          st));
    }
    note_launches(1);
    k_w_light<<<W.light_ctas, kLightThreads, light_smem(W), st>>>(c, W);
    W_TRY(cudaGetLastError());
    if (d_total) { /* report buffer; else stale windows := INIT and the shadow scan */
        W_TRY(launch_collect_reports(c, out, cap, d_total, st));
        W_TRY(launch_materialize(c, W, 1, sm_count, st));
        W_TRY(launch_collect(c, shadow_words, s, out, cap, d_total, st, 2));
    }
#undef W_TRY
    return cudaSuccess;
}

} // namespace hirace_impl
