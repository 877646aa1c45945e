/*
 * subwarp.cu — partial-mask warp synchronisation ("HiRace
 * tracks a bounded history of sub-warp synchronizations (essentially a warp-level vector clock)
 * and opportunistically prunes the history"; reading R20; include/hirace.h
 * hirace_set_warp_syncs).
 *
 * Split of the work.  A __syncwarp(mask) orders lanes of one warp only, so every relation the
 * three-level FSM decides across warps, blocks and epochs stays exact.  Only the WARP-level
 * question changes: inside one block epoch two accesses of different lanes are no longer
 * "concurrent iff same w".  The replay therefore
 *   1. runs the FSM with w read as the warp's sync number (event w = last sync its lane passed):
 *      equal numbers are truly concurrent (same-batch pairs, exact), different numbers are
 *      treated as ordered -- which misses exactly the pairs a partial mask left unordered;
 *   2. catches those pairs with a per-word sub-warp history: per lane and access class (read,
 *      atomic, write) the last sync number at which that lane accessed the word in this block
 *      epoch ("pruned" to one number per lane and class: the latest is the one most likely to
 *      be unordered, since e1 -> e2 iff V_e2[lane(e1)] > w1 is monotone in w1), compared with the
 *      warp vector clock V after the accessing lane's last sync;
 *   3. on such a race, turns the FSM's next state into the RACE state of its level (T/W ->
 *      RACE_W, B -> RACE_B, G -> RACE_G), storing the detecting accessor, so the class rules
 *      (C1.6) and the sticky upgrades work unchanged.
 * The history of a word belongs to the first warp that uses it in the block epoch; another warp
 * with partial syncs touching the same word in the same (g, b) makes every race of either warp a
 * BLOCK race the FSM finds by itself (a conflicting same-warp pair always conflicts with one of
 * the other warp's accesses), so its accesses skip the history.
 *
 * Kernels: k_ws_families (one CTA: log validation, (g,b,warp) families by a block scan),
 * k_ws_clocks (one warp per family: the vector clock after every listed sync, joins of 32
 * columns in shared memory), k_replay_masked (persistent cooperative replay, one event per
 * thread per step, contiguous warp shares, grid barrier between batches).
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"
#include "record.cuh"
#include "replay_core.cuh"

namespace hirace_impl {

using namespace hirace;

namespace {

constexpr int kFamThreads = 1024;
constexpr int kClockWarps = 8;
constexpr int kMaskedThreads = 256;
static_assert(kSlotWords == ws::kSlotWords, "history slot layout");
using ws::kEmpty;
using ws::mix64;

__device__ __forceinline__ unsigned long long fam_key(uint32_t g, uint32_t b, uint32_t warp)
{
    return ((unsigned long long)g << 50) | ((unsigned long long)b << 40) | warp;
}

/* Validation + families: one CTA walks the log in 1024-record tiles, flags family heads and
 * numbers them with a block scan. */
__global__ void __launch_bounds__(kFamThreads)
    k_ws_families(const hirace_warp_sync *__restrict__ s, uint32_t n, uint32_t total_warps, uint32_t warp_size,
                  WsDev W, unsigned int *err)
{
    __shared__ uint32_t sc[kFamThreads];
    __shared__ uint32_t s_base;
    const uint32_t t = threadIdx.x;
    if (t == 0)
        s_base = 0;
    __syncthreads();
    for (uint32_t base = 0; base < n; base += kFamThreads) {
        const uint32_t i = base + t;
        uint32_t head = 0;
        unsigned long long key = 0;
        if (i < n) {
            const hirace_warp_sync x = s[i];
            const uint32_t w = (x.meta >> 5) & 511u;
            key = fam_key(x.meta >> 24, (x.meta >> 14) & 1023u, x.warp);
            bool ok = w >= 1 && x.mask != 0 && (warp_size >= 32 || (x.mask >> warp_size) == 0) &&
                      x.warp < total_warps && (x.meta & 31u) == 0 && x.pad == 0;
            if (i == 0) {
                head = 1;
            } else {
                const hirace_warp_sync y = s[i - 1];
                const unsigned long long pk = fam_key(y.meta >> 24, (y.meta >> 14) & 1023u, y.warp);
                head = key != pk;
                ok = ok && (key > pk || (key == pk && w > ((y.meta >> 5) & 511u)));
            }
            if (!ok)
                atomicOr(err, ERR_BAD_TRACE);
            W.sync_w[i] = w;
            W.sync_mask[i] = x.mask;
        }
        sc[t] = head;
        __syncthreads();
        for (uint32_t d = 1; d < kFamThreads; d <<= 1) { /* inclusive Hillis-Steele scan */
            const uint32_t v = t >= d ? sc[t - d] : 0u;
            __syncthreads();
            sc[t] += v;
            __syncthreads();
        }
        if (i < n)
            W.sync_fam[i] = s_base + sc[t] - 1;
        if (head) {
            const uint32_t f = s_base + sc[t] - 1;
            W.fam_key[f] = key;
            W.fam_lo[f] = i;
        }
        __syncthreads();
        if (t == kFamThreads - 1)
            s_base += sc[t];
        __syncthreads();
    }
    if (t == 0) {
        *W.nfam = s_base;
        W.fam_lo[s_base] = n;
    }
}

/* Warp vector clocks: one warp per family, lane i owns column i of the 32 x 32 matrix
 * V[l][i] = the largest sync number of lane i that lane l knows of.  An unlisted number before a
 * listed sync is a full-mask sync: everyone knows everything up to it.  A listed sync s of mask M
 * joins the rows of M and stamps V[.][i] = s for i in M; the joined row is the clock after s. */
__global__ void __launch_bounds__(kClockWarps * 32) k_ws_clocks(WsDev W)
{
    __shared__ unsigned short V[kClockWarps][32][33];
    const uint32_t lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
    const uint32_t nfam = *W.nfam;
    for (uint32_t f = blockIdx.x * kClockWarps + wl; f < nfam; f += gridDim.x * kClockWarps) {
        for (int l = 0; l < 32; l++)
            V[wl][l][lane] = 0;
        uint32_t prev = 0;
        const uint32_t lo = W.fam_lo[f], hi = W.fam_lo[f + 1];
        for (uint32_t s = lo; s < hi; s++) {
            const uint32_t ws = W.sync_w[s], m = W.sync_mask[s];
            __syncwarp();
            if (ws - 1 > prev)
                for (int l = 0; l < 32; l++)
                    V[wl][l][lane] = (unsigned short)(ws - 1);
            __syncwarp();
            uint32_t j = 0;
            for (uint32_t r = m; r; r &= r - 1)
                j = max(j, (uint32_t)V[wl][__ffs(r) - 1][lane]);
            const uint32_t v = ((m >> lane) & 1u) ? ws : j;
            __syncwarp();
            for (uint32_t r = m; r; r &= r - 1)
                V[wl][__ffs(r) - 1][lane] = (unsigned short)v;
            W.vrow[(size_t)s * 32 + lane] = (unsigned short)v;
            prev = ws;
        }
        __syncwarp();
    }
}

/* lookup key of (family, sync number w): g:8 << 51 | b:10 << 41 | w:9 << 32 | warp:32 (w = 0: the
 * family record) */
__device__ __forceinline__ unsigned long long sync_hkey(uint32_t g, uint32_t b, uint32_t w, uint32_t warp)
{
    return ((unsigned long long)g << 51) | ((unsigned long long)b << 41) | ((unsigned long long)w << 32) | warp;
}


__device__ void fh_insert(const WsDev &W, unsigned long long hk, uint32_t row, uint32_t smax)
{
    for (unsigned long long h = mix64(hk) & W.fh_mask;; h = (h + 1) & W.fh_mask) {
        unsigned long long *e = reinterpret_cast<unsigned long long *>(W.fhash + h);
        if (atomicCAS(e, kEmpty, hk) == kEmpty) {
            W.fhash[h].z = row;
            W.fhash[h].w = smax;
            return;
        }
    }
}

/* One lookup table for the replay: (family, w) of every listed sync -> {row, smax}, and
 * (family, 0) -> {~0, smax} (smax = the family's last listed sync number).  Half full at most. */
__global__ void k_ws_hash(WsDev W, uint32_t n)
{
    for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < n; s += gridDim.x * blockDim.x) {
        const uint32_t f = W.sync_fam[s];
        const unsigned long long fk = W.fam_key[f];
        const uint32_t g = (uint32_t)(fk >> 50), b = (uint32_t)(fk >> 40) & 1023u, warp = (uint32_t)fk;
        const uint32_t smax = W.sync_w[W.fam_lo[f + 1] - 1];
        fh_insert(W, sync_hkey(g, b, W.sync_w[s], warp), s, smax);
        if (s == W.fam_lo[f])
            fh_insert(W, sync_hkey(g, b, 0, warp), ~0u, smax);
    }
}

__device__ __forceinline__ uint4 fh_find(const WsDev &W, unsigned long long hk)
{
    for (unsigned long long h = mix64(hk) & W.fh_mask;; h = (h + 1) & W.fh_mask) {
        const uint4 e = __ldg(W.fhash + h);
        const unsigned long long k = ((unsigned long long)e.y << 32) | e.x;
        if (k == hk || k == kEmpty)
            return k == hk ? e : make_uint4(0xffffffffu, 0xffffffffu, 0xffffffffu, 0);
    }
}

#ifndef HIRACE_MASKED_MINB
#define HIRACE_MASKED_MINB 4
#endif
template <bool P2, typename R>
__global__ void __launch_bounds__(kMaskedThreads, HIRACE_MASKED_MINB)
    k_replay_masked(hirace_dev_ctx c, WsDev W, const uint4 *__restrict__ ev, const uint32_t *__restrict__ off,
                    const uint32_t *__restrict__ nbp, unsigned int *bar)
{
    __shared__ __align__(16) unsigned char s_table[2048 + RAW_TABLE_BYTES];
    __shared__ unsigned long long s_stats[4];
    const uint32_t lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < (2048 + RAW_TABLE_BYTES) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(s_table)[i] = __ldg(reinterpret_cast<const uint4 *>(c.table) + i);
    if (threadIdx.x < 4)
        s_stats[threadIdx.x] = 0;
    __syncthreads();

    geom G = make_geom(c);
    G.pow2 = P2;
    const Rec<R> rec(c);
    const unsigned char *const raw = s_table + 2048;
    R *const shadow = shadow_as<R>(c);
    const uint32_t nb = *nbp;
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t tid_max = total_threads > 0xffffffffull ? 0xffffffffu : (uint32_t)(total_threads - 1);
    const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t gb = c.g_base ? *c.g_base : 0u;
    const uint32_t gran = c.gran_log2;
    unsigned int bar_epoch = 0;
    Counters cnt{0, 0, 0, 0};
    uint32_t bad = 0, clk = 0, full = 0;

    for (uint32_t bi = 0; bi < nb; bi++) {
        const uint32_t bstart = __ldg(&off[bi]), bend = __ldg(&off[bi + 1]);
        const Batch B = make_batch<R>(__ldg(&ev[bstart].w) >> 5, rec, gb);
        if (B.g == 255u)
            bad = 1;
        if (!B.fit)
            clk = 1;
        uint32_t i, iend;
        warp_share(bstart, bend, warp_global, nwarps, lane, i, iend);
        for (; B.fit && i < iend; i += 32) {
            const uint4 e = ld_event(ev + i);
            const uint32_t tid = e.z, meta = e.w, kind = meta & 3u, szl = (meta >> 2) & 7u;
            const bool sh = (int)e.y < 0;
            const uint64_t offb = (((uint64_t)(e.y & 0x7fffffffu)) << 32) | e.x;
            const uint64_t word = offb >> gran;
            const uint32_t nw = szl <= gran ? 1u : (1u << (szl - gran));
            const uint64_t lim = sh ? c.smem_words : c.global_words;
            if ((meta >> 5) != B.key || szl > 4 || tid > tid_max || word + nw > lim) {
                bad = 1;
                continue;
            }
            if (c.f_active && !((tid & c.f_tid_mask) == c.f_tid_match &&
                                (sh ? (c.f_spaces & 2u) != 0
                                    : ((c.f_spaces & 1u) != 0 && word >= c.f_glo && word < c.f_ghi))))
                continue;
            uint32_t blk, wib;
            coords(tid, G, &blk, &wib);
            const uint32_t lt = tid - blk * G.bt;
            const uint32_t ln = lt - wib * c.warp_size;
            /* the family of this warp in (g, b) and the listed sync this access follows */
            bool chk = false, upd = false;
            uint32_t row = 0;
            unsigned long long owner = 0;
            if (W.nsync) {
                const uint32_t gw = blk * W.wpb + wib;
                /* w == 0 (no sync passed yet) finds the family record {~0, smax} */
                uint4 fe = fh_find(W, sync_hkey(B.graw, B.b, B.w, gw));
                if (fe.z != 0xffffffffu) {
                    if (!((__ldg(W.sync_mask + fe.z) >> ln) & 1u)) {
                        bad = 1;
                        continue;
                    }
                    chk = true;
                    row = fe.z;
                } else if (B.w && fe.x == 0xffffffffu && fe.y == 0xffffffffu) {
                    fe = fh_find(W, sync_hkey(B.graw, B.b, 0, gw));
                }
                if (fe.x != 0xffffffffu || fe.y != 0xffffffffu) {
                    upd = B.w < fe.w;
                    owner = (1ull << 63) | ((unsigned long long)B.g << 50) | ((unsigned long long)B.b << 40) | gw;
                }
            }
            const uint32_t cls = kind == HIRACE_READ ? 0u : (kind == HIRACE_WRITE ? 2u : 1u);
            const uint32_t stamp = (1u << 18) | (B.g << 10) | B.b;
            for (uint32_t k = 0; k < nw; k++) {
                const uint64_t wk = word + k;
                const uint64_t idx = sh ? c.global_words + (uint64_t)blk * c.smem_words + wk : wk;
                const uint64_t key = sh ? (HIRACE_SHARED_BIT | ((uint64_t)blk << 32) | wk) : wk;
                /* a4 first: its latency overlaps the history work (a stale value costs a retry) */
                R *p = shadow + idx;
                R o = Rec<R>::load(p);
                bool side = false;
                if (chk || upd) {
                    ulonglong2 sv[4];
                    unsigned long long *slot = ws::hist_slot(W.H, key, owner, full, sv);
                    if (slot)
                        side = ws::side_step(W.H, slot, sv, ln, stamp, cls, W.H.confl[cls], B.w,
                                             W.vrow + (size_t)row * 32, chk, upd, B.w, full);
                }
                cnt.checked++;
                bool first = true;
                for (;;) {
                    uint32_t ent = raw[((uint32_t)(o & 31u) << 7) | rec.label(o, tid, kind, B.ep, G)];
                    if (side) {
                        const uint32_t ns = W.H.race_of[ent & E_STATE];
                        if (ns != (ent & E_STATE))
                            ent = ns | E_REPORT; /* store the detecting accessor */
                    }
                    const R n = rec.next(o, ent, tid, B.ep);
                    if (n == o)
                        break;
                    cnt.cas += first ? 1u : 0u;
                    cnt.retry += first ? 0u : 1u;
                    first = false;
                    const R prev = Rec<R>::cas(p, o, n);
                    if (prev == o) {
                        const uint32_t cn = race_class(st_of(n)), co = race_class(st_of(o));
                        if ((ent & E_REPORT) && cn > co) {
                            const unsigned long long pos = atomicAdd(c.report_count, 1ull);
                            if (pos < c.report_capacity) {
                                hirace_race rr;
                                rr.key = key;
                                rr.cls_and_epoch = cn | (B.graw << 8);
                                rr.detect_tid = tid;
                                c.reports[pos] = rr;
                            }
                        }
                        break;
                    }
                    o = prev;
                }
            }
        }
        if (bi + 1 < nb)
            grid_sync(bar, gridDim.x, bar_epoch);
    }
    if (bad)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
    if (clk)
        atomicOr(c.error_flags, ERR_CLOCK);
    if (full)
        atomicOr(c.error_flags, ERR_HISTORY);
    __syncwarp();
    flush_stats(c, cnt, s_stats, lane);
}

bool pow2_geom(const hirace_dev_ctx &c)
{
    return (c.block_threads & (c.block_threads - 1)) == 0 && (c.warp_size & (c.warp_size - 1)) == 0;
}

const void *masked_kernel(const hirace_dev_ctx &c)
{
    const bool p2 = pow2_geom(c);
    if (c.rec_bytes == 4)
        return p2 ? (const void *)k_replay_masked<true, unsigned int> : (const void *)k_replay_masked<false, unsigned int>;
    return p2 ? (const void *)k_replay_masked<true, unsigned long long>
              : (const void *)k_replay_masked<false, unsigned long long>;
}

} // namespace

cudaError_t launch_ws_prepare(const hirace_warp_sync *d_syncs, uint32_t n, uint32_t total_warps, uint32_t warp_size,
                              const WsDev &W, unsigned int *err, int sm_count, cudaStream_t st)
{
    note_launches(1);
    k_ws_families<<<1, kFamThreads, 0, st>>>(d_syncs, n, total_warps, warp_size, W, err);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess)
        return e;
    const uint32_t blocks = (n + kClockWarps - 1) / kClockWarps;
    const uint32_t grid = blocks < (uint32_t)(8 * sm_count) ? (blocks ? blocks : 1u) : (uint32_t)(8 * sm_count);
    k_ws_clocks<<<grid, kClockWarps * 32, 0, st>>>(W);
    if ((e = cudaGetLastError()) != cudaSuccess)
        return e;
    note_launches(2);
    const uint32_t hb = (n + 255) / 256;
    k_ws_hash<<<hb < (uint32_t)(8 * sm_count) ? hb : (uint32_t)(8 * sm_count), 256, 0, st>>>(W, n);
    return cudaGetLastError();
}

int masked_max_grid(int device)
{
    int sms = 0, occ = 1 << 30;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const void *fns[] = {(const void *)k_replay_masked<true, unsigned long long>,
                         (const void *)k_replay_masked<false, unsigned long long>,
                         (const void *)k_replay_masked<true, unsigned int>,
                         (const void *)k_replay_masked<false, unsigned int>};
    for (const void *f : fns) {
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, f, kMaskedThreads, 0);
        occ = o < occ ? o : occ;
    }
    return sms * (occ < 1 ? 1 : occ);
}

cudaError_t launch_replay_masked(const hirace_dev_ctx &c, const WsDev &W, const hirace_event *ev, const Scratch &s,
                                 int grid, cudaStream_t st)
{
    hirace_dev_ctx cc = c;
    WsDev ww = W;
    const uint4 *evp = reinterpret_cast<const uint4 *>(ev);
    const uint32_t *offp = s.batch_off;
    const uint32_t *nbp = s.nbatches;
    unsigned int *barp = s.grid_bar;
    void *args[] = {&cc, &ww, &evp, &offp, &nbp, &barp};
    note_launches(1);
    return cudaLaunchCooperativeKernel(masked_kernel(c), dim3(grid), dim3(kMaskedThreads), args, 0, st);
}

} // namespace hirace_impl
