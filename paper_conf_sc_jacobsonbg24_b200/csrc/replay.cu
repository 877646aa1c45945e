/*
 * replay.cu — the hot kernel: persistent, cooperative trace replay through the HiRace FSM
 * (§8(a) rows a1-a9; Algorithm 1).
 *
 * Work layout.  Batches (g,b,w) are processed in order with a grid barrier between them;
 * inside a batch any order is a linear extension of happens-before.  Each warp
 * owns a contiguous, balanced share of the batch and walks it in 32-event chunks (one event
 * per lane), keeping the next two chunks' 16-byte events in flight (a1).
 *
 * Per chunk, the common path is short and branch-free (optimistic concurrency):
 *   a2  decode: one compare checks batch key + access size, shadow index from the address;
 *   a4  each lane's coherent shadow load (ld.relaxed.gpu: never a stale L1 line);
 *   a5  relation/sync label by XOR+shift, one lookup in the raw-flag shared-memory table, pack;
 *   a6  one atom.cas per changed word; an unchanged record issues no CAS (the access is
 *       linearised at the load: no-write fast path, e.g. every read of a G_R word).
 * a3 warp aggregation happens only where it pays: lanes whose CAS lost (typically lanes of
 * the same warp on the same word) are grouped with __match_any_sync and the group leader folds
 * all members' accesses in lane order from the record its CAS returned, then commits them with
 * one CAS (Algorithm 1's retry loop).  Other rare cases also leave the
 * common path behind warp-uniform votes: 8/16-byte accesses, race reports (a7: warp-compacted
 * append, one atomicAdd per warp), invalid events.
 *
 * Every kernel is instantiated for both record layouts (record.cuh): the 8-byte record and the
 * compact 4-byte record of hirace_shadow_alloc_compact.
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "collect.cuh"
#include "internal.h"
#include "kernel_common.cuh"
#include "record.cuh"
#include "replay_core.cuh"


namespace hirace_impl {

using namespace hirace;

#ifdef HIRACE_BARRIER_TRACE
/* diagnostics build only: per (batch, CTA) globaltimer at arrival and after release */
__device__ unsigned long long g_bar_trace[128 * 2048 * 2];
__device__ unsigned int g_bar_smid[2048];
__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif

namespace {

/* chunks holding 8/16-byte accesses: word by word through the group commit (rare; the configs
 * emit 4-byte accesses).  `take` marks this lane's event as one to process here. */
template <typename R>
__device__ __noinline__ uint4 chunk_multiword(const hirace_dev_ctx c, const geom G, const unsigned char *raw,
                                              const Batch B, uint4 e, bool take, uint32_t lane)
{
    const Rec<R> rec(c);
    Counters cnt{0, 0, 0, 0};
    const uint64_t addr = ((uint64_t)e.y << 32) | e.x;
    const uint32_t szl = (e.w >> 2) & 7u, gran = c.gran_log2;
    const uint32_t nw = szl <= gran ? 1u : (1u << (szl - gran));
    const uint64_t word = (addr & ~HIRACE_SHARED_BIT) >> gran;
    const bool sh = (addr & HIRACE_SHARED_BIT) != 0;
    const uint64_t base = sh ? c.global_words + (uint64_t)block_of(e.z, G) * c.smem_words + word : word;
    R *const shadow = shadow_as<R>(c);
    const uint32_t maxnw = __reduce_max_sync(FULL, take ? nw : 0u);
    for (uint32_t k = 0; k < maxnw; k++) {
        const bool act = take && k < nw;
        const uint64_t my = act ? base + k : NONE;
        const uint32_t peers = __match_any_sync(FULL, my);
        cnt.checked += act;
        const bool lead = act && (peers & ((1u << lane) - 1)) == 0;
        const R o = lead ? Rec<R>::load(shadow + my) : (R)0;
        uint32_t rtid = 0;
        const uint32_t cls = commit_groups<R>(shadow + my, o, lead ? peers : 0u, e.z, e.w & 3u, G, raw, B, rec, cnt,
                                              rtid, true);
        if (__any_sync(FULL, cls != 0))
            append_reports(c, cls, key_of(G, e, k, gran), B.graw, rtid, lane);
    }
    return make_uint4(cnt.checked, cnt.retry, cnt.cas, cnt.nowrite);
}


/* a2: decode + validate one lane's event (sub-element accesses map to their element; the
 * element is 1 << gran_log2 bytes, a 4-byte word by default); accesses covering several
 * elements are committed right here, element by element.  W32: the whole shadow has
 * < 2^31 words and tracked byte offsets fit 32 bits, so index math and range checks are 32-bit
 * (fewer instructions on the hot path); otherwise 64-bit. */
template <bool W32, typename R>
__device__ __forceinline__ Lane decode(const uint4 &e, bool valid_in, uint32_t keysz, const Batch &B,
                                       uint32_t tid_max, const hirace_dev_ctx &c, const geom &G,
                                       const unsigned char *raw, Counters &cnt, uint32_t &bad, uint32_t lane)
{
    Lane L;
    bool valid = valid_in;
    L.tid = e.z;
    L.kind = e.w & 3u;
    const uint32_t meta = e.w;
    const bool sh = (int)e.y < 0;
    const uint32_t gran = c.gran_log2;
    const bool key_ok = (meta >> 2) - keysz <= gran; /* same batch, size <= one element */
    const bool tid_ok = L.tid <= tid_max;
    uint64_t word;
    bool in_range;
    if (W32) {
        const uint32_t w32 = e.x >> gran;
        word = w32;
        in_range = (e.y & 0x7fffffffu) == 0 && w32 < (sh ? c.smem_words : (uint32_t)c.global_words);
    } else {
        word = ((((uint64_t)(e.y & 0x7fffffffu)) << 32) | e.x) >> gran;
        in_range = sh ? word < c.smem_words : word < c.global_words;
    }
    if (c.f_active) { /* selective tracking (hirace_set_filter): unselected accesses are skipped */
        const uint64_t wsel = ((((uint64_t)(e.y & 0x7fffffffu)) << 32) | e.x) >> gran;
        valid = valid && (L.tid & c.f_tid_mask) == c.f_tid_match &&
                (sh ? (c.f_spaces & 2u) != 0 : ((c.f_spaces & 1u) != 0 && wsel >= c.f_glo && wsel < c.f_ghi));
    }
    L.ok = valid && key_ok && tid_ok && in_range;
    if (__any_sync(FULL, valid && !L.ok)) {
        const uint64_t wfull = ((((uint64_t)(e.y & 0x7fffffffu)) << 32) | e.x) >> gran;
        const uint32_t szl = (meta >> 2) & 7u;
        const bool multi = valid && (meta >> 5) == B.key && szl > gran && szl <= 4 && tid_ok &&
                           (sh ? wfull + (1u << (szl - gran)) <= c.smem_words
                               : wfull + (1u << (szl - gran)) <= c.global_words);
        if (valid && !L.ok && !multi)
            bad = 1;
        if (__any_sync(FULL, multi)) {
            const uint4 d = chunk_multiword<R>(c, G, raw, B, e, multi, lane);
            cnt.checked += d.x;
            cnt.retry += d.y;
            cnt.cas += d.z;
        }
    }
    if (W32)
        L.idx = !L.ok ? NONE
                      : (uint64_t)(sh ? (uint32_t)c.global_words + block_of(L.tid, G) * c.smem_words + (uint32_t)word
                                      : (uint32_t)word);
    else
        L.idx = !L.ok ? NONE : (sh ? c.global_words + (uint64_t)block_of(L.tid, G) * c.smem_words + word : word);
    return L;
}


/* out of line so the collect's registers do not raise the replay loop's allocation */
template <typename R>
__device__ __noinline__ unsigned int collect_call(const hirace_dev_ctx c, uint64_t nwords, hirace_race *out,
                                                  uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt,
                                                  unsigned int *bar, unsigned int epoch)
{
    if (!collect_phase_small<R>(c, nwords, out, cap, d_total, cta_cnt, bar, epoch))
        collect_phase<R>(c, nwords, out, cap, d_total, cta_cnt, bar, epoch);
    return epoch;
}


template <bool P2, bool W32, typename R>
__global__ void __launch_bounds__(kReplayThreads, kMinBlocks)
    k_replay(hirace_dev_ctx c, const uint4 *__restrict__ ev, const uint32_t *__restrict__ off,
             const uint32_t *__restrict__ nbp, unsigned int *bar, uint64_t shadow_words, hirace_race *out,
             uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt, int report_mode)
{
    __shared__ __align__(16) unsigned char s_table[2048 + RAW_TABLE_BYTES]; /* canonical | raw-flag */
    __shared__ unsigned long long s_stats[4];
    const uint32_t lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < (2048 + RAW_TABLE_BYTES) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(s_table)[i] = __ldg(reinterpret_cast<const uint4 *>(c.table) + i);
    if (threadIdx.x < 4)
        s_stats[threadIdx.x] = 0;

    geom G = make_geom(c);
    G.pow2 = P2; /* compile-time geometry mode: shifts (P2) or fast division */
    const Rec<R> rec(c);
    const unsigned char *const raw = s_table + 2048;
    const uint32_t nb = *nbp;
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t tid_max = total_threads > 0xffffffffull ? 0xffffffffu : (uint32_t)(total_threads - 1);
    const uint32_t below = (1u << lane) - 1;
    const uint32_t tab_s = smem_u32(s_table);
    const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    unsigned int bar_epoch = 0;
    Counters cnt{0, 0, 0, 0};
    uint32_t bad = 0, clk = 0;

    /* a1: events of the first chunks of every batch are requested before the barrier that
     * precedes the batch, so the HBM latency overlaps the barrier */
    uint32_t bstart = nb ? __ldg(&off[0]) : 0, bend = nb ? __ldg(&off[1]) : 0;
    __syncthreads();
    uint32_t i, iend; /* this warp's contiguous share of the batch: events [i - lane, iend) */
    warp_share(bstart, bend, warp_global, nwarps, lane, i, iend);
    uint4 e0 = i < iend ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
    uint4 e1 = i + 32 < iend ? ld_event(ev + i + 32) : make_uint4(0, 0, 0, 0);
    const uint32_t gb = c.g_base ? *c.g_base : 0u; /* epoch reset: offset of this check's epochs */
    /* the batch key is read before the barrier that precedes the batch (its load latency is
     * off the post-barrier critical path) */
    uint32_t key_next = nb ? __ldg(&ev[bstart].w) >> 5 : 0u;
    for (uint32_t bi = 0; bi < nb; bi++) {
        const Batch B = make_batch<R>(key_next, rec, gb);
        const uint32_t keysz = B.key << 3; /* (meta >> 2) - keysz = size_log2 for this batch */
        if (B.g == 255u)
            bad = 1; /* reserved for retired RACE records (R7) */
        if (!B.fit)
            clk = 1; /* compact record: epochs beyond the declared limits; batch not checked */

        for (; i - lane < iend; i += 32) {
            const uint4 e = e0;
            e0 = e1; /* a1: keep the next chunks' events in flight */
            ld_event_if(ev + i + 64, i + 64 < iend, e1);
            const bool valid = i < iend && B.fit;
            const Lane cur = decode<W32, R>(e, valid, keysz, B, tid_max, c, G, raw, cnt, bad, lane);
            process_decoded<R>(cur, B, c, G, rec, raw, tab_s, cnt, lane, below);
        }
        if (bi + 1 < nb) {
            bstart = __ldg(&off[bi + 1]);
            bend = __ldg(&off[bi + 2]);
            key_next = __ldg(&ev[bstart].w) >> 5;
            warp_share(bstart, bend, warp_global, nwarps, lane, i, iend);
            e0 = i < iend ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
            e1 = i + 32 < iend ? ld_event(ev + i + 32) : make_uint4(0, 0, 0, 0);
#ifdef HIRACE_BARRIER_TRACE
            __syncthreads();
            if (threadIdx.x == 0 && bi < 128 && blockIdx.x < 2048) {
                g_bar_trace[(bi * 2048 + blockIdx.x) * 2] = gtimer();
                unsigned int sm;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
                g_bar_smid[blockIdx.x] = sm;
            }
#endif
            grid_sync(bar, gridDim.x, bar_epoch);
#ifdef HIRACE_BARRIER_TRACE
            if (threadIdx.x == 0 && bi < 128 && blockIdx.x < 2048)
                g_bar_trace[(bi * 2048 + blockIdx.x) * 2 + 1] = gtimer();
#endif
        }
    }

    /* fused a7 collection (hirace_check_trace_device): one more barrier, then the shadow scan,
     * unless the report buffer covers every flagged word (report mode: k_collect_reports runs
     * next; every CTA reads the same final report count after the barrier) */
    if (d_total) {
        grid_sync(bar, gridDim.x, bar_epoch);
        if (!(report_mode && reports_cover(c)))
            bar_epoch = collect_call<R>(c, shadow_words, out, cap, d_total, cta_cnt, bar, bar_epoch);
    }

    if (__any_sync(FULL, bad) && lane == 0)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
    if (clk && threadIdx.x == 0)
        atomicOr(c.error_flags, ERR_CLOCK);
    flush_stats(c, cnt, s_stats, lane);
}

/* Single-batch replay of 8-byte wire records (sharded mode): word:31 |
 * shared:1 | tid:30 | kind:2; the batch's (g,b,w) is given, so no batch discovery and no grid
 * barrier — a plain launch.  Each warp walks a contiguous balanced share of 32-record chunks
 * with the same per-chunk path (a4-a7) as k_replay. */
template <bool P2, typename R>
__global__ void __launch_bounds__(kReplayThreads, kMinBlocks)
    k_replay_wire(hirace_dev_ctx c, const unsigned long long *__restrict__ wire, uint32_t n, uint32_t key)
{
    __shared__ __align__(16) unsigned char s_table[2048 + RAW_TABLE_BYTES]; /* canonical | raw-flag */
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
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t below = (1u << lane) - 1;
    const uint32_t tab_s = smem_u32(s_table);
    Counters cnt{0, 0, 0, 0};
    const Batch B = make_batch<R>(key, rec);
    const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t nchunks = (n + 31) / 32;
    const uint32_t c0 = (uint32_t)(((uint64_t)nchunks * warp_global) / nwarps);
    const uint32_t c1 = (uint32_t)(((uint64_t)nchunks * (warp_global + 1)) / nwarps);
    const uint32_t iend = min(n, c1 * 32);
    uint32_t bad = 0;
    uint32_t i = c0 * 32 + lane;
    unsigned long long w0 = i < iend ? __ldcs(wire + i) : 0ull;
    unsigned long long w1 = i + 32 < iend ? __ldcs(wire + i + 32) : 0ull;
    for (; i - lane < iend; i += 32) {
        const unsigned long long w = w0;
        const bool valid = i < iend && B.fit;
        w0 = w1;
        w1 = i + 64 < iend ? __ldcs(wire + i + 64) : 0ull;
        Lane L;
        const uint32_t lo = (uint32_t)w, hi = (uint32_t)(w >> 32);
        const uint32_t word = lo & 0x7fffffffu;
        const bool sh = (lo >> 31) != 0;
        L.tid = hi & 0x3fffffffu;
        L.kind = hi >> 30;
        L.ok = valid && L.tid < total_threads && (sh ? word < c.smem_words : word < c.global_words);
        bad |= (valid && !L.ok) ? 1u : 0u;
        L.idx = !L.ok ? NONE : (sh ? c.global_words + (uint64_t)block_of(L.tid, G) * c.smem_words + word : (uint64_t)word);
        process_decoded<R>(L, B, c, G, rec, raw, tab_s, cnt, lane, below);
    }
    if ((__any_sync(FULL, bad) || B.g == 255u) && lane == 0)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
    if (!B.fit && n && threadIdx.x == 0)
        atomicOr(c.error_flags, ERR_CLOCK);
    flush_stats(c, cnt, s_stats, lane);
}

/* standalone collect: one cooperative kernel running collect_phase (collect.cuh); in report
 * mode it stands down when k_collect_reports (launched before it) covered every flagged word */
template <typename R>
__global__ void __launch_bounds__(kCollectThreads) k_collect(hirace_dev_ctx c, uint64_t nwords, hirace_race *out,
                                                             uint64_t cap, unsigned long long *d_total,
                                                             uint32_t *cta_cnt, unsigned int *bar, int report_mode)
{
    if (report_mode && reports_cover(c))
        return;
    unsigned int epoch = 0;
    collect_phase<R>(c, nwords, out, cap, d_total, cta_cnt, bar, epoch);
}

/* report-buffer collect (collect.cuh collect_reports_cta): one CTA, keys sorted in smem */
template <typename R>
__global__ void __launch_bounds__(kReportThreads) k_collect_reports(hirace_dev_ctx c, hirace_race *out, uint64_t cap,
                                                                    unsigned long long *d_total)
{
    extern __shared__ unsigned long long s_keys[];
    collect_reports_cta<R>(c, out, cap, d_total, s_keys);
}

bool pow2_geometry(const hirace_dev_ctx &c)
{
    return (c.block_threads & (c.block_threads - 1)) == 0 && (c.warp_size & (c.warp_size - 1)) == 0;
}

template <bool P2, typename R> const void *replay_fn(bool w32)
{
    return w32 ? (const void *)k_replay<P2, true, R> : (const void *)k_replay<P2, false, R>;
}

const void *replay_kernel(const hirace_dev_ctx &c, bool w32)
{
    const bool p2 = pow2_geometry(c);
    if (c.rec_bytes == 4)
        return p2 ? replay_fn<true, unsigned int>(w32) : replay_fn<false, unsigned int>(w32);
    return p2 ? replay_fn<true, unsigned long long>(w32) : replay_fn<false, unsigned long long>(w32);
}

} // namespace

#ifdef HIRACE_BARRIER_TRACE
extern "C" int hirace_debug_barrier_trace(unsigned long long *host, uint64_t n)
{
    return (int)cudaMemcpyFromSymbol(host, g_bar_trace, n * sizeof(unsigned long long));
}
extern "C" int hirace_debug_barrier_smid(unsigned int *host, uint64_t n)
{
    return (int)cudaMemcpyFromSymbol(host, g_bar_smid, n * sizeof(unsigned int));
}
#endif

int replay_max_grid(int device)
{
    int sms = 0, occ = 1 << 30;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const void *fns[] = {(const void *)k_replay<true, false, unsigned long long>,
                         (const void *)k_replay<false, false, unsigned long long>,
                         (const void *)k_replay<true, true, unsigned long long>,
                         (const void *)k_replay<false, true, unsigned long long>,
                         (const void *)k_replay<true, false, unsigned int>,
                         (const void *)k_replay<false, false, unsigned int>,
                         (const void *)k_replay<true, true, unsigned int>,
                         (const void *)k_replay<false, true, unsigned int>};
    for (const void *f : fns) {
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, f, kReplayThreads, 0);
        occ = o < occ ? o : occ;
    }
    if (occ < 1)
        occ = 1;
    return sms * occ;
}

int collect_max_grid(int device)
{
    int sms = 0, occ = 0, occ2 = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_collect<unsigned long long>, kCollectThreads, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, k_collect<unsigned int>, kCollectThreads, 0);
    occ = occ2 < occ ? occ2 : occ;
    if (occ < 1)
        occ = 1;
    return sms * occ < kMaxCtas ? sms * occ : kMaxCtas;
}

cudaError_t replay_init()
{
    const int bytes = (int)(kReportSortCap * sizeof(unsigned long long));
    cudaError_t e = cudaFuncSetAttribute(k_collect_reports<unsigned long long>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess)
        return e;
    return cudaFuncSetAttribute(k_collect_reports<unsigned int>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

cudaError_t launch_collect_reports(const hirace_dev_ctx &c, hirace_race *out, uint64_t cap,
                                   unsigned long long *d_total, cudaStream_t st)
{
    const size_t bytes = kReportSortCap * sizeof(unsigned long long);
    note_launches(1);
    if (c.rec_bytes == 4)
        k_collect_reports<unsigned int><<<1, kReportThreads, bytes, st>>>(c, out, cap, d_total);
    else
        k_collect_reports<unsigned long long><<<1, kReportThreads, bytes, st>>>(c, out, cap, d_total);
    return cudaGetLastError();
}

cudaError_t launch_collect(const hirace_dev_ctx &c, uint64_t shadow_words, const Scratch &s, hirace_race *out,
                           uint64_t cap, unsigned long long *d_total, cudaStream_t st, int report_mode)
{
    if (report_mode == 1) {
        cudaError_t e = launch_collect_reports(c, out, cap, d_total, st);
        if (e != cudaSuccess)
            return e;
    }
    cudaError_t e = cudaMemsetAsync(s.grid_bar2, 0, sizeof(unsigned int), st);
    if (e != cudaSuccess)
        return e;
    const uint64_t tiles = (shadow_words + kCollectTile - 1) / kCollectTile;
    int grid = (int)(tiles < (uint64_t)s.collect_grid ? tiles : (uint64_t)s.collect_grid);
    if (grid < 1)
        grid = 1;
    hirace_dev_ctx cc = c;
    uint64_t nw = shadow_words, cp = cap;
    hirace_race *o = out;
    unsigned long long *dt = d_total;
    uint32_t *cnt = s.cta_cnt;
    unsigned int *bar = s.grid_bar2;
    int rm = report_mode;
    void *args[] = {&cc, &nw, &o, &cp, &dt, &cnt, &bar, &rm};
    const void *fn = c.rec_bytes == 4 ? (const void *)k_collect<unsigned int> : (const void *)k_collect<unsigned long long>;
    note_launches(1);
    return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kCollectThreads), args, 0, st);
}

cudaError_t launch_replay_wire(const hirace_dev_ctx &c, const unsigned long long *wire, uint32_t n, uint32_t batch_key,
                               int grid, cudaStream_t st)
{
    const bool p2 = pow2_geometry(c);
    const uint32_t need = (n + 31) / 32; /* no more warps than chunks */
    const uint64_t want = ((uint64_t)need * 32 + kReplayThreads - 1) / kReplayThreads;
    const int g2 = (int)(want < (uint64_t)grid ? want : (uint64_t)grid);
    note_launches(1);
    if (c.rec_bytes == 4) {
        if (p2)
            k_replay_wire<true, unsigned int><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
        else
            k_replay_wire<false, unsigned int><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
    } else {
        if (p2)
            k_replay_wire<true, unsigned long long><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
        else
            k_replay_wire<false, unsigned long long><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
    }
    return cudaGetLastError();
}

cudaError_t launch_replay(const hirace_dev_ctx &c, const hirace_event *ev, const Scratch &s, int grid,
                          cudaStream_t st, uint64_t shadow_words, hirace_race *out, uint64_t cap,
                          unsigned long long *d_total, int report_mode)
{
    cudaError_t e;
    /* s.grid_bar was zeroed by k_batches, which always runs right before on this stream */
    hirace_dev_ctx cc = c;
    const uint4 *evp = reinterpret_cast<const uint4 *>(ev);
    const uint32_t *offp = s.batch_off;
    const uint32_t *nbp = s.nbatches;
    unsigned int *barp = s.grid_bar;
    uint64_t nw = shadow_words, cp = cap;
    hirace_race *o = out;
    unsigned long long *dt = d_total;
    uint32_t *cnt = s.cta_cnt;
    int rm = d_total ? report_mode : 0;
    void *args[] = {&cc, &evp, &offp, &nbp, &barp, &nw, &o, &cp, &dt, &cnt, &rm};
    /* W32: every shadow index and tracked byte offset fits 32 bits (see decode) */
    const uint64_t sw = c.global_words + (uint64_t)c.grid_blocks * c.smem_words;
#ifdef HIRACE_NO_W32
    const bool w32 = false;
    (void)sw;
#else
    const bool w32 = sw < (1ull << 31) && c.global_words < (1ull << 30) && c.smem_words < (1u << 30);
#endif
    note_launches(1);
    e = cudaLaunchCooperativeKernel(replay_kernel(c, w32), dim3(grid), dim3(kReplayThreads), args, 0, st);
    if (e != cudaSuccess || !rm)
        return e;
    return launch_collect_reports(c, out, cap, d_total, st); /* stands down if the scan ran */
}

} // namespace hirace_impl
