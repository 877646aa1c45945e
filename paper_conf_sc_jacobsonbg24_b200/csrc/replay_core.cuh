/* replay_core.cuh — the per-chunk hot path shared by the replay kernels (replay.cu: batch-major
 * k_replay / k_replay_wire; window.cu: the heavy-window kernel of the window-major path):
 * a4 coherent shadow load, a5 raw-flag label + lookup, a6 CAS of changed records, a3 fold of
 * collided CASes (Algorithm 1's retry loop), a7 warp-compacted report append.
 * Included by one translation unit each (internal linkage). */
#ifndef HIRACE_REPLAY_CORE_CUH
#define HIRACE_REPLAY_CORE_CUH

#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"
#include "record.cuh"

namespace hirace_impl {

using namespace hirace;

namespace {

constexpr uint32_t FULL = 0xffffffffu;
constexpr uint64_t NONE = ~0ull;
#ifndef HIRACE_REPLAY_MINB
#define HIRACE_REPLAY_MINB 2 /* 2 x 16 warps per SM at <= 64 registers */
#endif
constexpr int kMinBlocks = HIRACE_REPLAY_MINB;

struct Batch {
    uint32_t key, g, b, w, ep; /* ep = epochs in record layout; g = trace g + epoch offset */
    uint32_t graw;             /* the trace's g (reports carry it)                          */
    bool fit;                  /* epochs within the record layout's fields (compact limits) */
};

/* gb: the epoch-reset offset (hirace_set_reset_mode EPOCH) added to the trace's g */
template <typename R> __device__ __forceinline__ Batch make_batch(uint32_t key, const Rec<R> &rec, uint32_t gb = 0)
{
    Batch B;
    B.key = key;
    B.graw = key >> 19;
    B.g = B.graw + gb;
    B.b = (key >> 9) & 1023u;
    B.w = key & 511u;
    B.ep = rec.ep(B.g, B.b, B.w);
    B.fit = rec.fits(B.g, B.b, B.w);
    return B;
}

struct Counters {
    uint32_t checked, retry, cas, nowrite; /* per thread; widened at the end */
};

__device__ __forceinline__ uint32_t lds_u8(uint32_t saddr)
{
    uint32_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(saddr));
    return v;
}

__device__ __forceinline__ uint4 ld_event(const uint4 *p)
{
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(p));
    return v;
}

/* predicated event load: v keeps its old contents when !pred (no zero-fill instructions;
 * such lanes are masked by `valid`) */
__device__ __forceinline__ void ld_event_if(const uint4 *p, bool pred, uint4 &v)
{
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %5, 0;\n\t"
                 "@q ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];\n\t}"
                 : "+r"(v.x), "+r"(v.y), "+r"(v.z), "+r"(v.w)
                 : "l"(p), "r"((uint32_t)pred));
}

/* race key (include/hirace.h) of element k of event e (elements of 1 << gran bytes) */
__device__ __forceinline__ uint64_t key_of(const geom &G, const uint4 &e, uint32_t k, uint32_t gran)
{
    const uint64_t addr = ((uint64_t)e.y << 32) | e.x;
    const uint64_t word = ((addr & ~HIRACE_SHARED_BIT) >> gran) + k;
    if (addr & HIRACE_SHARED_BIT)
        return HIRACE_SHARED_BIT | ((uint64_t)block_of(e.z, G) << 32) | word;
    return word;
}

/* Fold, for every lane with a non-zero `peers` (a group leader), its group's accesses into
 * record o in lane order: the same sequence of Algorithm-1 transitions as if their CASes had
 * won one after another.  Accessors are broadcast by shuffle, so all lanes must call it.
 * raw = the raw-flag table (label_raw layout). */
template <typename R>
__device__ __forceinline__ R fold_shfl(R o, uint32_t peers, uint32_t my_tid, uint32_t my_kind, const geom &G,
                                       const unsigned char *raw, const Batch &B, const Rec<R> &rec, uint32_t &rep,
                                       uint32_t &rtid)
{
    R n = o;
    for (uint32_t uni = __reduce_or_sync(FULL, peers); uni; uni &= uni - 1) {
        const int m = __ffs(uni) - 1;
        const uint32_t t = __shfl_sync(FULL, my_tid, m);
        const uint32_t k = __shfl_sync(FULL, my_kind, m);
        if ((peers >> m) & 1u) {
            const uint32_t e = raw[((uint32_t)(n & 31u) << 7) | rec.label(n, t, k, B.ep, G)];
            if (e & E_REPORT) {
                rep = 1;
                rtid = t;
            }
            n = rec.next(n, e, t, B.ep);
        }
    }
    return n;
}

/* Commit for group leaders (peers != 0 only in leaders) starting from observed records o:
 * fold, CAS, re-fold on failure until every leader's CAS sticks or the record is unchanged.
 * Returns the report class for this lane; counts into cnt. */
template <typename R>
__device__ __forceinline__ uint32_t commit_groups(R *p, R o, uint32_t peers, uint32_t tid, uint32_t kind,
                                                  const geom &G, const unsigned char *raw, const Batch &B,
                                                  const Rec<R> &rec, Counters &cnt, uint32_t &rtid, bool first)
{
    bool pending = peers != 0;
    uint32_t cls = 0;
    while (__any_sync(FULL, pending)) {
        uint32_t rep = 0, rt = 0;
        const R n = fold_shfl<R>(o, pending ? peers : 0u, tid, kind, G, raw, B, rec, rep, rt);
        if (pending) {
            if (n == o) {
                pending = false;
            } else {
                cnt.cas += first ? 1u : 0u; /* first attempt of this group, else a retry */
                cnt.retry += first ? 0u : 1u;
                const R prev = Rec<R>::cas(p, o, n);
                if (prev == o) {
                    pending = false;
                    const uint32_t cn = race_class(st_of(n)), co = race_class(st_of(o));
                    cls = (rep && cn > co) ? cn : 0u;
                    rtid = rt;
                } else {
                    o = prev;
                }
            }
        }
        first = false;
    }
    return cls;
}

/* a7: warp-compacted report append (one atomicAdd per warp) */
__device__ __forceinline__ void append_reports(const hirace_dev_ctx &c, uint32_t cls, uint64_t key, uint32_t g,
                                               uint32_t rtid, uint32_t lane)
{
    const uint32_t m = __ballot_sync(FULL, cls != 0);
    if (!m)
        return;
    unsigned long long base = 0;
    const int first = __ffs(m) - 1;
    if ((int)lane == first)
        base = atomicAdd(c.report_count, (unsigned long long)__popc(m));
    base = __shfl_sync(FULL, base, first);
    if (cls) {
        const unsigned long long pos = base + __popc(m & ((1u << lane) - 1));
        if (pos < c.report_capacity) {
            hirace_race r;
            r.key = key;
            r.cls_and_epoch = cls | (g << 8);
            r.detect_tid = rtid;
            c.reports[pos] = r;
        }
    }
}

/* Contiguous, balanced share of a batch [bstart, bend) for warp w of nw: whole 32-event
 * chunks [c0, c1).  Consecutive chunks of a batch are usually consecutive instructions of the
 * same traced warp and touch the same words; giving them to one replay warp processes them in
 * sequence instead of racing their CASes (grid-stride would run them concurrently). */
__device__ __forceinline__ void warp_share(uint32_t bstart, uint32_t bend, uint32_t w, uint32_t nw, uint32_t lane,
                                           uint32_t &i, uint32_t &iend)
{
    const uint32_t nchunks = (bend - bstart + 31) / 32;
    const uint32_t c0 = (uint32_t)(((uint64_t)nchunks * w) / nw);
    const uint32_t c1 = (uint32_t)(((uint64_t)nchunks * (w + 1)) / nw);
    i = bstart + c0 * 32 + lane;
    iend = min(bend, bstart + c1 * 32);
}


/* one lane's decoded access */
struct Lane {
    uint64_t idx;
    uint32_t tid, kind;
    bool ok;
};
/* race key of a decoded lane (include/hirace.h) */
__device__ __forceinline__ uint64_t key_of_idx(const Lane &L, const hirace_dev_ctx &c, const geom &G)
{
    if (L.idx < c.global_words)
        return L.idx;
    const uint32_t blk = block_of(L.tid, G);
    return HIRACE_SHARED_BIT | ((uint64_t)blk << 32) | (L.idx - c.global_words - (uint64_t)blk * c.smem_words);
}

/* a5 + a6 issue for one chunk whose records o were loaded: transition, then the CAS of every
 * changed word (the result is awaited in chunk_finish, so other work can overlap it) */
template <typename R> struct Issued {
    R n, prev;
    uint32_t ent;
    bool do_cas;
};

template <typename R>
__device__ __forceinline__ Issued<R> chunk_issue(const Lane &cur, R o, const Batch &B, const hirace_dev_ctx &c,
                                                 const geom &G, const Rec<R> &rec, uint32_t tab_s, Counters &cnt)
{
    Issued<R> I;
    I.ent = lds_u8(tab_s + 2048 + (((uint32_t)(o & 31u) << 7) | rec.label(o, cur.tid, cur.kind, B.ep, G)));
    I.n = rec.next(o, I.ent, cur.tid, B.ep);
    /* a6: one CAS per changed word; unchanged = linearised at the load */
    I.do_cas = cur.ok && I.n != o;
    cnt.cas += I.do_cas; /* main-path no-write accesses = checked - first CASes (counted at the end) */
    I.prev = Rec<R>::cas_if(shadow_as<R>(c) + cur.idx, o, I.n, I.do_cas);
    return I;
}

/* a6 result, a3 fold of the lost CASes, a7 report (warp-collective) */
template <typename R>
__device__ __forceinline__ void chunk_finish(const Lane &cur, R o, const Issued<R> &I, const Batch &B,
                                             const hirace_dev_ctx &c, const geom &G, const Rec<R> &rec,
                                             const unsigned char *raw, Counters &cnt, uint32_t lane, uint32_t below)
{
    const bool failed = I.do_cas && I.prev != o;
    /* common case: no lane lost its CAS and no lane's transition reports -> one vote */
    const bool rep = (I.ent & E_REPORT) && I.do_cas && !failed;
    if (!__any_sync(FULL, failed || rep))
        return;
    uint32_t cls = 0, rtid = cur.tid;
    if (rep) {
        const uint32_t cn = race_class(st_of(I.n)), co = race_class(st_of(o));
        cls = cn > co ? cn : 0u;
    }
    if (__any_sync(FULL, failed)) {
        /* Algorithm 1's retry for the lanes whose CAS lost: group them by word, the group
         * leader folds its members' accesses from the record it observed */
        const uint32_t peers = __match_any_sync(FULL, failed ? cur.idx : NONE);
        const bool lead = failed && (peers & below) == 0;
        cls |= commit_groups<R>(shadow_as<R>(c) + cur.idx, I.prev, lead ? peers : 0u, cur.tid, cur.kind, G, raw, B,
                                rec, cnt, rtid, false);
    }
    /* a7 */
    if (__any_sync(FULL, cls != 0))
        append_reports(c, cls, key_of_idx(cur, c, G), B.graw, rtid, lane);
}

/* One 32-event chunk (one event per lane) after decode: a4 load, a5 transition, a6 CAS, a3
 * collision fold, a7 report.  All lanes of the warp call it (warp-collective).  tab_s = shared
 * address of the canonical table; the raw-flag table follows it at +2048. */
template <typename R>
__device__ __forceinline__ void process_decoded(const Lane &cur, const Batch &B, const hirace_dev_ctx &c,
                                                const geom &G, const Rec<R> &rec, const unsigned char *raw,
                                                uint32_t tab_s, Counters &cnt, uint32_t lane, uint32_t below)
{
    /* a4: optimistic: every lane reads its own word (coherent load); lanes that share a word
     * are grouped only if their CAS collides (chunk_finish) */
    const R o = cur.ok ? Rec<R>::load(shadow_as<R>(c) + cur.idx) : (R)0;
    cnt.checked += cur.ok;
    const Issued<R> I = chunk_issue<R>(cur, o, B, c, G, rec, tab_s, cnt);
    chunk_finish<R>(cur, o, I, B, c, G, rec, raw, cnt, lane, below);
}

__device__ __forceinline__ void flush_stats(const hirace_dev_ctx &c, Counters cnt, unsigned long long *s_stats,
                                            uint32_t lane)
{
    cnt.nowrite = cnt.checked - cnt.cas; /* accesses that issued no CAS of their own */
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
        cnt.checked += __shfl_xor_sync(FULL, cnt.checked, d);
        cnt.retry += __shfl_xor_sync(FULL, cnt.retry, d);
        cnt.cas += __shfl_xor_sync(FULL, cnt.cas, d);
        cnt.nowrite += __shfl_xor_sync(FULL, cnt.nowrite, d);
    }
    if (lane == 0) {
        atomicAdd(&s_stats[0], (unsigned long long)cnt.checked);
        atomicAdd(&s_stats[1], (unsigned long long)cnt.retry);
        atomicAdd(&s_stats[2], (unsigned long long)cnt.cas);
        atomicAdd(&s_stats[3], (unsigned long long)cnt.nowrite);
    }
    __syncthreads();
    if (threadIdx.x < 4 && s_stats[threadIdx.x])
        atomicAdd(&c.stats[threadIdx.x], s_stats[threadIdx.x]);
}

} // namespace
} // namespace hirace_impl

#endif
