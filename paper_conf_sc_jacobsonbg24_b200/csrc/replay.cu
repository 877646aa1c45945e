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
 *   a4  each lane's coherent 8-byte shadow load (ld.relaxed.gpu: never a stale L1 line);
 *   a5  relation/sync label by XOR+shift, one lookup in the 2 KB shared-memory table, pack;
 *   a6  one atom.cas.b64 per changed word; an unchanged record issues no CAS (the access is
 *       linearised at the load: no-write fast path, e.g. every read of a G_R word).
 * a3 warp aggregation happens only where it pays: lanes whose CAS lost (typically lanes of
 * the same warp on the same word) are grouped with __match_any_sync and the group leader folds
 * all members' accesses in lane order from the record its CAS returned, then commits them with
 * one CAS (Algorithm 1's retry loop).  Other rare cases also leave the
 * common path behind warp-uniform votes: 8/16-byte accesses, race reports (a7: warp-compacted
 * append, one atomicAdd per warp), invalid events.
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace_device.cuh"
#include "collect.cuh"
#include "internal.h"
#include "kernel_common.cuh"

namespace hirace_impl {

using namespace hirace;

#ifdef HIRACE_WARP_TRACE
/* diagnostics build only: per (batch, replay warp) globaltimer when its share is done, and smid */
__device__ unsigned long long g_warp_trace[16 * 8192 * 4];
/* per replay warp: max (over all chunks of all batches) of load wait, CAS wait, fold time (ns) */
__device__ unsigned long long g_chunk_detail[8192 * 4];
#endif
#ifdef HIRACE_BARRIER_TRACE
/* diagnostics build only: per (batch, CTA) globaltimer at arrival and after release */
__device__ unsigned long long g_bar_trace[128 * 2048 * 2];
__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif

namespace {

constexpr uint32_t FULL = 0xffffffffu;
constexpr uint64_t NONE = ~0ull;
#ifndef HIRACE_REPLAY_MINB
#define HIRACE_REPLAY_MINB 2 /* 2 x 16 warps per SM at <= 64 registers */
#endif
constexpr int kMinBlocks = HIRACE_REPLAY_MINB;

struct Batch {
    uint32_t key, g, b, w, ep; /* ep = epochs in record layout */
};

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
#ifdef HIRACE_EV_EVICT_FIRST
    asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
                 "ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], pol;\n\t}"
#else
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
#endif
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

/* race key (include/hirace.h) of word k of event e */
__device__ __forceinline__ uint64_t key_of(const geom &G, const uint4 &e, uint32_t k)
{
    const uint64_t addr = ((uint64_t)e.y << 32) | e.x;
    const uint64_t word = ((addr & ~HIRACE_SHARED_BIT) >> 2) + k;
    if (addr & HIRACE_SHARED_BIT)
        return HIRACE_SHARED_BIT | ((uint64_t)block_of(e.z, G) << 32) | word;
    return word;
}

/* Fold, for every lane with a non-zero `peers` (a group leader), its group's accesses into
 * record o in lane order: the same sequence of Algorithm-1 transitions as if their CASes had
 * won one after another.  Accessors are broadcast by shuffle, so all lanes must call it. */
__device__ __forceinline__ uint64_t fold_shfl(uint64_t o, uint32_t peers, uint32_t my_tid, uint32_t my_kind,
                                              const geom &G, const unsigned char *tab, const Batch &B,
                                              uint32_t &rep, uint32_t &rtid)
{
    uint64_t n = o;
    for (uint32_t uni = __reduce_or_sync(FULL, peers); uni; uni &= uni - 1) {
        const int m = __ffs(uni) - 1;
        const uint32_t t = __shfl_sync(FULL, my_tid, m);
        const uint32_t k = __shfl_sync(FULL, my_kind, m);
        if ((peers >> m) & 1u) {
            access a{t, k, B.g, B.b, B.w};
            uint32_t r = 0;
            n = step(n, a, tab, G, &r);
            if (r) {
                rep = 1;
                rtid = t;
            }
        }
    }
    return n;
}

/* Commit for group leaders (peers != 0 only in leaders) starting from observed records o:
 * fold, CAS, re-fold on failure until every leader's CAS sticks or the record is unchanged.
 * Returns the report class for this lane; counts into cnt. */
__device__ __forceinline__ uint32_t commit_groups(unsigned long long *p, uint64_t o, uint32_t peers, uint32_t tid,
                                                  uint32_t kind, const geom &G, const unsigned char *tab,
                                                  const Batch &B, Counters &cnt, uint32_t &rtid, bool first)
{
    bool pending = peers != 0;
    uint32_t cls = 0;
    while (__any_sync(FULL, pending)) {
        uint32_t rep = 0, rt = 0;
        const uint64_t n = fold_shfl(o, pending ? peers : 0u, tid, kind, G, tab, B, rep, rt);
        if (pending) {
            if (n == o) {
                pending = false;
            } else {
                cnt.cas += first ? 1u : 0u; /* first attempt of this group, else a retry */
                cnt.retry += first ? 0u : 1u;
                const uint64_t prev = cas64(p, o, n);
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

/* chunks holding 8/16-byte accesses: word by word through the group commit (rare; the configs
 * emit 4-byte accesses).  `take` marks this lane's event as one to process here. */
__device__ __noinline__ uint4 chunk_multiword(const hirace_dev_ctx c, const geom G, const unsigned char *tab,
                                              const Batch B, uint4 e, bool take, uint32_t lane)
{
    Counters cnt{0, 0, 0, 0};
    const uint64_t addr = ((uint64_t)e.y << 32) | e.x;
    const uint32_t szl = (e.w >> 2) & 7u;
    const uint32_t nw = szl <= 2 ? 1u : (1u << (szl - 2));
    const uint64_t word = (addr & ~HIRACE_SHARED_BIT) >> 2;
    const bool sh = (addr & HIRACE_SHARED_BIT) != 0;
    const uint64_t base = sh ? c.global_words + (uint64_t)block_of(e.z, G) * c.smem_words + word : word;
    const uint32_t maxnw = __reduce_max_sync(FULL, take ? nw : 0u);
    for (uint32_t k = 0; k < maxnw; k++) {
        const bool act = take && k < nw;
        const uint64_t my = act ? base + k : NONE;
        const uint32_t peers = __match_any_sync(FULL, my);
        cnt.checked += act;
        const bool lead = act && (peers & ((1u << lane) - 1)) == 0;
        const uint64_t o = lead ? ld_coherent(c.shadow + my) : 0;
        uint32_t rtid = 0;
        const uint32_t cls =
            commit_groups(c.shadow + my, o, lead ? peers : 0u, e.z, e.w & 3u, G, tab, B, cnt, rtid, true);
        if (__any_sync(FULL, cls != 0))
            append_reports(c, cls, key_of(G, e, k), B.g, rtid, lane);
    }
    return make_uint4(cnt.checked, cnt.retry, cnt.cas, cnt.nowrite);
}

#ifndef HIRACE_STEAL
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
#endif

/* one lane's decoded access */
struct Lane {
    uint64_t idx;
    uint32_t tid, kind;
    bool ok;
};

/* a2: decode + validate one lane's event (sub-word accesses map to their word); 8/16-byte
 * accesses of the chunk are committed right here, word by word.  W32: the whole shadow has
 * < 2^31 words and tracked byte offsets fit 32 bits, so index math and range checks are 32-bit
 * (fewer instructions on the hot path); otherwise 64-bit. */
template <bool W32>
__device__ __forceinline__ Lane decode(const uint4 &e, bool valid, uint32_t keysz, const Batch &B,
                                       uint32_t tid_max, const hirace_dev_ctx &c, const geom &G,
                                       const unsigned char *tab, Counters &cnt, uint32_t &bad, uint32_t lane)
{
    Lane L;
    L.tid = e.z;
    L.kind = e.w & 3u;
    const uint32_t meta = e.w;
    const bool sh = (int)e.y < 0;
    const bool key_ok = (meta >> 2) - keysz <= 2u; /* same batch, size <= 4 bytes */
    const bool tid_ok = L.tid <= tid_max;
    uint64_t word;
    bool in_range;
    if (W32) {
        const uint32_t w32 = e.x >> 2;
        word = w32;
        in_range = (e.y & 0x7fffffffu) == 0 && w32 < (sh ? c.smem_words : (uint32_t)c.global_words);
    } else {
        word = ((uint64_t)(e.y & 0x7fffffffu) << 30) | (e.x >> 2);
        in_range = sh ? word < c.smem_words : word < c.global_words;
    }
    L.ok = valid && key_ok && tid_ok && in_range;
    if (__any_sync(FULL, valid && !L.ok)) {
        const uint64_t wfull = ((uint64_t)(e.y & 0x7fffffffu) << 30) | (e.x >> 2);
        const uint32_t szl = (meta >> 2) & 7u;
        const bool multi = valid && (meta >> 5) == B.key && (szl == 3 || szl == 4) && tid_ok &&
                           (sh ? wfull + (1u << (szl - 2)) <= c.smem_words : wfull + (1u << (szl - 2)) <= c.global_words);
        if (valid && !L.ok && !multi)
            bad = 1;
        if (__any_sync(FULL, multi)) {
            const uint4 d = chunk_multiword(c, G, tab, B, e, multi, lane);
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

/* race key of a decoded lane (include/hirace.h) */
__device__ __forceinline__ uint64_t key_of_idx(const Lane &L, const hirace_dev_ctx &c, const geom &G)
{
    if (L.idx < c.global_words)
        return L.idx;
    const uint32_t blk = block_of(L.tid, G);
    return HIRACE_SHARED_BIT | ((uint64_t)blk << 32) | (L.idx - c.global_words - (uint64_t)blk * c.smem_words);
}

/* out of line so the collect's registers do not raise the replay loop's allocation */
__device__ __noinline__ unsigned int collect_call(const hirace_dev_ctx c, uint64_t nwords, hirace_race *out, uint64_t cap,
                                                  unsigned long long *d_total, uint32_t *cta_cnt, unsigned int *bar,
                                                  unsigned int epoch)
{
    collect_phase(c, nwords, out, cap, d_total, cta_cnt, bar, epoch);
    return epoch;
}

/* One 32-event chunk (one event per lane): a2 decode, a4 load, a5 transition, a6 CAS, a3
 * collision fold, a7 report.  All lanes of the warp call it (warp-collective). */
__device__ __forceinline__ void process_decoded(const Lane &cur, const Batch &B, const hirace_dev_ctx &c,
                                                const geom &G, const unsigned char *s_table, uint32_t tab_s,
                                                Counters &cnt, uint32_t lane, uint32_t below);

template <bool W32>
__device__ __forceinline__ void process_chunk(const uint4 &e, bool valid, uint32_t keysz, const Batch &B,
                                              uint32_t tid_max, const hirace_dev_ctx &c, const geom &G,
                                              const unsigned char *s_table, uint32_t tab_s, Counters &cnt,
                                              uint32_t &bad, uint32_t lane, uint32_t below)
{
    const Lane cur = decode<W32>(e, valid, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
    process_decoded(cur, B, c, G, s_table, tab_s, cnt, lane, below);
}

__device__ __forceinline__ void process_decoded(const Lane &cur, const Batch &B, const hirace_dev_ctx &c,
                                                const geom &G, const unsigned char *s_table, uint32_t tab_s,
                                                Counters &cnt, uint32_t lane, uint32_t below)
{

    /* a4: optimistic: every lane reads its own word (coherent load); lanes that share a word
     * are grouped only if their CAS collides (below) */
    unsigned long long *const p = c.shadow + cur.idx;
#ifdef HIRACE_WARP_TRACE
    const unsigned long long tt0 = gtimer();
#endif
    const uint64_t o = cur.ok ? ld_coherent(p) : 0;
    cnt.checked += cur.ok;
#ifdef HIRACE_WARP_TRACE
    uint32_t dmy;
    asm volatile("add.u32 %0, %1, 0;" : "=r"(dmy) : "r"((uint32_t)o));
    const unsigned long long tt1 = gtimer();
#endif

    /* a5: transition */
    const access a{cur.tid, cur.kind, B.g, B.b, B.w};
    const uint32_t ent = lds_u8(tab_s + 2048 + ((st_of(o) << 7) | label_raw(o, a, G)));
    const uint64_t n = (ent & E_KEEP) ? ((o & ~(uint64_t)31) | (ent & E_STATE))
                                      : (((uint64_t)cur.tid << SH_TID) | B.ep | (ent & E_STATE));
    /* a6: one CAS per changed word; unchanged = linearised at the load */
    const bool do_cas = cur.ok && n != o;
    cnt.cas += do_cas; /* main-path no-write accesses = checked - first CASes (counted at the end) */
    const uint64_t prev = cas64_if(p, o, n, do_cas);
    const bool failed = do_cas && prev != o;
    /* common case: no lane lost its CAS and no lane's transition reports -> one vote */
    const bool rep = (ent & E_REPORT) && do_cas && !failed;
#ifndef HIRACE_WARP_TRACE
    if (!__any_sync(FULL, failed || rep))
        return;
#endif
    uint32_t cls = 0, rtid = cur.tid;
    if (rep) {
        const uint32_t cn = race_class(st_of(n)), co = race_class(st_of(o));
        cls = cn > co ? cn : 0u;
    }
#ifdef HIRACE_WARP_TRACE
    const unsigned long long tt2 = gtimer();
    const bool failed_any = __any_sync(FULL, failed);
#endif
    if (__any_sync(FULL, failed)) {
        /* Algorithm 1's retry for the lanes whose CAS lost: group them by word, the group
         * leader folds its members' accesses from the record it observed */
        const uint32_t peers = __match_any_sync(FULL, failed ? cur.idx : NONE);
        const bool lead = failed && (peers & below) == 0;
        cls |= commit_groups(p, prev, lead ? peers : 0u, cur.tid, cur.kind, G, s_table, B, cnt, rtid, false);
    }
    /* a7 */
    if (__any_sync(FULL, cls != 0))
        append_reports(c, cls, key_of_idx(cur, c, G), B.g, rtid, lane);
#ifdef HIRACE_WARP_TRACE
    const unsigned long long tt3 = gtimer();
    if (lane == 0) {
        const uint32_t wg = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
        if (wg < 8192) {
            unsigned long long *d = &g_chunk_detail[wg * 4];
            const bool anyf = __any_sync(1u, failed_any);
            if (!anyf && tt3 - tt0 > d[0]) d[0] = tt3 - tt0;
            if (anyf && tt3 - tt0 > d[1]) d[1] = tt3 - tt0;
            d[2] += anyf;
            if (tt1 - tt0 > d[3]) d[3] = tt1 - tt0;
        }
    }
#endif
}

#ifdef HIRACE_PIPE
/* Pipelined chunk processing (opt-in, -DHIRACE_PIPE; measured slower).  The shadow loads of chunk i+1 are issued right after
 * chunk i's CASes, before their results are awaited, so each chunk costs about one L2 round
 * trip instead of two (load, then CAS).  Issued after the CASes in program order, the loads
 * normally observe them; a load that does not (another lane's word, reordered in the memory
 * system) is only stale for a same-batch access, which is either linearised before the CAS
 * (no store) or fails its own CAS and retries: the same argument as for concurrent warps
 * (Algorithm 1; any in-batch order is a linear extension, L177). */
struct Staged {
    Lane L;
    uint64_t o; /* observed record */
};

__device__ __forceinline__ Staged stage_chunk(const uint4 &e, bool valid, uint32_t keysz, const Batch &B,
                                              uint32_t tid_max, const hirace_dev_ctx &c, const geom &G,
                                              const unsigned char *s_table, Counters &cnt, uint32_t &bad,
                                              uint32_t lane)
{
    Staged S;
    S.L = decode<false>(e, valid, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
    S.o = ld_coherent_if(c.shadow + S.L.idx, S.L.ok, 0); /* a4 */
    return S;
}

/* a5 + a6 issue: transition of the staged record and its CAS (result not awaited here) */
struct Issued {
    uint64_t n, prev;
    uint32_t ent;
    bool do_cas;
};

__device__ __forceinline__ Issued issue_chunk(const Staged &S, const Batch &B, const geom &G, uint32_t tab_s,
                                              const hirace_dev_ctx &c, Counters &cnt)
{
    Issued I;
    const access a{S.L.tid, S.L.kind, B.g, B.b, B.w};
    I.ent = lds_u8(tab_s + ((st_of(S.o) << 6) | label(S.o, a, G)));
    I.n = (I.ent & E_KEEP) ? ((S.o & ~(uint64_t)31) | (I.ent & E_STATE))
                           : (((uint64_t)S.L.tid << SH_TID) | B.ep | (I.ent & E_STATE));
    I.do_cas = S.L.ok && I.n != S.o;
    cnt.checked += S.L.ok;
    cnt.cas += I.do_cas;
    I.prev = cas64_if(c.shadow + S.L.idx, S.o, I.n, I.do_cas);
    return I;
}

/* a6 result, a3 fold of lost CASes, a7 report (warp-collective) */
__device__ __forceinline__ void finish_chunk(const Staged &S, const Issued &I, const Batch &B, const geom &G,
                                             const unsigned char *s_table, const hirace_dev_ctx &c, Counters &cnt,
                                             uint32_t lane, uint32_t below)
{
    uint32_t cls = 0, rtid = S.L.tid;
    if (I.do_cas && I.prev == S.o) {
        const uint32_t cn = race_class(st_of(I.n)), co = race_class(st_of(S.o));
        cls = ((I.ent & E_REPORT) && cn > co) ? cn : 0u;
    }
    const bool failed = I.do_cas && I.prev != S.o;
    if (__any_sync(FULL, failed)) {
        const uint32_t peers = __match_any_sync(FULL, failed ? S.L.idx : NONE);
        const bool lead = failed && (peers & below) == 0;
        cnt.retry += lead;
        cls |= commit_groups(c.shadow + S.L.idx, I.prev, lead ? peers : 0u, S.L.tid, S.L.kind, G, s_table, B, cnt,
                             rtid, true);
    }
    if (__any_sync(FULL, cls != 0))
        append_reports(c, cls, key_of_idx(S.L, c, G), B.g, rtid, lane);
}
#endif

#ifdef HIRACE_STEAL
/* Work stealing inside a CTA (cuts the batch tail before each grid barrier).  Each warp's
 * contiguous share [c0, c1) of the batch's chunks sits in one shared 32-bit word
 * back:16 | front:16 (relative to c0; native 32-bit shared atomics).  The owner claims from
 * the front with an atomic add of 1, issued one hand-out ahead so its latency is hidden (the
 * result is consumed a chunk later); a warp whose share is exhausted takes single chunks from
 * the back of the CTA's fullest share with an atomic add of -2^16.  Claims linearise on the
 * word, so every chunk is replayed exactly once; owner and thieves work at opposite ends of a
 * share, far apart until it is nearly drained (adjacent chunks touch the same words).  Any
 * order of a batch's events is a linear extension of happens-before.
 * Double-buffered by batch parity, so the next batch's shares are published (and the owners'
 * first claims issued) before the grid barrier.  Shares must stay below 2^15 chunks. */
__device__ __forceinline__ uint32_t atom_add_shared_if(uint32_t *p, uint32_t v, bool pred)
{
    uint32_t r = 0;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q atom.shared.add.u32 %0, [%1], %2;\n\t}"
                 : "+r"(r)
                 : "r"(smem_u32(p)), "r"(v), "r"((uint32_t)pred)
                 : "memory");
    return r;
}

__device__ __forceinline__ int share_begin(uint32_t nchunks, uint32_t w, uint32_t nw)
{
    return (int)(((uint64_t)nchunks * w) / nw);
}

__device__ __forceinline__ void share_init(uint32_t *s_rng, uint32_t bstart, uint32_t bend, uint32_t w, uint32_t nw,
                                           uint32_t wib, uint32_t lane, int &ca, int &cb, int &c0,
                                           uint32_t &pend)
{
    const uint32_t nchunks = (bend - bstart + 31) / 32;
    c0 = share_begin(nchunks, w, nw);
    const int len = share_begin(nchunks, w + 1, nw) - c0;
    ca = len > 0 ? c0 : -1;
    cb = len > 1 ? c0 + 1 : -1;
    if (lane == 0)
        s_rng[wib] = ((uint32_t)len << 16) | 2u;
    pend = atom_add_shared_if(&s_rng[wib], 1u, lane == 0); /* same thread: ordered after the store */
}

__device__ __forceinline__ uint4 chunk_event(const uint4 *ev, int ch, uint32_t bstart, uint32_t bend, uint32_t lane)
{
    const uint32_t i = bstart + (uint32_t)ch * 32u + lane;
    return (ch >= 0 && i < bend) ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
}

/* consume the pending front claim (lane 0's atomic result) and issue the next one */
__device__ __forceinline__ int claim_front(uint32_t *r, uint32_t &pend, int c0, uint32_t lane)
{
    const int f = (int)(int16_t)(pend & 0xffffu), bk = (int)(int16_t)(pend >> 16);
    const int ch = __shfl_sync(FULL, f < bk ? c0 + f : -1, 0);
    if (ch >= 0)
        pend = atom_add_shared_if(r, 1u, lane == 0);
    return ch;
}

/* a chunk from the back of the fullest share of this CTA, or -1 when all are drained */
__device__ __forceinline__ int steal_back(uint32_t *s_rng, uint32_t nwib, uint32_t lane, uint32_t nchunks,
                                          uint32_t warp0, uint32_t nw)
{
    for (;;) {
        int rem = -1;
        if (lane < nwib) {
            const uint32_t r = *(volatile uint32_t *)&s_rng[lane];
            rem = (int)(int16_t)(r >> 16) - (int)(int16_t)(r & 0xffffu);
        }
        const int best = __reduce_max_sync(FULL, rem);
        if (best <= 0)
            return -1;
        const uint32_t v = __ffs(__ballot_sync(FULL, rem == best)) - 1;
        int ch = -1;
        if (lane == 0) {
            const uint32_t old = atomicAdd(&s_rng[v], 0xffff0000u);
            const int f = (int)(int16_t)(old & 0xffffu), bk = (int)(int16_t)(old >> 16);
            ch = f < bk ? share_begin(nchunks, warp0 + v, nw) + bk - 1 : -1;
        }
        ch = __shfl_sync(FULL, ch, 0);
        if (ch >= 0)
            return ch;
    }
}
#endif

template <bool P2, bool W32>
__global__ void __launch_bounds__(kReplayThreads, kMinBlocks)
    k_replay(hirace_dev_ctx c, const uint4 *__restrict__ ev, const uint32_t *__restrict__ off,
             const uint32_t *__restrict__ nbp, unsigned int *bar, uint64_t shadow_words, hirace_race *out,
             uint64_t cap, unsigned long long *d_total, uint32_t *cta_cnt)
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
    const uint32_t nb = *nbp;
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t tid_max = total_threads > 0xffffffffull ? 0xffffffffu : (uint32_t)(total_threads - 1);
    const uint32_t below = (1u << lane) - 1;
    const uint32_t tab_s = smem_u32(s_table);
    const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    unsigned int bar_epoch = 0;
    Counters cnt{0, 0, 0, 0};
    uint32_t bad = 0;

    /* a1: events of the first chunks of every batch are requested before the barrier that
     * precedes the batch, so the HBM latency overlaps the barrier */
    uint32_t bstart = nb ? __ldg(&off[0]) : 0, bend = nb ? __ldg(&off[1]) : 0;
#ifdef HIRACE_STEAL
    __shared__ uint32_t s_rng[2][kReplayThreads / 32];
    const uint32_t wib = threadIdx.x >> 5, nwib = blockDim.x >> 5;
    int ca, cb, c0; /* this warp's next two chunks (batch-relative, -1 = none); share start */
    uint32_t pend;  /* lane 0: result of the in-flight front claim */
    const uint32_t warp0 = blockIdx.x * nwib;
    share_init(s_rng[0], bstart, bend, warp_global, nwarps, wib, lane, ca, cb, c0, pend);
    uint4 e0 = chunk_event(ev, ca, bstart, bend, lane);
    uint4 e1 = chunk_event(ev, cb, bstart, bend, lane);
    __syncthreads();
#else
    __syncthreads();
    uint32_t i, iend; /* this warp's contiguous share of the batch: events [i - lane, iend) */
    warp_share(bstart, bend, warp_global, nwarps, lane, i, iend);
    uint4 e0 = i < iend ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
    uint4 e1 = i + 32 < iend ? ld_event(ev + i + 32) : make_uint4(0, 0, 0, 0);
#endif
    for (uint32_t bi = 0; bi < nb; bi++) {
        Batch B;
        B.key = __ldg(&ev[bstart].w) >> 5;
        B.g = B.key >> 19;
        B.b = (B.key >> 9) & 1023u;
        B.w = B.key & 511u;
        B.ep = (B.g << SH_G) | (B.b << SH_B) | (B.w << SH_W);
        const uint32_t keysz = B.key << 3; /* (meta >> 2) - keysz = size_log2 for this batch */
        if (B.g == 255u)
            bad = 1; /* reserved for retired RACE records (R7) */

#ifdef HIRACE_STEAL
        uint32_t *const rng = s_rng[bi & 1];
        const uint32_t nchunks = (bend - bstart + 31) / 32;
        bool own = true; /* still claiming from this warp's own share */
        while (ca >= 0) {
            const uint4 e = e0;
            const bool valid = bstart + (uint32_t)ca * 32u + lane < bend;
            e0 = e1; /* a1: keep the next chunks' events in flight */
            ca = cb;
            if (own) { /* own share front to back, then the back ends of the CTA's other shares */
                cb = claim_front(&rng[wib], pend, c0, lane);
                own = cb >= 0;
            }
#ifndef HIRACE_STEAL_OFF
            if (!own)
                cb = steal_back(rng, nwib, lane, nchunks, warp0, nwarps);
#endif
            e1 = chunk_event(ev, cb, bstart, bend, lane);
            process_chunk<W32>(e, valid, keysz, B, tid_max, c, G, s_table, tab_s, cnt, bad, lane, below);
        }
#ifdef HIRACE_WARP_TRACE
        if (lane == 0 && bi < 16 && warp_global < 8192) {
            uint32_t smid;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            g_warp_trace[(bi * 8192 + warp_global) * 4] = gtimer();
            g_warp_trace[(bi * 8192 + warp_global) * 4 + 1] = smid;
        }
#endif
        if (bi + 1 < nb) {
            bstart = __ldg(&off[bi + 1]);
            bend = __ldg(&off[bi + 2]);
            share_init(s_rng[(bi + 1) & 1], bstart, bend, warp_global, nwarps, wib, lane, ca, cb, c0, pend);
            e0 = chunk_event(ev, ca, bstart, bend, lane);
            e1 = chunk_event(ev, cb, bstart, bend, lane);
#else
#if defined(HIRACE_UNROLL2) && !defined(HIRACE_PIPE)
        /* two chunks per trip: e0/e1 are refilled in place right after their decode, so the
         * prefetch pipeline costs no register moves */
        for (;;) {
            if (i - lane >= iend)
                break;
            Lane cur = decode<W32>(e0, i < iend, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
            ld_event_if(ev + i + 64, i + 64 < iend, e0);
            process_decoded(cur, B, c, G, s_table, tab_s, cnt, lane, below);
            i += 32;
            if (i - lane >= iend)
                break;
            cur = decode<W32>(e1, i < iend, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
            ld_event_if(ev + i + 64, i + 64 < iend, e1);
            process_decoded(cur, B, c, G, s_table, tab_s, cnt, lane, below);
            i += 32;
        }
#elif !defined(HIRACE_PIPE)
#ifdef HIRACE_WARP_TRACE
        unsigned long long t_prev = gtimer(), t_max = 0, t_at = 0, t_evmax = 0;
#endif
        for (; i - lane < iend; i += 32) {
            const uint4 e = e0;
            const bool valid = i < iend;
            e0 = e1; /* a1: keep the next chunks' events in flight */
            ld_event_if(ev + i + 64, i + 64 < iend, e1);
#ifdef HIRACE_WARP_TRACE
            {
                uint32_t dmy;
                asm volatile("add.u32 %0, %1, %2;" : "=r"(dmy) : "r"(e.x), "r"(e.w));
                const unsigned long long t_ev = gtimer();
                if (t_ev - t_prev > t_evmax)
                    t_evmax = t_ev - t_prev;
            }
#endif
            process_chunk<W32>(e, valid, keysz, B, tid_max, c, G, s_table, tab_s, cnt, bad, lane, below);
#ifdef HIRACE_WARP_TRACE
            const unsigned long long t_now = gtimer();
            if (t_now - t_prev > t_max) {
                t_max = t_now - t_prev;
                t_at = i - lane;
            }
            t_prev = t_now;
#endif
        }
#else
        if (i - lane < iend) {
            Staged cur = stage_chunk(e0, i < iend, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
            e0 = e1; /* a1: keep the next chunks' events in flight */
            e1 = i + 64 < iend ? ld_event(ev + i + 64) : make_uint4(0, 0, 0, 0);
            for (;; i += 32) {
                const Issued I = issue_chunk(cur, B, G, tab_s, c, cnt);
                const bool more = i + 32 - lane < iend; /* warp-uniform */
                Staged nxt;
                if (more) { /* next chunk's shadow loads go out behind this chunk's CASes */
                    nxt = stage_chunk(e0, i + 32 < iend, keysz, B, tid_max, c, G, s_table, cnt, bad, lane);
                    e0 = e1;
                    e1 = i + 96 < iend ? ld_event(ev + i + 96) : make_uint4(0, 0, 0, 0);
                }
                finish_chunk(cur, I, B, G, s_table, c, cnt, lane, below);
                if (!more)
                    break;
                cur = nxt;
            }
            i += 32;
        }
#endif
#ifdef HIRACE_WARP_TRACE
        if (lane == 0 && bi < 16 && warp_global < 8192) {
            uint32_t smid;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            g_warp_trace[(bi * 8192 + warp_global) * 4] = gtimer();
            g_warp_trace[(bi * 8192 + warp_global) * 4 + 1] = smid;
            g_warp_trace[(bi * 8192 + warp_global) * 4 + 2] = t_max;
            g_warp_trace[(bi * 8192 + warp_global) * 4 + 3] = t_at | (t_evmax << 32);
        }
#endif
        if (bi + 1 < nb) {
            bstart = __ldg(&off[bi + 1]);
            bend = __ldg(&off[bi + 2]);
            warp_share(bstart, bend, warp_global, nwarps, lane, i, iend);
            e0 = i < iend ? ld_event(ev + i) : make_uint4(0, 0, 0, 0);
            e1 = i + 32 < iend ? ld_event(ev + i + 32) : make_uint4(0, 0, 0, 0);
#endif
#ifdef HIRACE_BARRIER_TRACE
            __syncthreads();
            if (threadIdx.x == 0 && bi < 128 && blockIdx.x < 2048)
                g_bar_trace[(bi * 2048 + blockIdx.x) * 2] = gtimer();
#endif
            grid_sync(bar, gridDim.x, bar_epoch);
#ifdef HIRACE_BARRIER_TRACE
            if (threadIdx.x == 0 && bi < 128 && blockIdx.x < 2048)
                g_bar_trace[(bi * 2048 + blockIdx.x) * 2 + 1] = gtimer();
#endif
        }
    }

    /* fused a7 collection (hirace_check_trace_device): one more barrier, then the shadow scan */
    if (d_total) {
        grid_sync(bar, gridDim.x, bar_epoch);
        bar_epoch = collect_call(c, shadow_words, out, cap, d_total, cta_cnt, bar, bar_epoch);
    }

    if (__any_sync(FULL, bad) && lane == 0)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
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

/* Single-batch replay of 8-byte wire records (sharded mode): word:31 |
 * shared:1 | tid:30 | kind:2; the batch's (g,b,w) is given, so no batch discovery and no grid
 * barrier — a plain launch.  Each warp walks a contiguous balanced share of 32-record chunks
 * with the same per-chunk path (a4-a7) as k_replay. */
template <bool P2>
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
    const uint64_t total_threads = (uint64_t)c.grid_blocks * c.block_threads;
    const uint32_t below = (1u << lane) - 1;
    const uint32_t tab_s = smem_u32(s_table);
    Counters cnt{0, 0, 0, 0};
    Batch B;
    B.key = key;
    B.g = key >> 19;
    B.b = (key >> 9) & 1023u;
    B.w = key & 511u;
    B.ep = (B.g << SH_G) | (B.b << SH_B) | (B.w << SH_W);
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
        const bool valid = i < iend;
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
        process_decoded(L, B, c, G, s_table, tab_s, cnt, lane, below);
    }
    if ((__any_sync(FULL, bad) || B.g == 255u) && lane == 0)
        atomicOr(c.error_flags, ERR_BAD_TRACE);
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

#ifdef HIRACE_WARP_TRACE
extern "C" int hirace_debug_chunk_detail(unsigned long long *host, uint64_t n)
{
    return (int)cudaMemcpyFromSymbol(host, g_chunk_detail, n * sizeof(unsigned long long));
}
extern "C" int hirace_debug_warp_trace(unsigned long long *host, uint64_t n)
{
    return (int)cudaMemcpyFromSymbol(host, g_warp_trace, n * sizeof(unsigned long long));
}
#endif
#ifdef HIRACE_BARRIER_TRACE
extern "C" int hirace_debug_barrier_trace(unsigned long long *host, uint64_t n)
{
    return (int)cudaMemcpyFromSymbol(host, g_bar_trace, n * sizeof(unsigned long long));
}
#endif

int replay_max_grid(int device)
{
    int sms = 0, occ = 0, occ2 = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    int occ3 = 0, occ4 = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_replay<true, false>, kReplayThreads, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, k_replay<false, false>, kReplayThreads, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ3, k_replay<true, true>, kReplayThreads, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ4, k_replay<false, true>, kReplayThreads, 0);
    occ = occ < occ2 ? occ : occ2;
    occ = occ < occ3 ? occ : occ3;
    occ = occ < occ4 ? occ : occ4;
    if (occ < 1)
        occ = 1;
    return sms * occ;
}

int collect_max_grid(int device)
{
    int sms = 0, occ = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_collect, 256, 0);
    if (occ < 1)
        occ = 1;
    return sms * occ < kMaxCtas ? sms * occ : kMaxCtas;
}

cudaError_t launch_replay_wire(const hirace_dev_ctx &c, const unsigned long long *wire, uint32_t n, uint32_t batch_key,
                               int grid, cudaStream_t st)
{
    const bool p2 = (c.block_threads & (c.block_threads - 1)) == 0 && (c.warp_size & (c.warp_size - 1)) == 0;
    const uint32_t need = (n + 31) / 32; /* no more warps than chunks */
    const uint64_t want = ((uint64_t)need * 32 + kReplayThreads - 1) / kReplayThreads;
    const int g2 = (int)(want < (uint64_t)grid ? want : (uint64_t)grid);
    if (p2)
        k_replay_wire<true><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
    else
        k_replay_wire<false><<<g2, kReplayThreads, 0, st>>>(c, wire, n, batch_key);
    return cudaGetLastError();
}

cudaError_t launch_replay(const hirace_dev_ctx &c, const hirace_event *ev, const Scratch &s, int grid,
                          cudaStream_t st, uint64_t shadow_words, hirace_race *out, uint64_t cap,
                          unsigned long long *d_total)
{
    cudaError_t e = cudaMemsetAsync(s.grid_bar, 0, sizeof(unsigned int), st);
    if (e != cudaSuccess)
        return e;
    hirace_dev_ctx cc = c;
    const uint4 *evp = reinterpret_cast<const uint4 *>(ev);
    const uint32_t *offp = s.batch_off;
    const uint32_t *nbp = s.nbatches;
    unsigned int *barp = s.grid_bar;
    uint64_t nw = shadow_words, cp = cap;
    hirace_race *o = out;
    unsigned long long *dt = d_total;
    uint32_t *cnt = s.cta_cnt;
    void *args[] = {&cc, &evp, &offp, &nbp, &barp, &nw, &o, &cp, &dt, &cnt};
    const bool p2 = (c.block_threads & (c.block_threads - 1)) == 0 && (c.warp_size & (c.warp_size - 1)) == 0;
    /* W32: every shadow index and tracked byte offset fits 32 bits (see decode) */
    const uint64_t sw = c.global_words + (uint64_t)c.grid_blocks * c.smem_words;
#ifdef HIRACE_NO_W32
    const bool w32 = false;
    (void)sw;
#else
    const bool w32 = sw < (1ull << 31) && c.global_words < (1ull << 30) && c.smem_words < (1u << 30);
#endif
    const void *fn = p2 ? (w32 ? (const void *)k_replay<true, true> : (const void *)k_replay<true, false>)
                        : (w32 ? (const void *)k_replay<false, true> : (const void *)k_replay<false, false>);
    return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kReplayThreads), args, 0, st);
}

} // namespace hirace_impl
