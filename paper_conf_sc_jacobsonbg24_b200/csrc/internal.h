/* internal.h — launch wrappers shared by the C-ABI implementation and the kernels. */
#ifndef HIRACE_INTERNAL_H
#define HIRACE_INTERNAL_H

#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace.h"
#include "hirace_device.cuh"

namespace hirace_impl {

#ifndef HIRACE_REPLAY_THREADS
#define HIRACE_REPLAY_THREADS 512 /* 16 warps */
#endif
constexpr int kReplayThreads = HIRACE_REPLAY_THREADS;
constexpr int kCollectTile = 4096;     /* shadow words per collect CTA                 */
constexpr int kCollectThreads = 256;
constexpr uint32_t kFindChunk = 32768; /* top-level batch-boundary probe chunk (32^3)   */
constexpr int kMaxCtas = 4096;         /* upper bound on co-resident CTAs of our kernels */

struct Scratch {
    uint32_t *batch_off;     /* sorted batch offsets [0..nb], HIRACE_MAX_BATCHES + 1         */
    uint32_t *nbatches;      /* nb                                                            */
    uint32_t *batch_ctr;     /* per-batch tile-claim counters, HIRACE_MAX_BATCHES             */
    unsigned int *grid_bar;  /* grid barrier counter (replay)                                 */
    unsigned int *grid_bar2; /* grid barrier counter (standalone collect)                     */
    uint32_t *cta_cnt;       /* collect: per-CTA flagged-word counts, kMaxCtas                */
    int collect_grid;        /* co-resident CTAs of k_collect                                  */
};

/* batch discovery (one CTA): boundaries, sort, validation */
cudaError_t launch_find_batches(const hirace_event *ev, uint32_t n, const Scratch &s, unsigned int *err,
                                int sm_count, cudaStream_t st);
/* persistent cooperative replay over the discovered batches */
/* optional fused collect at the end of the replay (out == nullptr: none) */
/* report_mode: the fused collect uses the report buffer when it covers every flagged word
 * (collect.cuh; k_collect_reports is launched right after), else the shadow scan */
cudaError_t launch_replay(const hirace_dev_ctx &c, const hirace_event *ev, const Scratch &s, int grid,
                          cudaStream_t st, uint64_t shadow_words = 0, hirace_race *out = nullptr, uint64_t cap = 0,
                          unsigned long long *d_total = nullptr, int report_mode = 0);
int collect_max_grid(int device);
int replay_max_grid(int device);
/* order-preserving compaction of RACE records from the shadow; report_mode 1: the report
 * buffer first (k_collect_reports), the scan only if it does not cover; 2: the same, with
 * k_collect_reports already launched by the caller */
cudaError_t launch_collect(const hirace_dev_ctx &c, uint64_t shadow_words, const Scratch &s, hirace_race *out,
                           uint64_t cap, unsigned long long *d_total, cudaStream_t st, int report_mode = 0);
/* one-CTA report-buffer collect (sort + unique of the reported keys) */
cudaError_t launch_collect_reports(const hirace_dev_ctx &c, hirace_race *out, uint64_t cap,
                                   unsigned long long *d_total, cudaStream_t st);
/* report mode pays off above this shadow size (a scan of it costs more than a launch + sort) */
constexpr uint64_t kReportModeMinBytes = 64ull << 20;
cudaError_t replay_init();
cudaError_t launch_rebase(const hirace_dev_ctx &c, uint64_t shadow_words, cudaStream_t st);
/* shadow := INIT and report count, stats, error flags := 0, in one launch */
cudaError_t launch_reset(void *shadow, uint64_t bytes, unsigned long long *report_count, unsigned long long *stats,
                         unsigned int *err, int sm_count, cudaStream_t st);
cudaError_t launch_bucket(const hirace_dev_ctx &c, const hirace_event *in, uint32_t n, int nranks, int my_rank,
                          hirace_event *out, unsigned long long *d_counts, uint32_t *d_tile_hist, uint32_t ntiles,
                          cudaStream_t st);
/* one batch [lo, hi) of events -> owner-grouped 8-byte wire records at out[*running ...] */
cudaError_t launch_bucket_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, uint32_t block_threads,
                               unsigned long long *out, uint64_t cap, uint32_t *d_tile_hist,
                               unsigned long long *d_tile_off, unsigned long long *d_running,
                               unsigned long long *d_counts_row, unsigned int *err, cudaStream_t st);
/* one batch [lo, hi) -> wire records stored straight into their owners' receive buffers
 * d_peer[owner] starting at d_owner_base[owner] (peer dispatch; d_peer / d_owner_base are
 * device arrays of nranks entries) */
cudaError_t launch_dispatch_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, uint32_t block_threads,
                                 unsigned long long *const *d_peer, const unsigned long long *d_owner_base,
                                 uint32_t *d_tile_hist, unsigned long long *d_tile_off, unsigned int *err,
                                 cudaStream_t st);
/* epoch reset (hirace_set_reset_mode EPOCH): O(flagged) reset, and the pre-replay rebase
 * check (force: always rebase, e.g. before inline hooks); gep = device {gbase, gnext} */
cudaError_t launch_epoch_reset(const hirace_dev_ctx &c, uint64_t shadow_words, unsigned int *gep, int sm_count,
                               cudaStream_t st);
cudaError_t launch_epoch_prep(const hirace_dev_ctx &c, uint64_t shadow_words, unsigned int *gep,
                              const hirace_event *ev, const uint32_t *off, const uint32_t *nbp, int force,
                              int sm_count, cudaStream_t st);
/* per-batch completion flags of the peer dispatch: release [j0, j1] to every owner (d_flags:
 * device array of nranks flag-array addresses), or wait until flags[j] >= target */
cudaError_t launch_peer_release(unsigned int *const *d_flags, int nranks, uint32_t j0, uint32_t j1, cudaStream_t st);
cudaError_t launch_peer_wait(const unsigned int *flags, uint32_t j, uint32_t target, cudaStream_t st);
/* single-batch replay of 8-byte wire records (batch key given) */
cudaError_t launch_replay_wire(const hirace_dev_ctx &c, const unsigned long long *wire, uint32_t n, uint32_t batch_key,
                               int grid, cudaStream_t st);
constexpr int kWireTile = 4096;
cudaError_t kernels_init(int device);

/* ---- window-major replay (window.cu; DESIGN.md §8 "window-major path") ------------------
 * The shadow is cut into windows of 2^wl records.  Element accesses are partitioned by window
 * with one or two counting-sort passes (digits d0 = low d0b bits of the window id, d1 = the
 * rest), keeping batch order inside every window; each light window is then replayed by one
 * CTA with its records in shared memory (TMA bulk copies in and out, shared-memory CAS,
 * __syncthreads between batches instead of grid barriers), heavy windows by all CTAs through
 * the global shadow.  Lazy reset: a window whose gen[] differs from *cur_gen is all-INIT. */
struct WinDev {
    uint32_t wl, d0b, d1b, nw;   /* window = 2^wl records; nw windows; digits              */
    uint32_t p1, p2;             /* events per pass-1 item, records per pass-2 chunk       */
    uint32_t heavy_cap;          /* max heavy windows                                      */
    uint32_t heavy_force;        /* != 0: heavy threshold override (tests: HIRACE_WIN_HEAVY) */
    uint32_t light_ctas;         /* CTAs of the light kernel                               */
    uint64_t elem_cap;           /* capacity of rec1/rec2 (element accesses)               */
    uint32_t items1_cap, chunks2_cap;
    uint4 *items1;               /* pass-1 items {start, end, batch, 0}                    */
    uint32_t *item1_first;       /* [nb + 1] first item of each batch                      */
    uint32_t *batch_key;         /* [nb] batch key (g:8 | b:10 | w:9)                      */
    uint32_t *count1, *count2;   /* digit x item count matrices, scanned in place          */
    unsigned long long *rec1, *rec2;
    uint32_t *win_cnt;           /* [nw + 1] counts, scanned in place into window starts   */
    uint32_t *aux;               /* kAux* slots                                            */
    uint32_t *heavy, *light;     /* window lists                                           */
    uint32_t *hseg;              /* [heavy_cap][nb + 1] batch starts inside heavy windows  */
    uint32_t *gen, *cur_gen;     /* window generation (lazy reset)                         */
    uint32_t *partials;          /* scan scratch (kScanMaxCtas)                            */
    unsigned long long *elems;   /* element accesses counted by pass 1                     */
    unsigned int *bar;           /* grid-barrier counters (kBarSlots)                      */
};
enum : uint32_t { kAuxItems1 = 0, kAuxTotal1, kAuxChunks2, kAuxTotal2, kAuxNHeavy, kAuxNLight, kAuxQueue,
                  kAuxAbort, kAuxViolations, kAuxCount = 16 };
constexpr int kScanMaxCtas = 1024;
constexpr int kBarSlots = 8;
constexpr uint32_t kWinHeavyCap = 64;
constexpr uint32_t ERR_CAPACITY = 8u; /* window path: more element accesses than rec1/rec2 hold */
constexpr uint32_t ERR_HISTORY = 16u; /* masked replay: the sub-warp history table was full     */
/* the whole window-major check: partition, heavy + light replay, then (d_total != null) the
 * collect into out / d_total */
cudaError_t launch_window_check(const hirace_dev_ctx &c, const WinDev &W, const Scratch &s, const hirace_event *ev,
                                uint32_t n, int sm_count, int replay_grid, cudaStream_t st, uint64_t shadow_words,
                                hirace_race *out, uint64_t cap, unsigned long long *d_total);
/* lazy reset: ++*cur_gen, report count / stats / error flags := 0 */
cudaError_t launch_lazy_reset(const hirace_dev_ctx &c, const WinDev &W, cudaStream_t st);
/* stale windows := INIT (all of them, or only when the report buffer does not cover the
 * flagged words and a shadow scan will follow) */
cudaError_t launch_materialize(const hirace_dev_ctx &c, const WinDev &W, int only_if_scan, int sm_count,
                               cudaStream_t st);
const void *window_light_kernel();
int window_light_threads();
size_t window_light_smem(uint32_t wl);
cudaError_t window_init();
/* ---- partial-mask warp syncs (subwarp.cu; hirace_set_warp_syncs, R20) ----------
 * Families = (g, b, warp) with listed syncs, sorted by key g<<50 | b<<40 | warp; sync_w / mask
 * / vrow per listed sync (vrow: the warp vector clock after it, 32 u16); hist: open-addressing
 * table of kSlotWords-word slots [key, owner, spill, 5 entries] plus a pool of 32-lane spill
 * blocks (subwarp.cu). */
constexpr uint32_t kSlotWords = 8; /* = hirace::ws::kSlotWords (checked in subwarp.cu) */
struct WsDev {
    unsigned long long *fam_key;
    uint32_t *fam_lo;        /* [nfam + 1] first listed sync of each family */
    uint32_t *nfam;
    uint32_t *sync_w, *sync_mask, *sync_fam;
    unsigned short *vrow;
    uint4 *fhash;            /* (family, w) lookup: {key lo, key hi, row, smax}; 2x(n + families) */
    unsigned long long fh_mask;
    uint32_t nsync;
    hirace_ws_ctx H;          /* the sub-warp history (hirace_device.cuh hirace::ws)     */
    uint32_t wpb;            /* warps per block */
};
cudaError_t launch_ws_prepare(const hirace_warp_sync *d_syncs, uint32_t n, uint32_t total_warps, uint32_t warp_size,
                              const WsDev &W, unsigned int *err, int sm_count, cudaStream_t st);
cudaError_t launch_replay_masked(const hirace_dev_ctx &c, const WsDev &W, const hirace_event *ev, const Scratch &s,
                                 int grid, cudaStream_t st);
int masked_max_grid(int device);
/* fsm_table.cpp: per state, the RACE state of its hierarchy level under `policy` */
void fsm_race_of(int policy, unsigned char out[32]);

/* process-wide count of kernels the library has launched (hirace_launch_count) */
void note_launches(unsigned k);
unsigned long long launch_count();

} // namespace hirace_impl

#endif
