/* internal.h — launch wrappers shared by the C-ABI implementation and the kernels. */
#ifndef HIRACE_INTERNAL_H
#define HIRACE_INTERNAL_H

#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace.h"

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
/* order-preserving compaction of RACE records from the shadow */
cudaError_t launch_collect(const hirace_dev_ctx &c, uint64_t shadow_words, const Scratch &s, hirace_race *out,
                           uint64_t cap, unsigned long long *d_total, cudaStream_t st, int report_mode = 0);
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
cudaError_t launch_bucket_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, int my_rank,
                               unsigned long long *out, uint64_t cap, uint32_t *d_tile_hist,
                               unsigned long long *d_tile_off, unsigned long long *d_running,
                               unsigned long long *d_counts_row, unsigned int *err, cudaStream_t st);
/* one batch [lo, hi) -> wire records stored straight into their owners' receive buffers
 * d_peer[owner] starting at d_owner_base[owner] (peer dispatch; d_peer / d_owner_base are
 * device arrays of nranks entries) */
cudaError_t launch_dispatch_wire(const hirace_event *in, uint32_t lo, uint32_t hi, int nranks, int my_rank,
                                 unsigned long long *const *d_peer, const unsigned long long *d_owner_base,
                                 uint32_t *d_tile_hist, unsigned long long *d_tile_off, unsigned int *err,
                                 cudaStream_t st);
/* single-batch replay of 8-byte wire records (batch key given) */
cudaError_t launch_replay_wire(const hirace_dev_ctx &c, const unsigned long long *wire, uint32_t n, uint32_t batch_key,
                               int grid, cudaStream_t st);
constexpr int kWireTile = 4096;
cudaError_t kernels_init(int device);

} // namespace hirace_impl

#endif
