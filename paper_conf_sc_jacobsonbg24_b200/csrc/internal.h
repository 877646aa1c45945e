/* internal.h — launch wrappers shared by the C-ABI implementation and the kernels. */
#ifndef HIRACE_INTERNAL_H
#define HIRACE_INTERNAL_H

#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace.h"

namespace hirace_impl {

constexpr int kReplayThreads = 256;  /* 8 warps */
constexpr int kCollectTile = 4096;     /* shadow words per collect CTA                 */
constexpr int kCollectThreads = 256;
constexpr uint32_t kFindChunk = 32768; /* top-level batch-boundary probe chunk (32^3)   */

struct Scratch {
    uint32_t *raw_pos;       /* boundary positions found (unsorted), HIRACE_MAX_BATCHES      */
    uint32_t *raw_count;     /* number found (excluding position 0)                          */
    uint32_t *batch_off;     /* sorted batch offsets [0..nb], HIRACE_MAX_BATCHES + 1         */
    uint32_t *nbatches;      /* nb                                                            */
    uint32_t *batch_ctr;     /* per-batch tile-claim counters, HIRACE_MAX_BATCHES             */
    unsigned int *grid_bar;  /* grid barrier counter                                          */
    uint32_t *tile_counts;   /* collect: per-tile counts / offsets                           */
    uint64_t ntiles;
};

/* batch discovery: find_batches + sort_batches */
cudaError_t launch_find_batches(const hirace_event *ev, uint32_t n, const Scratch &s, unsigned int *err,
                                int sm_count, cudaStream_t st);
/* persistent cooperative replay over the discovered batches */
cudaError_t launch_replay(const hirace_dev_ctx &c, const hirace_event *ev, const Scratch &s, int grid,
                          cudaStream_t st);
int replay_max_grid(int device);
/* order-preserving compaction of RACE records from the shadow */
cudaError_t launch_collect(const hirace_dev_ctx &c, uint64_t shadow_words, const Scratch &s, hirace_race *out,
                           uint64_t cap, unsigned long long *d_total, cudaStream_t st);
cudaError_t launch_rebase(const hirace_dev_ctx &c, uint64_t shadow_words, cudaStream_t st);
cudaError_t launch_bucket(const hirace_dev_ctx &c, const hirace_event *in, uint32_t n, int nranks, int my_rank,
                          hirace_event *out, unsigned long long *d_counts, uint32_t *d_tile_hist, uint32_t ntiles,
                          cudaStream_t st);
cudaError_t kernels_init(int device);

} // namespace hirace_impl

#endif
