/*
 * hirace_api.cu — host implementation of the C-ABI declared in include/hirace.h.
 * Every step of the hot path runs in the kernels of hirace_kernels.cu; this file only
 * validates arguments, owns device memory and sequences launches on the caller's stream.
 * There is no CPU fallback: without a CUDA device every entry point that needs one fails
 * with HIRACE_E_CUDA.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "hirace.h"
#include "hirace_device.cuh"
#include "internal.h"

using namespace hirace_impl;

struct hirace_ctx {
    hirace_config cfg;
    int device = 0;
    int sm_count = 0;
    int replay_grid = 0;
    uint64_t global_words = 0, shadow_words = 0;
    unsigned long long *d_shadow = nullptr;
    unsigned char *d_table = nullptr;
    unsigned char h_table[2048 + hirace::RAW_TABLE_BYTES]; /* canonical | raw-flag expansion */
    int policy = HIRACE_POLICY_STRICT;
    hirace_race *d_reports = nullptr;
    unsigned long long *d_report_count = nullptr;
    unsigned long long *d_stats = nullptr;
    unsigned int *d_err = nullptr;
    Scratch scr{};
    /* collect staging (host API) */
    hirace_race *d_collect = nullptr;
    uint64_t collect_cap = 0;
    unsigned long long *d_total = nullptr;
    /* bucket scratch */
    uint32_t *d_bucket_hist = nullptr;
    uint64_t bucket_hist_cap = 0;
    unsigned long long *d_bucket_counts = nullptr;
    /* wire bucket scratch */
    unsigned long long *d_wire_off = nullptr;   /* per-tile offsets of one batch       */
    uint64_t wire_off_cap = 0;
    unsigned long long *d_wire_counts = nullptr; /* nb x nranks (+1: running total)    */
    uint64_t wire_counts_cap = 0;
    unsigned int *d_wire_flag = nullptr;
    /* host-trace staging ring */
    hirace_event *d_stage[2] = {nullptr, nullptr};
    uint64_t stage_cap = 0;
    cudaStream_t copy_stream = nullptr;
    cudaEvent_t ev_copied[2] = {nullptr, nullptr}, ev_used[2] = {nullptr, nullptr};
    hirace_dev_ctx dev{};
    uint32_t g = 0;
    cudaEvent_t t_start = nullptr, t_stop = nullptr;
    hirace_status sticky = HIRACE_OK;
};

namespace {

hirace_status set_sticky(hirace_ctx *c, hirace_status s)
{
    if (c && s != HIRACE_OK && c->sticky == HIRACE_OK)
        c->sticky = s;
    return s;
}

hirace_status from_cuda(hirace_ctx *c, cudaError_t e)
{
    if (e == cudaSuccess)
        return HIRACE_OK;
    return set_sticky(c, e == cudaErrorMemoryAllocation ? HIRACE_E_NOMEM : HIRACE_E_CUDA);
}

#define HR_CUDA(c, x)                                  \
    do {                                               \
        cudaError_t _e = (x);                          \
        if (_e != cudaSuccess)                         \
            return from_cuda((c), _e);                 \
    } while (0)

hirace_status device_errors(hirace_ctx *c)
{
    unsigned int flags = 0;
    cudaError_t e = cudaMemcpy(&flags, c->d_err, sizeof(flags), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess)
        return from_cuda(c, e);
    if (flags & hirace::ERR_BAD_TRACE)
        set_sticky(c, HIRACE_E_BAD_TRACE);
    if (flags & hirace::ERR_CLOCK)
        set_sticky(c, HIRACE_E_CLOCK_OVERFLOW);
    return c->sticky;
}

} // namespace

extern "C" {

const char *hirace_version(void) { return "hirace-b200 0.1 (sm_100a)"; }

const char *hirace_status_string(hirace_status s)
{
    switch (s) {
    case HIRACE_OK: return "ok";
    case HIRACE_E_INVAL: return "invalid argument";
    case HIRACE_E_NOMEM: return "out of memory";
    case HIRACE_E_CUDA: return "CUDA error";
    case HIRACE_E_CLOCK_OVERFLOW: return "epoch clock overflow: detection stopped";
    case HIRACE_E_REPORT_OVERFLOW: return "report overflow";
    case HIRACE_E_BAD_TRACE: return "bad trace";
    case HIRACE_E_COMM: return "communication error";
    }
    return "unknown";
}

hirace_status hirace_shadow_alloc(const hirace_config *cfg, hirace_ctx **out)
{
    if (!cfg || !out)
        return HIRACE_E_INVAL;
    *out = nullptr;
    if (cfg->grid_blocks == 0 || cfg->block_threads == 0 || cfg->warp_size == 0 || cfg->granularity_log2 != 2)
        return HIRACE_E_INVAL;
    if ((uint64_t)cfg->grid_blocks * cfg->block_threads > 0xffffffffull)
        return HIRACE_E_INVAL;
    if ((cfg->smem_bytes_per_block & 3) || (cfg->global_bytes & 3))
        return HIRACE_E_INVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0 || cfg->device < 0 || cfg->device >= ndev)
        return HIRACE_E_CUDA;
    hirace_ctx *c = new (std::nothrow) hirace_ctx();
    if (!c)
        return HIRACE_E_NOMEM;
    c->cfg = *cfg;
    if (c->cfg.report_capacity == 0)
        c->cfg.report_capacity = 1ull << 20;
    c->device = cfg->device;
    c->global_words = cfg->global_bytes >> 2;
    const uint64_t smem_words = cfg->smem_bytes_per_block >> 2;
    c->shadow_words = c->global_words + (uint64_t)cfg->grid_blocks * smem_words;
    if (c->shadow_words == 0)
        c->shadow_words = 1;
    hirace_status st = HIRACE_OK;
    auto fail = [&](cudaError_t e) {
        st = e == cudaErrorMemoryAllocation ? HIRACE_E_NOMEM : HIRACE_E_CUDA;
        hirace_shadow_free(c);
        return st;
    };
    cudaError_t e;
    if ((e = cudaSetDevice(c->device)) != cudaSuccess)
        return fail(e);
    static std::once_flag once[64];
    static cudaError_t init_err[64];
    std::call_once(once[c->device & 63], [&] { init_err[c->device & 63] = kernels_init(c->device); });
    if ((e = init_err[c->device & 63]) != cudaSuccess)
        return fail(e);
    cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, c->device);
    c->replay_grid = replay_max_grid(c->device);
    unsigned char table[2048 + hirace::RAW_TABLE_BYTES];
    if (hirace_fsm_table(table) != HIRACE_OK) {
        hirace_shadow_free(c);
        return HIRACE_E_INVAL;
    }
    c->scr.collect_grid = collect_max_grid(c->device);
    if ((e = cudaMalloc(&c->d_shadow, c->shadow_words * 8)) != cudaSuccess ||
        (e = cudaMalloc(&c->d_table, 2048 + hirace::RAW_TABLE_BYTES)) != cudaSuccess ||
        (e = cudaMalloc(&c->d_reports, c->cfg.report_capacity * sizeof(hirace_race))) != cudaSuccess ||
        (e = cudaMalloc(&c->d_report_count, sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&c->d_stats, 4 * sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&c->d_err, sizeof(unsigned int))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.batch_off, (HIRACE_MAX_BATCHES + 1) * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.nbatches, sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.batch_ctr, HIRACE_MAX_BATCHES * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.grid_bar, sizeof(unsigned int))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.grid_bar2, sizeof(unsigned int))) != cudaSuccess ||
        (e = cudaMalloc(&c->scr.cta_cnt, kMaxCtas * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&c->d_total, sizeof(unsigned long long))) != cudaSuccess)
        return fail(e);
    hirace::expand_raw_table(table, table + 2048); /* the replay kernel's label_raw layout */
    if ((e = cudaMemcpy(c->d_table, table, sizeof(table), cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e);
    hirace_dev_ctx &d = c->dev;
    d.shadow = c->d_shadow;
    d.table = c->d_table;
    d.reports = c->d_reports;
    d.report_count = c->d_report_count;
    d.stats = c->d_stats;
    d.error_flags = c->d_err;
    d.report_capacity = c->cfg.report_capacity;
    d.global_words = c->global_words;
    d.global_base = nullptr;
    d.smem_words = (unsigned int)smem_words;
    d.grid_blocks = cfg->grid_blocks;
    d.block_threads = cfg->block_threads;
    d.warp_size = cfg->warp_size;
    hirace::fastdiv_init(cfg->block_threads, &d.bt_magic, &d.bt_s1, &d.bt_s2);
    hirace::fastdiv_init(cfg->warp_size, &d.ws_magic, &d.ws_s1, &d.ws_s2);
    d.g = 0;
    if (hirace_shadow_reset(c, nullptr) != HIRACE_OK || cudaDeviceSynchronize() != cudaSuccess) {
        hirace_shadow_free(c);
        return HIRACE_E_CUDA;
    }
    *out = c;
    return HIRACE_OK;
}

hirace_status hirace_shadow_free(hirace_ctx *c)
{
    if (!c)
        return HIRACE_OK;
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    void *ptrs[] = {c->d_shadow, c->d_table, c->d_reports, c->d_report_count, c->d_stats, c->d_err,
                    c->scr.batch_off, c->scr.nbatches, c->scr.batch_ctr, c->scr.grid_bar,
                    c->scr.grid_bar2, c->scr.cta_cnt, c->d_collect, c->d_total, c->d_bucket_hist, c->d_bucket_counts,
                    c->d_stage[0], c->d_stage[1], c->d_wire_off, c->d_wire_counts, c->d_wire_flag};
    for (void *p : ptrs)
        if (p)
            cudaFree(p);
    for (int i = 0; i < 2; i++) {
        if (c->ev_copied[i])
            cudaEventDestroy(c->ev_copied[i]);
        if (c->ev_used[i])
            cudaEventDestroy(c->ev_used[i]);
    }
    if (c->copy_stream)
        cudaStreamDestroy(c->copy_stream);
    delete c;
    return HIRACE_OK;
}

hirace_status hirace_set_policy(hirace_ctx *c, int policy, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    if (policy == c->policy)
        return HIRACE_OK;
    if (hirace_fsm_table_policy(policy, c->h_table) != HIRACE_OK)
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    /* h_table is context-owned and only rewritten by a later policy change, which first waits */
    HR_CUDA(c, cudaStreamSynchronize((cudaStream_t)stream));
    hirace::expand_raw_table(c->h_table, c->h_table + 2048);
    HR_CUDA(c, cudaMemcpyAsync(c->d_table, c->h_table, sizeof(c->h_table), cudaMemcpyHostToDevice,
                               (cudaStream_t)stream));
    HR_CUDA(c, cudaStreamSynchronize((cudaStream_t)stream));
    c->policy = policy;
    return HIRACE_OK;
}

hirace_status hirace_shadow_reset(hirace_ctx *c, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, cudaMemsetAsync(c->d_shadow, 0, c->shadow_words * 8, st));
    HR_CUDA(c, cudaMemsetAsync(c->d_report_count, 0, sizeof(unsigned long long), st));
    HR_CUDA(c, cudaMemsetAsync(c->d_stats, 0, 4 * sizeof(unsigned long long), st));
    HR_CUDA(c, cudaMemsetAsync(c->d_err, 0, sizeof(unsigned int), st));
    c->g = 0;
    c->dev.g = 0;
    c->sticky = HIRACE_OK;
    return HIRACE_OK;
}

hirace_status hirace_barrier(hirace_ctx *c, hirace_scope scope, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (scope != HIRACE_SCOPE_GRID)
        return set_sticky(c, HIRACE_E_INVAL);
    HR_CUDA(c, cudaSetDevice(c->device));
    if (c->g + 1 >= 255u) {
        HR_CUDA(c, launch_rebase(c->dev, c->shadow_words, (cudaStream_t)stream));
        c->g = 0;
    } else {
        c->g++;
    }
    c->dev.g = c->g;
    return HIRACE_OK;
}

hirace_status hirace_replay_trace(hirace_ctx *c, const hirace_event *d_events, uint64_t n, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (n == 0)
        return HIRACE_OK;
    if (!d_events || n >= 0xffffffffull)
        return set_sticky(c, HIRACE_E_INVAL);
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, launch_find_batches(d_events, (uint32_t)n, c->scr, c->d_err, c->sm_count, st));
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    HR_CUDA(c, launch_replay(c->dev, d_events, c->scr, c->replay_grid, st));
    if (c->t_stop)
        HR_CUDA(c, cudaEventRecord(c->t_stop, st));
    return HIRACE_OK;
}

hirace_status hirace_set_kernel_timing(hirace_ctx *c, void *start_event, void *stop_event)
{
    if (!c || (!start_event) != (!stop_event))
        return HIRACE_E_INVAL;
    c->t_start = (cudaEvent_t)start_event;
    c->t_stop = (cudaEvent_t)stop_event;
    return HIRACE_OK;
}

hirace_status hirace_find_batches(hirace_ctx *c, const hirace_event *d_events, uint64_t n, uint32_t *h_offsets,
                                  uint32_t *h_keys, uint64_t cap, uint64_t *nbatches, void *stream)
{
    if (!c || !nbatches || (cap && (!h_offsets || !h_keys)) || (n && !d_events) || n >= 0xffffffffull)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    *nbatches = 0;
    if (n == 0)
        return HIRACE_OK;
    HR_CUDA(c, launch_find_batches(d_events, (uint32_t)n, c->scr, c->d_err, c->sm_count, st));
    uint32_t nb = 0;
    HR_CUDA(c, cudaMemcpyAsync(&nb, c->scr.nbatches, sizeof(nb), cudaMemcpyDeviceToHost, st));
    HR_CUDA(c, cudaStreamSynchronize(st));
    hirace_status s = device_errors(c);
    if (s != HIRACE_OK)
        return s;
    *nbatches = nb;
    if (nb + 1 > cap)
        return HIRACE_OK; /* caller retries with a bigger buffer */
    HR_CUDA(c, cudaMemcpy(h_offsets, c->scr.batch_off, (nb + 1) * sizeof(uint32_t), cudaMemcpyDeviceToHost));
    for (uint32_t i = 0; i < nb; i++) {
        uint32_t meta = 0;
        HR_CUDA(c, cudaMemcpy(&meta, &d_events[h_offsets[i]].meta, sizeof(meta), cudaMemcpyDeviceToHost));
        h_keys[i] = meta >> 5;
    }
    return HIRACE_OK;
}

hirace_status hirace_check_trace_device(hirace_ctx *c, const hirace_event *d_events, uint64_t n, hirace_race *d_out,
                                        uint64_t cap, unsigned long long *d_n_total, void *stream)
{
    if (!c || !d_n_total || (cap && !d_out))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (n >= 0xffffffffull || (n && !d_events))
        return set_sticky(c, HIRACE_E_INVAL);
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (n == 0)
        return hirace_collect_races_device(c, d_out, cap, d_n_total, stream);
    HR_CUDA(c, launch_find_batches(d_events, (uint32_t)n, c->scr, c->d_err, c->sm_count, st));
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    HR_CUDA(c, launch_replay(c->dev, d_events, c->scr, c->replay_grid, st, c->shadow_words, d_out, cap, d_n_total));
    if (c->t_stop)
        HR_CUDA(c, cudaEventRecord(c->t_stop, st));
    return HIRACE_OK;
}

hirace_status hirace_collect_races_device(hirace_ctx *c, hirace_race *d_out, uint64_t cap,
                                          unsigned long long *d_n_total, void *stream)
{
    if (!c || !d_n_total || (cap && !d_out))
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, launch_collect(c->dev, c->shadow_words, c->scr, d_out, cap, d_n_total, (cudaStream_t)stream));
    return c->sticky;
}

hirace_status hirace_collect_races(hirace_ctx *c, hirace_race *h_out, uint64_t cap, uint64_t *n_total, void *stream)
{
    if (!c || !n_total || (cap && !h_out))
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (cap > c->collect_cap) {
        if (c->d_collect)
            cudaFree(c->d_collect);
        c->d_collect = nullptr;
        c->collect_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_collect, cap * sizeof(hirace_race)));
        c->collect_cap = cap;
    }
    HR_CUDA(c, launch_collect(c->dev, c->shadow_words, c->scr, c->d_collect, cap, c->d_total, st));
    unsigned long long total = 0;
    HR_CUDA(c, cudaMemcpyAsync(&total, c->d_total, sizeof(total), cudaMemcpyDeviceToHost, st));
    HR_CUDA(c, cudaStreamSynchronize(st));
    *n_total = total;
    uint64_t m = total < cap ? total : cap;
    if (m)
        HR_CUDA(c, cudaMemcpy(h_out, c->d_collect, m * sizeof(hirace_race), cudaMemcpyDeviceToHost));
    return device_errors(c);
}

hirace_status hirace_check_trace_host(hirace_ctx *c, const hirace_event *h_events, uint64_t n, hirace_race *h_out,
                                      uint64_t cap, uint64_t *n_total, void *stream)
{
    if (!c || !n_total || (n && !h_events))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    const uint64_t chunk = 1ull << 22; /* 4 Mi events = 64 MiB per staging buffer */
    if (!c->copy_stream) {
        HR_CUDA(c, cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
        for (int i = 0; i < 2; i++) {
            HR_CUDA(c, cudaEventCreateWithFlags(&c->ev_copied[i], cudaEventDisableTiming));
            HR_CUDA(c, cudaEventCreateWithFlags(&c->ev_used[i], cudaEventDisableTiming));
        }
    }
    const uint64_t need = n < chunk ? (n ? n : 1) : chunk;
    if (need > c->stage_cap) {
        for (int i = 0; i < 2; i++) {
            if (c->d_stage[i])
                cudaFree(c->d_stage[i]);
            c->d_stage[i] = nullptr;
        }
        c->stage_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_stage[0], need * sizeof(hirace_event)));
        HR_CUDA(c, cudaMalloc(&c->d_stage[1], need * sizeof(hirace_event)));
        c->stage_cap = need;
    }
    /* the copy stream must not run ahead of work already queued on `st` */
    HR_CUDA(c, cudaEventRecord(c->ev_used[0], st));
    HR_CUDA(c, cudaStreamWaitEvent(c->copy_stream, c->ev_used[0], 0));
    HR_CUDA(c, cudaEventRecord(c->ev_used[1], st));
    for (uint64_t off = 0, k = 0; off < n; off += chunk, k++) {
        const int b = (int)(k & 1);
        const uint64_t m = n - off < chunk ? n - off : chunk;
        HR_CUDA(c, cudaStreamWaitEvent(c->copy_stream, c->ev_used[b], 0));
        HR_CUDA(c, cudaMemcpyAsync(c->d_stage[b], h_events + off, m * sizeof(hirace_event), cudaMemcpyHostToDevice,
                                   c->copy_stream));
        HR_CUDA(c, cudaEventRecord(c->ev_copied[b], c->copy_stream));
        HR_CUDA(c, cudaStreamWaitEvent(st, c->ev_copied[b], 0));
        hirace_status s = hirace_replay_trace(c, c->d_stage[b], m, stream);
        if (s != HIRACE_OK)
            return s;
        HR_CUDA(c, cudaEventRecord(c->ev_used[b], st));
    }
    return hirace_collect_races(c, h_out, cap, n_total, stream);
}

hirace_status hirace_get_stats(hirace_ctx *c, uint64_t *checked, uint64_t *cas_retries, uint64_t *cas_ops,
                               uint64_t *no_write, uint64_t *dropped_reports)
{
    if (!c)
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, cudaDeviceSynchronize());
    unsigned long long s[4] = {0, 0, 0, 0}, rc = 0;
    HR_CUDA(c, cudaMemcpy(s, c->d_stats, sizeof(s), cudaMemcpyDeviceToHost));
    HR_CUDA(c, cudaMemcpy(&rc, c->d_report_count, sizeof(rc), cudaMemcpyDeviceToHost));
    if (checked)
        *checked = s[0];
    if (cas_retries)
        *cas_retries = s[1];
    if (cas_ops)
        *cas_ops = s[2];
    if (no_write)
        *no_write = s[3];
    if (dropped_reports)
        *dropped_reports = rc > c->cfg.report_capacity ? rc - c->cfg.report_capacity : 0;
    device_errors(c);
    return HIRACE_OK;
}

hirace_status hirace_sync(hirace_ctx *c)
{
    if (!c)
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, cudaDeviceSynchronize());
    return device_errors(c);
}

hirace_status hirace_get_dev_ctx(hirace_ctx *c, const void *global_base, hirace_dev_ctx *out)
{
    if (!c || !out)
        return HIRACE_E_INVAL;
    *out = c->dev;
    out->global_base = global_base;
    out->g = c->g;
    return HIRACE_OK;
}

hirace_status hirace_bucket_events(hirace_ctx *c, const hirace_event *d_in, uint64_t n, int nranks, int my_rank,
                                   hirace_event *d_out, uint64_t *h_counts, void *stream)
{
    if (!c || !h_counts || nranks < 1 || nranks > 32 || my_rank < 0 || my_rank >= nranks || n >= 0xffffffffull ||
        (n && (!d_in || !d_out)))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (n == 0) {
        for (int r = 0; r < nranks; r++)
            h_counts[r] = 0;
        return HIRACE_OK;
    }
    const uint32_t ntiles = (uint32_t)((n + 4095) / 4096);
    const uint64_t need = (uint64_t)ntiles * nranks;
    if (need > c->bucket_hist_cap) {
        if (c->d_bucket_hist)
            cudaFree(c->d_bucket_hist);
        c->d_bucket_hist = nullptr;
        c->bucket_hist_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_bucket_hist, need * sizeof(uint32_t)));
        c->bucket_hist_cap = need;
    }
    if (!c->d_bucket_counts)
        HR_CUDA(c, cudaMalloc(&c->d_bucket_counts, 32 * sizeof(unsigned long long)));
    HR_CUDA(c, launch_bucket(c->dev, d_in, (uint32_t)n, nranks, my_rank, d_out, c->d_bucket_counts, c->d_bucket_hist,
                             ntiles, st));
    unsigned long long tmp[32];
    HR_CUDA(c, cudaMemcpyAsync(tmp, c->d_bucket_counts, nranks * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    HR_CUDA(c, cudaStreamSynchronize(st));
    for (int r = 0; r < nranks; r++)
        h_counts[r] = tmp[r];
    return HIRACE_OK;
}

hirace_status hirace_bucket_wire(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                 int nranks, int my_rank, uint64_t *d_out, uint64_t cap, uint64_t *h_counts,
                                 uint64_t *n_words, void *stream)
{
    if (!c || !h_offsets || !h_counts || !n_words || nranks < 1 || nranks > 32 || my_rank < 0 || my_rank >= nranks ||
        nb > HIRACE_MAX_BATCHES || (nb && !d_in) || (cap && !d_out))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    const uint64_t threads = (uint64_t)c->cfg.grid_blocks * c->cfg.block_threads;
    if (threads > HIRACE_WIRE_MAX_TIDS || (uint64_t)c->dev.smem_words > HIRACE_WIRE_MAX_WORDS)
        return HIRACE_E_INVAL;
    for (uint64_t b = 0; b < nb; b++)
        if (h_offsets[b + 1] < h_offsets[b] || h_offsets[b + 1] >= 0xffffffffu)
            return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    uint32_t maxlen = 0;
    for (uint64_t b = 0; b < nb; b++)
        maxlen = h_offsets[b + 1] - h_offsets[b] > maxlen ? h_offsets[b + 1] - h_offsets[b] : maxlen;
    const uint64_t ntiles = (maxlen + kWireTile - 1) / kWireTile;
    const uint64_t need_hist = ntiles * (uint64_t)nranks;
    if (need_hist > c->bucket_hist_cap) {
        if (c->d_bucket_hist)
            cudaFree(c->d_bucket_hist);
        c->d_bucket_hist = nullptr;
        c->bucket_hist_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_bucket_hist, need_hist * sizeof(uint32_t)));
        c->bucket_hist_cap = need_hist;
    }
    if (need_hist > c->wire_off_cap) {
        if (c->d_wire_off)
            cudaFree(c->d_wire_off);
        c->d_wire_off = nullptr;
        c->wire_off_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_wire_off, need_hist * sizeof(unsigned long long)));
        c->wire_off_cap = need_hist;
    }
    const uint64_t need_counts = nb * (uint64_t)nranks + 1;
    if (need_counts > c->wire_counts_cap) {
        if (c->d_wire_counts)
            cudaFree(c->d_wire_counts);
        c->d_wire_counts = nullptr;
        c->wire_counts_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_wire_counts, need_counts * sizeof(unsigned long long)));
        c->wire_counts_cap = need_counts;
    }
    if (!c->d_wire_flag)
        HR_CUDA(c, cudaMalloc(&c->d_wire_flag, sizeof(unsigned int)));
    unsigned long long *running = c->d_wire_counts + nb * (uint64_t)nranks;
    HR_CUDA(c, cudaMemsetAsync(running, 0, sizeof(unsigned long long), st));
    HR_CUDA(c, cudaMemsetAsync(c->d_wire_flag, 0, sizeof(unsigned int), st));
    for (uint64_t b = 0; b < nb; b++)
        HR_CUDA(c, launch_bucket_wire(d_in, h_offsets[b], h_offsets[b + 1], nranks, my_rank,
                                      reinterpret_cast<unsigned long long *>(d_out), cap, c->d_bucket_hist,
                                      c->d_wire_off, running, c->d_wire_counts + b * (uint64_t)nranks, c->d_wire_flag,
                                      st));
    HR_CUDA(c, cudaMemcpyAsync(h_counts, c->d_wire_counts, nb * (uint64_t)nranks * sizeof(uint64_t),
                               cudaMemcpyDeviceToHost, st));
    unsigned long long total = 0;
    unsigned int flag = 0;
    HR_CUDA(c, cudaMemcpyAsync(&total, running, sizeof(total), cudaMemcpyDeviceToHost, st));
    HR_CUDA(c, cudaMemcpyAsync(&flag, c->d_wire_flag, sizeof(flag), cudaMemcpyDeviceToHost, st));
    HR_CUDA(c, cudaStreamSynchronize(st));
    *n_words = total;
    if (flag & hirace::ERR_BAD_TRACE)
        return set_sticky(c, HIRACE_E_BAD_TRACE);
    if (total > cap)
        return HIRACE_E_INVAL;
    return HIRACE_OK;
}

hirace_status hirace_replay_wire(hirace_ctx *c, const uint64_t *d_wire, uint64_t n, uint32_t batch_key, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (n == 0)
        return HIRACE_OK;
    if (!d_wire || n >= 0xffffffffull || batch_key >= (1u << 27))
        return set_sticky(c, HIRACE_E_INVAL);
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    HR_CUDA(c, launch_replay_wire(c->dev, reinterpret_cast<const unsigned long long *>(d_wire), (uint32_t)n, batch_key,
                                  c->replay_grid, st));
    if (c->t_stop)
        HR_CUDA(c, cudaEventRecord(c->t_stop, st));
    return HIRACE_OK;
}

} /* extern "C" */
