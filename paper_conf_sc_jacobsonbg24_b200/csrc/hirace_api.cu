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

#include <nvtx3/nvToolsExt.h>

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
    uint32_t rec_bytes = 8; /* 8-byte records, or 4 (compact, hirace_shadow_alloc_compact) */
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
    /* peer dispatch: [nranks peer buffer pointers | nb x nranks destination offsets] */
    unsigned long long *d_peer_tab = nullptr;
    uint64_t peer_tab_cap = 0;
    void **d_flag_tab = nullptr; /* peer flag-array addresses (hirace_peer_release) */
    /* host-trace staging ring */
    hirace_event *d_stage[2] = {nullptr, nullptr};
    uint64_t stage_cap = 0;
    cudaStream_t copy_stream = nullptr;
    cudaEvent_t ev_copied[2] = {nullptr, nullptr}, ev_used[2] = {nullptr, nullptr};
    hirace_dev_ctx dev{};
    /* window-major path (window.cu) */
    int replay_mode = HIRACE_REPLAY_AUTO;
    uint32_t win_log2 = 14;
    WinDev win{};
    uint64_t win_events_cap = 0;  /* events the window scratch is sized for */
    hirace_event *d_trace = nullptr; /* whole-trace staging for hirace_check_trace_host */
    uint64_t trace_cap = 0;
    bool lazy = false;            /* a lazy reset left stale windows behind */
    int reset_mode = HIRACE_RESET_FULL;
    unsigned int *d_gepoch = nullptr; /* epoch reset: {gbase, gnext} (device) */
    uint32_t g = 0;
    cudaEvent_t t_start = nullptr, t_stop = nullptr;
    /* partial-mask warp syncs (hirace_set_warp_syncs) */
    WsDev ws{};
    uint64_t ws_n = 0, ws_slots = 0;
    hirace_ws_ctx iws{};        /* inline hooks' sub-warp history (hirace_inline_warp_syncs) */
    uint64_t iws_slots = 0;
    int masked_grid = 0;
    hirace_status sticky = HIRACE_OK;
};

namespace {

/* NVTX range over one API call (Nsight timelines; header-only nvtx3, near-free when no tool is
 * attached) */
struct Nvtx {
    explicit Nvtx(const char *name) { nvtxRangePushA(name); }
    ~Nvtx() { nvtxRangePop(); }
};

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

/* collect from the report buffer (falling back to the shadow scan on the device) when the
 * shadow is large enough for a full scan to cost more than the sort (collect.cuh) */
int report_mode(const hirace_ctx *c)
{
    if (const char *f = getenv("HIRACE_COLLECT")) /* "scan" / "reports": force a path (tests, A/B) */
        return f[0] == 'r' ? 1 : 0;
    return c->shadow_words * c->rec_bytes >= kReportModeMinBytes ? 1 : 0;
}

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
    if (flags & ERR_CAPACITY)
        set_sticky(c, HIRACE_E_NOMEM);
    if (flags & ERR_HISTORY)
        set_sticky(c, HIRACE_E_HISTORY_OVERFLOW);
    return c->sticky;
}

constexpr uint32_t kWindowPadLog2 = 14;           /* shadow allocation padded to 2^14 records */
constexpr uint32_t kWindowLog2Default = 12;       /* 32 KB windows: 4 light CTAs per SM (§8)    */

/* does this context replay window-major? (8-byte records, 4-byte elements) */
bool window_active(const hirace_ctx *c)
{
    if (c->rec_bytes != 8 || c->cfg.granularity_log2 != 2 || !c->win.gen || c->ws_n)
        return false; /* (a partial-sync log replays batch-major) */
    if (c->replay_mode == HIRACE_REPLAY_WINDOW)
        return true;
    /* AUTO: batch-major everywhere (measured faster on every config); the
     * HIRACE_WINDOW_AUTO_BYTES environment variable re-enables window-major above a size */
    const char *v = getenv("HIRACE_WINDOW_AUTO_BYTES");
    return c->replay_mode == HIRACE_REPLAY_AUTO && v && c->shadow_words * 8 >= strtoull(v, nullptr, 10);
}

/* window geometry + generation array for window size 2^wl records (all windows stale) */
cudaError_t window_geometry(hirace_ctx *c, uint32_t wl)
{
    WinDev &W = c->win;
    const uint64_t padded = ((c->shadow_words + (1ull << kWindowPadLog2) - 1) >> kWindowPadLog2) << kWindowPadLog2;
    const uint64_t nw = padded >> wl;
    if (nw + 1 >= (1ull << 31))
        return cudaErrorInvalidValue;
    uint32_t wb = 0;
    while ((1ull << wb) < nw)
        wb++;
    if (wb > 20)
        return cudaErrorInvalidValue; /* two passes of <= 1024 digits */
    if (W.gen)
        cudaFree(W.gen);
    W.gen = nullptr;
    cudaError_t e;
    if ((e = cudaMalloc(&W.gen, nw * sizeof(uint32_t))) != cudaSuccess)
        return e;
    if (!W.cur_gen && (e = cudaMalloc(&W.cur_gen, sizeof(uint32_t))) != cudaSuccess)
        return e;
    if ((e = cudaMemset(W.gen, 0, nw * sizeof(uint32_t))) != cudaSuccess)
        return e;
    const uint32_t one = 1;
    if ((e = cudaMemcpy(W.cur_gen, &one, sizeof(one), cudaMemcpyHostToDevice)) != cudaSuccess)
        return e;
    W.wl = wl;
    W.nw = (uint32_t)nw;
    /* digits: one pass up to 2^9 windows, else two balanced passes of <= 2^10 digits */
    W.d0b = wb <= 9 ? wb : (wb + 1) / 2;
    W.d1b = wb - W.d0b;
    W.p1 = 1u << 16;
    W.p2 = 1u << 16;
    W.heavy_cap = kWinHeavyCap;
    const char *hf = getenv("HIRACE_WIN_HEAVY"); /* tests: force the heavy-window path */
    W.heavy_force = hf ? (uint32_t)strtoul(hf, nullptr, 10) : 0u;
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, window_light_kernel(), window_light_threads(),
                                                  window_light_smem(wl));
    W.light_ctas = (uint32_t)(c->sm_count * (occ > 0 ? occ : 1));
    c->win_log2 = wl;
    c->win_events_cap = 0; /* per-size scratch is (re)allocated on the next check */
    return cudaSuccess;
}

void window_free_scratch(WinDev &W)
{
    void *ptrs[] = {W.items1, W.item1_first, W.batch_key, W.count1, W.count2, W.rec1,
                    W.rec2 != W.rec1 ? W.rec2 : nullptr, W.win_cnt, W.aux, W.heavy, W.light, W.hseg,
                    W.partials, W.bar, W.elems};
    for (void *p : ptrs)
        if (p)
            cudaFree(p);
    W.items1 = nullptr;
    W.item1_first = W.batch_key = W.count1 = W.count2 = W.win_cnt = W.aux = W.heavy = W.light = W.hseg = nullptr;
    W.partials = nullptr;
    W.rec1 = W.rec2 = nullptr;
    W.bar = nullptr;
    W.elems = nullptr;
}

/* per-check scratch sized for n events (grown on demand; never inside a graph capture: the
 * warm-up call allocates) */
cudaError_t window_scratch(hirace_ctx *c, uint64_t n)
{
    WinDev &W = c->win;
    if (n <= c->win_events_cap && W.rec1)
        return cudaSuccess;
    cudaDeviceSynchronize();
    window_free_scratch(W);
    const uint64_t nb_max = HIRACE_MAX_BATCHES;
    const uint64_t items1 = n / W.p1 + (n < nb_max ? n : nb_max) + 1;
    const uint64_t elem_cap = n + n / 4 + 65536;
    const uint64_t chunks2 = elem_cap / W.p2 + 2;
    const uint64_t R0 = 1ull << W.d0b, R1 = 1ull << W.d1b;
    if (items1 > 0xffffffffull || R0 * items1 > 0xffffffffull || R1 * chunks2 > 0xffffffffull ||
        elem_cap >= 0xffffffffull)
        return cudaErrorInvalidValue;
    W.elem_cap = elem_cap;
    W.items1_cap = (uint32_t)items1;
    W.chunks2_cap = (uint32_t)chunks2;
    cudaError_t e;
#define WA(ptr, bytes)                                                                                              \
    if ((e = cudaMalloc((void **)&(ptr), (bytes))) != cudaSuccess) {                                                 \
        window_free_scratch(W);                                                                                      \
        return e;                                                                                                    \
    }
    WA(W.items1, items1 * sizeof(uint4));
    WA(W.item1_first, (nb_max + 1) * sizeof(uint32_t));
    WA(W.batch_key, nb_max * sizeof(uint32_t));
    WA(W.count1, R0 * items1 * sizeof(uint32_t));
    WA(W.count2, W.d1b ? R1 * chunks2 * sizeof(uint32_t) : sizeof(uint32_t));
    WA(W.rec1, (elem_cap + 2) * sizeof(unsigned long long)); /* +2: 16-byte aligned bulk reads */
    if (W.d1b) {
        WA(W.rec2, (elem_cap + 2) * sizeof(unsigned long long));
    } else {
        W.rec2 = W.rec1;
    }
    WA(W.win_cnt, ((uint64_t)W.nw + 1) * sizeof(uint32_t));
    WA(W.aux, kAuxCount * sizeof(uint32_t));
    WA(W.heavy, W.heavy_cap * sizeof(uint32_t));
    WA(W.light, (uint64_t)W.nw * sizeof(uint32_t));
    WA(W.hseg, (uint64_t)W.heavy_cap * (nb_max + 1) * sizeof(uint32_t));
    WA(W.partials, kScanMaxCtas * sizeof(uint32_t));
    WA(W.bar, kBarSlots * sizeof(unsigned int));
    WA(W.elems, sizeof(unsigned long long));
#undef WA
    if ((e = cudaMemset(W.aux, 0, kAuxCount * sizeof(uint32_t))) != cudaSuccess)
        return e;
    c->win_events_cap = n;
    return cudaSuccess;
}

/* epoch reset: bring the shadow back to offset 0 (records keep the trace's g) before a path
 * that does not add the offset (inline hooks, wire replay, hirace_barrier) */
hirace_status ensure_epoch_normal(hirace_ctx *c, cudaStream_t st)
{
    if (c->reset_mode != HIRACE_RESET_EPOCH)
        return HIRACE_OK;
    HR_CUDA(c, launch_epoch_prep(c->dev, c->shadow_words, c->d_gepoch, nullptr, nullptr, nullptr, 1, c->sm_count, st));
    return HIRACE_OK;
}

/* stale windows := INIT before a path that reads or writes the shadow directly */
hirace_status ensure_materialized(hirace_ctx *c, cudaStream_t st)
{
    if (!c->lazy)
        return HIRACE_OK;
    HR_CUDA(c, launch_materialize(c->dev, c->win, 0, c->sm_count, st));
    c->lazy = false;
    return HIRACE_OK;
}

/* a7 collection into device memory: the report buffer when it covers every flagged word (large
 * shadows), else the ordered shadow scan; after a lazy reset the stale windows are made INIT
 * first, and only when the scan actually runs */
hirace_status collect_into(hirace_ctx *c, hirace_race *d_out, uint64_t cap, unsigned long long *d_total,
                           cudaStream_t st)
{
    const int rm = report_mode(c);
    if (c->lazy && rm) {
        HR_CUDA(c, launch_collect_reports(c->dev, d_out, cap, d_total, st));
        HR_CUDA(c, launch_materialize(c->dev, c->win, 1, c->sm_count, st));
        HR_CUDA(c, launch_collect(c->dev, c->shadow_words, c->scr, d_out, cap, d_total, st, 2));
        return HIRACE_OK;
    }
    if (ensure_materialized(c, st) != HIRACE_OK)
        return c->sticky;
    HR_CUDA(c, launch_collect(c->dev, c->shadow_words, c->scr, d_out, cap, d_total, st, rm));
    return HIRACE_OK;
}

/* classes R 0, A 1, X 2 inside one block (C1.3): strict R-A, R-X, A-X, X-X conflict; relaxed only
 * pairs with X; and the FSM state -> RACE-of-its-level table of the policy */
void ws_policy_tables(int policy, hirace_ws_ctx &H)
{
    const bool relaxed = policy == HIRACE_POLICY_RELAXED_READ_ATOMIC;
    H.confl[0] = relaxed ? 4u : 6u;
    H.confl[1] = relaxed ? 4u : 5u;
    H.confl[2] = 7u;
    fsm_race_of(policy, H.race_of);
}

/* masked replay launch: the policy-dependent tables are refreshed from the context */
cudaError_t launch_masked(hirace_ctx *c, const hirace_event *d_events, cudaStream_t st)
{
    WsDev W = c->ws;
    ws_policy_tables(c->policy, W.H);
    return launch_replay_masked(c->dev, W, d_events, c->scr, c->masked_grid, st);
}

/* empty history: every slot free, no spill block handed out, the pool's lane words stale */
cudaError_t hist_clear(const hirace_ws_ctx &H, uint64_t slots, cudaStream_t st)
{
    cudaError_t e = cudaMemsetAsync(H.hist, 0xff, slots * kSlotWords * sizeof(unsigned long long), st);
    if (e == cudaSuccess)
        e = cudaMemsetAsync(H.spill, 0xff, H.nspill * 32 * sizeof(unsigned long long), st);
    if (e == cudaSuccess)
        e = cudaMemsetAsync(H.spill_count, 0, sizeof(unsigned long long), st);
    return e;
}

cudaError_t ws_clear(hirace_ctx *c, cudaStream_t st)
{
    return hist_clear(c->ws.H, c->ws_slots, st);
}

void ws_free(hirace_ctx *c)
{
    void *ptrs[] = {c->ws.fam_key, c->ws.fam_lo, c->ws.nfam, c->ws.sync_w, c->ws.sync_mask, c->ws.sync_fam,
                    c->ws.vrow, c->ws.fhash, c->ws.H.hist, c->ws.H.spill, c->ws.H.spill_count};
    for (void *p : ptrs)
        if (p)
            cudaFree(p);
    c->ws = WsDev{};
    c->ws_n = 0;
    c->ws_slots = 0;
}

} // namespace

extern "C" {

hirace_status hirace_set_warp_syncs(hirace_ctx *c, const hirace_warp_sync *d_syncs, uint64_t n, uint64_t history_slots,
                                    void *stream)
{
    Nvtx nvtx_range("hirace_set_warp_syncs");
    if (!c || (n && !d_syncs) || n >= (1ull << 31) || history_slots > (1ull << 32))
        return HIRACE_E_INVAL;
    if (n && (c->cfg.warp_size > 32 || c->cfg.granularity_log2 != 2))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (ensure_materialized(c, st) != HIRACE_OK) /* from here on: batch-major, shadow explicit */
        return c->sticky;
    HR_CUDA(c, cudaStreamSynchronize(st));
    ws_free(c);
    if (n == 0)
        return HIRACE_OK;
    uint64_t slots = 64;
    while (slots < (history_slots ? history_slots : 65536ull))
        slots <<= 1;
    uint64_t fh_slots = 64;
    while (fh_slots < 4 * n) /* listed syncs + family records (<= n) at most half full */
        fh_slots <<= 1;
    WsDev &W = c->ws;
    cudaError_t e;
    if ((e = cudaMalloc(&W.fam_key, n * sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&W.fam_lo, (n + 1) * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&W.nfam, sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&W.sync_w, n * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&W.sync_mask, n * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&W.sync_fam, n * sizeof(uint32_t))) != cudaSuccess ||
        (e = cudaMalloc(&W.vrow, n * 32 * sizeof(unsigned short))) != cudaSuccess ||
        (e = cudaMalloc(&W.fhash, fh_slots * sizeof(uint4))) != cudaSuccess ||
        (e = cudaMalloc(&W.H.hist, slots * kSlotWords * sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&W.H.spill, (slots / 8) * 32 * sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&W.H.spill_count, sizeof(unsigned long long))) != cudaSuccess) {
        ws_free(c);
        return from_cuda(c, e);
    }
    W.H.slots_mask = slots - 1;
    W.H.nspill = slots / 8;
    W.fh_mask = fh_slots - 1;
    W.nsync = (uint32_t)n;
    W.wpb = (c->cfg.block_threads + c->cfg.warp_size - 1) / c->cfg.warp_size;
    c->ws_slots = slots;
    if (!c->masked_grid)
        c->masked_grid = masked_max_grid(c->device);
    HR_CUDA(c, ws_clear(c, st));
    HR_CUDA(c, cudaMemsetAsync(W.fhash, 0xff, fh_slots * sizeof(uint4), st));
    HR_CUDA(c, launch_ws_prepare(d_syncs, (uint32_t)n, c->cfg.grid_blocks * W.wpb, c->cfg.warp_size, W, c->d_err,
                                 c->sm_count, st));
    HR_CUDA(c, cudaStreamSynchronize(st));
    hirace_status s = device_errors(c);
    if (s != HIRACE_OK) {
        ws_free(c);
        return s;
    }
    c->ws_n = n;
    return HIRACE_OK;
}

hirace_status hirace_inline_warp_syncs(hirace_ctx *c, uint64_t history_slots, hirace_ws_ctx *out)
{
    if (!c || !out || c->rec_bytes != 8 || c->cfg.warp_size > 32 || c->cfg.granularity_log2 != 2 ||
        history_slots > (1ull << 32))
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (!c->iws.hist) {
        uint64_t slots = 64;
        while (slots < (history_slots ? history_slots : 65536ull))
            slots <<= 1;
        hirace_ws_ctx &H = c->iws;
        cudaError_t e;
        if ((e = cudaMalloc(&H.hist, slots * kSlotWords * sizeof(unsigned long long))) != cudaSuccess ||
            (e = cudaMalloc(&H.spill, (slots / 8) * 32 * sizeof(unsigned long long))) != cudaSuccess ||
            (e = cudaMalloc(&H.spill_count, sizeof(unsigned long long))) != cudaSuccess) {
            void *ptrs[] = {H.hist, H.spill, H.spill_count};
            for (void *p : ptrs)
                if (p)
                    cudaFree(p);
            H = hirace_ws_ctx{};
            return from_cuda(c, e);
        }
        H.slots_mask = slots - 1;
        H.nspill = slots / 8;
        c->iws_slots = slots;
        HR_CUDA(c, hist_clear(H, slots, nullptr));
        HR_CUDA(c, cudaDeviceSynchronize());
    }
    ws_policy_tables(c->policy, c->iws);
    *out = c->iws;
    return HIRACE_OK;
}

const char *hirace_version(void) { return "hirace-b200 0.2 (sm_100a)"; }

hirace_status hirace_set_replay_mode(hirace_ctx *c, int mode, uint32_t window_log2)
{
    if (!c || mode < HIRACE_REPLAY_AUTO || mode > HIRACE_REPLAY_WINDOW || (window_log2 && (window_log2 < 5 || window_log2 > 14)))
        return HIRACE_E_INVAL;
    if (mode == HIRACE_REPLAY_WINDOW && (c->rec_bytes != 8 || c->cfg.granularity_log2 != 2))
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, cudaDeviceSynchronize());
    const uint32_t wl = window_log2 ? window_log2 : kWindowLog2Default;
    if (c->win.gen && wl != c->win_log2) {
        window_free_scratch(c->win);
        HR_CUDA(c, window_geometry(c, wl));
    }
    c->replay_mode = mode;
    c->lazy = false;
    if (window_active(c)) { /* window-major has its own (lazy) reset */
        c->reset_mode = HIRACE_RESET_FULL;
        c->dev.g_base = nullptr;
    }
    /* the mode change starts from an all-INIT shadow (full reset: every window current) */
    HR_CUDA(c, launch_reset(c->d_shadow, c->shadow_words * c->rec_bytes, c->d_report_count, c->d_stats, c->d_err,
                            c->sm_count, nullptr));
    HR_CUDA(c, cudaDeviceSynchronize());
    c->g = 0;
    c->dev.g = 0;
    c->sticky = HIRACE_OK;
    return HIRACE_OK;
}

hirace_status hirace_set_reset_mode(hirace_ctx *c, int mode)
{
    if (!c || (mode != HIRACE_RESET_FULL && mode != HIRACE_RESET_EPOCH))
        return HIRACE_E_INVAL;
    if (mode == HIRACE_RESET_EPOCH && (c->rec_bytes != 8 || window_active(c)))
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, cudaDeviceSynchronize());
    if (mode == HIRACE_RESET_EPOCH) {
        if (!c->d_gepoch)
            HR_CUDA(c, cudaMalloc(&c->d_gepoch, 4 * sizeof(unsigned int)));
        HR_CUDA(c, cudaMemset(c->d_gepoch, 0, 4 * sizeof(unsigned int)));
        c->dev.g_base = c->d_gepoch;
    } else {
        c->dev.g_base = nullptr;
    }
    c->reset_mode = mode;
    HR_CUDA(c, launch_reset(c->d_shadow, c->shadow_words * c->rec_bytes, c->d_report_count, c->d_stats, c->d_err,
                            c->sm_count, nullptr));
    HR_CUDA(c, cudaDeviceSynchronize());
    c->sticky = HIRACE_OK;
    return HIRACE_OK;
}

hirace_status hirace_get_replay_mode(const hirace_ctx *c, int *active_window)
{
    if (!c || !active_window)
        return HIRACE_E_INVAL;
    *active_window = window_active(c) ? 1 : 0;
    return HIRACE_OK;
}

hirace_status hirace_launch_count(uint64_t *out)
{
    if (!out)
        return HIRACE_E_INVAL;
    *out = launch_count();
    return HIRACE_OK;
}

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
    case HIRACE_E_HISTORY_OVERFLOW: return "sub-warp history full: masked-warp accesses not all compared";
    }
    return "unknown";
}

namespace {

/* shared by hirace_shadow_alloc (lim == NULL: 8-byte records) and hirace_shadow_alloc_compact */
hirace_status shadow_alloc_impl(const hirace_config *cfg, const hirace_epoch_limits *lim, hirace_ctx **out)
{
    if (!cfg || !out)
        return HIRACE_E_INVAL;
    *out = nullptr;
    if (cfg->grid_blocks == 0 || cfg->block_threads == 0 || cfg->warp_size == 0 || cfg->granularity_log2 > 2)
        return HIRACE_E_INVAL;
    if ((uint64_t)cfg->grid_blocks * cfg->block_threads > 0xffffffffull)
        return HIRACE_E_INVAL;
    if ((cfg->smem_bytes_per_block & 3) || (cfg->global_bytes & 3))
        return HIRACE_E_INVAL;
    hirace::clay lay{};
    if (lim) {
        if (lim->max_g > 254u || lim->max_b > 1023u || lim->max_w > 511u)
            return HIRACE_E_INVAL;
        if (!hirace::make_clay(lim->max_g, lim->max_b, lim->max_w, cfg->grid_blocks * cfg->block_threads, &lay))
            return HIRACE_E_INVAL; /* the record would not fit 32 bits */
    }
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
    c->rec_bytes = lim ? 4u : 8u;
    c->global_words = cfg->global_bytes >> cfg->granularity_log2;
    const uint64_t smem_words = cfg->smem_bytes_per_block >> cfg->granularity_log2;
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
    const uint64_t padded = ((c->shadow_words + (1ull << kWindowPadLog2) - 1) >> kWindowPadLog2) << kWindowPadLog2;
    if ((e = cudaMalloc(&c->d_shadow, padded * c->rec_bytes)) != cudaSuccess ||
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
    d.rec_bytes = c->rec_bytes;
    d.gran_log2 = cfg->granularity_log2;
    d.f_active = 0;
    d.f_tid_mask = 0;
    d.f_tid_match = 0;
    d.f_spaces = 3;
    d.f_glo = 0;
    d.f_ghi = ~0ull;
    d.f_smem_words = d.smem_words;
    d.f_pad = 0;
    d.g_base = nullptr;
    d.c_sh_b = lay.sh_b;
    d.c_sh_w = lay.sh_w;
    d.c_sh_t = lay.sh_t;
    d.c_max_g = lim ? lim->max_g : 254u;
    d.c_max_b = lim ? lim->max_b : 1023u;
    d.c_max_w = lim ? lim->max_w : 511u;
    if (c->rec_bytes == 8 && cfg->granularity_log2 == 2 && (e = window_geometry(c, kWindowLog2Default)) != cudaSuccess)
        return fail(e);
    if (hirace_shadow_reset(c, nullptr) != HIRACE_OK || cudaDeviceSynchronize() != cudaSuccess) {
        hirace_shadow_free(c);
        return HIRACE_E_CUDA;
    }
    *out = c;
    return HIRACE_OK;
}

} // namespace

hirace_status hirace_shadow_alloc(const hirace_config *cfg, hirace_ctx **out)
{
    return shadow_alloc_impl(cfg, nullptr, out);
}

hirace_status hirace_shadow_alloc_compact(const hirace_config *cfg, const hirace_epoch_limits *lim, hirace_ctx **out)
{
    if (!lim)
        return HIRACE_E_INVAL;
    return shadow_alloc_impl(cfg, lim, out);
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
                    c->d_stage[0], c->d_stage[1], c->d_wire_off, c->d_wire_counts, c->d_wire_flag,
                    c->d_peer_tab, c->d_flag_tab, c->d_gepoch, c->ws.fam_key, c->ws.fam_lo, c->ws.nfam,
                    c->ws.sync_w, c->ws.sync_mask, c->ws.sync_fam, c->ws.vrow, c->ws.fhash, c->ws.H.hist,
                    c->ws.H.spill, c->ws.H.spill_count, c->iws.hist, c->iws.spill, c->iws.spill_count};
    for (void *p : ptrs)
        if (p)
            cudaFree(p);
    window_free_scratch(c->win);
    if (c->win.gen)
        cudaFree(c->win.gen);
    if (c->win.cur_gen)
        cudaFree(c->win.cur_gen);
    if (c->d_trace)
        cudaFree(c->d_trace);
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

hirace_status hirace_set_filter(hirace_ctx *c, uint32_t tid_mask, uint32_t tid_match, uint32_t spaces,
                                uint64_t global_lo, uint64_t global_hi)
{
    if (!c || (tid_match & ~tid_mask) || spaces > 3 || global_lo > global_hi)
        return HIRACE_E_INVAL;
    hirace_dev_ctx &d = c->dev;
    d.f_tid_mask = tid_mask;
    d.f_tid_match = tid_match;
    d.f_spaces = spaces;
    d.f_glo = (spaces & 1u) ? global_lo : 0;
    d.f_ghi = (spaces & 1u) ? global_hi : 0;
    d.f_smem_words = (spaces & 2u) ? d.smem_words : 0;
    d.f_active = (tid_mask != 0 || spaces != 3 || global_lo != 0 || global_hi < c->global_words) ? 1u : 0u;
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
    Nvtx nvtx_range("hirace_shadow_reset");
    if (!c)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (window_active(c)) { /* lazy: the generation moves on, windows read as INIT (O(1)) */
        HR_CUDA(c, launch_lazy_reset(c->dev, c->win, st));
        c->lazy = true;
    } else if (c->reset_mode == HIRACE_RESET_EPOCH) { /* O(flagged): epochs move on */
        HR_CUDA(c, launch_epoch_reset(c->dev, c->shadow_words, c->d_gepoch, c->sm_count, st));
        c->lazy = false;
    } else {
        HR_CUDA(c, launch_reset(c->d_shadow, c->shadow_words * c->rec_bytes, c->d_report_count, c->d_stats, c->d_err,
                                c->sm_count, st));
        c->lazy = false;
    }
    if (c->ws.H.hist) /* the sub-warp histories belong to the check */
        HR_CUDA(c, ws_clear(c, st));
    if (c->iws.hist)
        HR_CUDA(c, hist_clear(c->iws, c->iws_slots, st));
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
    return hirace_advance_grid_epochs(c, 1, stream);
}

hirace_status hirace_advance_grid_epochs(hirace_ctx *c, uint32_t count, void *stream)
{
    if (!c)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (c->rec_bytes != 8) /* compact contexts are replay-only */
        return set_sticky(c, HIRACE_E_INVAL);
    HR_CUDA(c, cudaSetDevice(c->device));
    if (count && ensure_epoch_normal(c, (cudaStream_t)stream) != HIRACE_OK)
        return c->sticky;
    for (uint32_t k = 0; k < count; k++) {
        if (c->g + 1 >= 255u) {
            if (ensure_materialized(c, (cudaStream_t)stream) != HIRACE_OK)
                return c->sticky;
            HR_CUDA(c, launch_rebase(c->dev, c->shadow_words, (cudaStream_t)stream));
            c->g = 0;
        } else {
            c->g++;
        }
    }
    c->dev.g = c->g;
    return HIRACE_OK;
}

hirace_status hirace_replay_trace(hirace_ctx *c, const hirace_event *d_events, uint64_t n, void *stream)
{
    Nvtx nvtx_range("hirace_replay_trace");
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
    const bool win = window_active(c);
    if (win)
        HR_CUDA(c, window_scratch(c, n));
    else if (ensure_materialized(c, st) != HIRACE_OK)
        return c->sticky;
    HR_CUDA(c, launch_find_batches(d_events, (uint32_t)n, c->scr, c->d_err, c->sm_count, st));
    if (!win && c->reset_mode == HIRACE_RESET_EPOCH)
        HR_CUDA(c, launch_epoch_prep(c->dev, c->shadow_words, c->d_gepoch, d_events, c->scr.batch_off,
                                     c->scr.nbatches, 0, c->sm_count, st));
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    if (win)
        HR_CUDA(c, launch_window_check(c->dev, c->win, c->scr, d_events, (uint32_t)n, c->sm_count, c->replay_grid, st,
                                       c->shadow_words, nullptr, 0, nullptr));
    else if (c->ws_n)
        HR_CUDA(c, launch_masked(c, d_events, st));
    else
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
    Nvtx nvtx_range("hirace_check_trace_device");
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
    const bool win = window_active(c);
    if (win)
        HR_CUDA(c, window_scratch(c, n));
    else if (ensure_materialized(c, st) != HIRACE_OK)
        return c->sticky;
    HR_CUDA(c, launch_find_batches(d_events, (uint32_t)n, c->scr, c->d_err, c->sm_count, st));
    if (!win && c->reset_mode == HIRACE_RESET_EPOCH)
        HR_CUDA(c, launch_epoch_prep(c->dev, c->shadow_words, c->d_gepoch, d_events, c->scr.batch_off,
                                     c->scr.nbatches, 0, c->sm_count, st));
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    if (win)
        HR_CUDA(c, launch_window_check(c->dev, c->win, c->scr, d_events, (uint32_t)n, c->sm_count, c->replay_grid, st,
                                       c->shadow_words, d_out, cap, d_n_total));
    else if (c->ws_n) {
        HR_CUDA(c, launch_masked(c, d_events, st));
        if (collect_into(c, d_out, cap, d_n_total, st) != HIRACE_OK)
            return c->sticky;
    } else
        HR_CUDA(c, launch_replay(c->dev, d_events, c->scr, c->replay_grid, st, c->shadow_words, d_out, cap, d_n_total,
                                 report_mode(c)));
    if (win && getenv("HIRACE_WIN_VALIDATE")) { /* diagnostics: synchronous */
        uint32_t aux[kAuxCount];
        HR_CUDA(c, cudaStreamSynchronize(st));
        HR_CUDA(c, cudaMemcpy(aux, c->win.aux, sizeof(aux), cudaMemcpyDeviceToHost));
        fprintf(stderr, "window check: items1 %u total1 %u chunks2 %u heavy %u light %u abort %u violations %u\n",
                aux[kAuxItems1], aux[kAuxTotal1], aux[kAuxChunks2], aux[kAuxNHeavy], aux[kAuxNLight], aux[kAuxAbort],
                aux[kAuxViolations]);
    }
    if (c->t_stop)
        HR_CUDA(c, cudaEventRecord(c->t_stop, st));
    return HIRACE_OK;
}

hirace_status hirace_collect_races_device(hirace_ctx *c, hirace_race *d_out, uint64_t cap,
                                          unsigned long long *d_n_total, void *stream)
{
    Nvtx nvtx_range("hirace_collect_races_device");
    if (!c || !d_n_total || (cap && !d_out))
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (collect_into(c, d_out, cap, d_n_total, (cudaStream_t)stream) != HIRACE_OK)
        return c->sticky;
    return c->sticky;
}

hirace_status hirace_collect_races(hirace_ctx *c, hirace_race *h_out, uint64_t cap, uint64_t *n_total, void *stream)
{
    Nvtx nvtx_range("hirace_collect_races");
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
    if (collect_into(c, c->d_collect, cap, c->d_total, st) != HIRACE_OK)
        return c->sticky;
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
    Nvtx nvtx_range("hirace_check_trace_host");
    if (!c || !n_total || (n && !h_events))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (window_active(c) && n) {
        /* window-major: the partition needs the whole trace; stage it in HBM (chunked copies on
         * the copy stream), then one check */
        if (n > c->trace_cap) {
            HR_CUDA(c, cudaStreamSynchronize(st));
            if (c->d_trace)
                cudaFree(c->d_trace);
            c->d_trace = nullptr;
            c->trace_cap = 0;
            HR_CUDA(c, cudaMalloc(&c->d_trace, n * sizeof(hirace_event)));
            c->trace_cap = n;
        }
        HR_CUDA(c, cudaMemcpyAsync(c->d_trace, h_events, n * sizeof(hirace_event), cudaMemcpyHostToDevice, st));
        hirace_status s = hirace_replay_trace(c, c->d_trace, n, stream);
        if (s != HIRACE_OK)
            return s;
        return hirace_collect_races(c, h_out, cap, n_total, stream);
    }
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
    if (!c || !out || c->rec_bytes != 8 || c->ws_n) /* inline hooks: 8-byte record, no sync log */
        return HIRACE_E_INVAL;
    if (c->lazy || c->reset_mode == HIRACE_RESET_EPOCH) { /* inline hooks use the trace's epochs */
        HR_CUDA(c, cudaSetDevice(c->device));
        if (ensure_materialized(c, nullptr) != HIRACE_OK || ensure_epoch_normal(c, nullptr) != HIRACE_OK)
            return c->sticky;
    }
    *out = c->dev;
    out->global_base = global_base;
    out->g = c->g;
    return HIRACE_OK;
}

hirace_status hirace_bucket_events(hirace_ctx *c, const hirace_event *d_in, uint64_t n, int nranks, int my_rank,
                                   hirace_event *d_out, uint64_t *h_counts, void *stream)
{
    if (!c || !h_counts || nranks < 1 || nranks > 32 || my_rank < 0 || my_rank >= nranks || n >= 0xffffffffull ||
        (n && (!d_in || !d_out)) || c->cfg.granularity_log2 != 2 || c->ws_n)
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

} /* extern "C" */

namespace {

/* scratch for per-batch wire bucketing of up to maxlen events into nranks owners */
hirace_status wire_scratch(hirace_ctx *c, uint64_t nb, int nranks, uint32_t maxlen)
{
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
    return HIRACE_OK;
}

hirace_status bucket_wire_impl(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                               int nranks, int my_rank, uint64_t *d_out, uint64_t cap, uint64_t *h_counts,
                               uint64_t *n_words, void *stream);

hirace_status wire_args_ok(hirace_ctx *c, const uint32_t *h_offsets, uint64_t nb, int nranks, int my_rank,
                           uint32_t *maxlen)
{
    if (nranks < 1 || nranks > 32 || my_rank < 0 || my_rank >= nranks || nb > HIRACE_MAX_BATCHES ||
        c->cfg.granularity_log2 != 2 || c->ws_n)
        return HIRACE_E_INVAL;
    const uint64_t threads = (uint64_t)c->cfg.grid_blocks * c->cfg.block_threads;
    if (threads > HIRACE_WIRE_MAX_TIDS || (uint64_t)c->dev.smem_words > HIRACE_WIRE_MAX_WORDS)
        return HIRACE_E_INVAL;
    *maxlen = 0;
    for (uint64_t b = 0; b < nb; b++) {
        if (h_offsets[b + 1] < h_offsets[b] || h_offsets[b + 1] >= 0xffffffffu)
            return HIRACE_E_INVAL;
        *maxlen = h_offsets[b + 1] - h_offsets[b] > *maxlen ? h_offsets[b + 1] - h_offsets[b] : *maxlen;
    }
    return HIRACE_OK;
}

} // namespace

extern "C" {

hirace_status hirace_count_wire(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                int nranks, int my_rank, uint64_t *h_counts, void *stream)
{
    Nvtx nvtx_range("hirace_count_wire");
    uint64_t n = 0;
    if (!c || !h_counts || !h_offsets || (nb && !d_in))
        return HIRACE_E_INVAL;
    return bucket_wire_impl(c, d_in, h_offsets, nb, nranks, my_rank, nullptr, 0, h_counts, &n, stream);
}

hirace_status hirace_dispatch_wire(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                   int nranks, int my_rank, void *const *h_peer, const uint64_t *h_dst, void *stream)
{
    Nvtx nvtx_range("hirace_dispatch_wire");
    if (!c || !h_offsets || !h_peer || !h_dst || (nb && !d_in))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    uint32_t maxlen = 0;
    hirace_status s = wire_args_ok(c, h_offsets, nb, nranks, my_rank, &maxlen);
    if (s != HIRACE_OK)
        return s;
    for (int r = 0; r < nranks; r++)
        if (!h_peer[r])
            return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if ((s = wire_scratch(c, nb, nranks, maxlen)) != HIRACE_OK)
        return s;
    /* device copies of the peer table and every batch's per-owner destinations; the host
     * arrays may be reused by the caller as soon as this call returns (staged, then synced) */
    const uint64_t need = (uint64_t)nranks + nb * (uint64_t)nranks;
    if (need > c->peer_tab_cap) {
        if (c->d_peer_tab)
            cudaFree(c->d_peer_tab);
        c->d_peer_tab = nullptr;
        c->peer_tab_cap = 0;
        HR_CUDA(c, cudaMalloc(&c->d_peer_tab, need * sizeof(unsigned long long)));
        c->peer_tab_cap = need;
    }
    HR_CUDA(c, cudaMemcpyAsync(c->d_peer_tab, h_peer, nranks * sizeof(void *), cudaMemcpyHostToDevice, st));
    if (nb)
        HR_CUDA(c, cudaMemcpyAsync(c->d_peer_tab + nranks, h_dst, nb * nranks * sizeof(uint64_t),
                                   cudaMemcpyHostToDevice, st));
    /* asynchronous: a bad record raises the context's sticky device error (BAD_TRACE at the
     * next synchronising call), so the dispatch -> replay path never drains the stream */
    for (uint64_t b = 0; b < nb; b++)
        HR_CUDA(c, launch_dispatch_wire(d_in, h_offsets[b], h_offsets[b + 1], nranks, c->cfg.block_threads,
                                        reinterpret_cast<unsigned long long *const *>(c->d_peer_tab),
                                        c->d_peer_tab + nranks + b * (uint64_t)nranks, c->d_bucket_hist,
                                        c->d_wire_off, c->d_err, st));
    return HIRACE_OK;
}

hirace_status hirace_peer_release(hirace_ctx *c, void *const *h_peer_flags, int nranks, uint32_t j0, uint32_t j1,
                                  void *stream)
{
    Nvtx nvtx_range("hirace_peer_release");
    if (!c || !h_peer_flags || nranks < 1 || nranks > 32 || j1 < j0 || j1 >= HIRACE_MAX_BATCHES)
        return HIRACE_E_INVAL;
    for (int r = 0; r < nranks; r++)
        if (!h_peer_flags[r])
            return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (!c->d_flag_tab)
        HR_CUDA(c, cudaMalloc(&c->d_flag_tab, 32 * sizeof(void *)));
    /* pinned staging: the copy is stream-ordered behind the previous release's kernel */
    HR_CUDA(c, cudaMemcpyAsync(c->d_flag_tab, h_peer_flags, nranks * sizeof(void *), cudaMemcpyHostToDevice, st));
    HR_CUDA(c, launch_peer_release(reinterpret_cast<unsigned int *const *>(c->d_flag_tab), nranks, j0, j1, st));
    return HIRACE_OK;
}

hirace_status hirace_peer_wait(hirace_ctx *c, const void *d_flags, uint32_t j, uint32_t target, void *stream)
{
    Nvtx nvtx_range("hirace_peer_wait");
    if (!c || !d_flags || j >= HIRACE_MAX_BATCHES)
        return HIRACE_E_INVAL;
    HR_CUDA(c, cudaSetDevice(c->device));
    HR_CUDA(c, launch_peer_wait(static_cast<const unsigned int *>(d_flags), j, target, (cudaStream_t)stream));
    return HIRACE_OK;
}

hirace_status hirace_peer_buffer_alloc(int device, uint64_t bytes, void **d_ptr, unsigned char handle[64])
{
    if (!d_ptr || !handle || bytes == 0)
        return HIRACE_E_INVAL;
    *d_ptr = nullptr;
    if (cudaSetDevice(device) != cudaSuccess)
        return HIRACE_E_CUDA;
    void *p = nullptr;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess)
        return e == cudaErrorMemoryAllocation ? HIRACE_E_NOMEM : HIRACE_E_CUDA;
    if (cudaMemset(p, 0, bytes) != cudaSuccess) { /* zero-initialised (completion flags start at 0) */
        cudaFree(p);
        return HIRACE_E_CUDA;
    }
    cudaIpcMemHandle_t h;
    static_assert(sizeof(h) == 64, "CUDA IPC handles are 64 bytes");
    if (cudaIpcGetMemHandle(&h, p) != cudaSuccess) {
        cudaFree(p);
        return HIRACE_E_CUDA;
    }
    memcpy(handle, &h, 64);
    *d_ptr = p;
    return HIRACE_OK;
}

hirace_status hirace_peer_buffer_free(void *d_ptr)
{
    return cudaFree(d_ptr) == cudaSuccess ? HIRACE_OK : HIRACE_E_CUDA;
}

hirace_status hirace_peer_open(int device, const unsigned char handle[64], void **d_ptr)
{
    if (!handle || !d_ptr)
        return HIRACE_E_INVAL;
    *d_ptr = nullptr;
    if (cudaSetDevice(device) != cudaSuccess)
        return HIRACE_E_CUDA;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, 64);
    return cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess) == cudaSuccess ? HIRACE_OK : HIRACE_E_CUDA;
}

hirace_status hirace_peer_close(void *d_ptr)
{
    return cudaIpcCloseMemHandle(d_ptr) == cudaSuccess ? HIRACE_OK : HIRACE_E_CUDA;
}

} /* extern "C" */

namespace {

/* hirace_bucket_wire; d_out == NULL counts only (hirace_count_wire: no capacity check) */
hirace_status bucket_wire_impl(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                               int nranks, int my_rank, uint64_t *d_out, uint64_t cap, uint64_t *h_counts,
                               uint64_t *n_words, void *stream)
{
    if (!c || !h_offsets || !h_counts || !n_words || (nb && !d_in) || (cap && !d_out))
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    uint32_t maxlen = 0;
    hirace_status s = wire_args_ok(c, h_offsets, nb, nranks, my_rank, &maxlen);
    if (s != HIRACE_OK)
        return s;
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if ((s = wire_scratch(c, nb, nranks, maxlen)) != HIRACE_OK)
        return s;
    unsigned long long *running = c->d_wire_counts + nb * (uint64_t)nranks;
    HR_CUDA(c, cudaMemsetAsync(running, 0, sizeof(unsigned long long), st));
    HR_CUDA(c, cudaMemsetAsync(c->d_wire_flag, 0, sizeof(unsigned int), st));
    for (uint64_t b = 0; b < nb; b++)
        HR_CUDA(c, launch_bucket_wire(d_in, h_offsets[b], h_offsets[b + 1], nranks, c->cfg.block_threads,
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
    if (d_out && total > cap)
        return HIRACE_E_INVAL;
    return HIRACE_OK;
}

} // namespace

extern "C" {

hirace_status hirace_bucket_wire(hirace_ctx *c, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                 int nranks, int my_rank, uint64_t *d_out, uint64_t cap, uint64_t *h_counts,
                                 uint64_t *n_words, void *stream)
{
    Nvtx nvtx_range("hirace_bucket_wire");
    if (cap && !d_out)
        return HIRACE_E_INVAL;
    uint64_t dummy = 0;
    const hirace_status s = bucket_wire_impl(c, d_in, h_offsets, nb, nranks, my_rank, d_out, cap, h_counts,
                                             n_words ? n_words : &dummy, stream);
    if (s == HIRACE_OK && !d_out && n_words && *n_words > 0)
        return HIRACE_E_INVAL; /* not sticky: call again with a buffer of *n_words records */
    return s;
}

hirace_status hirace_replay_wire(hirace_ctx *c, const uint64_t *d_wire, uint64_t n, uint32_t batch_key, void *stream)
{
    Nvtx nvtx_range("hirace_replay_wire");
    if (!c || c->ws_n)
        return HIRACE_E_INVAL;
    if (c->sticky != HIRACE_OK)
        return c->sticky;
    if (n == 0)
        return HIRACE_OK;
    if (!d_wire || n >= 0xffffffffull || batch_key >= (1u << 27) || c->cfg.granularity_log2 != 2)
        return set_sticky(c, HIRACE_E_INVAL);
    cudaStream_t st = (cudaStream_t)stream;
    HR_CUDA(c, cudaSetDevice(c->device));
    if (ensure_materialized(c, st) != HIRACE_OK || ensure_epoch_normal(c, st) != HIRACE_OK)
        return c->sticky;
    if (c->t_start)
        HR_CUDA(c, cudaEventRecord(c->t_start, st));
    HR_CUDA(c, launch_replay_wire(c->dev, reinterpret_cast<const unsigned long long *>(d_wire), (uint32_t)n, batch_key,
                                  c->replay_grid, st));
    if (c->t_stop)
        HR_CUDA(c, cudaEventRecord(c->t_stop, st));
    return HIRACE_OK;
}

} /* extern "C" */
