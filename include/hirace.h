/*
 * hirace.h — C-ABI of the B200-native HiRace hot path (libhirace.so).
 *
 * HiRace (Jacobson, Burtscher, Gopalakrishnan, SC'24; /root/reference/PAPER.md) keeps ONE
 * constant-size shadow record per tracked memory word — an FSM state plus the last accessor's
 * id and barrier epochs (Fig. 3) — and advances it on every read, write or
 * atomic with a lock-free atomicCAS loop (Algorithm 1).  A word whose record
 * reaches RACE has two accesses that are not ordered by the bulk-synchronous barrier hierarchy
 * (data-race definition PAPER.md; barriers L120-122, L211-213; atomics/scopes L215-229).
 *
 * Plain C: pointers are host or device as stated per argument, sizes are counts, streams are
 * `cudaStream_t` passed as `void*` (0 = legacy default stream).  No torch types.
 *
 * ERRORS.  Every host function returns hirace_status.  Errors are STICKY per context: once a
 * call returns (or a kernel records) an error, later calls on that context return it too,
 * except hirace_shadow_free / hirace_get_stats / hirace_status_string.  Races collected before
 * HIRACE_E_CLOCK_OVERFLOW stay valid ("detection is discontinued with a warning ... after
 * reporting identified races", PAPER.md L227 fn. 3).  Errors found by kernels (bad trace,
 * clock overflow) surface at the next synchronising call (collect / get_stats / sync).
 *
 * OWNERSHIP.  The context owns the shadow array, the FSM table, the race-report buffer and all
 * scratch.  The caller owns event buffers and output buffers.
 *
 * STREAMS.  Calls taking a stream are asynchronous on it, except where noted.  One context
 * must not be used from two streams concurrently.
 */
#ifndef HIRACE_H
#define HIRACE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    HIRACE_OK = 0,
    HIRACE_E_INVAL = -1,          /* bad argument / config / unsupported combination          */
    HIRACE_E_NOMEM = -2,          /* device or host allocation failed                          */
    HIRACE_E_CUDA = -3,           /* a CUDA runtime call failed (no device, launch error, ...) */
    HIRACE_E_CLOCK_OVERFLOW = -4, /* an epoch counter exceeded its field (g 8 / b 10 / w 9 bits)
                                     in an inline hook; detection stopped, races so far valid
                                     (PAPER.md L227 fn. 3, L458)                               */
    HIRACE_E_REPORT_OVERFLOW = -5,/* reserved: collection never loses races (shadow scan)     */
    HIRACE_E_BAD_TRACE = -6,      /* replay input not sorted by (g,b,w), tid/address out of
                                     range, access size > 16 B, or > HIRACE_MAX_BATCHES batches */
    HIRACE_E_COMM = -7,           /* sharded mode exchange failure (set by the Python layer)   */
    HIRACE_E_HISTORY_OVERFLOW = -8/* the sub-warp access history (hirace_set_warp_syncs) was
                                     full: some masked-warp accesses were not compared with
                                     their lanes' history, races among them may be missed   */
} hirace_status;

/* Access kinds: the paper's 4 memory access types. */
typedef enum {
    HIRACE_READ = 0,
    HIRACE_WRITE = 1,
    HIRACE_ATOMIC_BLOCK = 2, /* block-scope atomic (atomicAdd_block, ...) */
    HIRACE_ATOMIC_GRID = 3   /* device-scope atomic (atomicMin, ...)       */
} hirace_kind;

/* Barrier scopes.  GRID = grid-wide sync or kernel boundary. */
typedef enum { HIRACE_SCOPE_WARP = 1, HIRACE_SCOPE_BLOCK = 2, HIRACE_SCOPE_GRID = 3,
               HIRACE_SCOPE_CLUSTER = 4 /* barrier.cluster / cluster.sync(): cluster contexts only */ } hirace_scope;

/* Race class = the coarsest hierarchy level of the first racing epoch (R6). */
typedef enum { HIRACE_RACE_WARP = 1, HIRACE_RACE_BLOCK = 2, HIRACE_RACE_GRID = 3 } hirace_race_class;

/* Conflict policy (R2 / SURVEY §8(f) f2).  STRICT (default, the paper's Table 1
 * reading): a plain read conflicts with an atomic; atomics of different blocks conflict unless
 * both are grid-scope.  RELAXED_READ_ATOMIC: a plain read never conflicts with an atomic and
 * atomics of one block never conflict; across blocks AB-AB and AB-AG still do.  Writes conflict
 * with everything under both. */
typedef enum { HIRACE_POLICY_STRICT = 0, HIRACE_POLICY_RELAXED_READ_ATOMIC = 1 } hirace_policy;

#define HIRACE_MAX_BATCHES 32767u   /* distinct (g,b,w) batch keys per replay call */
#define HIRACE_SHARED_BIT (1ull << 63)

/* Tracked geometry.  warp_size may be any value >= 1 (2 reproduces the paper's Fig. 1 toy
 * hierarchy).  One shadow record per tracked element ("for each element",
 * PAPER.md L162) of 1 << granularity_log2 bytes: 2 = 4-byte words (default, every sharded /
 * wire entry point requires it), 1 = half-words, 0 = bytes (arrays of char: neighbouring bytes
 * written by different threads do not race).  Race keys and "word" indices below count elements.
 * Accesses smaller than an element map to their element; larger ones cover size >> granularity
 * elements.  report_capacity = device race-report records
 * (16 B each); 0 selects a default of 1<<20. */
typedef struct {
    uint32_t grid_blocks;          /* blocks of the checked kernel                        */
    uint32_t block_threads;        /* threads per block (blockDim.x*y*z)                   */
    uint32_t warp_size;            /* threads per warp (32 on NVIDIA hardware)             */
    uint32_t smem_bytes_per_block; /* tracked shared-memory window per block, bytes        */
    uint64_t global_bytes;         /* tracked global extent, bytes from the tracked base   */
    uint32_t granularity_log2;     /* 0, 1 or 2: element = 1, 2 or 4 bytes                  */
    int32_t device;                /* CUDA device ordinal                                  */
    uint64_t report_capacity;      /* race-report ring entries (0 = default)               */
} hirace_config;

/* One traced access, 16 bytes.
 *   addr: bit 63 = shared space.  Shared: byte offset inside the accessing block's tracked
 *         shared window.  Global: byte offset from the tracked global base.
 *   tid:  global thread id = block * block_threads + thread-in-block.
 *   meta: kind:2 | size_log2:3 | w:9 | b:10 | g:8  (bit 0 upward); size = 1 << size_log2 bytes
 *         (<= 16); g = grid epochs (kernel boundaries / grid syncs) passed, b = __syncthreads
 *         passed since the last g, w = full-warp syncs passed since the last b. */
typedef struct {
    uint64_t addr;
    uint32_t tid;
    uint32_t meta;
} hirace_event;

/* One flagged word.  key: global -> word index; shared -> 1<<63 | block<<32 | word.
 * cls_and_epoch = class (1..3) | (g* mod 256) << 8, g* = grid epoch of the first race.
 * detect_tid = the thread whose access moved the record into RACE (not unique across
 * interleavings; never compared). */
typedef struct {
    uint64_t key;
    uint32_t cls_and_epoch;
    uint32_t detect_tid;
} hirace_race;

typedef struct hirace_ctx hirace_ctx;

/* Device-side context handed by value to instrumented kernels (include/hirace_device.cuh).
 * All pointers are device pointers owned by the hirace_ctx. */
typedef struct {
    unsigned long long *shadow;       /* [global_words | grid_blocks * smem_words] records   */
    const unsigned char *table;       /* 2048-entry FSM transition table, followed by its
                                         4096-entry raw-flag expansion (hirace_device.cuh)     */
    hirace_race *reports;             /* race-report ring                                     */
    unsigned long long *report_count; /* records appended (may exceed capacity)               */
    unsigned long long *stats;        /* [checked, cas_retries, cas_ops, no_write]            */
    unsigned int *error_flags;        /* bit0 bad trace, bit1 clock overflow                  */
    unsigned long long report_capacity;
    unsigned long long global_words;
    const void *global_base;          /* tracked global base for inline hooks (may be NULL)   */
    unsigned int smem_words;
    unsigned int grid_blocks, block_threads, warp_size;
    unsigned int bt_magic, bt_s1, bt_s2; /* fast division by block_threads                    */
    unsigned int ws_magic, ws_s1, ws_s2; /* fast division by warp_size                        */
    unsigned int g;                   /* current grid epoch for inline hooks                  */
    /* record layout: rec_bytes = 8 (the 64-bit record of hirace_device.cuh) or 4 (compact
     * record of hirace_shadow_alloc_compact: state:5 | g | b | w | tid, fields starting at
     * bits 5, c_sh_b, c_sh_w, c_sh_t; epochs up to c_max_g / c_max_b / c_max_w)            */
    unsigned int rec_bytes;
    unsigned int c_sh_b, c_sh_w, c_sh_t;
    unsigned int c_max_g, c_max_b, c_max_w;
    unsigned int gran_log2;           /* tracked element = 1 << gran_log2 bytes               */
    /* selective tracking (hirace_set_filter): an access is checked iff f_active == 0, or
     * (tid & f_tid_mask) == f_tid_match and its space is enabled in f_spaces (bit 0 global,
     * bit 1 shared) and, for global, its first element index lies in [f_glo, f_ghi) (an empty
     * range when global memory is disabled).  f_smem_words = smem_words, or 0 when shared
     * memory is disabled (the inline hook's bound).                                          */
    unsigned int f_active, f_tid_mask, f_tid_match, f_spaces;
    unsigned long long f_glo, f_ghi;
    unsigned int f_smem_words, f_pad;
    /* epoch reset (hirace_set_reset_mode): device word holding the grid-epoch offset the
     * replay adds to every trace g (records store g + offset); NULL = 0                     */
    const unsigned int *g_base;
} hirace_dev_ctx;

/* ---- lifecycle (a11: shadow alloc/init, "Initially, all State values are set
 *      to INIT") -------------------------------------------------------------------------- */

/* Allocates shadow = 8 B per tracked word (global_bytes/4 + grid_blocks*smem_bytes/4 words),
 * all INIT, plus the FSM table and report buffer on cfg->device.  Synchronous.
 * Errors: INVAL (NULL args, zero geometry, granularity_log2 > 2, extents not multiples of 4
 * bytes, tid space > 2^32), NOMEM, CUDA. */
hirace_status hirace_shadow_alloc(const hirace_config *cfg, hirace_ctx **out);

/* ---- compact 32-bit shadow ("the shadow-memory footprint
 *      ... can be reduced", L419-423) ------------------------------------------------------ */

/* Declared upper bounds of the epoch counters of the traces a compact context will replay:
 * g <= max_g (grid epochs / kernel boundaries), b <= max_b (__syncthreads since the last g),
 * w <= max_w (full-warp syncs since the last b).  0 = that barrier level never occurs. */
typedef struct {
    uint32_t max_g, max_b, max_w;
} hirace_epoch_limits;

/* hirace_shadow_alloc with 4-byte records: half the shadow footprint (4 B per tracked 4-byte
 * word = 1.0x the tracked bytes, vs 2.0x for 8-byte records).  The record is
 *     state:5 | g:Gb | b:Bb | w:Wb | tid:T     (bit 0 upward, all-zero = INIT)
 * with Gb/Bb/Wb = bits needed for max_g/max_b/max_w and T = bits needed for the largest global
 * thread id.  It holds exactly the fields of the 8-byte record, never truncated, so every
 * transition is the same (same FSM table, same label); verdicts are identical.
 * Replay only: inline hooks (hirace_get_dev_ctx) and hirace_barrier need the 8-byte record.
 * A replayed batch whose (g,b,w) exceeds the declared limits is not checked and raises sticky
 * HIRACE_E_CLOCK_OVERFLOW (races found in earlier batches stay valid).
 * Errors: INVAL (as hirace_shadow_alloc; NULL lim; max_g > 254, max_b > 1023, max_w > 511;
 * 5 + Gb + Bb + Wb + T > 32 — the trace does not fit 32 bits, use hirace_shadow_alloc),
 * NOMEM, CUDA. */
hirace_status hirace_shadow_alloc_compact(const hirace_config *cfg, const hirace_epoch_limits *lim,
                                          hirace_ctx **out);

/* Frees everything the context owns (synchronises the device first).  NULL is a no-op. */
hirace_status hirace_shadow_free(hirace_ctx *ctx);

/* Sets every shadow record to INIT, clears reports, stats and sticky errors; g := 0. Async. */
hirace_status hirace_shadow_reset(hirace_ctx *ctx, void *stream);

/* How hirace_shadow_reset returns the shadow to all-INIT (reading R19).
 * FULL (default): every record is rewritten (a memset of the shadow: 32 GiB on config 5).
 * EPOCH: O(flagged words) - the next check's grid epochs start past every epoch used since the
 * last sweep (the replay adds an offset to the trace's g), so a record left by an earlier
 * check has a different g and reads as INIT by the FSM's own rule (a different grid epoch
 * restarts a record, reading R4); only the RACE records (sticky) are cleared, from the report
 * buffer.  A full sweep still happens when the report buffer overflowed, and a rebase sweep
 * (records of the current check keep their epochs minus the offset, older ones become INIT)
 * when the offset plus a trace's largest g would pass 254 - once per ~254 / (epochs per
 * check) checks.  Race sets and classes are identical in both modes; the g in reported
 * cls_and_epoch is the trace's g in both.  EPOCH applies to the batch-major replay of 8-byte
 * records; inline hooks, wire replay and hirace_barrier first normalise the shadow (a rebase
 * sweep).  INVAL for compact contexts or window-major mode, or an unknown mode.  Waits for the
 * device, then resets the shadow. */
typedef enum { HIRACE_RESET_FULL = 0, HIRACE_RESET_EPOCH = 1 } hirace_reset_mode;
hirace_status hirace_set_reset_mode(hirace_ctx *ctx, int mode);

/* Host barrier hook.  Only HIRACE_SCOPE_GRID is meaningful on the host: a kernel boundary /
 * grid sync advances the context's grid epoch g used by inline hooks.  When g
 * would wrap its 8-bit field the library first runs a rebase sweep (non-RACE records -> INIT,
 * RACE records retired) so equality-only epoch comparisons stay exact (R7).
 * WARP/BLOCK scopes are device-side (hirace::barrier) -> INVAL.  Async. */
hirace_status hirace_barrier(hirace_ctx *ctx, hirace_scope scope, void *stream);

/* Advances the context's grid epoch g by `count` grid-wide synchronisations the host did not
 * see (same rebase rule as hirace_barrier).  A cooperative kernel whose threads call
 * hirace::barrier(GRID) k times ends in epoch g + k on the device; before the next inline
 * kernel the host must therefore advance g by k + 1 (k device grid syncs + the kernel
 * boundary), e.g. hirace_advance_grid_epochs(ctx, k + 1, stream), so no epoch is reused
 * (reused epochs would make ordered cross-kernel accesses look concurrent).  Compact contexts:
 * INVAL.  Async. */
hirace_status hirace_advance_grid_epochs(hirace_ctx *ctx, uint32_t count, void *stream);

/* ---- replay (a1-a9) ------------------------------------------------------------------- */

/* Replays n DEVICE-resident events through the shadow FSM.  Events must be sorted by batch
 * key (g,b,w) = meta >> 5; inside a batch any order (all such events are pairwise concurrent
 * or same-thread, so any order is a linear extension of happens-before).
 * Batches are found on the device and validated (any unsorted input, out-of-range tid or
 * address, size > 16 B -> sticky HIRACE_E_BAD_TRACE, reported at the next sync).  At most
 * HIRACE_MAX_BATCHES batches and n < 2^32 per call; consecutive calls on one stream continue
 * the same linearisation.  Async on `stream`. */
hirace_status hirace_replay_trace(hirace_ctx *ctx, const hirace_event *d_events, uint64_t n, void *stream);

/* hirace_replay_trace + hirace_collect_races_device fused into one persistent kernel: the
 * collection runs as a final grid-wide phase of the replay kernel (no extra launches).  Writes
 * min(cap, total) unique key-sorted records to DEVICE d_out and the total to DEVICE
 * *d_n_total.  Async on `stream`.  Kernel-detected errors surface at the next sync. */
hirace_status hirace_check_trace_device(hirace_ctx *ctx, const hirace_event *d_events, uint64_t n,
                                        hirace_race *d_out, uint64_t cap, unsigned long long *d_n_total,
                                        void *stream);

/* Batch discovery only (a9, as run by hirace_replay_trace): writes the batch start offsets
 * (nb + 1 entries, last = n) and batch keys (g<<19 | b<<9 | w) of DEVICE events to HOST arrays
 * of capacity cap and *nbatches = nb.  Synchronises `stream`.  Used by the sharded driver to
 * exchange events batch by batch.  BAD_TRACE if the keys do not strictly increase. */
hirace_status hirace_find_batches(hirace_ctx *ctx, const hirace_event *d_events, uint64_t n, uint32_t *h_offsets,
                                  uint32_t *h_keys, uint64_t cap, uint64_t *nbatches, void *stream);

/* Same work from HOST events (pinned or pageable): copies through a device staging ring in
 * chunks, overlapping H2D with replay, then collects like hirace_collect_races.  Synchronous.
 * This is the end-to-end entry point. */
hirace_status hirace_check_trace_host(hirace_ctx *ctx, const hirace_event *h_events, uint64_t n,
                                      hirace_race *h_out, uint64_t cap, uint64_t *n_total, void *stream);

/* ---- results (a7) -------------------------------------------------------------------- */

/* How the flagged words are gathered (same output either way): every word entering RACE or
 * upgrading its class appends a report, so for a shadow of >= 64 MiB whose report buffer did
 * not overflow and holds <= 16,384 reports, one CTA sorts the reported keys in shared memory and
 * reads each word's final record ("device sort + unique"); otherwise an
 * order-preserving compaction of the RACE records of the whole shadow runs (single-read,
 * register-resident for small shadows).  Keys come out sorted (global words, then shared words
 * block-major) because the shadow is laid out in key order. */

/* Copies min(cap, n_total) flagged words, sorted by key, unique, to HOST memory h_out and sets
 * *n_total (call again with a bigger buffer if n_total > cap).  Synchronises `stream`.
 * Returns the sticky status (e.g. BAD_TRACE) after copying. */
hirace_status hirace_collect_races(hirace_ctx *ctx, hirace_race *h_out, uint64_t cap, uint64_t *n_total,
                                   void *stream);

/* Device-side variant: writes min(cap, total) records to DEVICE memory d_out and the total to
 * DEVICE *d_n_total.  Async (for timed loops / CUDA graphs). */
hirace_status hirace_collect_races_device(hirace_ctx *ctx, hirace_race *d_out, uint64_t cap,
                                          unsigned long long *d_n_total, void *stream);

/* Counters since the last reset: word-level accesses checked, CAS retries, CAS issued,
 * accesses linearised without a store (no-write fast path), reports appended beyond capacity.
 * Synchronises the device.  Any pointer may be NULL. */
hirace_status hirace_get_stats(hirace_ctx *ctx, uint64_t *checked, uint64_t *cas_retries, uint64_t *cas_ops,
                               uint64_t *no_write, uint64_t *dropped_reports);

/* Synchronises and returns the sticky status (HIRACE_OK if none). */
hirace_status hirace_sync(hirace_ctx *ctx);

/* Copies the device context for inline hooks into *out (host memory).  global_base is the
 * device address tracked global offsets are measured from (may be NULL for replay-only). */
hirace_status hirace_get_dev_ctx(hirace_ctx *ctx, const void *global_base, hirace_dev_ctx *out);

/* Measurement hook: when both are non-NULL, every later hirace_replay_trace records `start`
 * immediately before and `stop` immediately after its replay-kernel launch on the call's
 * stream (cudaEvent_t handles owned by the caller), so the caller can time the dominant
 * kernel alone with cudaEventElapsedTime.  NULL, NULL disables it. */
hirace_status hirace_set_kernel_timing(hirace_ctx *ctx, void *start_event, void *stop_event);

/* ---- sharded mode (a10) ---------------------------------------------------------------- */

/* Buckets n DEVICE events by owner rank for address sharding across nranks GPUs
 * (SURVEY §8(e)): owner(global word) = (word >> 14) mod nranks (64 KiB chunks, so coalesced
 * runs stay on one owner); shared-space events stay on `my_rank` (shared memory is per block,
 * PAPER.md L118).  Writes the events grouped by owner — stable inside each owner, so batch
 * order is preserved — to DEVICE d_out (n records), with every global address rewritten to
 * the owner's shard-local word ((word >> 14) / nranks) << 14 | (word mod 2^14), so the owner's
 * context tracks ceil(global_words / (2^14 nranks)) * 2^14 words.  Per-owner counts go to HOST
 * h_counts[nranks].  Synchronises `stream` (the counts size the exchange).  nranks <= 32.
 * A global 8/16-byte access that straddles two owner chunks cannot be routed as one 16-byte
 * event: it raises sticky BAD_TRACE (hirace_bucket_wire splits such accesses per word). */
hirace_status hirace_bucket_events(hirace_ctx *ctx, const hirace_event *d_in, uint64_t n, int nranks, int my_rank,
                                   hirace_event *d_out, uint64_t *h_counts, void *stream);

/* ---- sharded mode, 8-byte wire format (a10) -------------------------------- */

/* Wire record, 8 bytes (half the 16-byte event on the NVLink exchange):
 *   bits  0..30  word: the owner's shard-local global word, or (bit 31 set) the word inside the
 *                accessing block's shared window (shared events stay on my_rank)
 *   bit  31      shared
 *   bits 32..61  tid (global thread id, < 2^30)
 *   bits 62..63  kind
 * The batch (g,b,w) is implied: records travel and replay one batch at a time.  Global words
 * are owned as in hirace_bucket_events (64 KiB chunks, owner = (word >> 14) mod nranks, local
 * word = ((word >> 14) / nranks) << 14 | word mod 2^14).  8/16-byte accesses are expanded into
 * one record per word, each routed to its own word's owner (an access may straddle chunks). */
#define HIRACE_WIRE_MAX_TIDS (1ull << 30)
#define HIRACE_WIRE_MAX_WORDS (1ull << 31)

/* Buckets the nb batches of DEVICE events d_in (batch b = [h_offsets[b], h_offsets[b+1]),
 * HOST offsets as returned by hirace_find_batches) into wire records at DEVICE d_out
 * (capacity cap records): batch-major, owner-grouped inside a batch (order inside a
 * (batch, owner) segment is unspecified).  Writes HOST h_counts[nb * nranks]
 * (row b = batch b's records per owner) and *n_words = total records.  If *n_words > cap the
 * counts are still written and HIRACE_E_INVAL is returned (not sticky): call again with a
 * buffer of *n_words records.  Synchronises `stream`.
 * Errors: INVAL (NULL args, nranks not in 1..32, my_rank out of range, grid threads > 2^30 or
 * shared-window words > 2^31 — such configurations use hirace_bucket_events), BAD_TRACE
 * (sticky: access size > 16 B, or a shard-local word >= 2^31 — those records are dropped), CUDA. */
hirace_status hirace_bucket_wire(hirace_ctx *ctx, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                 int nranks, int my_rank, uint64_t *d_out, uint64_t cap, uint64_t *h_counts,
                                 uint64_t *n_words, void *stream);

/* Replays n DEVICE wire records of ONE batch, key = g<<19 | b<<9 | w, on ctx (the owner's shard
 * context: its global extent is the shard's).  Successive calls must follow the global batch
 * order.  Records with tid or word out of range -> sticky BAD_TRACE at the next sync.  Async. */
hirace_status hirace_replay_wire(hirace_ctx *ctx, const uint64_t *d_wire, uint64_t n, uint32_t batch_key, void *stream);

/* ---- sharded mode, peer-memory dispatch (a10 fused with the exchange) --------
 * The bucketing kernel stores every wire record DIRECTLY into its owner's receive buffer — on
 * the owner's GPU over NVLink/NVSwitch (CUDA IPC mapping + P2P), or in another process on the
 * same GPU — so the exchange is the scatter itself: no local staging copy, no separate
 * all_to_all.  Protocol per trace (sharded.run_sharded_p2p):
 *   1. hirace_count_wire: per-batch per-owner record counts (no output);
 *   2. the ranks all-gather their count matrices; every rank derives, for each batch b and
 *      owner r, where its segment starts in r's buffer: batches in the global order, inside a
 *      batch the senders in rank order;
 *   3. hirace_dispatch_wire with the peer table (each rank's buffer from
 *      hirace_peer_buffer_alloc, opened by the others with hirace_peer_open);
 *   4. every rank records an interprocess CUDA event after its dispatch; after a host barrier
 *      (which only orders the records) each owner's stream waits on all the peers' events and
 *      replays its buffer batch by batch with hirace_replay_wire — no stream drains. */

/* Per-batch per-owner wire-record counts of nb batches of DEVICE events (h_offsets as from
 * hirace_find_batches): HOST h_counts[nb * nranks], row b = batch b.  Exactly the records
 * hirace_dispatch_wire / hirace_bucket_wire produce.  Synchronises `stream`.
 * Errors: as hirace_bucket_wire. */
hirace_status hirace_count_wire(hirace_ctx *ctx, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                int nranks, int my_rank, uint64_t *h_counts, void *stream);

/* Buckets nb batches of DEVICE events into wire records and stores each one into its owner's
 * receive buffer: h_peer[r] (HOST array of nranks device addresses valid in this process, 8-byte
 * aligned) at record index h_dst[b * nranks + r] + k, k = 0 .. count(b, r) - 1 in unspecified
 * order.  The caller owns the buffers and guarantees the index ranges are
 * inside them and disjoint across senders.  Asynchronous on `stream`; the host arrays may be
 * reused on return.  The owners may read the records once the stream has passed this call
 * (e.g. an interprocess CUDA event recorded after it, waited on by the owners' streams).
 * Errors: INVAL (NULL args, a NULL peer, nranks not in 1..32, geometry beyond the wire format),
 * CUDA; a record beyond the wire format (access size > 16 B, shard-local word >= 2^31) is
 * dropped and raises sticky BAD_TRACE at the next synchronising call. */
hirace_status hirace_dispatch_wire(hirace_ctx *ctx, const hirace_event *d_in, const uint32_t *h_offsets, uint64_t nb,
                                   int nranks, int my_rank, void *const *h_peer, const uint64_t *h_dst,
                                   void *stream);

/* Per-batch completion of the peer dispatch (instead of one event for the whole dispatch):
 * after its dispatch of global batch j (which may be empty), every sender calls
 * hirace_peer_release(ctx, h_peer_flags, nranks, j, j, stream): h_peer_flags[r] = owner r's flag
 * array (a hirace_peer_buffer_alloc buffer of >= HIRACE_MAX_BATCHES u32, zero-initialised by its
 * owner, mapped here with hirace_peer_open) - a system-scope release fence, then +1 on flag j of
 * every owner.  An owner queues hirace_peer_wait(ctx, d_my_flags, j, target, stream) before its
 * replay of batch j: the stream waits (acquire loads, no host involvement) until flag j >= target,
 * target = nranks x (runs so far that used batch j, this one included; flags only grow).  The
 * replay of batch j then overlaps the senders' dispatch of later batches.  Errors: INVAL (NULL
 * args, nranks not in 1..32, j beyond HIRACE_MAX_BATCHES), CUDA.  Asynchronous. */
hirace_status hirace_peer_release(hirace_ctx *ctx, void *const *h_peer_flags, int nranks, uint32_t j0, uint32_t j1,
                                  void *stream);
hirace_status hirace_peer_wait(hirace_ctx *ctx, const void *d_flags, uint32_t j, uint32_t target, void *stream);

/* A zero-initialised receive buffer of `bytes` on `device` that other processes can map:
 * *d_ptr = its device address here, handle = its 64-byte CUDA IPC handle (to be sent to the peers).  The caller
 * frees it with hirace_peer_buffer_free after every peer closed it.  Errors: INVAL, NOMEM, CUDA. */
hirace_status hirace_peer_buffer_alloc(int device, uint64_t bytes, void **d_ptr, unsigned char handle[64]);
hirace_status hirace_peer_buffer_free(void *d_ptr);

/* Maps a peer's receive buffer (handle from hirace_peer_buffer_alloc in ANOTHER process) into
 * this process on `device`, enabling peer access when it lives on another GPU.  Unmap with
 * hirace_peer_close.  Errors: INVAL, CUDA (e.g. no P2P path, or the handle is this process's). */
hirace_status hirace_peer_open(int device, const unsigned char handle[64], void **d_ptr);
hirace_status hirace_peer_close(void *d_ptr);

/* ---- microbenchmarks for the roofline (diagnostics; not part of the checking path) -------- */

/* Rate of 64-bit operations on `nwords` distinct words of a fresh device array (nwords*8 bytes;
 * <= ~64 MiB stays L2-resident), coalesced (random = 0) or uniformly random (random = 1).
 * op: 0 atomicCAS, 1 atomicAdd, 2 coherent load (ld.relaxed.gpu), 3 load + CAS pair.
 * Writes operations per second to *ops_per_s.  Synchronous. */
hirace_status hirace_microbench_atomics(int device, uint64_t nwords, int random, int op, uint64_t nops,
                                        double *ops_per_s, void *stream);

/* Cost of one grid barrier at the persistent replay kernel's grid size, microseconds.
 * mode 0 = the library's barrier; 1 = busy polling; 2 = generation flag set by the last CTA. */
hirace_status hirace_microbench_grid_sync(int device, int iters, int mode, double *us_per_barrier, void *stream);
/* Diagnostics: op 2 (coherent load) or 3 (load + CAS) on the 8-byte words words[idx[i]],
 * i < n, grid-stride over the list with ctas_per_sm x 256-thread CTAs per SM; the list order is
 * the access pattern.  *ms_out = kernel time (CUDA events on `stream`).  Caller owns both
 * device buffers.  HIRACE_E_INVAL on null pointers or another op. */
hirace_status hirace_microbench_indexed(int device, void *words, const void *idx, uint64_t n, int op,
                                        int ctas_per_sm, double *ms_out, void *stream);

/* Selective tracking ("Individual threads or test data
 * addresses may have their instrumentation enabled or disabled dynamically.  The memory
 * footprint can be reduced by tracking only representative threads from a symmetric group").
 * Later replays (hirace_replay_trace / hirace_check_trace_*) and inline launches (the device
 * context copied after this call) check an access only if
 *     (tid & tid_mask) == tid_match                 -- e.g. mask 31, match 0: lane 0 of every warp
 *     and its space is in `spaces` (1 = global, 2 = shared, 3 = both)
 *     and, for a global access, its first element index is in [global_lo, global_hi).
 * Unselected accesses are skipped (not counted as checked, never BAD_TRACE).  Races are then
 * those among the selected accesses.  hirace_set_filter(ctx, 0, 0, 3, 0, UINT64_MAX) selects
 * everything (the default).  Host-side; takes effect at the next launch.  The wire replay
 * (sharded mode) ignores the filter.  Errors: INVAL (NULL ctx, tid_match outside tid_mask,
 * spaces > 3, global_lo > global_hi). */
hirace_status hirace_set_filter(hirace_ctx *ctx, uint32_t tid_mask, uint32_t tid_match, uint32_t spaces,
                                uint64_t global_lo, uint64_t global_hi);

/* Selects the conflict policy of a context by uploading that policy's FSM table (stream-ordered
 * on `stream`).  Takes effect for later replays and inline launches; call it on a reset shadow
 * (records written under one policy are states of that policy's automaton).
 * Errors: INVAL (NULL ctx, unknown policy), CUDA. */
hirace_status hirace_set_policy(hirace_ctx *ctx, int policy, void *stream);

/* ---- verification hooks (host-only, NOT a replay path) --------------------------------- */

/* Writes the 2048-byte FSM transition table: entry[state<<6 | kind<<4 | sync<<2 | rel] =
 * next_state:5 | keep_record:1 | report:1 (PAPER.md L295 flat-array encoding). */
hirace_status hirace_fsm_table(unsigned char out[2048]);

/* hirace_fsm_table for a given hirace_policy.  Errors: INVAL (NULL out, unknown policy). */
hirace_status hirace_fsm_table_policy(int policy, unsigned char out[2048]);

/* One FSM step on the host with the same inline function the kernels use, for model checking:
 * returns the new 64-bit record for old record `old_shadow` and one access. *report is set to
 * 1 if the step enters or upgrades a RACE state. */
uint64_t hirace_fsm_step(uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t b, uint32_t w,
                         uint32_t block_threads, uint32_t warp_size, int *report);

/* hirace_fsm_step under a given hirace_policy (unknown values select STRICT). */
uint64_t hirace_fsm_step_policy(int policy, uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t b,
                                uint32_t w, uint32_t block_threads, uint32_t warp_size, int *report);

/* One FSM step on a compact 4-byte record (hirace_shadow_alloc_compact layout for grid_threads
 * threads and limits *lim), with the same inline functions the compact replay kernels use.
 * Inputs must lie within the limits.  Returns 0xffffffff if the layout does not fit 32 bits. */
uint32_t hirace_fsm_step_compact(int policy, uint32_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t b,
                                 uint32_t w, uint32_t block_threads, uint32_t warp_size, uint32_t grid_threads,
                                 const hirace_epoch_limits *lim, int *report);

/* Cluster level (reading R16): host model of the
 * derived cluster-level FSM (hirace_device.cuh, namespace hirace::cluster), 34 reachable states;
 * the replay path is hirace_cluster_replay below.
 * hirace_fsm_table_cluster writes the 16384-byte table (entry[state<<8 | kind<<6 | sync<<3 | rel]
 * = next:6 | keep:1 | report:1) and the number of live states.  Errors: INVAL (NULL out, or the
 * rules reaching more than 64 states).
 * hirace_fsm_cluster_class: race class of a state code (0 = not RACE; 4 = CLUSTER).
 * hirace_fsm_step_cluster: one step on the record state:6 | g:8 | c:7 | b:8 | w:8 | tid:27;
 * returns ~0 for a zero geometry or an epoch / tid beyond its field. */
hirace_status hirace_fsm_table_cluster(unsigned char out[16384], uint32_t *n_states);
uint32_t hirace_fsm_cluster_class(uint32_t state);
uint64_t hirace_fsm_step_cluster(uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t c, uint32_t b,
                                 uint32_t w, uint32_t block_threads, uint32_t warp_size, uint32_t cluster_blocks,
                                 int *report);

/* ---- partial-mask warp synchronisation ------------------
 * "masked warp synchronization primitives may be used to implement non-hierarchical barrier
 * points, which are not amenable to representation within HiRace's FSM.  In these cases,
 * HiRace ... tracks a bounded history of sub-warp synchronizations (essentially a warp-level
 * vector clock) and opportunistically prunes the history" (R20).
 *
 * Trace convention.  Inside one block epoch (g, b) each warp numbers its synchronisations --
 * full-mask __syncwarp / votes and partial __syncwarp(mask) alike -- 1, 2, 3, ... in a linear
 * order consistent with every lane's program order.  An event's w is the number of the LAST warp
 * sync its lane passed (0 = none), so traces without partial masks keep their meaning (w =
 * full-warp syncs since the last b).  The partial syncs are listed in a log of
 * hirace_warp_sync records sorted by (g, b, warp, w), strictly increasing; numbers not listed
 * are full-mask syncs.
 *   warp  global warp id = block * ceil(block_threads / warp_size) + warp in block
 *   mask  the participating lanes (bit i = lane i), non-zero, lanes < warp_size
 *   meta  w:9 << 5 | b:10 << 14 | g:8 << 24  (the event meta layout with kind = size = 0)
 * An access of lane j after sync w1 happens before an access of lane i != j after sync w2 > w1
 * iff a chain of syncs w1 < s_1 < ... < s_m <= w2 links lane j to lane i (consecutive syncs
 * share a lane); every other ordering is the three-level one. */
typedef struct {
    uint32_t warp;
    uint32_t mask;
    uint32_t meta;
    uint32_t pad; /* 0 */
} hirace_warp_sync;

/* Sets the partial-sync log for the following hirace_replay_trace / hirace_check_trace_*
 * calls of ctx (until replaced; n == 0 removes it).  d_syncs: DEVICE array of n records (read
 * during this call only; the context keeps its own derived copy).  The library derives, per
 * (g, b, warp) family, the warp vector clock after every listed sync (one warp per family),
 * and allocates a sub-warp access history of history_slots slots (rounded up to a power of two;
 * 0 = 65,536; 64 B each, plus a pool of slots/8 spill blocks of 256 B): one slot per word that
 * masked-family accesses touch in a block epoch, holding for up to five (lane, access class)
 * pairs the last sync number (read / atomic / write), more pairs in a spill block.  The replay
 * then runs the per-access FSM as usual with w read as the sync number, and additionally
 * compares each access of a family at a listed sync with its lanes' history against the vector
 * clock: a conflicting access not ordered before it is a race of the FSM state's level (WARP
 * while one warp touched the word in the block epoch, else BLOCK / GRID; R20).
 * The log drives the replay (batch-major: while a log is set, window-major mode replays
 * batch-major, and the wire / sharded entry points and hirace_get_dev_ctx return
 * HIRACE_E_INVAL); instrumented kernels take partial syncs live through
 * hirace_inline_warp_syncs instead.  The history is
 * cleared by hirace_shadow_reset.  Synchronises `stream`.
 * Errors: INVAL (NULL ctx / n && !d_syncs, warp_size > 32, granularity_log2 != 2), BAD_TRACE
 * (unsorted or duplicate records, w == 0, mask 0 or beyond warp_size, warp id beyond the grid;
 * sticky), NOMEM, CUDA.  During replay: an access after a listed sync whose mask lacks its lane
 * -> sticky BAD_TRACE; a full history -> sticky HIRACE_E_HISTORY_OVERFLOW. */
hirace_status hirace_set_warp_syncs(hirace_ctx *ctx, const hirace_warp_sync *d_syncs, uint64_t n,
                                    uint64_t history_slots, void *stream);

/* Partial-mask syncs in the INLINE hooks (the paper's setting): the
 * sub-warp history of an instrumented kernel (device pointers owned by the context; the same
 * 64-B bounded-history slots and spill pool as the replay), passed by value next to the
 * hirace_dev_ctx.  Device side (include/hirace_device.cuh, namespace hirace::ws): a per-warp
 * vector clock in a caller-provided __shared__ buffer (ws_smem_bytes(blockDim)),
 * thread_init_ws, syncwarp (call right after every __syncwarp(mask) / tile.sync(), also the
 * full-mask ones), barrier_ws (after __syncthreads / at a grid sync), on_access_ws.  The sync
 * numbering is the order in which the warp reaches its syncs (an atomic per-warp counter), so
 * any schedule gives the relation of R20. */
typedef struct {
    unsigned long long *hist;        /* slots_mask + 1 slots of 8 words                       */
    unsigned long long slots_mask;
    unsigned long long *spill;       /* nspill blocks of 32 lane words                        */
    unsigned long long *spill_count;
    unsigned long long nspill;
    unsigned int confl[3];           /* per class (R, A, X): the classes it conflicts with    */
    unsigned char race_of[32];       /* FSM state -> RACE state of its level                   */
} hirace_ws_ctx;

/* Allocates (first call) the context's inline sub-warp history with history_slots slots (power
 * of two, 0 = 65,536) and writes its device handle.  The conflict and level tables follow the
 * context's policy at the time of the call.  Cleared by hirace_shadow_reset.  Synchronous.
 * Errors: INVAL (NULL args, compact record, warp_size > 32, granularity_log2 != 2), NOMEM, CUDA.
 * During the kernel: a full history -> sticky HIRACE_E_HISTORY_OVERFLOW, a warp sync number
 * beyond 511 -> sticky HIRACE_E_CLOCK_OVERFLOW. */
hirace_status hirace_inline_warp_syncs(hirace_ctx *ctx, uint64_t history_slots, hirace_ws_ctx *out);

/* ---- cluster-level replay (reading R16) ----------------------------
 * A context whose hierarchy has a thread-block-cluster level between the block and the grid:
 * blocks [k*cluster_blocks, (k+1)*cluster_blocks) form cluster k (cluster_blocks must divide
 * grid_blocks, <= 255; granularity_log2 must be 2; grid_blocks*block_threads <= 2^27).
 * Events are hirace_event with two extra address fields:
 *   addr bits 56..62  c: cluster barriers (barrier.cluster arrive+wait) passed since the last g;
 *                     __syncthreads counts b restart at each c;
 *   addr bits 48..55  shared accesses only: DSMEM target, 0 = the accessing block's own window,
 *                     r+1 = the window of the block with cluster rank r;
 *   addr bits 0..47   byte offset (global from the tracked base, shared in the target window).
 * Records: 8 bytes, state:6 | g:8 | c:7 | b:8 | w:8 | tid:27 (so b, w <= 255), the derived cluster
 * FSM (hirace_fsm_table_cluster).  Race classes add HIRACE_RACE_CLUSTER = 4.
 *
 * hirace_cluster_alloc   context + shadow (all INIT) on cfg->device; caller frees with
 *                        hirace_cluster_free.  Errors: INVAL (geometry as above), NOMEM, CUDA.
 * hirace_cluster_reset   shadow := INIT, errors and stats := 0, stream-ordered.
 * hirace_cluster_replay  d_events (device, n < 2^32) sorted by (g, c, b, w); asynchronous on
 *                        `stream`; one cooperative launch.  Events that are not batch-sorted or
 *                        out of range (tid, address, DSMEM target outside the cluster, b or w
 *                        > 255) are skipped and make the next collect return BAD_TRACE (sticky
 *                        until reset).
 * hirace_cluster_collect synchronises the device, writes min(cap, n_total) flagged words in key
 *                        order (hirace_race; class 1 WARP, 2 BLOCK, 3 GRID, 4 CLUSTER) to
 *                        host memory and sets *n_total.
 * hirace_cluster_get_stats  checked word accesses and CAS retries since the last reset. */
typedef struct hirace_cluster_ctx hirace_cluster_ctx;
#define HIRACE_RACE_CLUSTER 4
hirace_status hirace_cluster_alloc(const hirace_config *cfg, uint32_t cluster_blocks, hirace_cluster_ctx **out);
hirace_status hirace_cluster_free(hirace_cluster_ctx *ctx);
hirace_status hirace_cluster_reset(hirace_cluster_ctx *ctx, void *stream);
hirace_status hirace_cluster_replay(hirace_cluster_ctx *ctx, const hirace_event *d_events, uint64_t n, void *stream);
hirace_status hirace_cluster_collect(hirace_cluster_ctx *ctx, hirace_race *h_out, uint64_t cap, uint64_t *n_total);
hirace_status hirace_cluster_get_stats(hirace_cluster_ctx *ctx, uint64_t *checked, uint64_t *cas_retries);

/* Inline hooks for a cluster context (the paper's wrapper, with the cluster level
 * of R16): device context handed by value to instrumented cluster kernels; the device side is
 * hirace::cluster::thread_init / on_access / barrier in include/hirace_device.cuh.  DSMEM
 * accesses are recognised from the generic address (an address another block of the cluster
 * maps through cluster.map_shared_rank / __cluster_map_shared_rank).  All pointers are device
 * pointers owned by the cluster context; g = grid epoch of the launch (0 here: the caller sets
 * it per launch, <= 254, one per kernel boundary).  Results: hirace_cluster_collect.
 * Errors (inline): out-of-range thread ids / epochs set the context's range flag (BAD_TRACE at
 * the next collect) and stop checking in that thread. */
typedef struct {
    unsigned long long *shadow;  /* [global_words | grid_blocks * smem_words] cluster records */
    const unsigned char *table;  /* 16 KB cluster FSM table (hirace_fsm_table_cluster)       */
    unsigned int *error_flags;   /* bit0 bad trace, bit1 range                               */
    unsigned long long *stats;   /* [checked word accesses, CAS retries]                     */
    const void *global_base;     /* tracked global base (may be NULL)                        */
    unsigned long long global_words;
    unsigned int smem_words, grid_blocks, block_threads, warp_size, cluster_blocks;
    unsigned int g;
} hirace_cluster_dev_ctx;
hirace_status hirace_cluster_get_dev_ctx(hirace_cluster_ctx *ctx, const void *global_base,
                                         hirace_cluster_dev_ctx *out);

const char *hirace_status_string(hirace_status s);

/* Library version string and the compile target ("sm_100a"). */
const char *hirace_version(void);

/* Replay strategy.  BATCH: the batch-major persistent kernel (k_replay: every
 * batch's events in trace order, grid barrier between batches).  WINDOW: window-major (the
 * element accesses are partitioned by shadow window with two counting-sort passes that keep
 * batch order inside each window, and each window is replayed by one CTA in shared memory;
 * PAPER.md L177 allows any order inside a batch, L162 makes records per element).  AUTO
 * (default): BATCH, which measured faster on every config (config 5: 34 vs 39 ms per check);
 * the environment variable HIRACE_WINDOW_AUTO_BYTES=<n> makes AUTO pick WINDOW for shadows of
 * at least n bytes.  WINDOW needs 8-byte records and 4-byte elements (granularity_log2 == 2).
 * In window mode hirace_shadow_reset is O(1) (a generation counter: every window reads as INIT
 * until replayed; paths that touch the shadow directly first make stale windows INIT).  The
 * window path holds up to 1.25 x n + 65536 element accesses per check (8/16-byte accesses
 * count 2/4); beyond that the check stops with HIRACE_E_NOMEM (sticky) and the caller can
 * switch to BATCH.  window_log2: 2^window_log2 records per window, 5..14 (0 = 12).  Setting
 * the mode waits for the device and resets the shadow (all INIT).  HIRACE_E_INVAL on an
 * unknown mode or a context WINDOW does not support. */
typedef enum { HIRACE_REPLAY_AUTO = 0, HIRACE_REPLAY_BATCH = 1, HIRACE_REPLAY_WINDOW = 2 } hirace_replay_mode;
hirace_status hirace_set_replay_mode(hirace_ctx *ctx, int mode, uint32_t window_log2);
/* *active_window = 1 if the next check runs window-major. */
hirace_status hirace_get_replay_mode(const hirace_ctx *ctx, int *active_window);

/* Process-wide number of kernels the library has launched so far (every replay, reset,
 * collect, bucketing ... kernel; captured CUDA-graph replays are not counted).  bench.py takes
 * the difference around one eager step.  HIRACE_E_INVAL if out is null. */
hirace_status hirace_launch_count(uint64_t *out);

#ifdef __cplusplus
}
#endif
#endif /* HIRACE_H */
