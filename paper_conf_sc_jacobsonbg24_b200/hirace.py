"""Thin ctypes binding over libhirace.so (include/hirace.h).  Argument marshalling only:
every step of the hot path runs in the library's sm_100a kernels.  PyTorch provides device
memory and streams.  There is no CPU fallback: if the library or a CUDA device is missing,
every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("HIRACE_LIB") or os.path.join(_PKG, "lib", "libhirace.so")  # override: A/B builds

EVENT_DTYPE = np.dtype([("addr", "<u8"), ("tid", "<u4"), ("meta", "<u4")])
RACE_DTYPE = np.dtype([("key", "<u8"), ("cls_and_epoch", "<u4"), ("detect_tid", "<u4")])
WARP_SYNC_DTYPE = np.dtype([("warp", "<u4"), ("mask", "<u4"), ("meta", "<u4"), ("pad", "<u4")])  # hirace_warp_sync

READ, WRITE, ATOMIC_BLOCK, ATOMIC_GRID = 0, 1, 2, 3
SCOPE_WARP, SCOPE_BLOCK, SCOPE_GRID = 1, 2, 3
RACE_WARP, RACE_BLOCK, RACE_GRID = 1, 2, 3
MAX_BATCHES = 32767

STATUS = {0: "HIRACE_OK", -1: "HIRACE_E_INVAL", -2: "HIRACE_E_NOMEM", -3: "HIRACE_E_CUDA",
          -4: "HIRACE_E_CLOCK_OVERFLOW", -5: "HIRACE_E_REPORT_OVERFLOW", -6: "HIRACE_E_BAD_TRACE",
          -7: "HIRACE_E_COMM", -8: "HIRACE_E_HISTORY_OVERFLOW"}

POLICY_STRICT, POLICY_RELAXED_READ_ATOMIC = 0, 1
REPLAY_AUTO, REPLAY_BATCH, REPLAY_WINDOW = 0, 1, 2
RESET_FULL, RESET_EPOCH = 0, 1

# every symbol include/hirace.h declares (checked by tests/test_abi.py against the header)
EXPORTS = ("hirace_shadow_alloc", "hirace_shadow_alloc_compact", "hirace_shadow_free", "hirace_shadow_reset", "hirace_barrier",
           "hirace_replay_trace", "hirace_find_batches", "hirace_check_trace_device", "hirace_check_trace_host", "hirace_collect_races",
           "hirace_collect_races_device", "hirace_get_stats", "hirace_sync", "hirace_get_dev_ctx",
           "hirace_bucket_events", "hirace_bucket_wire", "hirace_replay_wire", "hirace_count_wire",
           "hirace_dispatch_wire", "hirace_peer_buffer_alloc", "hirace_peer_buffer_free", "hirace_peer_open",
           "hirace_peer_close", "hirace_set_kernel_timing", "hirace_microbench_atomics", "hirace_microbench_grid_sync", "hirace_microbench_indexed", "hirace_set_policy", "hirace_set_filter",
           "hirace_fsm_table", "hirace_fsm_table_policy", "hirace_fsm_step", "hirace_fsm_step_policy", "hirace_fsm_step_compact",
           "hirace_fsm_table_cluster", "hirace_fsm_cluster_class", "hirace_fsm_step_cluster",
           "hirace_cluster_alloc", "hirace_cluster_free", "hirace_cluster_reset", "hirace_cluster_replay",
           "hirace_cluster_collect", "hirace_cluster_get_stats", "hirace_status_string",
           "hirace_version", "hirace_launch_count", "hirace_set_replay_mode", "hirace_get_replay_mode",
           "hirace_advance_grid_epochs", "hirace_peer_release", "hirace_peer_wait", "hirace_set_reset_mode",
           "hirace_set_warp_syncs", "hirace_cluster_get_dev_ctx", "hirace_inline_warp_syncs")


class HiraceError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}")


class Config(ctypes.Structure):
    _fields_ = [("grid_blocks", ctypes.c_uint32), ("block_threads", ctypes.c_uint32),
                ("warp_size", ctypes.c_uint32), ("smem_bytes_per_block", ctypes.c_uint32),
                ("global_bytes", ctypes.c_uint64), ("granularity_log2", ctypes.c_uint32),
                ("device", ctypes.c_int32), ("report_capacity", ctypes.c_uint64)]


class DevCtx(ctypes.Structure):
    _fields_ = [("shadow", ctypes.c_void_p), ("table", ctypes.c_void_p), ("reports", ctypes.c_void_p),
                ("report_count", ctypes.c_void_p), ("stats", ctypes.c_void_p),
                ("error_flags", ctypes.c_void_p), ("report_capacity", ctypes.c_uint64),
                ("global_words", ctypes.c_uint64), ("global_base", ctypes.c_void_p),
                ("smem_words", ctypes.c_uint32), ("grid_blocks", ctypes.c_uint32),
                ("block_threads", ctypes.c_uint32), ("warp_size", ctypes.c_uint32),
                ("bt_magic", ctypes.c_uint32), ("bt_s1", ctypes.c_uint32), ("bt_s2", ctypes.c_uint32),
                ("ws_magic", ctypes.c_uint32), ("ws_s1", ctypes.c_uint32), ("ws_s2", ctypes.c_uint32),
                ("g", ctypes.c_uint32), ("rec_bytes", ctypes.c_uint32), ("c_sh_b", ctypes.c_uint32),
                ("c_sh_w", ctypes.c_uint32), ("c_sh_t", ctypes.c_uint32), ("c_max_g", ctypes.c_uint32),
                ("c_max_b", ctypes.c_uint32), ("c_max_w", ctypes.c_uint32), ("gran_log2", ctypes.c_uint32),
                ("f_active", ctypes.c_uint32), ("f_tid_mask", ctypes.c_uint32), ("f_tid_match", ctypes.c_uint32),
                ("f_spaces", ctypes.c_uint32), ("f_glo", ctypes.c_uint64), ("f_ghi", ctypes.c_uint64),
                ("f_smem_words", ctypes.c_uint32), ("f_pad", ctypes.c_uint32), ("g_base", ctypes.c_void_p)]


class ClusterDevCtx(ctypes.Structure):
    """hirace_cluster_dev_ctx (include/hirace.h): handed by value to instrumented cluster kernels."""
    _fields_ = [("shadow", ctypes.c_void_p), ("table", ctypes.c_void_p), ("error_flags", ctypes.c_void_p),
                ("stats", ctypes.c_void_p), ("global_base", ctypes.c_void_p), ("global_words", ctypes.c_uint64),
                ("smem_words", ctypes.c_uint32), ("grid_blocks", ctypes.c_uint32), ("block_threads", ctypes.c_uint32),
                ("warp_size", ctypes.c_uint32), ("cluster_blocks", ctypes.c_uint32), ("g", ctypes.c_uint32)]


class WsCtx(ctypes.Structure):
    """hirace_ws_ctx (include/hirace.h): the inline hooks' sub-warp history."""
    _fields_ = [("hist", ctypes.c_void_p), ("slots_mask", ctypes.c_uint64), ("spill", ctypes.c_void_p),
                ("spill_count", ctypes.c_void_p), ("nspill", ctypes.c_uint64), ("confl", ctypes.c_uint32 * 3),
                ("race_of", ctypes.c_uint8 * 32)]


class EpochLimits(ctypes.Structure):
    """hirace_epoch_limits: declared maxima of the g / b / w epoch counters (compact records)."""
    _fields_ = [("max_g", ctypes.c_uint32), ("max_b", ctypes.c_uint32), ("max_w", ctypes.c_uint32)]


_lib = None


def load():
    """Loads the in-tree library; raises if it was not built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise RuntimeError(f"{SO_PATH} missing: build it with `python -m paper_conf_sc_jacobsonbg24_b200.build` "
                           "(the CUDA path has no fallback)")
    lib = ctypes.CDLL(SO_PATH)
    P, U64, U32, I32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    sig = {
        "hirace_shadow_alloc": (I32, [ctypes.POINTER(Config), ctypes.POINTER(P)]),
        "hirace_shadow_alloc_compact": (I32, [ctypes.POINTER(Config), ctypes.POINTER(EpochLimits), ctypes.POINTER(P)]),
        "hirace_shadow_free": (I32, [P]),
        "hirace_shadow_reset": (I32, [P, P]),
        "hirace_barrier": (I32, [P, I32, P]),
        "hirace_replay_trace": (I32, [P, P, U64, P]),
        "hirace_check_trace_host": (I32, [P, P, U64, P, U64, ctypes.POINTER(U64), P]),
        "hirace_check_trace_device": (I32, [P, P, U64, P, U64, P, P]),
        "hirace_find_batches": (I32, [P, P, U64, P, P, U64, ctypes.POINTER(U64), P]),
        "hirace_collect_races": (I32, [P, P, U64, ctypes.POINTER(U64), P]),
        "hirace_collect_races_device": (I32, [P, P, U64, P, P]),
        "hirace_get_stats": (I32, [P] + [ctypes.POINTER(U64)] * 5),
        "hirace_sync": (I32, [P]),
        "hirace_get_dev_ctx": (I32, [P, P, ctypes.POINTER(DevCtx)]),
        "hirace_bucket_events": (I32, [P, P, U64, I32, I32, P, ctypes.POINTER(U64), P]),
        "hirace_bucket_wire": (I32, [P, P, P, U64, I32, I32, P, U64, P, ctypes.POINTER(U64), P]),
        "hirace_replay_wire": (I32, [P, P, U64, U32, P]),
        "hirace_count_wire": (I32, [P, P, P, U64, I32, I32, P, P]),
        "hirace_dispatch_wire": (I32, [P, P, P, U64, I32, I32, P, P, P]),
        "hirace_peer_buffer_alloc": (I32, [I32, U64, ctypes.POINTER(P), P]),
        "hirace_peer_buffer_free": (I32, [P]),
        "hirace_peer_open": (I32, [I32, P, ctypes.POINTER(P)]),
        "hirace_peer_close": (I32, [P]),
        "hirace_set_kernel_timing": (I32, [P, P, P]),
        "hirace_microbench_atomics": (I32, [I32, U64, I32, I32, U64, ctypes.POINTER(ctypes.c_double), P]),
        "hirace_microbench_grid_sync": (I32, [I32, I32, I32, ctypes.POINTER(ctypes.c_double), P]),
        "hirace_microbench_indexed": (I32, [I32, P, P, U64, I32, I32, ctypes.POINTER(ctypes.c_double), P]),
        "hirace_set_policy": (I32, [P, I32, P]),
        "hirace_set_filter": (I32, [P, U32, U32, U32, U64, U64]),
        "hirace_fsm_table": (I32, [P]),
        "hirace_fsm_table_policy": (I32, [I32, P]),
        "hirace_fsm_step": (U64, [U64, U32, U32, U32, U32, U32, U32, U32, ctypes.POINTER(I32)]),
        "hirace_fsm_step_policy": (U64, [I32, U64, U32, U32, U32, U32, U32, U32, U32, ctypes.POINTER(I32)]),
        "hirace_fsm_step_compact": (U32, [I32, U32, U32, U32, U32, U32, U32, U32, U32, U32,
                                          ctypes.POINTER(EpochLimits), ctypes.POINTER(I32)]),
        "hirace_fsm_table_cluster": (I32, [P, ctypes.POINTER(U32)]),
        "hirace_fsm_cluster_class": (U32, [U32]),
        "hirace_fsm_step_cluster": (U64, [U64, U32, U32, U32, U32, U32, U32, U32, U32, U32, ctypes.POINTER(I32)]),
        "hirace_cluster_alloc": (I32, [ctypes.POINTER(Config), U32, ctypes.POINTER(ctypes.c_void_p)]),
        "hirace_cluster_free": (I32, [P]),
        "hirace_cluster_reset": (I32, [P, P]),
        "hirace_cluster_replay": (I32, [P, P, U64, P]),
        "hirace_cluster_collect": (I32, [P, P, U64, ctypes.POINTER(U64)]),
        "hirace_cluster_get_stats": (I32, [P, ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "hirace_status_string": (ctypes.c_char_p, [I32]),
        "hirace_version": (ctypes.c_char_p, []),
        "hirace_launch_count": (I32, [ctypes.POINTER(U64)]),
        "hirace_set_replay_mode": (I32, [P, I32, U32]),
        "hirace_advance_grid_epochs": (I32, [P, U32, P]),
        "hirace_peer_release": (I32, [P, P, I32, U32, U32, P]),
        "hirace_peer_wait": (I32, [P, P, U32, U32, P]),
        "hirace_set_reset_mode": (I32, [P, I32]),
        "hirace_get_replay_mode": (I32, [P, ctypes.POINTER(I32)]),
        "hirace_set_warp_syncs": (I32, [P, P, U64, U64, P]),
        "hirace_cluster_get_dev_ctx": (I32, [P, P, ctypes.POINTER(ClusterDevCtx)]),
        "hirace_inline_warp_syncs": (I32, [P, U64, ctypes.POINTER(WsCtx)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype, f.argtypes = res, args
    _lib = lib
    return lib


def _check(st: int, where: str):
    if st != 0:
        raise HiraceError(st, where)


def fsm_table(policy: int = 0) -> np.ndarray:
    t = np.zeros(2048, np.uint8)
    if policy == POLICY_STRICT:
        _check(load().hirace_fsm_table(t.ctypes.data), "hirace_fsm_table")
    else:
        _check(load().hirace_fsm_table_policy(policy, t.ctypes.data), "hirace_fsm_table_policy")
    return t


def fsm_step(old: int, tid: int, kind: int, g: int, b: int, w: int, block_threads: int, warp_size: int,
             policy: int = 0):
    rep = ctypes.c_int(0)
    if policy == POLICY_STRICT:
        n = load().hirace_fsm_step(old, tid, kind, g, b, w, block_threads, warp_size, ctypes.byref(rep))
    else:
        n = load().hirace_fsm_step_policy(policy, old, tid, kind, g, b, w, block_threads, warp_size,
                                          ctypes.byref(rep))
    return int(n), int(rep.value)


def fsm_step_compact(old: int, tid: int, kind: int, g: int, b: int, w: int, block_threads: int, warp_size: int,
                     grid_threads: int, limits, policy: int = 0):
    """One step on a compact 4-byte record (include/hirace.h hirace_fsm_step_compact)."""
    rep = ctypes.c_int(0)
    lim = EpochLimits(*limits)
    n = load().hirace_fsm_step_compact(policy, old, tid, kind, g, b, w, block_threads, warp_size, grid_threads,
                                       ctypes.byref(lim), ctypes.byref(rep))
    return int(n), int(rep.value)


def fsm_table_cluster():
    """(16384-byte cluster-level table, number of live states) (hirace_fsm_table_cluster)."""
    t = np.zeros(16384, np.uint8)
    n = ctypes.c_uint32(0)
    _check(load().hirace_fsm_table_cluster(t.ctypes.data, ctypes.byref(n)), "hirace_fsm_table_cluster")
    return t, int(n.value)


def fsm_cluster_class(state: int) -> int:
    return int(load().hirace_fsm_cluster_class(state))


def fsm_step_cluster(old: int, tid: int, kind: int, g: int, c: int, b: int, w: int, block_threads: int,
                     warp_size: int, cluster_blocks: int):
    """One cluster-level FSM step on the host (include/hirace.h hirace_fsm_step_cluster)."""
    rep = ctypes.c_int(0)
    n = load().hirace_fsm_step_cluster(old, tid, kind, g, c, b, w, block_threads, warp_size, cluster_blocks,
                                       ctypes.byref(rep))
    if n == (1 << 64) - 1:
        raise HiraceError(-1, "hirace_fsm_step_cluster")
    return int(n), int(rep.value)


def trace_epoch_limits(events: np.ndarray) -> tuple[int, int, int]:
    """(max g, max b, max w) over a trace's events: the limits a compact context needs."""
    meta = events["meta"]
    if meta.shape[0] == 0:
        return (0, 0, 0)
    return (int((meta >> 24).max()), int(((meta >> 14) & 1023).max()), int(((meta >> 5) & 511).max()))


def microbench_atomics(nwords: int, random: bool, op: int, nops: int, device: int = 0, stream=None) -> float:
    """64-bit op rate on distinct words (op 0 CAS, 1 add, 2 coherent load, 3 load+CAS)."""
    r = ctypes.c_double(0)
    _check(load().hirace_microbench_atomics(device, nwords, int(random), op, nops, ctypes.byref(r),
                                            _stream_handle(stream)), "hirace_microbench_atomics")
    return r.value


def microbench_grid_sync(iters: int = 200, mode: int = 0, device: int = 0, stream=None) -> float:
    """Microseconds per grid barrier of the persistent replay kernel (mode: see hirace.h)."""
    r = ctypes.c_double(0)
    _check(load().hirace_microbench_grid_sync(device, iters, mode, ctypes.byref(r), _stream_handle(stream)),
           "hirace_microbench_grid_sync")
    return r.value


def microbench_indexed(words_ptr: int, idx_ptr: int, n: int, op: int = 3, ctas_per_sm: int = 8, device: int = 0,
                       stream=None) -> float:
    """ms of one load (op 2) / load+CAS (op 3) pass over words[idx[i]] (diagnostics)."""
    ms = ctypes.c_double()
    _check(load().hirace_microbench_indexed(device, words_ptr, idx_ptr, n, op, ctas_per_sm, ctypes.byref(ms),
                                            _stream_handle(stream)), "microbench_indexed")
    return ms.value


def launch_count() -> int:
    v = ctypes.c_uint64(0)
    _check(load().hirace_launch_count(ctypes.byref(v)), "hirace_launch_count")
    return int(v.value)


def _stream_handle(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def events_to_device(events: np.ndarray, device="cuda"):
    """Copies an EVENT_DTYPE array into a CUDA uint8 tensor (16 bytes per event)."""
    import torch
    ev = np.ascontiguousarray(events)
    assert ev.dtype == EVENT_DTYPE
    return torch.from_numpy(ev.view(np.uint8).reshape(-1)).to(device)


class Checker:
    """One hirace_ctx: shadow (8 B per tracked 4-byte word, or 4 B with compact=(max_g, max_b,
    max_w): hirace_shadow_alloc_compact), FSM table, report buffer."""

    def __init__(self, grid_blocks: int, block_threads: int, warp_size: int = 32, global_words: int = 0,
                 smem_words: int = 0, report_capacity: int = 0, device: int = 0, policy: int = 0,
                 compact=None, granularity_log2: int = 2):
        """Extents are given in 4-byte words (global_words, smem_words per block); the shadow has
        one record per element of 1 << granularity_log2 bytes."""
        self.lib = load()
        cfg = Config(grid_blocks, block_threads, warp_size, 4 * smem_words, 4 * global_words, granularity_log2,
                     device, report_capacity)
        h = ctypes.c_void_p()
        if compact is None:
            _check(self.lib.hirace_shadow_alloc(ctypes.byref(cfg), ctypes.byref(h)), "hirace_shadow_alloc")
        else:
            lim = EpochLimits(*compact)
            _check(self.lib.hirace_shadow_alloc_compact(ctypes.byref(cfg), ctypes.byref(lim), ctypes.byref(h)),
                   "hirace_shadow_alloc_compact")
        self.h = h
        self.compact = None if compact is None else tuple(int(x) for x in compact)
        self.rec_bytes = 8 if compact is None else 4
        self.geometry = dict(grid_blocks=grid_blocks, block_threads=block_threads, warp_size=warp_size,
                             global_words=global_words, smem_words=smem_words)
        self.granularity_log2 = granularity_log2
        self.device = device
        self.policy = POLICY_STRICT
        if policy != POLICY_STRICT:
            self.set_policy(policy)

    @classmethod
    def for_trace(cls, trace, report_capacity: int = 0, device: int = 0, policy: int = 0, compact: bool = False,
                  history_slots: int = 0):
        """compact=True: 4-byte records sized by the trace's own epoch maxima.  A trace with a
        partial-mask warp-sync log (trace.warp_syncs) gets it set (hirace_set_warp_syncs)."""
        lim = trace_epoch_limits(trace.events) if compact else None
        c = cls(trace.grid_blocks, trace.block_threads, trace.warp_size, trace.global_words, trace.smem_words,
                report_capacity, device, policy, compact=lim,
                granularity_log2=getattr(trace, "granularity_log2", 2))
        syncs = getattr(trace, "warp_syncs", None)
        if syncs is not None and len(syncs):
            c.set_warp_syncs(syncs, history_slots or trace.info.get("history_slots", 0))
        return c

    def set_warp_syncs(self, syncs, history_slots: int = 0, stream=None):
        """hirace_set_warp_syncs: syncs = WARP_SYNC_DTYPE numpy array (copied to the device for
        the call) or a CUDA tensor of 16-byte records; empty / None removes the log."""
        import torch
        if syncs is None or len(syncs) == 0:
            _check(self.lib.hirace_set_warp_syncs(self.h, None, 0, 0, _stream_handle(stream)),
                   "hirace_set_warp_syncs")
            return
        if isinstance(syncs, np.ndarray):
            arr = np.ascontiguousarray(syncs)
            assert arr.dtype.itemsize == 16
            dev = torch.from_numpy(arr.view(np.uint8).reshape(-1)).to(f"cuda:{self.device}")
            n = arr.shape[0]
        else:
            dev = syncs
            n = dev.numel() * dev.element_size() // 16
        _check(self.lib.hirace_set_warp_syncs(self.h, ctypes.c_void_p(dev.data_ptr()), n, history_slots,
                                              _stream_handle(stream)), "hirace_set_warp_syncs")

    def set_filter(self, tid_mask: int = 0, tid_match: int = 0, spaces: int = 3, global_lo: int = 0,
                   global_hi: int = (1 << 64) - 1):
        """Selective tracking (include/hirace.h hirace_set_filter); defaults select everything."""
        _check(self.lib.hirace_set_filter(self.h, tid_mask, tid_match, spaces, global_lo, global_hi),
               "hirace_set_filter")

    def set_policy(self, policy: int, stream=None):
        """POLICY_STRICT or POLICY_RELAXED_READ_ATOMIC (include/hirace.h hirace_policy)."""
        _check(self.lib.hirace_set_policy(self.h, policy, _stream_handle(stream)), "hirace_set_policy")
        self.policy = policy

    @property
    def shadow_bytes(self) -> int:
        g = self.geometry
        per_word = 4 >> self.granularity_log2   # records per 4-byte word
        return self.rec_bytes * per_word * (g["global_words"] + g["grid_blocks"] * g["smem_words"])

    def close(self):
        if getattr(self, "h", None):
            self.lib.hirace_shadow_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset(self, stream=None):
        _check(self.lib.hirace_shadow_reset(self.h, _stream_handle(stream)), "hirace_shadow_reset")

    def barrier(self, scope=SCOPE_GRID, stream=None):
        _check(self.lib.hirace_barrier(self.h, scope, _stream_handle(stream)), "hirace_barrier")

    def advance_grid_epochs(self, count: int, stream=None):
        """hirace_advance_grid_epochs: count grid syncs the host did not see (k device grid
        syncs of a cooperative kernel + its boundary = k + 1)."""
        _check(self.lib.hirace_advance_grid_epochs(self.h, count, _stream_handle(stream)),
               "hirace_advance_grid_epochs")

    def replay(self, events_dev, n: int | None = None, stream=None):
        """events_dev: CUDA tensor holding 16-byte events (uint8 [16n] or int64 [n,2])."""
        nbytes = events_dev.numel() * events_dev.element_size()
        if n is None:
            n = nbytes // 16
        _check(self.lib.hirace_replay_trace(self.h, ctypes.c_void_p(events_dev.data_ptr()), n,
                                            _stream_handle(stream)), "hirace_replay_trace")

    def replay_ptr(self, ptr: int, n: int, stream=None):
        _check(self.lib.hirace_replay_trace(self.h, ctypes.c_void_p(ptr), n, _stream_handle(stream)),
               "hirace_replay_trace")

    def find_batches(self, events_dev, n: int | None = None, stream=None):
        """(offsets[nb+1], keys[nb]) of device events (batch discovery as the replay does it)."""
        if n is None:
            n = events_dev.numel() * events_dev.element_size() // 16
        cap = 64
        while True:
            offs = np.zeros(cap, np.uint32)
            keys = np.zeros(cap, np.uint32)
            nb = ctypes.c_uint64(0)
            _check(self.lib.hirace_find_batches(self.h, ctypes.c_void_p(events_dev.data_ptr()), n, offs.ctypes.data,
                                                keys.ctypes.data, cap, ctypes.byref(nb), _stream_handle(stream)),
                   "hirace_find_batches")
            if nb.value + 1 <= cap:
                return offs[: nb.value + 1].copy(), keys[: nb.value].copy()
            cap = int(nb.value) + 1

    def collect(self, cap: int | None = None, stream=None) -> np.ndarray:
        """Flagged words sorted by key (RACE_DTYPE).  Raises on a sticky error."""
        total = ctypes.c_uint64(0)
        cap = 1 << 16 if cap is None else cap
        while True:
            out = np.empty(max(cap, 1), RACE_DTYPE)
            st = self.lib.hirace_collect_races(self.h, out.ctypes.data, cap, ctypes.byref(total),
                                               _stream_handle(stream))
            _check(st, "hirace_collect_races")
            if total.value <= cap:
                return out[: total.value]
            cap = int(total.value)

    def collect_device(self, out_dev, cap: int, total_dev, stream=None):
        _check(self.lib.hirace_collect_races_device(self.h, ctypes.c_void_p(out_dev.data_ptr()), cap,
                                                    ctypes.c_void_p(total_dev.data_ptr()),
                                                    _stream_handle(stream)), "hirace_collect_races_device")

    def check_device(self, events_dev, out_dev, cap: int, total_dev, n: int | None = None, stream=None):
        """Fused replay + collect on device-resident events (one persistent kernel)."""
        if n is None:
            n = events_dev.numel() * events_dev.element_size() // 16
        _check(self.lib.hirace_check_trace_device(self.h, ctypes.c_void_p(events_dev.data_ptr()), n,
                                                  ctypes.c_void_p(out_dev.data_ptr()), cap,
                                                  ctypes.c_void_p(total_dev.data_ptr()), _stream_handle(stream)),
               "hirace_check_trace_device")

    def check_host(self, events: np.ndarray, cap: int | None = None, stream=None) -> np.ndarray:
        """End-to-end from HOST events: H2D (chunked, overlapped) + replay + collect + D2H."""
        ev = np.ascontiguousarray(events)
        cap = max(1 << 16, 0) if cap is None else cap
        total = ctypes.c_uint64(0)
        while True:
            out = np.empty(max(cap, 1), RACE_DTYPE)
            st = self.lib.hirace_check_trace_host(self.h, ev.ctypes.data, ev.shape[0], out.ctypes.data, cap,
                                                  ctypes.byref(total), _stream_handle(stream))
            _check(st, "hirace_check_trace_host")
            if total.value <= cap:
                return out[: total.value]
            cap = int(total.value)
            self.reset(stream)

    def check_host_ptr(self, ptr: int, n: int, out_ptr: int, cap: int, stream=None) -> int:
        total = ctypes.c_uint64(0)
        _check(self.lib.hirace_check_trace_host(self.h, ctypes.c_void_p(ptr), n, ctypes.c_void_p(out_ptr), cap,
                                                ctypes.byref(total), _stream_handle(stream)),
               "hirace_check_trace_host")
        return int(total.value)

    def set_kernel_timing(self, start=None, stop=None):
        """torch.cuda.Event pair (already recorded once) or None: times the replay kernel."""
        a = ctypes.c_void_p(start.cuda_event if start is not None else 0)
        b = ctypes.c_void_p(stop.cuda_event if stop is not None else 0)
        _check(self.lib.hirace_set_kernel_timing(self.h, a, b), "hirace_set_kernel_timing")

    def set_replay_mode(self, mode: int, window_log2: int = 0):
        """REPLAY_AUTO / REPLAY_BATCH / REPLAY_WINDOW (include/hirace.h); resets the shadow."""
        _check(self.lib.hirace_set_replay_mode(self.h, mode, window_log2), "hirace_set_replay_mode")

    def set_reset_mode(self, mode: int):
        """RESET_FULL / RESET_EPOCH (include/hirace.h hirace_set_reset_mode)."""
        _check(self.lib.hirace_set_reset_mode(self.h, mode), "hirace_set_reset_mode")

    @property
    def window_active(self) -> bool:
        v = ctypes.c_int(0)
        _check(self.lib.hirace_get_replay_mode(self.h, ctypes.byref(v)), "hirace_get_replay_mode")
        return bool(v.value)

    def launches(self) -> int:
        """Kernels the library has launched so far (process-wide, hirace_launch_count)."""
        return launch_count()

    def stats(self) -> dict:
        v = [ctypes.c_uint64(0) for _ in range(5)]
        _check(self.lib.hirace_get_stats(self.h, *[ctypes.byref(x) for x in v]), "hirace_get_stats")
        return dict(checked=v[0].value, cas_retries=v[1].value, cas_ops=v[2].value, no_write=v[3].value,
                    dropped_reports=v[4].value)

    def sync(self) -> int:
        return int(self.lib.hirace_sync(self.h))

    def dev_ctx(self, global_base: int = 0) -> DevCtx:
        d = DevCtx()
        _check(self.lib.hirace_get_dev_ctx(self.h, ctypes.c_void_p(global_base), ctypes.byref(d)),
               "hirace_get_dev_ctx")
        return d

    def inline_ws(self, history_slots: int = 0) -> WsCtx:
        """hirace_inline_warp_syncs: the sub-warp history handle for inline hooks with
        partial-mask syncs (hirace::ws::*)."""
        w = WsCtx()
        _check(self.lib.hirace_inline_warp_syncs(self.h, history_slots, ctypes.byref(w)), "hirace_inline_warp_syncs")
        return w

    def bucket(self, events_dev, n: int, nranks: int, my_rank: int, out_dev, stream=None) -> list[int]:
        counts = (ctypes.c_uint64 * nranks)()
        _check(self.lib.hirace_bucket_events(self.h, ctypes.c_void_p(events_dev.data_ptr()), n, nranks, my_rank,
                                             ctypes.c_void_p(out_dev.data_ptr()), counts, _stream_handle(stream)),
               "hirace_bucket_events")
        return [int(x) for x in counts]

    def bucket_wire(self, events_dev, offsets: np.ndarray, nranks: int, my_rank: int, stream=None):
        """8-byte wire records of all batches (include/hirace.h hirace_bucket_wire).
        offsets: batch start offsets (nb + 1, as from find_batches).  Returns (wire int64 CUDA
        tensor [m], counts uint64 [nb, nranks]); batch-major, owner-grouped."""
        import torch
        offs = np.ascontiguousarray(offsets, dtype=np.uint32)
        nb = max(len(offs) - 1, 0)
        counts = np.zeros((max(nb, 1), nranks), np.uint64)
        total = ctypes.c_uint64(0)
        n_ev = int(offs[-1]) if nb else 0
        cap = n_ev + n_ev // 8 + 64
        dev = events_dev.device
        while True:
            out = torch.empty(cap, dtype=torch.int64, device=dev)
            st = self.lib.hirace_bucket_wire(self.h, ctypes.c_void_p(events_dev.data_ptr() if nb else 0),
                                             offs.ctypes.data, nb, nranks, my_rank, ctypes.c_void_p(out.data_ptr()),
                                             cap, counts.ctypes.data, ctypes.byref(total), _stream_handle(stream))
            if st == -1 and total.value > cap:
                cap = int(total.value)
                continue
            _check(st, "hirace_bucket_wire")
            return out[: total.value], counts[:nb]

    def count_wire(self, events_dev, offsets: np.ndarray, nranks: int, my_rank: int, stream=None) -> np.ndarray:
        """Per-batch per-owner wire-record counts [nb, nranks] (hirace_count_wire)."""
        offs = np.ascontiguousarray(offsets, dtype=np.uint32)
        nb = max(len(offs) - 1, 0)
        counts = np.zeros((max(nb, 1), nranks), np.uint64)
        _check(self.lib.hirace_count_wire(self.h, ctypes.c_void_p(events_dev.data_ptr() if nb else 0),
                                          offs.ctypes.data, nb, nranks, my_rank, counts.ctypes.data,
                                          _stream_handle(stream)), "hirace_count_wire")
        return counts[:nb]

    def dispatch_wire(self, events_dev, offsets: np.ndarray, nranks: int, my_rank: int, peers, dst: np.ndarray,
                      stream=None):
        """Stores every batch's wire records into the owners' buffers (hirace_dispatch_wire).
        peers: nranks device addresses; dst: uint64 [nb, nranks] record offsets."""
        offs = np.ascontiguousarray(offsets, dtype=np.uint32)
        nb = max(len(offs) - 1, 0)
        if nb == 0:
            return
        tab = (ctypes.c_void_p * nranks)(*[ctypes.c_void_p(int(p)) for p in peers])
        d = np.ascontiguousarray(dst, dtype=np.uint64).reshape(-1)
        _check(self.lib.hirace_dispatch_wire(self.h, ctypes.c_void_p(events_dev.data_ptr() if nb else 0),
                                             offs.ctypes.data, nb, nranks, my_rank, tab,
                                             d.ctypes.data, _stream_handle(stream)),
               "hirace_dispatch_wire")

    def peer_release(self, peer_flags, j0: int, j1: int, stream=None):
        """hirace_peer_release: +1 on flags [j0, j1] of every owner (after this rank's dispatch)."""
        tab = (ctypes.c_void_p * len(peer_flags))(*[ctypes.c_void_p(int(p)) for p in peer_flags])
        _check(self.lib.hirace_peer_release(self.h, tab, len(peer_flags), j0, j1, _stream_handle(stream)),
               "hirace_peer_release")

    def peer_wait(self, flags_ptr: int, j: int, target: int, stream=None):
        """hirace_peer_wait: the stream waits until this rank's flag j >= target."""
        _check(self.lib.hirace_peer_wait(self.h, ctypes.c_void_p(flags_ptr), j, target, _stream_handle(stream)),
               "hirace_peer_wait")

    def replay_wire(self, wire_dev, n: int, batch_key: int, stream=None):
        """Replays n wire records of one batch (key g<<19 | b<<9 | w)."""
        _check(self.lib.hirace_replay_wire(self.h, ctypes.c_void_p(wire_dev.data_ptr() if n else 0), n, batch_key,
                                           _stream_handle(stream)), "hirace_replay_wire")

    def replay_wire_ptr(self, ptr: int, n: int, batch_key: int, stream=None):
        _check(self.lib.hirace_replay_wire(self.h, ctypes.c_void_p(ptr if n else 0), n, batch_key,
                                           _stream_handle(stream)), "hirace_replay_wire")


class PeerBuffer:
    """A receive buffer other processes can map (hirace_peer_buffer_alloc): `ptr` here, `handle`
    (64 bytes) for the peers, who map it with peer_open()."""

    def __init__(self, nbytes: int, device: int = 0):
        self.lib = load()
        p = ctypes.c_void_p()
        h = (ctypes.c_ubyte * 64)()
        _check(self.lib.hirace_peer_buffer_alloc(device, max(int(nbytes), 8), ctypes.byref(p), h),
               "hirace_peer_buffer_alloc")
        self.ptr, self.handle, self.nbytes, self.device = int(p.value), bytes(h), max(int(nbytes), 8), device

    def free(self):
        if self.ptr:
            self.lib.hirace_peer_buffer_free(ctypes.c_void_p(self.ptr))
            self.ptr = 0


def peer_open(handle: bytes, device: int = 0) -> int:
    p = ctypes.c_void_p()
    h = (ctypes.c_ubyte * 64).from_buffer_copy(handle)
    _check(load().hirace_peer_open(device, h, ctypes.byref(p)), "hirace_peer_open")
    return int(p.value)


def peer_close(ptr: int):
    _check(load().hirace_peer_close(ctypes.c_void_p(ptr)), "hirace_peer_close")


class ClusterChecker:
    """One hirace_cluster_ctx (include/hirace.h, cluster-level replay): the
    hierarchy thread < warp < block < cluster < grid, events with the cluster epoch and DSMEM
    target in their address bits (tracegen.pack_cluster_addr)."""

    def __init__(self, grid_blocks: int, block_threads: int, cluster_blocks: int, warp_size: int = 32,
                 global_words: int = 0, smem_words: int = 0, device: int = 0):
        self.lib = load()
        cfg = Config(grid_blocks, block_threads, warp_size, 4 * smem_words, 4 * global_words, 2, device, 0)
        h = ctypes.c_void_p()
        _check(self.lib.hirace_cluster_alloc(ctypes.byref(cfg), cluster_blocks, ctypes.byref(h)),
               "hirace_cluster_alloc")
        self.h = h
        self.device = device

    @classmethod
    def for_trace(cls, trace, device: int = 0):
        return cls(trace.grid_blocks, trace.block_threads, trace.cluster_blocks, trace.warp_size,
                   trace.global_words, trace.smem_words, device)

    def close(self):
        if getattr(self, "h", None):
            self.lib.hirace_cluster_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset(self, stream=None):
        _check(self.lib.hirace_cluster_reset(self.h, _stream_handle(stream)), "hirace_cluster_reset")

    def replay(self, events_dev, n: int | None = None, stream=None):
        if n is None:
            n = events_dev.numel() * events_dev.element_size() // 16
        _check(self.lib.hirace_cluster_replay(self.h, ctypes.c_void_p(events_dev.data_ptr()), n,
                                              _stream_handle(stream)), "hirace_cluster_replay")

    def collect(self, cap: int = 1 << 16) -> np.ndarray:
        total = ctypes.c_uint64(0)
        while True:
            out = np.empty(max(cap, 1), RACE_DTYPE)
            _check(self.lib.hirace_cluster_collect(self.h, out.ctypes.data, cap, ctypes.byref(total)),
                   "hirace_cluster_collect")
            if total.value <= cap:
                return out[: total.value]
            cap = int(total.value)

    def dev_ctx(self, global_base: int = 0) -> ClusterDevCtx:
        """hirace_cluster_get_dev_ctx: the device context of the cluster inline hooks."""
        d = ClusterDevCtx()
        _check(self.lib.hirace_cluster_get_dev_ctx(self.h, ctypes.c_void_p(global_base), ctypes.byref(d)),
               "hirace_cluster_get_dev_ctx")
        return d

    def stats(self):
        a, b = ctypes.c_uint64(0), ctypes.c_uint64(0)
        _check(self.lib.hirace_cluster_get_stats(self.h, ctypes.byref(a), ctypes.byref(b)), "hirace_cluster_get_stats")
        return int(a.value), int(b.value)


def races_to_dict(races: np.ndarray) -> dict:
    """{key: class} from collected records."""
    return {int(k): int(c) & 0xFF for k, c in zip(races["key"], races["cls_and_epoch"])}
