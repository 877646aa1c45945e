"""ORACLE: plain CPU implementations of what the HiRace hot path must compute.

TEST INFRASTRUCTURE ONLY.  Only `tests/`, `__graft_entry__.smoke()` and `bench.py`
(`cpu_baseline` leg and `--impl reference`) may import, call, link or execute anything under
`oracle/`.  The product package (`paper_conf_sc_jacobsonbg24_b200/`) never imports it and the
two share no code.

  oracle_d.c  Oracle-D: the race definition, sort + per-level scan, C.
  oracle_par.c  all-core driver: splits the element-level accesses by key into shards and runs
              oracle_d.c's oracle_races_gran on each (a key's verdict depends only on its own
              accesses); pinned against the single-thread function.
  brute.py    literal O(n^2) pairwise enumeration of C1, for tiny traces.
  races_cluster / brute.races_cluster: the definition with a thread-block-cluster level
              (reading R16); class CLUSTER = 4.
  races_masked / brute.races_masked: the definition with partial-mask __syncwarp(mask)
              (reading R20; C1.1''/C1.2'' in
              oracle_d.c): the oracle by forward knowledge propagation along the sync log, the
              brute force by per-lane vector clocks.

Pins (tests/test_oracle_pins.py): brute force on random tiny traces, the paper's listings
(closed forms, tests/golden/), configs 1/2/4 closed forms, read-only invariants.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_d.c")
_SRCS = [_SRC, os.path.join(_HERE, "oracle_par.c")]
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

WARP, BLOCK, GRID, CLUSTER = 1, 2, 3, 4
CLASS_NAMES = {1: "WARP", 2: "BLOCK", 3: "GRID", 4: "CLUSTER"}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or any(os.path.getmtime(_SO) < os.path.getmtime(p) for p in _SRCS):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread", *_SRCS, "-o", _SO + ".tmp"])
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.oracle_races_policy.restype = ctypes.c_int64
        lib.oracle_races_policy.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                            ctypes.c_int]
        lib.oracle_races_gran.restype = ctypes.c_int64
        lib.oracle_races_gran.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                          ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                          ctypes.c_int, ctypes.c_uint32]
        lib.oracle_races_par.restype = ctypes.c_int64
        lib.oracle_races_par.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                         ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                         ctypes.c_int, ctypes.c_uint32, ctypes.c_int, ctypes.c_int]
        lib.oracle_races_masked.restype = ctypes.c_int64
        lib.oracle_races_masked.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                            ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int]
        lib.oracle_races_cluster.restype = ctypes.c_int64
        lib.oracle_races_cluster.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                             ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                             ctypes.c_uint64]
        _lib = lib
    return _lib


def races(events: np.ndarray, block_threads: int, warp_size: int, policy: int = 0, granularity_log2: int = 2):
    """Oracle-D.  Returns (keys u64[], cls u8[], gstar u8[]) sorted by key.  policy 0 = strict
    conflict rule (C1.3), 1 = relaxed read-vs-atomic (R2b).  granularity_log2: the
    tracked element is 1 << granularity_log2 bytes (2 = 4-byte words; keys are element indices)."""
    lib = _load()
    ev = np.ascontiguousarray(events)
    n = int(ev.shape[0])
    cap = max(1024, n)
    while True:
        keys = np.empty(cap, np.uint64)
        cls = np.empty(cap, np.uint8)
        gs = np.empty(cap, np.uint8)
        r = lib.oracle_races_gran(ev.ctypes.data if n else None, n, block_threads, warp_size,
                                  keys.ctypes.data, cls.ctypes.data, gs.ctypes.data, cap, policy, granularity_log2)
        if r < 0:
            raise RuntimeError(f"oracle_races failed ({r})")
        if r <= cap:
            return keys[:r], cls[:r], gs[:r]
        cap = int(r)


def hardware_threads() -> int:
    """std::thread::hardware_concurrency() equivalent: the CPUs this process may run on."""
    try:
        return len(os.sched_getaffinity(0))
    except (AttributeError, OSError):
        return os.cpu_count() or 1


def races_parallel(events: np.ndarray, block_threads: int, warp_size: int, policy: int = 0,
                   granularity_log2: int = 2, threads: int | None = None, shards: int | None = None):
    """Oracle-D over address shards on `threads` cores (default: all).  Same result as races()
    (oracle_par.c; pinned by tests/test_oracle_par.py)."""
    lib = _load()
    ev = np.ascontiguousarray(events)
    n = int(ev.shape[0])
    t = int(threads or hardware_threads())
    s = int(shards or max(4 * t, min(4096, n // (1 << 22) + 1)))
    cap = 1 << 16
    while True:
        keys = np.empty(cap, np.uint64)
        cls = np.empty(cap, np.uint8)
        gs = np.empty(cap, np.uint8)
        r = lib.oracle_races_par(ev.ctypes.data if n else None, n, block_threads, warp_size, keys.ctypes.data,
                                 cls.ctypes.data, gs.ctypes.data, cap, policy, granularity_log2, t, s)
        if r < 0:
            raise RuntimeError(f"oracle_races_par failed ({r})")
        if r <= cap:
            return keys[:r], cls[:r], gs[:r]
        cap = int(r)


def races_of(trace, policy: int = 0):
    return races(trace.events, trace.block_threads, trace.warp_size, policy, getattr(trace, "granularity_log2", 2))


def races_dict(trace, policy: int = 0) -> dict:
    k, c, _ = races_of(trace, policy)
    return {int(a): int(b) for a, b in zip(k, c)}


def races_cluster(events: np.ndarray, block_threads: int, warp_size: int, cluster_blocks: int):
    """Oracle-D with the cluster level (C1.1'-C1.6' in oracle_d.c; strict conflict rule, 4-byte
    words).  Returns (keys u64[], cls u8[], gstar u8[]) sorted by key; cls 4 = CLUSTER."""
    lib = _load()
    ev = np.ascontiguousarray(events)
    n = int(ev.shape[0])
    cap = max(1024, n)
    while True:
        keys = np.empty(cap, np.uint64)
        cls = np.empty(cap, np.uint8)
        gs = np.empty(cap, np.uint8)
        r = lib.oracle_races_cluster(ev.ctypes.data if n else None, n, block_threads, warp_size, cluster_blocks,
                                     keys.ctypes.data, cls.ctypes.data, gs.ctypes.data, cap)
        if r < 0:
            raise RuntimeError(f"oracle_races_cluster failed ({r})")
        if r <= cap:
            return keys[:r], cls[:r], gs[:r]
        cap = int(r)


def races_cluster_dict(trace) -> dict:
    k, c, _ = races_cluster(trace.events, trace.block_threads, trace.warp_size, trace.cluster_blocks)
    return {int(a): int(b) for a, b in zip(k, c)}


class BadSyncLog(ValueError):
    """oracle_races_masked returned -4: malformed partial-sync log, or an access after a partial
    sync its lane is not in."""


def races_masked(events: np.ndarray, block_threads: int, warp_size: int, syncs, policy: int = 0):
    """Oracle-D with partial-mask warp syncs (C1.1''/C1.2'' in oracle_d.c; 4-byte words).
    syncs: tracegen.SYNC_DTYPE log (None/empty = none).  Returns (keys, cls, gstar) by key."""
    lib = _load()
    ev = np.ascontiguousarray(events)
    n = int(ev.shape[0])
    sy = np.ascontiguousarray(syncs) if syncs is not None else None
    ns = 0 if sy is None else int(sy.shape[0])
    cap = max(1024, n)
    while True:
        keys = np.empty(cap, np.uint64)
        cls = np.empty(cap, np.uint8)
        gs = np.empty(cap, np.uint8)
        r = lib.oracle_races_masked(ev.ctypes.data if n else None, n, block_threads, warp_size,
                                    sy.ctypes.data if ns else None, ns, keys.ctypes.data, cls.ctypes.data,
                                    gs.ctypes.data, cap, policy)
        if r == -4:
            raise BadSyncLog("malformed partial-sync log or an access outside its sync's mask")
        if r < 0:
            raise RuntimeError(f"oracle_races_masked failed ({r})")
        if r <= cap:
            return keys[:r], cls[:r], gs[:r]
        cap = int(r)


def races_masked_dict(trace, policy: int = 0) -> dict:
    k, c, _ = races_masked(trace.events, trace.block_threads, trace.warp_size, trace.warp_syncs, policy)
    return {int(a): int(b) for a, b in zip(k, c)}
