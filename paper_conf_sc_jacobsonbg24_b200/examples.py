"""ctypes binding of libhirace_examples.so: native CUDA programs (configs 1-4) that run either
uninstrumented or checked inline by the HiRace device hooks (paper_conf_sc_jacobsonbg24_b200/
examples/examples.cu).  Used for the inline-mode parity tests and the instrumented-slowdown
metric."""
from __future__ import annotations

import ctypes
import os

from .hirace import DevCtx, _stream_handle

_LIBDIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "lib")
_SO = {False: os.path.join(_LIBDIR, "libhirace_examples.so"),       # per-thread inline hooks
       True: os.path.join(_LIBDIR, "libhirace_examples_agg.so")}    # warp-aggregated (HIRACE_INLINE_AGGREGATE)
_libs = {}
_aggregate = False


def use_aggregated_hooks(flag: bool):
    """Selects the build of the native programs whose hooks aggregate same-element accesses of a
    warp (hirace::on_access_warp) instead of checking thread by thread."""
    global _aggregate
    _aggregate = bool(flag)


def load():
    if _aggregate not in _libs:
        so = _SO[_aggregate]
        if not os.path.exists(so):
            raise RuntimeError(f"{so} missing: python -m paper_conf_sc_jacobsonbg24_b200.build")
        lib = ctypes.CDLL(so)
        P, I, U = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint
        lib.hx_stencil.argtypes = [P, P, I, I, I, U, I, P]
        lib.hx_reduce.argtypes = [P, P, I, I, I, U, I, P]
        lib.hx_multiphase.argtypes = [P, P, I, I, I, I, I, P, U, I, P]
        lib.hx_bfs.argtypes = [P, P, P, P, I, I, U, ctypes.POINTER(I), P]
        lib.hx_cluster_halo.argtypes = [P, P, I, I, I, I, P]
        lib.hx_tiled.argtypes = [P, P, P, I, I, I, I, I, I, P]
        lib.hx_cluster_hist.argtypes = [P, P, I, I, I, I, I, I, P]
        for f in (lib.hx_stencil, lib.hx_reduce, lib.hx_multiphase, lib.hx_bfs, lib.hx_cluster_halo,
                  lib.hx_cluster_hist, lib.hx_tiled):
            f.restype = I
        _libs[_aggregate] = lib
    return _libs[_aggregate]


def _ctx(checker, base_ptr):
    if checker is None:
        return None, None
    d = checker.dev_ctx(base_ptr)
    return d, ctypes.byref(d)


def _ok(rc, name):
    if rc != 0:
        raise RuntimeError(f"{name}: CUDA error {rc}")


def stencil(checker, buf, n: int, steps: int, racy: bool, g0: int = 0, smem_shadow: bool = True, stream=None):
    """buf: CUDA float32 tensor of 2 n^2 (A then B; the tracked global base).  smem_shadow: keep the
    tile's shadow records in shared memory (else in the context's global shadow)."""
    d, p = _ctx(checker, buf.data_ptr())
    _ok(load().hx_stencil(p, ctypes.c_void_p(buf.data_ptr()), n, steps, int(racy), g0, int(smem_shadow),
                          _stream_handle(stream)), "hx_stencil")


def reduce(checker, out, block_threads: int, passes: int, racy: int, g0: int = 0, smem_shadow: bool = True,
           stream=None):
    """racy: 0 clean, 1 post-init barrier dropped, 2 first level barrier dropped."""
    d, p = _ctx(checker, out.data_ptr())
    _ok(load().hx_reduce(p, ctypes.c_void_p(out.data_ptr()), block_threads, passes, racy, g0, int(smem_shadow),
                         _stream_handle(stream)), "hx_reduce")


def multiphase(checker, AB, grid: int, phases: int, racy: int, bar, racy_phase_g: int = 31, racy_phase_b: int = 7,
               g0: int = 0, smem_shadow: bool = True, stream=None):
    """racy: 0 clean, 1 grid barrier after racy_phase_g demoted, 2 tile barrier of racy_phase_b dropped."""
    d, p = _ctx(checker, AB.data_ptr())
    bar.zero_()
    _ok(load().hx_multiphase(p, ctypes.c_void_p(AB.data_ptr()), grid, phases, racy, racy_phase_g, racy_phase_b,
                             ctypes.c_void_p(bar.data_ptr()), g0, int(smem_shadow), _stream_handle(stream)),
        "hx_multiphase")


def bfs(checker, base, nindex, nlist, dist, V: int, racy: bool, g0: int = 0, stream=None) -> int:
    """CSR arrays and dist are int32 CUDA tensors laid out contiguously from `base`."""
    d, p = _ctx(checker, base)
    levels = ctypes.c_int(0)
    _ok(load().hx_bfs(p, ctypes.c_void_p(nindex.data_ptr()), ctypes.c_void_p(nlist.data_ptr()),
                      ctypes.c_void_p(dist.data_ptr()), V, int(racy), g0, ctypes.byref(levels),
                      _stream_handle(stream)), "hx_bfs")
    return levels.value


__all__ = ["stencil", "reduce", "multiphase", "bfs", "load", "use_aggregated_hooks", "DevCtx"]


def cluster_halo(checker, out, nclusters: int, cluster_blocks: int, block_threads: int, sync: str, stream=None):
    """DSMEM halo (tracegen.cluster_halo) under the cluster inline hooks; checker: ClusterChecker
    or None (uninstrumented); out: CUDA float32 tensor of nclusters*cluster_blocks*block_threads.
    sync: "cluster", "block" or "none"."""
    d, p = _ctx(checker, out.data_ptr())
    mode = {"none": 0, "cluster": 1, "block": 2}[sync]
    _ok(load().hx_cluster_halo(p, ctypes.c_void_p(out.data_ptr()), nclusters, cluster_blocks, block_threads, mode,
                               _stream_handle(stream)), "hx_cluster_halo")


def cluster_hist(checker, out, nclusters: int, cluster_blocks: int, block_threads: int, bins: int,
                 block_scope: bool, drop: int | None, stream=None):
    """DSMEM histogram (tracegen.cluster_histogram); out: CUDA int32 tensor of nclusters*bins (the
    tracked global base)."""
    d, p = _ctx(checker, out.data_ptr())
    _ok(load().hx_cluster_hist(p, ctypes.c_void_p(out.data_ptr()), nclusters, cluster_blocks, block_threads, bins,
                               int(block_scope), int(drop or 0), _stream_handle(stream)), "hx_cluster_hist")


def tiled(checker, out, grid: int, block_threads: int, tile: int, rounds: int, racy: str | None,
          history_slots: int = 0, smem_tracking: bool = True, stream=None):
    """tiled_partition<tile> reduction (tracegen.tiled_reduce's program) under the inline hooks with
    partial-mask syncs; checker None = uninstrumented.  out: CUDA float32 tensor of
    grid*block_threads/tile (the tracked global base).  racy: None, "half_mask" or "pair".
    smem_tracking: the shared words' history slots and FSM records in shared memory (else in the
    context's global table and shadow)."""
    mode = {None: 0, "half_mask": 1, "pair": 2}[racy]
    if checker is None:
        p = w = None
    else:
        d = checker.dev_ctx(out.data_ptr())
        ws = checker.inline_ws(history_slots)
        p, w = ctypes.byref(d), ctypes.byref(ws)
    _ok(load().hx_tiled(p, w, ctypes.c_void_p(out.data_ptr()), grid, block_threads, tile, rounds, mode,
                        int(smem_tracking), _stream_handle(stream)), "hx_tiled")
