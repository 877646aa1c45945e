"""B200-native HiRace hot path: per-access shadow-state update for GPU data-race checking.

The compute path is libhirace.so (sm_100a CUDA kernels behind the C-ABI in include/hirace.h);
`hirace` is its ctypes binding, `sharded` the address-sharded multi-GPU driver.
"""
from .hirace import (ATOMIC_BLOCK, ATOMIC_GRID, EVENT_DTYPE, RACE_DTYPE, READ, WRITE, Checker, ClusterChecker,  # noqa: F401
                     HiraceError, POLICY_RELAXED_READ_ATOMIC, POLICY_STRICT, REPLAY_AUTO, REPLAY_BATCH,
                     REPLAY_WINDOW, RESET_EPOCH, RESET_FULL, events_to_device, launch_count, fsm_step,
                     fsm_cluster_class, fsm_step_cluster, fsm_step_compact, fsm_table,
                     fsm_table_cluster, load, races_to_dict, trace_epoch_limits)

__all__ = ["Checker", "ClusterChecker", "HiraceError", "EVENT_DTYPE", "RACE_DTYPE", "events_to_device", "fsm_step", "fsm_step_compact",
           "fsm_table", "fsm_table_cluster", "fsm_step_cluster", "fsm_cluster_class", "trace_epoch_limits",
           "load", "races_to_dict", "READ", "WRITE", "ATOMIC_BLOCK", "ATOMIC_GRID",
           "POLICY_STRICT", "POLICY_RELAXED_READ_ATOMIC", "REPLAY_AUTO", "REPLAY_BATCH", "REPLAY_WINDOW",
           "RESET_FULL", "RESET_EPOCH", "launch_count"]
