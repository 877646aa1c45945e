"""Address-sharded multi-GPU mode.

One process per GPU.  Each rank holds some of the trace's events (any partition works: by
block, by thread, by time slice).  Global words are owned by rank (word >> 14) mod P (64 KiB
chunks, so coalesced runs stay together); the shared-memory words of block k are owned by rank
k mod P, so all accesses to one shared word meet on one rank whichever rank traced them.
Batch by batch — in the global (g,b,w) order every rank agrees on — each rank

  1. buckets its events of the batch by owner on the GPU (`hirace_bucket_events`: a stable
     partition that also rewrites global addresses to the owner's shard-local word index),
  2. exchanges them with `all_to_all_single` (counts, then payload; NCCL over NVLink/NVSwitch
     with device tensors, or gloo through host staging for CPU tests / single-GPU runs),
  3. replays what it received on its own shard of the shadow (`hirace_replay_trace`).

Every word's events therefore reach exactly one rank, in batch order, so each rank's race set
is exact for the words it owns; the union (keys mapped back to global words) is the answer.
Inside a batch any order is a linear extension of happens-before, so the
received segments need no merge.

`run_sharded_p2p` fuses the bucketing with the exchange (the B200-native path): the dispatch
kernel stores every wire record straight into its owner's receive buffer, mapped from the
owner's GPU with CUDA IPC (NVLink/NVSwitch P2P stores; on one GPU, another process's buffer),
at an offset every rank derives from one all-gather of the count matrices — no staging copy
and no all_to_all (`PeerExchange`; include/hirace.h hirace_dispatch_wire).

`run_sharded_wire` is the NCCL pipeline: ONE bucketing launch sequence over
all local batches into 8-byte wire records (hirace_bucket_wire; g,b,w implied by the batch),
ONE all_to_all of the [ranks x batches] count matrix, then every batch's payload
all_to_all posted asynchronously up front while the replays (hirace_replay_wire) consume
them in batch order — the exchange of batch k+1 overlaps the replay of batch k, and the host
never waits on the exchange with NCCL (work.wait() orders the streams).  `run_sharded` (16-byte
events, per-batch synchronous exchange) remains for geometries beyond the wire format's
limits (> 2^30 threads or > 2^31 words per shard).

The orchestration is written against three small interfaces (`ops`: find_batches / bucket /
replay / collect, and an exchange) so the host logic can be tested on CPU with gloo and
world_size > 1; the GPU ops are the library's kernels, there is no CPU fallback for them.
"""
from __future__ import annotations

import numpy as np

CHUNK_LOG2 = 14


def _nvtx_push(msg: str):
    """NVTX range per batch (Nsight timelines; a no-op without CUDA)."""
    try:
        import torch
        if torch.cuda.is_available():
            torch.cuda.nvtx.range_push(msg)
    except Exception:
        pass


def _nvtx_pop():
    try:
        import torch
        if torch.cuda.is_available():
            torch.cuda.nvtx.range_pop()
    except Exception:
        pass
SHARED_BIT = np.uint64(1) << np.uint64(63)


def shard_words(global_words: int, nranks: int) -> int:
    """Shadow words a rank must track for its shard of `global_words` tracked global words."""
    chunk = 1 << CHUNK_LOG2
    nchunks = -(-global_words // chunk)
    return max(1, -(-nchunks // nranks)) * chunk


def owner_of_words(words: np.ndarray, nranks: int) -> np.ndarray:
    return (np.asarray(words, np.uint64) >> np.uint64(CHUNK_LOG2)) % np.uint64(nranks)


def owner_of_blocks(blocks: np.ndarray, nranks: int) -> np.ndarray:
    """Owner rank of the shared-memory words of each block (block mod P; owner_of in
    csrc/hirace_kernels.cu)."""
    return np.asarray(blocks, np.uint64) % np.uint64(nranks)


def local_to_global_keys(keys: np.ndarray, rank: int, nranks: int) -> np.ndarray:
    """Shard-local race keys -> global keys (shared keys are unchanged)."""
    keys = np.asarray(keys, dtype=np.uint64)
    sh = (keys & SHARED_BIT) != 0
    c = np.uint64(CHUNK_LOG2)
    mask = np.uint64((1 << CHUNK_LOG2) - 1)
    glob = (((keys >> c) * np.uint64(nranks) + np.uint64(rank)) << c) | (keys & mask)
    return np.where(sh, keys, glob)


# ---------------------------------------------------------------------------------------------
# exchanges
# ---------------------------------------------------------------------------------------------

class NcclExchange:
    """all_to_all_single on device tensors (NCCL over NVLink 5 / NVSwitch)."""

    def __init__(self, group, device):
        import torch
        import torch.distributed as dist
        self.dist, self.torch, self.group, self.device = dist, torch, group, device

    def counts(self, send_counts: list[int]) -> list[int]:
        t = self.torch.tensor(send_counts, dtype=self.torch.int64, device=self.device)
        r = self.torch.empty_like(t)
        self.dist.all_to_all_single(r, t, group=self.group)
        return [int(x) for x in r.cpu()]

    def payload(self, send, send_counts: list[int], recv_counts: list[int]):
        """send: int64 tensor [n, 2] (16-byte events) grouped by destination rank."""
        out = self.torch.empty((sum(recv_counts), 2), dtype=self.torch.int64, device=self.device)
        self.dist.all_to_all_single(out, send, output_split_sizes=recv_counts, input_split_sizes=send_counts,
                                    group=self.group)
        return out

    def counts_matrix(self, send):
        """send: int64 numpy [P, nb] (row = destination) -> recv [P, nb] (row = source)."""
        P, nb = send.shape
        t = self.torch.from_numpy(np.ascontiguousarray(send, dtype=np.int64).reshape(-1)).to(self.device)
        r = self.torch.empty_like(t)
        if nb:
            self.dist.all_to_all_single(r, t, group=self.group)
        return r.cpu().numpy().reshape(P, nb)

    def payload_async(self, send, send_counts: list[int], recv_counts: list[int]):
        """Posts one batch's exchange of 8-byte wire records (int64 [n]); returns a handle for
        finish().  NCCL: device tensors, the collective runs on NCCL's stream."""
        out = self.torch.empty(sum(recv_counts), dtype=self.torch.int64, device=self.device)
        work = self.dist.all_to_all_single(out, send, output_split_sizes=recv_counts, input_split_sizes=send_counts,
                                           group=self.group, async_op=True)
        return out, work

    def finish(self, handle):
        out, work = handle
        work.wait()  # NCCL: the current stream waits on the collective; the host does not block
        return out


class HostExchange(NcclExchange):
    """The same exchange through host memory (gloo): CPU tests and several ranks on one GPU."""

    def __init__(self, group, device=None):
        super().__init__(group, "cpu")
        self.out_device = device

    def payload(self, send, send_counts, recv_counts):
        cpu = send.cpu() if hasattr(send, "cpu") else send
        out = super().payload(cpu, send_counts, recv_counts)
        return out.to(self.out_device) if self.out_device is not None else out

    def payload_async(self, send, send_counts, recv_counts):
        cpu = send.cpu() if hasattr(send, "cpu") else send
        return super().payload_async(cpu, send_counts, recv_counts)

    def finish(self, handle):
        out = super().finish(handle)
        return out.to(self.out_device) if self.out_device is not None else out


class PeerExchange:
    """Receive buffers in peer memory for run_sharded_p2p: this rank's buffer is a
    hirace_peer_buffer_alloc allocation, the other ranks' are mapped with hirace_peer_open (CUDA
    IPC; P2P over NVLink between GPUs).  Host-side agreement (count matrices, handles, the
    barrier that orders the completion events) goes through the process group (gloo or NCCL).
    Reusing the buffers run after run is safe: run_sharded_p2p's count pass synchronises each
    rank's stream before the count all-gather, so every owner has finished replaying the
    previous run before any rank dispatches into its buffer again."""

    def __init__(self, group, dist, device: int = 0, per_batch: bool = True):
        """per_batch: run_sharded_p2p completes batch by batch with device flags (one GPU per
        rank); False: one fence after the whole dispatch (ranks time-sliced on one GPU, where a
        spinning wait only burns the other ranks' time slices)."""
        import torch
        self.per_batch = per_batch
        self.group, self.dist, self.device = group, dist, device
        self.buf = None
        self.opened = {}   # rank -> (handle, ptr)
        self.ptrs = None
        self.flags = None          # this rank's flag array (peer buffer, zeroed once)
        self.flag_ptrs = None      # every owner's flag array, mapped here
        self.flag_opened = {}
        self.uses = {}             # global batch index -> runs that used it
        # completion: an interprocess event per rank, recorded after its dispatch; the owners'
        # streams wait on the peers' events (GPU-side ordering, no stream drain)
        with torch.cuda.device(device):
            self.done = torch.cuda.Event(interprocess=True)
        self.peer_done = None

    def _gather(self, obj):
        objs = [None] * self.dist.get_world_size(self.group)
        self.dist.all_gather_object(objs, obj, group=self.group)
        return objs

    def all_counts(self, counts):
        """counts: int64 [nbg, P] of this rank -> [P_sender, nbg, P_owner] of all ranks: one
        all_gather of tensors (device tensors over NCCL; host tensors over gloo)."""
        import torch
        P = self.dist.get_world_size(self.group)
        c = torch.from_numpy(np.ascontiguousarray(counts, dtype=np.int64))
        if self.dist.get_backend(self.group) == "nccl":
            c = c.to(f"cuda:{self.device}")
        out = [torch.empty_like(c) for _ in range(P)]
        self.dist.all_gather(out, c, group=self.group)
        return np.stack([o.cpu().numpy() for o in out])

    def setup(self, need_bytes: int):
        """Every rank's buffer holds at least its own need; returns the peer table (device
        addresses in this process, index = owner rank)."""
        from .hirace import PeerBuffer, peer_close, peer_open
        me = self.dist.get_rank(self.group)
        grow = self.buf is None or self.buf.nbytes < need_bytes
        if any(self._gather(grow)):  # a remapped buffer: everyone drops stale mappings first
            for _, (_, ptr) in self.opened.items():
                peer_close(ptr)
            self.opened = {}
            self.dist.barrier(group=self.group)
            if grow:
                if self.buf is not None:
                    self.buf.free()
                self.buf = PeerBuffer(max(need_bytes, 1 << 20), self.device)
        handles = self._gather(self.buf.handle)
        ptrs = []
        for r, h in enumerate(handles):
            if r == me:
                ptrs.append(self.buf.ptr)
                continue
            if r not in self.opened or self.opened[r][0] != h:
                if r in self.opened:
                    peer_close(self.opened[r][1])
                self.opened[r] = (h, peer_open(h, self.device))
            ptrs.append(self.opened[r][1])
        self.ptrs = ptrs
        return ptrs

    def _setup_flags(self):
        from .hirace import MAX_BATCHES, PeerBuffer, peer_open
        if self.flag_ptrs is not None:
            return
        self.flags = PeerBuffer(4 * (MAX_BATCHES + 1), self.device)  # zero-initialised
        handles = self._gather(self.flags.handle)
        me = self.dist.get_rank(self.group)
        ptrs = []
        for r, h in enumerate(handles):
            if r == me:
                ptrs.append(self.flags.ptr)
            else:
                self.flag_opened[r] = peer_open(h, self.device)
                ptrs.append(self.flag_opened[r])
        self.flag_ptrs = ptrs
        self.dist.barrier(group=self.group)  # every owner's flags exist before any release

    def dispatch_batch(self, ops, events, offs, i, dst_row):
        """This rank's local batch i (or None: nothing to send for this global batch)."""
        self._setup_flags()
        if i is not None:
            ops.dispatch_wire(events, offs[i:i + 2], self.ptrs, dst_row.reshape(1, -1))

    def release(self, ops, j):
        ops.ctx.peer_release(self.flag_ptrs, j, j)

    def wait(self, ops, j):
        P = self.dist.get_world_size(self.group)
        ops.ctx.peer_wait(self.flags.ptr, j, (self.uses.get(j, 0) + 1) * P)

    def end_run(self, nbg):
        for j in range(nbg):
            self.uses[j] = self.uses.get(j, 0) + 1

    def fence(self):
        """Every rank's dispatch stores are complete and visible before any replay: each rank
        records its interprocess event after its dispatch, a host barrier orders those records
        before the waits, and this rank's stream waits on every peer's event."""
        import torch
        stream = torch.cuda.current_stream(self.device)
        if self.peer_done is None:
            handles = self._gather(self.done.ipc_handle())
            me = self.dist.get_rank(self.group)
            self.peer_done = [None if r == me else torch.cuda.Event.from_ipc_handle(self.device, h)
                              for r, h in enumerate(handles)]
        self.done.record(stream)
        self.dist.barrier(group=self.group)
        for ev in self.peer_done:
            if ev is not None:
                stream.wait_event(ev)

    def dispatch(self, ops, events, offs, dst_local):
        ops.dispatch_wire(events, offs, self.ptrs, dst_local)

    def received(self, ops, start: int, n: int, key: int):
        """Replays records [start, start + n) of this rank's buffer as batch `key`."""
        ops.replay_wire_ptr(self.buf.ptr + 8 * start, n, key)

    def close(self):
        from .hirace import peer_close
        for _, (_, ptr) in self.opened.items():
            peer_close(ptr)
        self.opened = {}
        for _, ptr in self.flag_opened.items():
            peer_close(ptr)
        self.flag_opened = {}
        self.dist.barrier(group=self.group)
        if self.buf is not None:
            self.buf.free()
            self.buf = None
        if self.flags is not None:
            self.flags.free()
            self.flags = None


# ---------------------------------------------------------------------------------------------
# GPU ops (the library's kernels)
# ---------------------------------------------------------------------------------------------

class GpuOps:
    """Per-rank shard context on one GPU; every step is a libhirace kernel."""

    def __init__(self, grid_blocks, block_threads, warp_size, global_words, smem_words, nranks, rank,
                 device=0, report_capacity=0):
        import torch

        from .hirace import Checker
        self.torch = torch
        self.nranks, self.rank, self.device = nranks, rank, device
        self.ctx = Checker(grid_blocks, block_threads, warp_size, shard_words(global_words, nranks), smem_words,
                           report_capacity, device)
        self.ctx.reset()

    def find_batches(self, events):
        """events: CUDA int64 tensor [n, 2] -> (offsets[nb+1], keys[nb]) numpy."""
        if events.shape[0] == 0:
            return np.zeros(1, np.uint32), np.zeros(0, np.uint32)
        return self.ctx.find_batches(events, events.shape[0])

    def bucket(self, events):
        out = self.torch.empty_like(events)
        counts = self.ctx.bucket(events, events.shape[0], self.nranks, self.rank, out) if events.shape[0] else \
            [0] * self.nranks
        return out, counts

    def replay(self, events):
        if events.shape[0]:
            self.ctx.replay(events, events.shape[0])

    def bucket_wire(self, events, offsets):
        """All local batches -> (wire int64 [m], counts [nb, P]) (hirace_bucket_wire)."""
        if len(offsets) <= 1:
            return self.torch.empty(0, dtype=self.torch.int64, device=events.device), np.zeros((0, self.nranks),
                                                                                                np.uint64)
        return self.ctx.bucket_wire(events, offsets, self.nranks, self.rank)

    def replay_wire(self, wire, key: int):
        if wire.shape[0]:
            self.ctx.replay_wire(wire, int(wire.shape[0]), key)

    def count_wire(self, events, offsets):
        """Per-batch per-owner wire-record counts [nb, P] (hirace_count_wire)."""
        if len(offsets) <= 1:
            return np.zeros((0, self.nranks), np.uint64)
        return self.ctx.count_wire(events, offsets, self.nranks, self.rank)

    def dispatch_wire(self, events, offsets, peers, dst):
        self.ctx.dispatch_wire(events, offsets, self.nranks, self.rank, peers, dst)

    def replay_wire_ptr(self, ptr: int, n: int, key: int):
        if n:
            self.ctx.replay_wire_ptr(ptr, n, key)

    def collect(self):
        r = self.ctx.collect()
        keys = local_to_global_keys(r["key"], self.rank, self.nranks)
        out = r.copy()
        out["key"] = keys
        return out


# ---------------------------------------------------------------------------------------------
# orchestration
# ---------------------------------------------------------------------------------------------

def all_batch_keys(local_keys: np.ndarray, group, dist) -> np.ndarray:
    """Union of every rank's batch keys, sorted: the global batch order all ranks follow."""
    objs = [None] * dist.get_world_size(group)
    dist.all_gather_object(objs, [int(k) for k in local_keys], group=group)
    return np.array(sorted(set().union(*[set(o) for o in objs])), dtype=np.uint32)


def run_sharded(local_events, ops, exchange, group, dist, on_batch=None):
    """Replays this rank's events (int64 tensor [n, 2], sorted by batch key) across all ranks.
    Returns the number of events this rank replayed (received).  `on_batch(key, n_recv)` is an
    optional hook for tests/telemetry."""
    offs, keys = ops.find_batches(local_events)
    order = all_batch_keys(keys, group, dist)
    where = {int(k): i for i, k in enumerate(keys)}
    received = 0
    for key in order:
        _nvtx_push(f"hirace batch key {int(key)}")
        i = where.get(int(key))
        part = local_events[int(offs[i]):int(offs[i + 1])] if i is not None else local_events[0:0]
        send, send_counts = ops.bucket(part)
        recv_counts = exchange.counts(send_counts)
        recv = exchange.payload(send, send_counts, recv_counts)
        ops.replay(recv)
        received += int(recv.shape[0])
        _nvtx_pop()
        if on_batch is not None:
            on_batch(int(key), int(recv.shape[0]))
    return received


def run_sharded_wire(local_events, ops, exchange, group, dist, on_batch=None):
    """The default sharded pipeline (module docstring): bucket all batches once, exchange the
    count matrix once, post every batch's payload exchange asynchronously, replay in the global
    batch order as each arrives.  Returns the number of wire records (word accesses) replayed
    on this rank."""
    offs, keys = ops.find_batches(local_events)
    order = all_batch_keys(keys, group, dist)
    P = dist.get_world_size(group)
    wire, counts = ops.bucket_wire(local_events, offs)
    counts = np.asarray(counts, dtype=np.int64).reshape(-1, P)
    row_start = np.concatenate(([0], np.cumsum(counts.sum(axis=1)))).astype(np.int64)
    where = {int(k): i for i, k in enumerate(keys)}
    nbg = len(order)
    send = np.zeros((P, nbg), np.int64)
    seg = np.zeros(nbg, np.int64)
    for j, k in enumerate(order):
        i = where.get(int(k))
        if i is not None:
            send[:, j] = counts[i]
            seg[j] = row_start[i]
    recv = exchange.counts_matrix(send)
    handles = []
    for j in range(nbg):  # all payload exchanges in flight; the replays below consume them in order
        n = int(send[:, j].sum())
        handles.append(exchange.payload_async(wire[int(seg[j]):int(seg[j]) + n], send[:, j].tolist(),
                                              recv[:, j].tolist()))
    received = 0
    for j, k in enumerate(order):
        _nvtx_push(f"hirace wire batch {j} (key {int(k)})")
        got = exchange.finish(handles[j])
        handles[j] = None
        ops.replay_wire(got, int(k))
        _nvtx_pop()
        received += int(got.shape[0])
        if on_batch is not None:
            on_batch(int(k), int(got.shape[0]))
    return received


def p2p_layout(all_counts: np.ndarray, me: int):
    """Receive-buffer layout of run_sharded_p2p from every rank's count matrix
    all_counts[s, j, r] (sender s, global batch j, owner r): owner r's buffer holds batch 0's
    records, then batch 1's, ...; inside a batch the senders in rank order.  Returns
    (dst [nbg, P]: where this rank's segment of batch j starts in owner r's buffer,
     base [nbg]: where batch j starts in this rank's own buffer, n_recv [nbg])."""
    per_batch = all_counts.sum(axis=0)                                   # [nbg, P]
    base_all = np.cumsum(per_batch, axis=0) - per_batch                  # exclusive over batches
    before = all_counts[:me].sum(axis=0) if me else np.zeros_like(per_batch)
    return base_all + before, base_all[:, me], per_batch[:, me]


def run_sharded_p2p(local_events, ops, exchange, group, dist, on_batch=None):
    """Fused bucket + exchange over peer memory (module docstring).  Returns the number of wire
    records (word accesses) replayed on this rank."""
    offs, keys = ops.find_batches(local_events)
    order = all_batch_keys(keys, group, dist)
    P = dist.get_world_size(group)
    me = dist.get_rank(group)
    counts = np.asarray(ops.count_wire(local_events, offs), dtype=np.int64).reshape(-1, P)
    gidx = np.array([int(np.searchsorted(order, k)) for k in keys], dtype=np.int64)
    nbg = len(order)
    mine = np.zeros((nbg, P), np.int64)
    if len(keys):
        mine[gidx] = counts
    dst, base, n_recv = p2p_layout(exchange.all_counts(mine), me)
    exchange.setup(8 * int(n_recv.sum()))
    received = 0
    if getattr(exchange, "per_batch", False):
        # per-batch completion: this rank dispatches global batch j (possibly nothing) and
        # releases it to every owner; its stream then waits until every sender released j and
        # replays it - batch j's replay overlaps the peers' dispatch of later batches
        local = {int(g): i for i, g in enumerate(gidx)}
        for j, k in enumerate(order):
            i = local.get(j)
            _nvtx_push(f"hirace p2p batch {j} (key {int(k)})")
            exchange.dispatch_batch(ops, local_events, offs, i, dst[j] if i is not None else None)
            exchange.release(ops, j)
            exchange.wait(ops, j)
            n = int(n_recv[j])
            exchange.received(ops, int(base[j]), n, int(k))
            _nvtx_pop()
            received += n
            if on_batch is not None:
                on_batch(int(k), n)
        exchange.end_run(nbg)
        return received
    exchange.dispatch(ops, local_events, offs, dst[gidx] if len(keys) else np.zeros((0, P), np.int64))
    exchange.fence()
    for j, k in enumerate(order):
        n = int(n_recv[j])
        exchange.received(ops, int(base[j]), n, int(k))
        received += n
        if on_batch is not None:
            on_batch(int(k), n)
    return received


def wire_fits(grid_threads: int, global_words: int, smem_words: int, nranks: int) -> bool:
    """Whether the 8-byte wire format covers this geometry (include/hirace.h limits)."""
    return grid_threads <= (1 << 30) and shard_words(global_words, nranks) <= (1 << 31) and smem_words <= (1 << 31)


def gather_races(races: np.ndarray, group, dist, dst: int = 0):
    """Union of the per-rank race sets (disjoint by owner), sorted by key, on rank `dst`."""
    objs = [None] * dist.get_world_size(group)
    dist.all_gather_object(objs, races.tobytes(), group=group)
    if dist.get_rank(group) != dst:
        return None
    allr = np.concatenate([np.frombuffer(b, dtype=races.dtype) for b in objs]) if objs else races[:0]
    return allr[np.argsort(allr["key"], kind="stable")]
