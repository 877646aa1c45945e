"""Address-sharded mode: the multi-process host logic on CPU with gloo.

Each rank holds the events of its own blocks; run_sharded exchanges them batch by batch with
all_to_all_single so that every global word's events land on its owner rank, with addresses
rewritten to the owner's shard-local words.  Here the per-rank ops are test doubles (numpy
partition + the oracle on what a rank received); the GPU ops are the library kernels
(tests/test_gpu_sharded.py).  The union of the per-rank race sets, mapped back to global keys,
must equal the oracle on the whole trace, bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import tracegen as tg
from paper_conf_sc_jacobsonbg24_b200 import sharded

RACE_DTYPE = np.dtype([("key", "<u8"), ("cls_and_epoch", "<u4"), ("detect_tid", "<u4")])


def _to_tensor(ev):
    return torch.from_numpy(np.ascontiguousarray(ev).view(np.int64).reshape(-1, 2).copy())


def _to_events(t):
    return t.numpy().reshape(-1).view(tg.EVENT_DTYPE) if t.numel() else np.empty(0, tg.EVENT_DTYPE)


class CpuTestOps:
    """Test double of sharded.GpuOps: numpy bucketing (same contract as hirace_bucket_events)
    and the oracle on the received events."""

    def __init__(self, trace, nranks, rank):
        self.t, self.P, self.r = trace, nranks, rank
        self.got = []

    def find_batches(self, events):
        ev = _to_events(events)
        if ev.shape[0] == 0:
            return np.zeros(1, np.uint32), np.zeros(0, np.uint32)
        k = ev["meta"] >> 5
        starts = np.flatnonzero(np.concatenate(([True], k[1:] != k[:-1])))
        return np.append(starts, ev.shape[0]).astype(np.uint32), k[starts].astype(np.uint32)

    def bucket(self, events):
        ev = _to_events(events).copy()
        sh = (ev["addr"] & tg.SHARED_BIT) != 0
        words = (ev["addr"] & ~tg.SHARED_BIT) >> np.uint64(2)
        owner = np.where(sh, sharded.owner_of_blocks(ev["tid"] // self.t.block_threads, self.P),
                         sharded.owner_of_words(words, self.P)).astype(np.int64)
        c = np.uint64(sharded.CHUNK_LOG2)
        local = (((words >> c) // np.uint64(self.P)) << c) | (words & np.uint64((1 << sharded.CHUNK_LOG2) - 1))
        ev["addr"] = np.where(sh, ev["addr"], (local << np.uint64(2)) | (ev["addr"] & np.uint64(3)))
        order = np.argsort(owner, kind="stable")
        counts = np.bincount(owner, minlength=self.P).tolist()
        return _to_tensor(ev[order]), counts

    def replay(self, events):
        self.got.append(_to_events(events).copy())

    def bucket_wire(self, events, offsets):
        return wire_bucket_np(_to_events(events), offsets, self.P, self.t.block_threads)

    def replay_wire(self, wire, key):
        self.got.append(wire_to_events(np.asarray(wire), key))

    def count_wire(self, events, offsets):
        return wire_bucket_np(_to_events(events), offsets, self.P, self.t.block_threads)[1]

    def collect(self):
        ev = np.concatenate(self.got) if self.got else np.empty(0, tg.EVENT_DTYPE)
        k, c, g = oracle.races(ev, self.t.block_threads, self.t.warp_size)
        out = np.empty(len(k), RACE_DTYPE)
        out["key"] = sharded.local_to_global_keys(k, self.r, self.P)
        out["cls_and_epoch"] = c.astype(np.uint32) | (g.astype(np.uint32) << 8)
        out["detect_tid"] = 0
        return out


class CpuPeerExchange:
    """Test double of sharded.PeerExchange: the receive buffer is a numpy array, and the
    "remote stores" of the dispatch travel as (offset, records) messages over gloo; the layout
    arithmetic (sharded.p2p_layout) and the orchestration are the product's."""

    def __init__(self, group, dist_mod):
        self.group, self.dist = group, dist_mod
        self.buf = None

    def _gather(self, obj):
        objs = [None] * self.dist.get_world_size(self.group)
        self.dist.all_gather_object(objs, obj, group=self.group)
        return objs

    def all_counts(self, counts):
        return np.stack([np.asarray(c, np.int64) for c in self._gather(np.asarray(counts, np.int64))])

    def setup(self, need_bytes):
        self.buf = np.full(need_bytes // 8, -1, np.int64)
        return None

    def dispatch(self, ops, events, offs, dst_local):
        wire, counts = ops.bucket_wire(events, offs)
        w = wire.numpy()
        flat = np.asarray(counts, np.int64).reshape(-1)
        pos = np.concatenate(([0], np.cumsum(flat)))
        P = self.dist.get_world_size(self.group)
        msgs = [[] for _ in range(P)]
        for i in range(len(flat)):            # segment (local batch i // P, owner i % P)
            b, r = divmod(i, P)
            if flat[i]:
                msgs[r].append((int(dst_local[b, r]), w[pos[i]:pos[i + 1]].copy()))
        me = self.dist.get_rank(self.group)
        for src, m in enumerate(self._gather(msgs)):
            for off, recs in m[me]:
                assert (self.buf[off:off + len(recs)] == -1).all()   # disjoint segments
                self.buf[off:off + len(recs)] = recs

    def fence(self):
        self.dist.barrier(group=self.group)
        assert (self.buf != -1).all()                                # every slot written once

    def received(self, ops, start, n, key):
        if n:
            ops.replay_wire(torch.from_numpy(self.buf[start:start + n]), key)


class CpuPeerExchangePerBatch(CpuPeerExchange):
    """The per-batch completion protocol of sharded.PeerExchange (hirace_peer_release /
    hirace_peer_wait): every rank dispatches global batch j (possibly nothing), releases it,
    and its replay of j waits until every sender's records of j are in its buffer."""

    per_batch = True

    def setup(self, need_bytes):
        super().setup(need_bytes)
        self.released = []

    def dispatch_batch(self, ops, events, offs, i, dst_row):
        P = self.dist.get_world_size(self.group)
        msgs = [[] for _ in range(P)]
        if i is not None:
            wire, counts = ops.bucket_wire(events, offs[i:i + 2])
            w = wire.numpy()
            flat = np.asarray(counts, np.int64).reshape(-1)
            pos = np.concatenate(([0], np.cumsum(flat)))
            for r in range(P):
                if flat[r]:
                    msgs[r].append((int(dst_row[r]), w[pos[r]:pos[r + 1]].copy()))
        me = self.dist.get_rank(self.group)
        self.pending = [m[me] for m in self._gather(msgs)]

    def release(self, ops, j):
        for m in self.pending:                   # the peers' stores of batch j land here
            for off, recs in m:
                assert (self.buf[off:off + len(recs)] == -1).all()
                self.buf[off:off + len(recs)] = recs
        self.released.append(j)

    def wait(self, ops, j):
        assert self.released and self.released[-1] == j

    def received(self, ops, start, n, key):
        assert (self.buf[start:start + n] != -1).all()   # batch j complete before its replay
        super().received(ops, start, n, key)

    def end_run(self, nbg):
        assert self.released == list(range(nbg))
        assert (self.buf != -1).all()


def wire_bucket_np(ev, offsets, P, bt):
    """Reference of the hirace_bucket_wire contract (include/hirace.h): per batch, one record per
    covered word, routed to its word's owner, shard-local words, owner-grouped (stable here;
    the kernel's order inside a (batch, owner) segment is unspecified)."""
    nb = len(offsets) - 1
    counts = np.zeros((max(nb, 0), P), np.uint64)
    parts = []
    for b in range(nb):
        e = ev[int(offsets[b]):int(offsets[b + 1])]
        szl = (e["meta"] >> 2) & 7
        nw = np.where(szl <= 2, 1, 1 << np.maximum(szl.astype(np.int64) - 2, 0)).astype(np.int64)
        rep = np.repeat(e, nw)
        k = np.arange(rep.shape[0]) - np.repeat(np.cumsum(nw) - nw, nw)
        sh = (rep["addr"] & tg.SHARED_BIT) != 0
        word = ((rep["addr"] & ~tg.SHARED_BIT) >> np.uint64(2)) + k.astype(np.uint64)
        c = np.uint64(sharded.CHUNK_LOG2)
        owner = np.where(sh, sharded.owner_of_blocks(rep["tid"] // bt, P), (word >> c) % np.uint64(P)).astype(np.int64)
        local = np.where(sh, word, (((word >> c) // np.uint64(P)) << c) | (word & np.uint64((1 << 14) - 1)))
        w = (local | (sh.astype(np.uint64) << np.uint64(31)) | (rep["tid"].astype(np.uint64) << np.uint64(32)) |
             ((rep["meta"] & 3).astype(np.uint64) << np.uint64(62)))
        order = np.argsort(owner, kind="stable")
        parts.append(w[order])
        counts[b] = np.bincount(owner, minlength=P)
    wire = np.concatenate(parts) if parts else np.zeros(0, np.uint64)
    return torch.from_numpy(wire.view(np.int64).copy()), counts


def wire_to_events(wire, key):
    """Wire records of batch `key` back to 4-byte events (for the oracle)."""
    w = np.asarray(wire).view(np.uint64)
    ev = np.empty(w.shape[0], tg.EVENT_DTYPE)
    word = w & np.uint64(0x7FFFFFFF)
    sh = (w >> np.uint64(31)) & np.uint64(1)
    ev["addr"] = (word << np.uint64(2)) | (sh << np.uint64(63))
    ev["tid"] = (w >> np.uint64(32)) & np.uint64(0x3FFFFFFF)
    g, b, ww = key >> 19, (key >> 9) & 1023, key & 511
    ev["meta"] = tg.pack_meta((w >> np.uint64(62)).astype(np.uint32), 2, ww, b, g)
    return ev


def _make(name):
    if name == "cfg2":
        return tg.cfg2(True, n=128, steps=3)
    if name == "cfg3":
        return tg.cfg3("bfs", True, scale=11, edge_factor=8)
    if name == "cfg4":
        return tg.cfg4("G", 6, 64, 34)
    if name == "wide":
        # global words spread over many 64 KiB chunks, all kinds, several epochs
        rng = np.random.default_rng(5)
        n = 30000
        ev = np.empty(n, dtype=tg.EVENT_DTYPE)
        ev["tid"] = rng.integers(0, 8 * 64, n)
        ev["addr"] = rng.integers(0, 1 << 20, n).astype(np.uint64) << np.uint64(2)  # 64 owner chunks
        ev["meta"] = tg.pack_meta(rng.choice(4, n, p=[.5, .3, .1, .1]), 2, 0, rng.integers(0, 3, n),
                                  rng.integers(0, 3, n))
        return tg.Trace("wide", tg.sort_by_batch(ev), 8, 64, 32, 1 << 20, 0)
    if name == "multi":
        # 8- and 16-byte accesses, many straddling a 64 KiB owner chunk, plus shared words
        rng = np.random.default_rng(11)
        n = 20000
        ev = np.empty(n, dtype=tg.EVENT_DTYPE)
        ev["tid"] = rng.integers(0, 8 * 64, n)
        chunk_edge = (rng.integers(1, 16, n).astype(np.uint64) << np.uint64(14)) - rng.integers(0, 3, n).astype(
            np.uint64)
        words = np.where(rng.random(n) < 0.5, chunk_edge, rng.integers(0, 1 << 18, n).astype(np.uint64))
        sh = rng.random(n) < 0.15
        szl = rng.choice([2, 3, 4], n, p=[.4, .3, .3])
        words = np.where(sh, rng.integers(0, 60, n).astype(np.uint64), words)
        ev["addr"] = (words << np.uint64(2)) | (sh.astype(np.uint64) << np.uint64(63))
        ev["meta"] = tg.pack_meta(rng.choice(4, n, p=[.5, .3, .1, .1]), szl, 0, rng.integers(0, 2, n),
                                  rng.integers(0, 3, n))
        return tg.Trace("multi", tg.sort_by_batch(ev), 8, 64, 32, 1 << 18, 64)
    raise ValueError(name)


def _words(t):
    szl = (t.events["meta"] >> 2) & 7
    return int(np.where(szl <= 2, 1, 1 << np.maximum(szl.astype(np.int64) - 2, 0)).sum())


def _worker(rank, world, port, name, q, wire=False, split="block"):
    """wire: False = 16-byte events, True = 8-byte wire + all_to_all, "p2p" = peer dispatch.
    split: which events a rank holds: its blocks, or its threads (a block's shared accesses then
    come from several ranks and must meet on the block's owner)."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        t = _make(name)
        blk = t.events["tid"] // t.block_threads
        part = blk if split == "block" else t.events["tid"]
        mine = t.events[(part % world) == rank]         # this rank's blocks / threads, batch order kept
        ops = CpuTestOps(t, world, rank)
        if wire == "p2p":
            ex, run = CpuPeerExchange(None, dist), sharded.run_sharded_p2p
        elif wire == "p2p_batch":
            ex, run = CpuPeerExchangePerBatch(None, dist), sharded.run_sharded_p2p
        else:
            ex = sharded.HostExchange(None)
            run = sharded.run_sharded_wire if wire else sharded.run_sharded
        n = run(_to_tensor(mine), ops, ex, None, dist)
        races = sharded.gather_races(ops.collect(), None, dist)
        tot = torch.tensor([n])
        dist.all_reduce(tot)
        if rank == 0:
            q.put((int(tot.item()), races["key"].tolist(), (races["cls_and_epoch"] & 0xFF).tolist()))
    finally:
        dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world,name", [(2, "cfg2"), (2, "cfg4"), (3, "cfg3"), (3, "wide")])
def test_sharded_exchange_reproduces_the_oracle(world, name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == t.n                   # every event replayed exactly once
    assert keys == [int(x) for x in k]    # same words
    assert cls == [int(x) for x in c]     # same classes


@pytest.mark.parametrize("world,name,split", [(2, "cfg2", "block"), (3, "cfg4", "block"), (2, "cfg3", "block"),
                                              (3, "wide", "block"), (2, "multi", "block"), (4, "multi", "block"),
                                              (2, "cfg2", "thread"), (3, "cfg4", "thread")])
def test_sharded_wire_pipeline_reproduces_the_oracle(world, name, split):
    """8-byte wire records, one count-matrix exchange, async per-batch payloads.
    split="thread": every block's events are spread over the ranks; its shared words still meet
    on the block's owner rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q, True, split)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == _words(t)              # every covered word replayed exactly once
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]
    assert len(k) > 0


@pytest.mark.parametrize("mode", ["p2p", "p2p_batch"])
@pytest.mark.parametrize("world,name", [(2, "cfg2"), (3, "cfg4"), (2, "cfg3"), (3, "wide"), (4, "multi")])
def test_sharded_p2p_pipeline_reproduces_the_oracle(world, name, mode):
    """Peer-memory dispatch (run_sharded_p2p): count matrices all-gathered once, every rank
    stores its records at sharded.p2p_layout offsets of the owners' buffers (disjoint, every
    slot written), owners replay batch by batch."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q, mode)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == _words(t)
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]


def test_p2p_layout_closed_form():
    # 3 ranks, 2 batches: owner r's buffer = batch-major, sender-minor segments
    a = np.arange(18).reshape(3, 2, 3) % 5
    for me in range(3):
        dst, base, n = sharded.p2p_layout(a, me)
        for j in range(2):
            for r in range(3):
                want = sum(a[s, jj, r] for s in range(3) for jj in range(j)) + sum(a[s, j, r] for s in range(me))
                assert dst[j, r] == want
            assert base[j] == sum(a[s, jj, me] for s in range(3) for jj in range(j))
            assert n[j] == a[:, j, me].sum()


def test_wire_reference_roundtrip():
    """The wire encoding is lossless for in-range records: decode(encode(e)) gives the event's
    shard-local word, tid, kind and the batch's epochs."""
    t = _make("multi")
    offs = np.flatnonzero(np.concatenate(([True], np.diff(t.events["meta"] >> 5) != 0)))
    offs = np.append(offs, t.n)
    wire, counts = wire_bucket_np(t.events, offs, 1, t.block_threads)
    assert int(counts.sum()) == _words(t) == wire.shape[0]
    keys = t.events["meta"][offs[:-1]] >> 5
    back = np.concatenate([wire_to_events(wire.numpy()[int(s):int(s + n)], int(k)) for s, n, k in
                           zip(np.concatenate(([0], np.cumsum(counts.sum(1))[:-1])), counts.sum(1), keys)])
    k1, c1, _ = oracle.races(back, t.block_threads, t.warp_size)
    k0, c0, _ = oracle.races_of(t)
    assert k1.tolist() == k0.tolist() and c1.tolist() == c0.tolist()


def test_shard_geometry():
    assert sharded.shard_words(1 << 20, 3) == 22 * (1 << 14)
    w = np.array([0, 1 << 14, 5 << 14 | 7, (1 << 32) - 1], dtype=np.uint64)
    for P in (1, 2, 3, 8):
        own = sharded.owner_of_words(w, P)
        local = (((w >> np.uint64(14)) // np.uint64(P)) << np.uint64(14)) | (w & np.uint64(16383))
        back = np.concatenate([sharded.local_to_global_keys(local[i:i + 1], int(own[i]), P) for i in range(len(w))])
        assert back.tolist() == w.tolist()
    shared = np.array([np.uint64(1) << np.uint64(63) | np.uint64(5 << 32 | 9)], dtype=np.uint64)
    assert sharded.local_to_global_keys(shared, 1, 4).tolist() == shared.tolist()
