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
        owner = np.where(sh, self.r, sharded.owner_of_words(words, self.P)).astype(np.int64)
        c = np.uint64(sharded.CHUNK_LOG2)
        local = (((words >> c) // np.uint64(self.P)) << c) | (words & np.uint64((1 << sharded.CHUNK_LOG2) - 1))
        ev["addr"] = np.where(sh, ev["addr"], (local << np.uint64(2)) | (ev["addr"] & np.uint64(3)))
        order = np.argsort(owner, kind="stable")
        counts = np.bincount(owner, minlength=self.P).tolist()
        return _to_tensor(ev[order]), counts

    def replay(self, events):
        self.got.append(_to_events(events).copy())

    def collect(self):
        ev = np.concatenate(self.got) if self.got else np.empty(0, tg.EVENT_DTYPE)
        k, c, g = oracle.races(ev, self.t.block_threads, self.t.warp_size)
        out = np.empty(len(k), RACE_DTYPE)
        out["key"] = sharded.local_to_global_keys(k, self.r, self.P)
        out["cls_and_epoch"] = c.astype(np.uint32) | (g.astype(np.uint32) << 8)
        out["detect_tid"] = 0
        return out


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
    raise ValueError(name)


def _worker(rank, world, port, name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        t = _make(name)
        blk = t.events["tid"] // t.block_threads
        mine = t.events[(blk % world) == rank]          # this rank's blocks, batch order kept
        ops = CpuTestOps(t, world, rank)
        ex = sharded.HostExchange(None)
        n = sharded.run_sharded(_to_tensor(mine), ops, ex, None, dist)
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
