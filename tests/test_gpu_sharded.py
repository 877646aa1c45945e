"""Address-sharded mode on the GPU: the bucket kernel's contract, and run_sharded with the real
kernels (several ranks sharing the one GPU through gloo host staging; one rank through NCCL)."""
import os
import socket

import numpy as np
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
from paper_conf_sc_jacobsonbg24_b200 import sharded  # noqa: E402
from tests.test_sharded import CpuTestOps, _make, _to_events, _to_tensor, _words, wire_bucket_np  # noqa: E402


@pytest.mark.parametrize("nranks,rank", [(1, 0), (2, 1), (3, 2), (8, 5), (32, 17)])
def test_bucket_kernel_matches_contract(nranks, rank):
    rng = np.random.default_rng(nranks * 100 + rank)
    n = 100_003
    ev = np.empty(n, dtype=tg.EVENT_DTYPE)
    ev["tid"] = rng.integers(0, 1 << 20, n)
    words = rng.integers(0, 1 << 30, n).astype(np.uint64)
    sh = rng.random(n) < 0.2
    ev["addr"] = (words << np.uint64(2)) | rng.integers(0, 4, n).astype(np.uint64)
    ev["addr"][sh] = (ev["addr"][sh] & np.uint64(0xFFFF)) | tg.SHARED_BIT
    ev["meta"] = tg.pack_meta(rng.choice(4, n), 2, 0, 0, 0)
    c = hr.Checker(4096, 256, 32, 1 << 20, 64)
    d = torch.from_numpy(ev.view(np.int64).reshape(-1, 2).copy()).cuda()
    out = torch.empty_like(d)
    counts = c.bucket(d, n, nranks, rank, out)
    geom = tg.Trace("bucket", ev, 4096, 256, 32, 1 << 20, 64)
    want_t, want_counts = CpuTestOps(geom, nranks, rank).bucket(torch.from_numpy(ev.view(np.int64).reshape(-1, 2)))
    assert counts == want_counts
    assert np.array_equal(out.cpu().numpy(), want_t.numpy())
    c.close()


@pytest.mark.parametrize("nranks,rank", [(1, 0), (2, 1), (3, 0), (8, 5), (32, 31)])
def test_bucket_wire_kernel_matches_contract(nranks, rank):
    t = _make("multi")
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    d = _to_tensor(t.events).cuda()
    offs, keys = c.find_batches(d)
    wire, counts = c.bucket_wire(d, offs, nranks, rank)
    want, want_counts = wire_bucket_np(t.events, offs, nranks, t.block_threads)
    assert np.array_equal(counts, want_counts)
    got = wire.cpu().numpy()
    ref = want.numpy()
    assert got.shape == ref.shape == (_words(t),)
    flat = want_counts.reshape(-1)
    pos = np.concatenate(([0], np.cumsum(flat.astype(np.int64))))
    for i in range(len(flat)):  # every (batch, owner) segment holds the same records
        a, b = int(pos[i]), int(pos[i + 1])
        assert np.array_equal(np.sort(got[a:b]), np.sort(ref[a:b]))
    c.close()


def test_bucket_wire_capacity_and_bad_sizes():
    t = _make("multi")
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    d = _to_tensor(t.events).cuda()
    offs, _ = c.find_batches(d)
    wire, counts = c.bucket_wire(d, offs, 2, 0)   # the binding grows its buffer on INVAL
    assert wire.shape[0] == _words(t) > t.n
    ev = t.events.copy()
    ev["meta"][5] = (ev["meta"][5] & ~np.uint32(7 << 2)) | np.uint32(5 << 2)  # 32-byte access
    with pytest.raises(hr.HiraceError):
        c.bucket_wire(_to_tensor(ev).cuda(), offs, 2, 0)
    c.close()


@pytest.mark.parametrize("compact", [False, True])
def test_replay_wire_matches_replay_trace(compact):
    """Single rank: wire replay of every batch == the 16-byte replay (same race set), with the
    8-byte and the compact 4-byte record."""
    for name in ("cfg2", "multi", "cfg4"):
        t = _make(name)
        d = _to_tensor(t.events).cuda()
        a = hr.Checker.for_trace(t)
        a.replay(d, t.n)
        want = a.collect()
        b = hr.Checker.for_trace(t, compact=compact)
        offs, keys = b.find_batches(d)
        wire, counts = b.bucket_wire(d, offs, 1, 0)
        start = 0
        for k, n in zip(keys, counts.sum(axis=1)):
            b.replay_wire(wire[start:start + int(n)], int(n), int(k))
            start += int(n)
        got = b.collect()
        assert got["key"].tolist() == want["key"].tolist()
        assert ((got["cls_and_epoch"] & 0xFF) == (want["cls_and_epoch"] & 0xFF)).all()
        assert b.stats()["checked"] == _words(t)
        a.close()
        b.close()


def test_replay_wire_rejects_out_of_range():
    c = hr.Checker(4, 64, 32, 1 << 14, 16)
    bad = torch.tensor([np.int64(1 << 20)], dtype=torch.int64, device="cuda")  # word 2^20 > 2^14 tracked
    c.replay_wire(bad, 1, 0)
    assert c.sync() == -6
    c.close()


def _gpu_worker(rank, world, port, name, q, wire=False, split="block", multi_gpu=False):
    """multi_gpu: one GPU per rank and NCCL (the real multi-GPU path); else every rank on GPU 0
    with gloo for the host-side agreement."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = rank if multi_gpu else 0
    torch.cuda.set_device(dev)
    if multi_gpu:
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        t = _make(name)
        blk = t.events["tid"] // t.block_threads
        part = blk if split == "block" else t.events["tid"]
        mine = t.events[(part % world) == rank]
        ops = sharded.GpuOps(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, world,
                             rank, device=dev)
        if wire == "p2p":   # peer dispatch into CUDA-IPC-mapped buffers of the other processes
            ex, run = sharded.PeerExchange(None, dist, device=dev), sharded.run_sharded_p2p
        elif multi_gpu:
            ex = sharded.NcclExchange(None, f"cuda:{dev}")
            run = sharded.run_sharded_wire if wire else sharded.run_sharded
        else:
            ex = sharded.HostExchange(None, device="cuda:0")
            run = sharded.run_sharded_wire if wire else sharded.run_sharded
        n = run(_to_tensor(mine).to(f"cuda:{dev}"), ops, ex, None, dist)
        if wire == "p2p":   # a second trace on the same buffers (handles cached, no regrowth)
            n2 = run(_to_tensor(mine).to(f"cuda:{dev}"), ops, ex, None, dist)
            assert n2 == n
            ex.close()
        races = sharded.gather_races(ops.collect(), None, dist)
        tot = torch.tensor([n], device=f"cuda:{dev}" if multi_gpu else "cpu")
        dist.all_reduce(tot)
        if rank == 0:
            q.put((int(tot.item()), races["key"].tolist(), (races["cls_and_epoch"] & 0xFF).tolist()))
    finally:
        dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world,name", [(2, "cfg2"), (3, "wide"), (2, "cfg3"), (4, "cfg4")])
def test_sharded_gpu_ranks_reproduce_the_oracle(world, name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == t.n
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]


@pytest.mark.parametrize("world,name", [(2, "cfg2"), (3, "multi"), (4, "cfg4"), (2, "cfg3")])
def test_sharded_wire_gpu_ranks_reproduce_the_oracle(world, name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_worker, args=(r, world, port, name, q, True)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == _words(t)
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]


@pytest.mark.parametrize("world,name,split", [(1, "multi", "block"), (2, "cfg2", "block"), (3, "multi", "block"),
                                              (2, "cfg3", "block"), (4, "cfg4", "block"), (2, "cfg2", "thread")])
def test_sharded_p2p_gpu_ranks_reproduce_the_oracle(world, name, split):
    """Peer dispatch with the real kernels: `world` processes share the GPU, each maps the
    others' receive buffers through CUDA IPC, the dispatch kernel stores straight into them and
    every batch is released per owner (hirace_peer_release / hirace_peer_wait).  The trace is
    replayed twice (RACE is sticky, so the race set is unchanged).  split="thread": each block's
    events come from several ranks."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_worker, args=(r, world, port, name, q, "p2p", split)) for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = _make(name)
    k, c, _ = oracle.races_of(t)
    assert total == _words(t)
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 GPUs (one rank per GPU over NCCL)")
@pytest.mark.parametrize("mode", ["wire", "p2p"])
def test_sharded_multi_gpu_nccl_ranks_reproduce_the_oracle(mode):
    """The real multi-GPU path: one process per GPU, NCCL all_to_all (wire) or peer dispatch
    over NVLink with per-batch release flags (p2p)."""
    world = min(4, torch.cuda.device_count())
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    wire = True if mode == "wire" else "p2p"
    procs = [ctx.Process(target=_gpu_worker, args=(r, world, port, "cfg2", q, wire, "thread", True))
             for r in range(world)]
    for p in procs:
        p.start()
    total, keys, cls = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = _make("cfg2")
    k, c, _ = oracle.races_of(t)
    assert total == _words(t)
    assert keys == [int(x) for x in k]
    assert cls == [int(x) for x in c]


def test_dispatch_wire_matches_bucket_wire():
    """One process: the dispatch kernel's stores (own buffer as every owner's destination,
    at disjoint offsets) hold exactly hirace_bucket_wire's (batch, owner) segments."""
    t = _make("multi")
    P, me = 4, 1
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    d = _to_tensor(t.events).cuda()
    offs, _ = c.find_batches(d)
    counts = c.count_wire(d, offs, P, me).astype(np.int64)
    wire, counts2 = c.bucket_wire(d, offs, P, me)
    assert np.array_equal(counts, counts2.astype(np.int64))
    flat = counts.reshape(-1)
    dst = (np.cumsum(flat) - flat).reshape(counts.shape)          # segment (b, r) at its bucket_wire position
    buf = torch.full((int(flat.sum()),), -1, dtype=torch.int64, device="cuda")
    c.dispatch_wire(d, offs, P, me, [buf.data_ptr()] * P, dst)
    got, ref = buf.cpu().numpy(), wire.cpu().numpy()
    assert (got != -1).all()
    for i in range(len(flat)):
        a, b = int(dst.reshape(-1)[i]), int(dst.reshape(-1)[i] + flat[i])
        assert np.array_equal(np.sort(got[a:b]), np.sort(ref[a:b]))
    c.close()


def test_sharded_wire_single_rank_nccl():
    port = _free_port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        t = _make("multi")
        ops = sharded.GpuOps(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, 1, 0)
        ex = sharded.NcclExchange(None, "cuda:0")
        n = sharded.run_sharded_wire(_to_tensor(t.events).cuda(), ops, ex, None, dist)
        races = sharded.gather_races(ops.collect(), None, dist)
    finally:
        dist.destroy_process_group()
    k, c, _ = oracle.races_of(t)
    assert n == _words(t)
    assert races["key"].tolist() == [int(x) for x in k]
    assert (races["cls_and_epoch"] & 0xFF).tolist() == [int(x) for x in c]


def test_sharded_single_rank_nccl():
    port = _free_port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        t = _make("wide")
        ops = sharded.GpuOps(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, 1, 0)
        ex = sharded.NcclExchange(None, "cuda:0")
        n = sharded.run_sharded(_to_tensor(t.events).cuda(), ops, ex, None, dist)
        races = sharded.gather_races(ops.collect(), None, dist)
    finally:
        dist.destroy_process_group()
    k, c, _ = oracle.races_of(t)
    assert n == t.n
    assert races["key"].tolist() == [int(x) for x in k]
    assert (races["cls_and_epoch"] & 0xFF).tolist() == [int(x) for x in c]
    assert _to_events  # imported helper used by the CPU tests


def test_bucket_events_flags_straddling_access():
    """The 16-byte path cannot split an access across owners: it must say so (BAD_TRACE)."""
    t = _make("multi")
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    d = _to_tensor(t.events).cuda()
    out = torch.empty_like(d)
    c.bucket(d, t.n, 2, 0, out)
    assert c.sync() == -6
    c.close()
    ok = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    ok.bucket(d, t.n, 1, 0, out)  # one rank: nothing to split
    assert ok.sync() == 0
    ok.close()
