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
from tests.test_sharded import CpuTestOps, _make, _to_events, _to_tensor  # noqa: E402


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
    want_t, want_counts = CpuTestOps(None, nranks, rank).bucket(torch.from_numpy(ev.view(np.int64).reshape(-1, 2)))
    assert counts == want_counts
    assert np.array_equal(out.cpu().numpy(), want_t.numpy())
    c.close()


def _gpu_worker(rank, world, port, name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        t = _make(name)
        blk = t.events["tid"] // t.block_threads
        mine = t.events[(blk % world) == rank]
        ops = sharded.GpuOps(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, world,
                             rank, device=0)
        ex = sharded.HostExchange(None, device="cuda:0")
        n = sharded.run_sharded(_to_tensor(mine).cuda(), ops, ex, None, dist)
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
