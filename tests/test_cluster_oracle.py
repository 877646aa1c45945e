"""Pins of the cluster-level oracle (reading R16).

Oracle-D's `oracle_races_cluster` (C, sort + per-level scan) is checked against the literal pair
loop `brute.races_cluster` (Python), against the two special cases that reduce to the pinned
three-level definition (one block per cluster; one cluster whose barriers play the grid epoch),
against barrier-semantics closed forms on two accesses, and against the closed forms of two
DSMEM programs (halo exchange, distributed histogram)."""
import numpy as np
import pytest

import oracle
import tracegen as tg
from oracle import brute
from tests.helpers import skey

W_, C_, B_, G_ = 1, 4, 2, 3  # class codes: WARP, CLUSTER, BLOCK, GRID


def _oracle(t):
    k, c, g = oracle.races_cluster(t.events, t.block_threads, t.warp_size, t.cluster_blocks)
    return {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}


@pytest.mark.parametrize("chunk", range(6))
def test_cluster_oracle_matches_bruteforce(chunk):
    for seed in range(chunk * 400, (chunk + 1) * 400):
        t = tg.random_tiny_cluster(seed)
        want = brute.races_cluster(t.events, t.block_threads, t.warp_size, t.cluster_blocks)
        assert _oracle(t) == want, seed


def test_cluster_bruteforce_hits_every_class():
    seen = set()
    for seed in range(600):
        t = tg.random_tiny_cluster(seed)
        seen |= {c for c, _ in brute.races_cluster(t.events, t.block_threads, t.warp_size,
                                                   t.cluster_blocks).values()}
    assert seen == {W_, B_, G_, C_}


def test_one_block_per_cluster_reduces_to_three_levels():
    """cluster_blocks = 1, c = 0, no DSMEM: a cluster is a block, so the verdict (classes and g*)
    is the pinned three-level oracle's."""
    for seed in range(800):
        t = tg.random_tiny(seed)
        k, c, g = oracle.races_of(t)
        want = {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}
        got = oracle.races_cluster(t.events, t.block_threads, t.warp_size, 1)
        assert {int(a): (int(b), int(x)) for a, b, x in zip(*got)} == want, seed


def test_single_cluster_barrier_plays_the_grid_epoch():
    """All blocks in one cluster, g = 0 and c := the three-level trace's g: barrier.cluster then
    separates exactly what the grid epoch separated, and GRID becomes CLUSTER."""
    for seed in range(800):
        t = tg.random_tiny(seed)
        m = tg.unpack_meta(t.events["meta"])
        ev = t.events.copy()
        sh = (ev["addr"] & tg.SHARED_BIT) != 0
        ev["addr"] = tg.pack_cluster_addr(ev["addr"] & ~tg.SHARED_BIT, sh, m["g"])
        ev["meta"] = tg.pack_meta(m["kind"], m["size_log2"], m["w"], m["b"], 0)
        k, c, _ = oracle.races_of(t)
        want = {int(a): {G_: C_}.get(int(b), int(b)) for a, b in zip(k, c)}
        kc, cc, gc = oracle.races_cluster(ev, t.block_threads, t.warp_size, t.grid_blocks)
        assert {int(a): int(b) for a, b in zip(kc, cc)} == want, seed
        assert not np.any(gc)
        bw = brute.races_cluster(ev, t.block_threads, t.warp_size, t.grid_blocks)
        assert {a: v[0] for a, v in bw.items()} == want, seed


def _two(bs, ws, cb, a, b):
    """Two accesses (tid, kind, g, c, b, shared, target, word) -> events."""
    ev = np.empty(2, dtype=tg.EVENT_DTYPE)
    for i, (tid, kind, g, c, bb, sh, tgt, word) in enumerate((a, b)):
        ev[i]["tid"] = tid
        ev[i]["addr"] = tg.pack_cluster_addr(word * 4, sh, c, tgt)
        ev[i]["meta"] = tg.pack_meta(kind, 2, 0, bb, g)
    return ev


R, W, AB, AG = tg.READ, tg.WRITE, tg.ATOMIC_BLOCK, tg.ATOMIC_GRID
# geometry: 4 threads per block, 2 threads per warp, 2 blocks per cluster -> blocks 0,1 = cluster 0
TWO = [
    # same block, two warps: barrier.cluster orders them (it is a rendezvous of the block too)
    ((0, W, 0, 0, 0, True, 0, 0), (2, R, 0, 1, 0, True, 0, 0), None),
    ((0, W, 0, 0, 0, True, 0, 0), (2, R, 0, 0, 0, True, 0, 0), B_),
    ((0, W, 0, 0, 0, True, 0, 0), (1, R, 0, 0, 0, True, 0, 0), W_),
    # two blocks of one cluster: __syncthreads does not order them, barrier.cluster does
    ((0, W, 0, 0, 0, False, 0, 5), (4, R, 0, 0, 1, False, 0, 5), C_),
    ((0, W, 0, 0, 0, False, 0, 5), (4, R, 0, 1, 0, False, 0, 5), None),
    # two clusters: a cluster barrier orders nothing between them, the grid epoch does
    ((0, W, 0, 0, 0, False, 0, 5), (8, R, 0, 1, 0, False, 0, 5), G_),
    ((0, W, 0, 0, 0, False, 0, 5), (8, R, 1, 0, 0, False, 0, 5), None),
    # DSMEM: block 1 writes block 0's shared word 3 (target rank 0 -> 1); block 0 reads it
    ((4, W, 0, 0, 0, True, 1, 3), (0, R, 0, 0, 0, True, 0, 3), C_),
    ((4, W, 0, 0, 0, True, 1, 3), (0, R, 0, 1, 0, True, 0, 3), None),
    ((4, W, 0, 0, 0, True, 2, 3), (0, R, 0, 0, 0, True, 0, 3), None),   # block 1's own word: other key
    # atomics through DSMEM: device scope never conflicts; block scope across blocks does (R3)
    ((4, AG, 0, 0, 0, True, 1, 3), (0, AG, 0, 0, 0, True, 0, 3), None),
    ((4, AB, 0, 0, 0, True, 1, 3), (0, AB, 0, 0, 0, True, 0, 3), C_),
    ((4, AB, 0, 0, 0, True, 1, 3), (6, AB, 0, 0, 0, True, 1, 3), None),  # same (remote) block's threads
    ((4, AG, 0, 0, 0, True, 1, 3), (0, R, 0, 0, 0, True, 0, 3), C_),      # plain read vs atomic (R2)
]


@pytest.mark.parametrize("a,b,cls", TWO)
def test_cluster_two_access_closed_forms(a, b, cls):
    ev = _two(4, 2, 2, a, b)
    got = oracle.races_cluster(ev, 4, 2, 2)
    assert [int(x) for x in got[1]] == ([] if cls is None else [cls])
    bw = brute.races_cluster(ev, 4, 2, 2)
    assert [v[0] for v in bw.values()] == ([] if cls is None else [cls])


@pytest.mark.parametrize("nclusters,cb,bs", [(2, 4, 64), (3, 2, 96), (1, 8, 32)])
@pytest.mark.parametrize("sync", ["cluster", "block", "none"])
def test_cluster_halo_closed_form(nclusters, cb, bs, sync):
    """Racy iff the cluster barrier is missing; then each cluster's 2(cb-1) edge words read by a
    neighbour rank are CLUSTER races (the owner's write vs the neighbour's DSMEM read)."""
    t = tg.cluster_halo(nclusters, cb, bs, sync)
    want = {}
    if sync != "cluster":
        for blk in range(nclusters * cb):
            r = blk % cb
            if r < cb - 1:
                want[skey(blk, bs - 1)] = C_
            if r > 0:
                want[skey(blk, 0)] = C_
    assert oracle.races_cluster_dict(t) == want


@pytest.mark.parametrize("nclusters,cb,bs,bins", [(2, 4, 64, 16), (3, 2, 32, 32), (2, 1, 64, 16)])
@pytest.mark.parametrize("atomic,drop", [(AG, None), (AG, 1), (AG, 2), (AB, None)])
def test_cluster_histogram_closed_form(nclusters, cb, bs, bins, atomic, drop):
    """Device-scope DSMEM atomics between two cluster barriers are race-free; dropping either
    barrier or using block-scope atomics makes every bin of each cluster's rank-0 block a
    CLUSTER race -- unless the cluster is one block, where only a dropped barrier races, at
    BLOCK level (bins written by warp 0 and added to by every warp)."""
    t = tg.cluster_histogram(nclusters, cb, bs, bins, atomic, drop)
    want = {}
    if drop is not None or (atomic == AB and cb > 1):
        cls = C_ if cb > 1 else B_
        for cl in range(nclusters):
            for j in range(bins):
                want[skey(cl * cb, j)] = cls
    assert oracle.races_cluster_dict(t) == want


def test_dsmem_target_outside_the_cluster_is_rejected():
    ev = _two(4, 2, 2, (0, W, 0, 0, 0, True, 3, 0), (1, R, 0, 0, 0, True, 0, 0))
    with pytest.raises(RuntimeError):
        oracle.races_cluster(ev, 4, 2, 2)
