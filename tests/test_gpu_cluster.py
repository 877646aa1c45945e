"""GPU parity of the cluster-level replay (hirace_cluster_*, DESIGN.md reading
R16) against the cluster oracle (oracle.races_cluster), element by element on the same seeded
traces: random tiny cluster traces with DSMEM targets, the DSMEM halo / histogram programs, a
random medium trace spanning many batches and CTAs, the one-block-per-cluster reduction on a
config-2 stencil, and the error paths."""
import numpy as np
import pytest

import oracle
import tracegen as tg

h = pytest.importorskip("paper_conf_sc_jacobsonbg24_b200")
torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _run(t, cb=None):
    c = h.ClusterChecker(t.grid_blocks, t.block_threads, cb or t.cluster_blocks, t.warp_size, t.global_words,
                         t.smem_words)
    try:
        c.replay(h.events_to_device(t.events, "cuda:0"))
        r = c.collect()
        return {int(k): (int(x) & 255, int(x) >> 8) for k, x in zip(r["key"], r["cls_and_epoch"])}, c.stats()
    finally:
        c.close()


def _want(t, cb=None):
    k, c, g = oracle.races_cluster(t.events, t.block_threads, t.warp_size, cb or t.cluster_blocks)
    return {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}


def test_cluster_random_tiny_parity():
    for seed in range(300):
        t = tg.random_tiny_cluster(seed)
        got, _ = _run(t)
        assert got == _want(t), seed


@pytest.mark.parametrize("sync", ["cluster", "block", "none"])
@pytest.mark.parametrize("shuffle", [None, 5])
def test_cluster_halo_parity(sync, shuffle):
    t = tg.cluster_halo(64, 4, 128, sync)
    if shuffle is not None:
        t.events = _shuffle(t.events, shuffle)
    got, (checked, _) = _run(t)
    assert got == _want(t)
    assert checked == t.n
    assert (len(got) == 0) == (sync == "cluster")


@pytest.mark.parametrize("atomic,drop", [(tg.ATOMIC_GRID, None), (tg.ATOMIC_GRID, 1), (tg.ATOMIC_GRID, 2),
                                         (tg.ATOMIC_BLOCK, None)])
def test_cluster_histogram_parity(atomic, drop):
    t = tg.cluster_histogram(32, 8, 256, 64, atomic, drop)
    got, _ = _run(t)
    assert got == _want(t)
    assert (len(got) == 0) == (atomic == tg.ATOMIC_GRID and drop is None)


def _shuffle(ev, seed):
    """another legal interleaving: permute inside each (g, c, b, w) batch"""
    rng = np.random.default_rng(seed)
    c = (ev["addr"] >> np.uint64(56)) & np.uint64(127)
    key = ((ev["meta"] >> 24).astype(np.uint64) << np.uint64(26)) | (c << np.uint64(19)) | \
        ((ev["meta"] >> 5) & ((1 << 19) - 1)).astype(np.uint64)
    return ev[np.lexsort((rng.random(ev.shape[0]), key))]


def _random_medium(seed, nb=64, bs=128, cb=4, n=300_000, gw=4096, sw=256):
    rng = np.random.default_rng(seed)
    ev = np.empty(n, dtype=tg.EVENT_DTYPE)
    shared = rng.random(n) < 0.5
    target = np.where(shared & (rng.random(n) < 0.3), rng.integers(0, cb, n) + 1, 0)
    words = np.where(shared, rng.integers(0, sw, n), rng.integers(0, gw, n))
    kind = rng.choice(4, n, p=(.6, .1, .15, .15))
    ev["addr"] = tg.pack_cluster_addr(words * 4, shared, rng.integers(0, 3, n), target)
    ev["tid"] = rng.integers(0, nb * bs, n)
    ev["meta"] = tg.pack_meta(kind, 2, rng.integers(0, 2, n), rng.integers(0, 3, n), rng.integers(0, 2, n))
    return tg.Trace(f"cmed{seed}", tg.sort_by_cluster_batch(ev), nb, bs, 32, gw, sw, cluster_blocks=cb)


@pytest.mark.parametrize("seed", [1, 2])
def test_cluster_random_medium_parity(seed):
    t = _random_medium(seed)
    got, _ = _run(t)
    want = _want(t)
    assert len(want) > 100
    assert got == want


def test_one_block_per_cluster_matches_three_level_oracle():
    t = tg.cfg2(True, n=64, steps=2)
    got, _ = _run(t, cb=1)
    k, c, g = oracle.races_of(t)
    assert got == {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}
    assert len(got) > 0


def test_cluster_reset_and_replay_again():
    t = tg.cluster_halo(16, 4, 64, "none")
    c = h.ClusterChecker.for_trace(t)
    try:
        ev = h.events_to_device(t.events, "cuda:0")
        c.replay(ev)
        a = h.races_to_dict(c.collect())
        c.reset()
        c.replay(ev)
        assert h.races_to_dict(c.collect()) == a == oracle.races_cluster_dict(t)
    finally:
        c.close()


def test_cluster_bad_traces():
    t = tg.cluster_halo(4, 4, 64, "cluster")
    bad = t.events[::-1].copy()       # not batch-sorted
    c = h.ClusterChecker.for_trace(t)
    try:
        c.replay(h.events_to_device(bad, "cuda:0"))
        with pytest.raises(h.HiraceError):
            c.collect()
    finally:
        c.close()
    ev = t.events.copy()
    sh = (ev["addr"] >> np.uint64(63)) != 0
    ev["addr"][sh] |= np.uint64(9) << np.uint64(48)   # DSMEM target rank 8 of a 4-block cluster
    c = h.ClusterChecker.for_trace(t)
    try:
        c.replay(h.events_to_device(ev, "cuda:0"))
        with pytest.raises(h.HiraceError):
            c.collect()
    finally:
        c.close()
    with pytest.raises(h.HiraceError):
        h.ClusterChecker(6, 64, 4, 32, 0, 64)   # 4 does not divide 6 blocks


def test_cluster_empty_trace():
    t = tg.cluster_halo(2, 2, 32, "none")
    c = h.ClusterChecker.for_trace(t)
    try:
        c.replay(h.events_to_device(t.events[:0], "cuda:0"), n=0)
        assert c.collect().shape[0] == 0
    finally:
        c.close()
