"""The derived cluster-level FSM (reading R16) checked on CPU through
the C-ABI host hook hirace_fsm_step_cluster (the inline step of hirace_device.cuh's
hirace::cluster namespace): the Murphi-style bisimulation of PAPER.md L233, strengthened to the
race class, over random tiny cluster traces (with DSMEM targets) x random linear extensions of
the cluster happens-before order, against the literal pair loop brute.races_cluster."""
import numpy as np
import pytest

import tracegen as tg
from oracle import brute

h = pytest.importorskip("paper_conf_sc_jacobsonbg24_b200")


def _hb(a, d):
    """a happens-before d: grid epochs, then (same cluster) cluster epochs, then (same block)
    block epochs, then (same warp) warp epochs."""
    if a["g"] != d["g"]:
        return a["g"] < d["g"]
    if a["cl"] != d["cl"]:
        return False
    if a["c"] != d["c"]:
        return a["c"] < d["c"]
    if a["block"] != d["block"]:
        return False
    if a["b"] != d["b"]:
        return a["b"] < d["b"]
    return a["warp"] == d["warp"] and a["w"] < d["w"]


def _linear_extension(acc, rng):
    n = len(acc)
    preds = [sum(1 for j in range(n) if _hb(acc[j], acc[i])) for i in range(n)]
    done, order = [False] * n, []
    for _ in range(n):
        ready = [i for i in range(n) if not done[i] and preds[i] == 0]
        i = ready[rng.integers(len(ready))]
        done[i] = True
        order.append(i)
        for j in range(n):
            if not done[j] and _hb(acc[i], acc[j]):
                preds[j] -= 1
    return order


def _simulate(acc, order, t):
    shadow = {}
    for i in order:
        a = acc[i]
        shadow[a["key"]], _ = h.fsm_step_cluster(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"], a["c"],
                                                 a["b"], a["w"], t.block_threads, t.warp_size, t.cluster_blocks)
    got = {}
    for k, v in shadow.items():
        cls = h.fsm_cluster_class(v & 63)
        if cls:
            got[k] = cls
    return got, {v & 63 for v in shadow.values()}


@pytest.mark.parametrize("chunk", range(6))
def test_cluster_bisimulation_random_linear_extensions(chunk):
    rng = np.random.default_rng(7000 + chunk)
    for seed in range(chunk * 350, (chunk + 1) * 350):
        t = tg.random_tiny_cluster(seed)
        want = {k: c for k, (c, _) in brute.races_cluster(t.events, t.block_threads, t.warp_size,
                                                          t.cluster_blocks).items()}
        acc = brute.accesses_cluster(t.events, t.block_threads, t.warp_size, t.cluster_blocks)
        for _ in range(4):
            got, _ = _simulate(acc, _linear_extension(acc, rng), t)
            assert got == want, (seed, got, want)


def test_cluster_every_state_reached():
    _, n = h.fsm_table_cluster()
    rng = np.random.default_rng(11)
    reached = set()
    for seed in range(2500):
        t = tg.random_tiny_cluster(seed, max_events=30)
        acc = brute.accesses_cluster(t.events, t.block_threads, t.warp_size, t.cluster_blocks)
        shadow = {}
        for i in _linear_extension(acc, rng):
            a = acc[i]
            shadow[a["key"]], _ = h.fsm_step_cluster(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"], a["c"],
                                                     a["b"], a["w"], t.block_threads, t.warp_size, t.cluster_blocks)
            reached.add(shadow[a["key"]] & 63)
    assert reached == set(range(1, n))  # every non-INIT state


def test_cluster_table_structure():
    t, n = h.fsm_table_cluster()
    assert n <= 64
    assert [h.fsm_cluster_class(s) for s in range(n - 4, n)] == [1, 2, 3, 4]
    assert all(h.fsm_cluster_class(s) == 0 for s in range(n - 4))
    ent = t.reshape(64, 256)
    assert np.all((ent[:n] & 63) < n)
    # RACE states are absorbing with a frozen record
    for s in range(n - 4, n):
        assert np.all(ent[s] & 64)
        assert all(h.fsm_cluster_class(int(x) & 63) >= 1 for x in ent[s])


def test_cluster_halo_and_histogram_through_the_fsm():
    """The DSMEM programs' closed forms (tests/test_cluster_oracle.py) reached by the FSM in the
    generators' natural batch order."""
    for t in (tg.cluster_halo(2, 4, 64, "block"), tg.cluster_halo(2, 4, 64, "cluster"),
              tg.cluster_histogram(2, 4, 64, 16, tg.ATOMIC_BLOCK), tg.cluster_histogram(2, 4, 64, 16, tg.ATOMIC_GRID),
              tg.cluster_histogram(2, 4, 64, 16, tg.ATOMIC_GRID, 2)):
        want = {k: c for k, (c, _) in brute.races_cluster(t.events, t.block_threads, t.warp_size,
                                                          t.cluster_blocks).items()}
        acc = brute.accesses_cluster(t.events, t.block_threads, t.warp_size, t.cluster_blocks)
        got, _ = _simulate(acc, range(len(acc)), t)
        assert got == want, t.name


def test_cluster_step_rejects_out_of_range_fields():
    with pytest.raises(h.HiraceError):
        h.fsm_step_cluster(0, 1 << 27, 0, 0, 0, 0, 0, 32, 32, 2)
    with pytest.raises(h.HiraceError):
        h.fsm_step_cluster(0, 0, 0, 0, 128, 0, 0, 32, 32, 2)
