"""Pins for the all-core Oracle-D driver (oracle/oracle_par.c), CPU only.

The driver splits the element-level accesses by key into shards and runs the pinned
single-thread oracle_races_gran on each shard (a race is a property of one memory location,
PAPER.md L101; SURVEY.md §8(c) C2 "multi-threaded over address shards").  Its result must equal
the single-thread function's on every input: random tiny traces (every class, shared keys,
several threads per shard layout), multi-element accesses that straddle shards, sub-word
granularity, the relaxed policy, and configs 1, 2 and 4 at full size.  The single-thread
function itself is pinned by tests/test_oracle_pins.py (brute force, closed forms).
"""
import numpy as np
import pytest

import oracle
import tracegen as tg


def _same(a, b):
    return all(np.array_equal(x, y) for x, y in zip(a, b))


@pytest.mark.parametrize("threads,shards", [(1, 1), (1, 7), (3, 5), (8, 64), (16, 3)])
def test_par_equals_single_random_tiny(threads, shards):
    for seed in range(300):
        t = tg.random_tiny(seed)
        a = oracle.races(t.events, t.block_threads, t.warp_size)
        b = oracle.races_parallel(t.events, t.block_threads, t.warp_size, threads=threads, shards=shards)
        assert _same(a, b), seed


@pytest.mark.parametrize("gran", [0, 1, 2])
def test_par_equals_single_multi_element_and_granularity(gran):
    # 1-16 byte accesses: wide accesses expand to several elements, which land in different shards
    for seed in range(300):
        t = tg.random_tiny_bytes(seed, gran)
        a = oracle.races(t.events, t.block_threads, t.warp_size, 0, gran)
        b = oracle.races_parallel(t.events, t.block_threads, t.warp_size, 0, gran, threads=4, shards=9)
        assert _same(a, b), seed


def test_par_equals_single_relaxed_policy():
    for seed in range(300):
        t = tg.random_tiny(seed)
        a = oracle.races(t.events, t.block_threads, t.warp_size, policy=1)
        b = oracle.races_parallel(t.events, t.block_threads, t.warp_size, policy=1, threads=4, shards=6)
        assert _same(a, b), seed


def test_par_empty_and_single_event():
    t = tg.random_tiny(0)
    for ev in (t.events[:0], t.events[:1]):
        a = oracle.races(ev, t.block_threads, t.warp_size)
        b = oracle.races_parallel(ev, t.block_threads, t.warp_size, threads=4, shards=4)
        assert _same(a, b)


@pytest.mark.parametrize("make", [lambda: tg.cfg1("post_init"), lambda: tg.cfg1(None), lambda: tg.cfg2(True),
                                  lambda: tg.cfg4("B", grid_blocks=64), lambda: tg.cfg4("G", grid_blocks=64)],
                         ids=["cfg1_racy", "cfg1_clean", "cfg2_racyA", "cfg4_racyB_nb64", "cfg4_racyG_nb64"])
def test_par_equals_single_configs(make):
    t = make()
    a = oracle.races_of(t)
    b = oracle.races_parallel(t.events, t.block_threads, t.warp_size, threads=8)
    assert _same(a, b)
    assert len(a[0]) == len(b[0])


def test_par_cfg5_reduced_matches_construction():
    # config 5's construction (injected non-decoy pairs) at reduced scale, through the driver
    t = tg.cfg5(grid_blocks=64, block_threads=256, words_log2=24, npatterns=300, workers=1)
    k, c, _ = oracle.races_parallel(t.events, t.block_threads, t.warp_size, threads=4)
    want = {w: {"WARP": 1, "BLOCK": 2, "GRID": 3}[c] for w, c in t.info["expected"].items()}
    assert {int(a): int(b) for a, b in zip(k, c)} == want
    assert _same(oracle.races_of(t), (k, c, _))
