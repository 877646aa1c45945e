"""Pins of the partial-mask __syncwarp(mask) oracle (DESIGN.md
reading R20; oracle_d.c C1.1''/C1.2'').

The oracle decides same-warp happens-before by forward knowledge propagation along the sync log;
the brute force (oracle/brute.py) by per-lane vector clocks over every pair.  The two are also
pinned by hand-derived cases (tests/golden/masked.json), the closed forms of the tiled
reduction generator, the reduction to the full-mask oracle, and the refinement invariant.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from oracle import brute

from .helpers import CLS, SHARED, load_golden


def _golden_trace(case):
    ev = np.empty(len(case["events"]), dtype=tg.EVENT_DTYPE)
    for i, (word, shared, tid, kind, w, b, g) in enumerate(case["events"]):
        ev[i]["addr"] = (word << 2) | (SHARED if shared else 0)
        ev[i]["tid"] = tid
        ev[i]["meta"] = int(tg.pack_meta(kind, 2, w, b, g))
    ev = tg.sort_by_batch(ev)
    sy = tg.make_syncs(*zip(*case["syncs"])) if case["syncs"] else np.empty(0, dtype=tg.SYNC_DTYPE)
    return tg.Trace(case["name"], ev, 1, case["block_threads"], case["warp_size"], 4, 4, warp_syncs=sy)


@pytest.mark.parametrize("case", load_golden("masked.json")["cases"], ids=lambda c: c["name"])
def test_golden_cases(case):
    t = _golden_trace(case)
    if case["expected"] is None:
        with pytest.raises(oracle.BadSyncLog):
            oracle.races_masked_dict(t)
        return
    want = {int(k): CLS[v] for k, v in case["expected"].items()}
    assert oracle.races_masked_dict(t) == want
    assert {k: v[0] for k, v in brute.races_masked(t.events, t.warp_syncs, t.block_threads, t.warp_size).items()} == want


@pytest.mark.parametrize("policy", [0, 1])
def test_oracle_equals_brute_force_on_random_programs(policy):
    for seed in range(1200):
        t = tg.random_tiny_masked(seed)
        k, c, g = oracle.races_masked(t.events, t.block_threads, t.warp_size, t.warp_syncs, policy)
        got = {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}
        assert got == brute.races_masked(t.events, t.warp_syncs, t.block_threads, t.warp_size, policy), t.name


def test_random_programs_exercise_partial_syncs():
    """the generator produces traces where the partial masks change the verdict"""
    differ = sum(oracle.races_masked_dict(tg.random_tiny_masked(s)) != oracle.races_dict(tg.random_tiny_masked(s))
                 for s in range(300))
    assert differ >= 30


def test_full_masks_reduce_to_the_plain_definition():
    """a log that lists every sync number with the full mask is C1.2 (w1 == w2 <=> concurrent)"""
    for seed in range(1500):
        t = tg.random_tiny(seed)
        m = t.events["meta"]
        w, b, g = (m >> 5) & 511, (m >> 14) & 1023, m >> 24
        tid = t.events["tid"]
        wpb = -(-t.block_threads // t.warp_size)
        warp = (tid // t.block_threads) * wpb + (tid % t.block_threads) // t.warp_size
        fams = {}
        for ww, bb, gg, wp in zip(w, b, g, warp):
            fams[(int(gg), int(bb), int(wp))] = max(fams.get((int(gg), int(bb), int(wp)), 0), int(ww))
        rows = [(wp, (1 << t.warp_size) - 1, s, bb, gg) for (gg, bb, wp), top in fams.items() for s in range(1, top + 1)]
        sy = tg.make_syncs(*zip(*rows)) if rows else None
        for policy in (0, 1):
            k0, c0, g0 = oracle.races(t.events, t.block_threads, t.warp_size, policy)
            k1, c1, g1 = oracle.races_masked(t.events, t.block_threads, t.warp_size, sy, policy)
            assert np.array_equal(k0, k1) and np.array_equal(c0, c1) and np.array_equal(g0, g1), t.name


def test_partial_masks_only_add_races():
    """fewer happens-before edges than the full-mask reading: every plain race stays a race"""
    for seed in range(600):
        t = tg.random_tiny_masked(seed)
        plain, masked = oracle.races_dict(t), oracle.races_masked_dict(t)
        assert set(plain) <= set(masked), t.name


@pytest.mark.parametrize("nb,bs,ws,tile", [(2, 64, 32, 4), (3, 64, 32, 8), (2, 64, 32, 16), (2, 64, 32, 32),
                                           (2, 32, 8, 4), (4, 128, 32, 8)])
def test_tiled_reduction_closed_forms(nb, bs, ws, tile):
    """tracegen.tiled_reduce: clean -> none; half_mask -> the upper half of every tile's words
    (written before a sync the upper lanes skip, read by the lower lanes), WARP; pair -> word
    t + tile of every even tile's leader, WARP when both tiles share a warp, else BLOCK"""
    clean = tg.tiled_reduce(nb, bs, tile, 2, None, ws)
    assert oracle.races_masked_dict(clean) == {}
    half = tg.tiled_reduce(nb, bs, tile, 2, "half_mask", ws)
    want = {SHARED | (blk << 32) | t: CLS["WARP"] for blk in range(nb) for t in range(bs) if t % tile >= tile // 2}
    assert oracle.races_masked_dict(half) == want
    pair = tg.tiled_reduce(nb, bs, tile, 2, "pair", ws)
    cls = CLS["WARP"] if 2 * tile <= ws else CLS["BLOCK"]
    want = {SHARED | (blk << 32) | (t + tile): cls for blk in range(nb) for t in range(0, bs, 2 * tile)
            if t + tile < bs}
    assert oracle.races_masked_dict(pair) == want


def test_tiled_reduction_half_mask_hidden_without_the_log():
    """sanity of the generator: the plain (full-mask) reading orders the tiles' steps, so the
    half-mask bug is invisible without the log -- the partial masks are what expose it"""
    half = tg.tiled_reduce(2, 64, 8, 2, "half_mask")
    assert oracle.races_dict(half) == {}


@pytest.mark.parametrize("bad", ["unsorted", "zero_w", "zero_mask", "wide_mask"])
def test_malformed_logs_are_rejected(bad):
    t = tg.random_tiny_masked(7)
    sy = tg.make_syncs([0, 0], [1, 3], [1, 2], [0, 0], [0, 0])
    if bad == "unsorted":
        sy = sy[::-1].copy()
    elif bad == "zero_w":
        sy["meta"][0] = tg.pack_meta(0, 0, 0, 0, 0)
    elif bad == "zero_mask":
        sy["mask"][0] = 0
    else:
        sy["mask"][0] = 1 << t.warp_size
    with pytest.raises(oracle.BadSyncLog):
        oracle.races_masked(t.events, t.block_threads, t.warp_size, sy)


def _lane_in_listed_mask(t):
    """every access after a listed (partial) sync comes from a lane of that sync's mask"""
    m = t.events["meta"]
    w, b, g = (m >> 5) & 511, (m >> 14) & 1023, m >> 24
    tid = t.events["tid"].astype(np.int64)
    wpb = -(-t.block_threads // t.warp_size)
    warp = (tid // t.block_threads) * wpb + (tid % t.block_threads) // t.warp_size
    lane = (tid % t.block_threads) % t.warp_size
    sy = t.warp_syncs
    listed = {(int(s["meta"]) >> 24, (int(s["meta"]) >> 14) & 1023, int(s["warp"]), (int(s["meta"]) >> 5) & 511):
              int(s["mask"]) for s in sy}
    for i in range(t.n):
        k = (int(g[i]), int(b[i]), int(warp[i]), int(w[i]))
        if k in listed:
            assert (listed[k] >> int(lane[i])) & 1, (t.name, i)


def test_generators_emit_well_formed_logs():
    """tracegen side of R20: logs sorted by (g, b, warp, w), strictly increasing, non-empty masks
    inside the warp, and accesses only after syncs their lane took part in"""
    traces = [tg.random_tiny_masked(s) for s in range(200)]
    traces += [tg.tiled_reduce(4, 64, tl, 2, r) for tl in (4, 8, 32) for r in (None, "half_mask", "pair")]
    for t in traces:
        sy = t.warp_syncs
        key = [(int(s["meta"]) >> 24, (int(s["meta"]) >> 14) & 1023, int(s["warp"]), (int(s["meta"]) >> 5) & 511)
               for s in sy]
        assert key == sorted(key) and len(set(key)) == len(key), t.name
        assert all(k[3] >= 1 for k in key)
        assert all(0 < int(s["mask"]) < (1 << t.warp_size) for s in sy)
        _lane_in_listed_mask(t)


def test_wide_accesses_oracle_equals_brute_force():
    """8- and 16-byte accesses cover 2 / 4 words (C1.1), each checked with the partial syncs"""
    for seed in range(600):
        t = tg.random_tiny_masked(seed, wide=True)
        k, c, g = oracle.races_masked(t.events, t.block_threads, t.warp_size, t.warp_syncs)
        got = {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}
        assert got == brute.races_masked(t.events, t.warp_syncs, t.block_threads, t.warp_size), t.name
