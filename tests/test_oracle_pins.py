"""Pins for the oracle (CPU only): the oracle is checked against things other than itself.

* literal brute-force pair enumeration of the definition on random tiny traces (PAPER.md L101,
  L233 'RACE iff the driver witnesses a data race');
* closed forms of the paper's Listings 2-5 (tests/golden/listings.json, each entry cited);
* the paper's worked scenarios' verdicts (tests/golden/scenarios.json);
* closed forms of configs 1, 2 and 4 (derived from the generators' shapes);
* invariants: read-only / grid-atomic-only histories never race (C1.3);
  the verdict is independent of the interleaving inside a batch (order-independence, Q14).
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from oracle import brute
from tests.helpers import (CLS, as_dict, expand_expected, listing_trace, load_golden,
                           scenario_trace, skey)


def _oracle(trace):
    k, c, g = oracle.races_of(trace)
    return {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}


@pytest.mark.parametrize("chunk", range(8))
def test_oracle_matches_bruteforce_random_tiny(chunk):
    for seed in range(chunk * 400, (chunk + 1) * 400):
        t = tg.random_tiny(seed)
        want = brute.races(t.events, t.block_threads, t.warp_size)
        got = _oracle(t)
        assert got == want, (seed, got, want)


def test_bruteforce_random_tiny_hits_every_class():
    seen = set()
    for seed in range(400):
        t = tg.random_tiny(seed)
        seen |= {c for c, _ in brute.races(t.events, t.block_threads, t.warp_size).values()}
    assert seen == {1, 2, 3}


@pytest.mark.parametrize("entry", load_golden("listings.json")["cases"],
                         ids=lambda e: e["case"] + "-" + "-".join(f"{k}{v}" for k, v in e["params"].items()))
def test_listing_closed_forms(entry):
    t = listing_trace(entry["case"], entry["params"])
    got = {k: c for k, (c, _) in _oracle(t).items()}
    assert got == expand_expected(entry["expected"]), entry["cite"]
    small = t.n <= 400
    if small:
        assert got == {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size).items()}


@pytest.mark.parametrize("sc", load_golden("scenarios.json")["scenarios"], ids=lambda s: s["name"])
def test_paper_scenarios_verdict(sc):
    geom = load_golden("scenarios.json")["geometry"]
    t = scenario_trace(geom, sc["steps"])
    got = {k: c for k, (c, _) in _oracle(t).items()}
    want = {} if sc["race"] is None else {0: CLS[sc["race"]]}
    assert got == want, sc["cite"]


def test_cfg1_closed_forms():
    # SURVEY §8(c) C3 / Listing 4: dropping the post-init barrier races
    # s[bs/2..bs-1]; WARP for one warp, BLOCK for two.
    assert as_dict(*oracle.races_of(tg.cfg1(None))[:2]) == {}
    want32 = {skey(0, w): CLS["WARP"] for w in range(16, 32)}
    t = tg.cfg1("post_init")
    assert t.n == 1016 and t.batch_count() == 48
    assert as_dict(*oracle.races_of(t)[:2]) == want32
    assert tg.cfg1(None).batch_count() == 56
    want64 = {skey(0, w): CLS["BLOCK"] for w in range(32, 64)}
    assert as_dict(*oracle.races_of(tg.cfg1("post_init", block_threads=64))[:2]) == want64
    # dropping the barrier after level 16 -> level 8 reads s[8..15] written at level 16
    assert as_dict(*oracle.races_of(tg.cfg1("level"))[:2]) == {skey(0, w): 1 for w in range(8, 16)}
    assert all(g == 0 for g in oracle.races_of(t)[2])


def _cfg2_expected(n, tile=16):
    nbx = n // tile
    T = tile + 2
    out = {}
    for blk in range(nbx * nbx):
        for ty in range(tile):
            cls = CLS["WARP"] if ty in (0, tile - 1) else CLS["BLOCK"]
            for tx in range(tile):
                out[skey(blk, (ty + 1) * T + tx + 1)] = cls
    return out


def test_cfg2_small_closed_forms():
    assert as_dict(*oracle.races_of(tg.cfg2(False, n=64, steps=3))[:2]) == {}
    t = tg.cfg2(True, n=64, steps=3)
    assert as_dict(*oracle.races_of(t)[:2]) == _cfg2_expected(64)
    for seed in range(3):
        ts = tg.cfg2(True, n=64, steps=3, shuffle_seed=seed)
        assert as_dict(*oracle.races_of(ts)[:2]) == _cfg2_expected(64)


@pytest.mark.slow
def test_cfg2_full_closed_form():
    # The bench workload: 1024 blocks x 256 threads, 8 steps = 17,825,792 events;
    # expected 32,768 WARP + 229,376 BLOCK shared keys.
    t = tg.cfg2(True)
    assert t.n == 17_825_792
    k, c, g = oracle.races_of(t)
    assert np.bincount(c, minlength=4).tolist() == [0, 32768, 229376, 0]
    assert as_dict(k, c) == _cfg2_expected(512)


def test_cfg4_closed_forms():
    nb, bs, ph = 4, 128, 34
    assert as_dict(*oracle.races_of(tg.cfg4(None, nb, bs, ph))[:2]) == {}
    # racy-G: grid.sync after phase 31 demoted -> block-edge halo words of A and B race (GRID)
    t = tg.cfg4("G", nb, bs, ph)
    d = as_dict(*oracle.races_of(t)[:2])
    total = nb * bs
    A0, B0 = 0, 2 * total
    want = {}
    for k in range(1, nb):
        for base in (A0, B0):
            want[base + 2 * k * bs - 1] = CLS["GRID"]   # last word of block k-1, read by block k
            want[base + 2 * k * bs] = CLS["GRID"]       # first word of block k, read by block k-1
    assert d == want and len(d) == 2 * (2 * nb - 2)
    # racy-B: tile barrier dropped in phase 7 -> tile cells 2..2bs-1 of every block
    t = tg.cfg4("B", nb, bs, ph)
    d = as_dict(*oracle.races_of(t)[:2])
    want = {}
    for blk in range(nb):
        for cell in range(2, 2 * bs):
            want[skey(blk, cell)] = CLS["WARP"]
        for lt in range(32, bs, 32):
            want[skey(blk, 2 * lt)] = CLS["BLOCK"]      # written by lt-1, read by lt
            want[skey(blk, 2 * lt + 1)] = CLS["BLOCK"]  # written by lt, read by lt-1
    assert d == want
    assert sum(v == CLS["BLOCK"] for v in d.values()) == nb * 2 * (bs // 32 - 1)


def test_read_only_and_grid_atomic_histories_never_race():
    rng = np.random.default_rng(7)
    for seed in range(300):
        t = tg.random_tiny(seed)
        ev = t.events.copy()
        kinds = rng.choice([tg.READ, tg.ATOMIC_GRID], 1)[0]
        ev["meta"] = (ev["meta"] & ~np.uint32(3)) | np.uint32(kinds)
        t2 = tg.Trace("ro", ev, t.grid_blocks, t.block_threads, t.warp_size, 4, 4)
        assert as_dict(*oracle.races_of(t2)[:2]) == {}


def test_verdict_independent_of_batch_interleaving():
    for seed in range(200):
        t = tg.random_tiny(seed, max_events=30)
        base = _oracle(t)
        ev = tg._shuffle_within_batches(t.events, seed + 1)
        t2 = tg.Trace("s", ev, t.grid_blocks, t.block_threads, t.warp_size, 4, 4)
        assert _oracle(t2) == base


def test_multiword_accesses_expand_to_words():
    # an 8-byte write at word 2 covers words 2,3; a 16-byte read at word 0 covers 0..3
    ev = np.empty(2, dtype=tg.EVENT_DTYPE)
    ev[0] = (8, 0, tg.pack_meta(tg.WRITE, 3, 0, 0, 0))
    ev[1] = (0, 1, tg.pack_meta(tg.READ, 4, 0, 0, 0))
    t = tg.Trace("mw", ev, 1, 32, 32, 4, 0)
    assert as_dict(*oracle.races_of(t)[:2]) == {2: 1, 3: 1}
    assert as_dict(*oracle.races_of(t)[:2]) == {k: c for k, (c, _) in brute.races(ev, 32, 32).items()}


def test_cfg3_clean_graph_kernels_never_race():
    # the atomic (clean) BFS/CC variants must give the empty set
    for kind in ("bfs", "cc"):
        t = tg.cfg3(kind, racy=False, scale=12, edge_factor=8)
        assert t.n > 10_000
        assert as_dict(*oracle.races_of(t)[:2]) == {}


@pytest.mark.parametrize("kind", ["bfs", "cc"])
def test_cfg3_racy_small_graph_oracle_matches_bruteforce(kind):
    t = tg.cfg3(kind, racy=True, scale=4, edge_factor=2, bs=8, ws=4)
    assert 20 < t.n < 700
    want = {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size).items()}
    assert want, "the racy graph kernels must race"
    assert as_dict(*oracle.races_of(t)[:2]) == want


def test_cfg5_construction_and_rank_partition():
    # config 5 (App. C): the injected pairs race with their class, decoys (separated by the
    # matching barrier) do not, and the filler regions never race; rank slices partition it
    kw = dict(grid_blocks=64, block_threads=256, words_log2=24, npatterns=300)
    t = tg.cfg5(**kw)
    want = {w: CLS[c] for w, c in t.info["expected"].items()}
    assert len(want) == 150 and set(want.values()) == {1, 2, 3}
    assert as_dict(*oracle.races_of(t)[:2]) == want
    parts = [tg.cfg5(nranks=3, rank=r, **kw) for r in range(3)]
    allev = np.concatenate([p.events for p in parts])
    assert allev.shape[0] == t.n
    key = lambda e: np.sort(e.view(np.dtype((np.void, 16))))  # noqa: E731
    assert np.array_equal(key(allev), key(t.events))
    assert all(p.batch_count() == 32 for p in parts)


# ---- element granularity (per-element shadow; reading R8) ----------

@pytest.mark.parametrize("gran", [0, 1, 2])
def test_granularity_oracle_vs_brute_force(gran):
    for seed in range(300):
        t = tg.random_tiny_bytes(seed, gran)
        want = {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size, 0, gran).items()}
        k, c, _ = oracle.races_of(t)
        assert {int(a): int(b) for a, b in zip(k, c)} == want, (gran, seed)


def _two_threads(off1, sz1, off2, sz2, kind1=1, kind2=1):
    """thread 0 and thread 32 (another warp of block 0) access bytes of one shared window,
    concurrently (same epochs)."""
    ev = np.empty(2, dtype=tg.EVENT_DTYPE)
    ev["addr"] = np.array([off1, off2], np.uint64) | tg.SHARED_BIT
    ev["tid"] = [0, 32]
    ev["meta"] = tg.pack_meta(np.array([kind1, kind2]), np.array([sz1, sz2]), 0, 0, 0)
    return ev


@pytest.mark.parametrize("off1,sz1,off2,sz2,flagged", [
    # (byte offset, size_log2) of two concurrent writes -> flagged elements per granularity 0/1/2
    (0, 0, 1, 0, ([], [0], [0])),            # adjacent bytes: race only when they share an element
    (1, 0, 2, 0, ([], [], [0])),             # bytes 1 and 2: different half-words
    (0, 2, 2, 0, ([2], [1], [0])),           # a word write and a byte write inside it
    (0, 3, 6, 1, ([6, 7], [3], [1])),        # 8-byte write vs half-word at bytes 6-7
    (4, 2, 8, 2, ([], [], [])),              # disjoint words never race
])
def test_granularity_closed_forms(off1, sz1, off2, sz2, flagged):
    ev = _two_threads(off1, sz1, off2, sz2)
    for gran in (0, 1, 2):
        k, c, _ = oracle.races(ev, 64, 32, 0, gran)
        assert [int(x) & 0xFFFFFFFF for x in k] == flagged[gran], gran
        assert all(int(x) == 2 for x in c)   # two warps of one block: BLOCK class


def test_finer_granularity_only_removes_races():
    """A racing pair on an element is a racing pair on the word holding it, so the words of the
    byte-granularity race set are a subset of the word-granularity race set."""
    for seed in range(300):
        t = tg.random_tiny_bytes(seed, 0)
        k0, _, _ = oracle.races(t.events, t.block_threads, t.warp_size, 0, 0)
        k2, _, _ = oracle.races(t.events, t.block_threads, t.warp_size, 0, 2)
        hi = np.uint64(0xFFFFFFFF00000000)
        words0 = {int((x & hi) | ((x & ~hi) >> np.uint64(2))) for x in k0}
        assert words0 <= {int(x) for x in k2}, seed
