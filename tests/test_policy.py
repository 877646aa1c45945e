"""the relaxed read-vs-atomic conflict policy (reading R2b), on CPU.

Under RELAXED_READ_ATOMIC a plain read never conflicts with an atomic and atomics of one block
never conflict; writes conflict with everything and, across blocks, AB-AB and AB-AG still do.

Pins of the two oracles (oracle_d.c and brute.py) under this policy, independent of both:
hand-evaluated pairs, and invariants the definition fixes (the conflict relation is a subset of
the strict one, so flagged keys are a subset; traces without plain reads, or without atomics,
have identical verdicts under both policies).  Then the product's relaxed FSM table is checked
by the same bisimulation property as the strict one (tests/test_fsm.py) against brute force.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from oracle import brute
from tests.test_fsm import _random_linear_extension, _unpack

h = pytest.importorskip("paper_conf_sc_jacobsonbg24_b200")

R, W, AB, AG = 0, 1, 2, 3
RELAXED = 1


def _trace(accs, bt=4, ws=2, nb=2):
    """accs: (tid, kind, g, b, w) on word 0."""
    ev = np.empty(len(accs), dtype=tg.EVENT_DTYPE)
    for i, (tid, k, g, b, w) in enumerate(accs):
        ev[i]["addr"] = 0
        ev[i]["tid"] = tid
        ev[i]["meta"] = int(tg.pack_meta(np.array([k]), 2, np.array([w]), np.array([b]), np.array([g]))[0])
    return tg.Trace("pin", tg.sort_by_batch(ev), nb, bt, ws, 1, 1)


# (accesses, strict verdict, relaxed verdict): class of word 0 or None; geometry bt=4, ws=2
PINS = [
    ([(0, R, 0, 0, 0), (4, AG, 0, 0, 0)], 3, None),       # read vs grid atomic, other block
    ([(0, R, 0, 0, 0), (1, AB, 0, 0, 0)], 1, None),       # read vs block atomic, same warp
    ([(0, R, 0, 0, 0), (2, AG, 0, 0, 0)], 2, None),       # read vs atomic, other warp
    ([(0, AB, 0, 0, 0), (4, AB, 0, 0, 0)], 3, 3),         # block atomics of two blocks
    ([(0, AB, 0, 0, 0), (4, AG, 0, 0, 0)], 3, 3),
    ([(0, AG, 0, 0, 0), (4, AG, 0, 0, 0)], None, None),   # grid atomics never conflict
    ([(0, AB, 0, 0, 0), (1, AB, 0, 0, 0)], None, None),   # same block
    ([(0, W, 0, 0, 0), (4, AG, 0, 0, 0)], 3, 3),          # write conflicts with everything
    ([(0, W, 0, 0, 0), (1, R, 0, 0, 0)], 1, 1),
    ([(0, R, 0, 0, 0), (4, AG, 0, 0, 0), (1, AB, 0, 0, 0)], 3, 3),   # AG vs AB across blocks
    # read/atomic pair in g0 (strict: grid race in g0), write race only in g1 (relaxed: g* = 1)
    ([(0, R, 0, 0, 0), (4, AG, 0, 0, 0), (0, W, 1, 0, 0), (1, W, 1, 0, 0)], 3, 1),
]


@pytest.mark.parametrize("i", range(len(PINS)))
def test_hand_evaluated_pairs(i):
    accs, strict, relaxed = PINS[i]
    t = _trace(accs)
    for pol, want in ((0, strict), (RELAXED, relaxed)):
        b = brute.races(t.events, t.block_threads, t.warp_size, pol)
        assert {k: c for k, (c, _) in b.items()} == ({} if want is None else {0: want}), (pol, b)
        assert oracle.races_dict(t, pol) == ({} if want is None else {0: want})


@pytest.mark.parametrize("chunk", range(4))
def test_relaxed_oracle_matches_bruteforce(chunk):
    for seed in range(chunk * 400, (chunk + 1) * 400):
        t = tg.random_tiny(seed)
        want = brute.races(t.events, t.block_threads, t.warp_size, RELAXED)
        k, c, g = oracle.races_of(t, RELAXED)
        got = {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}
        assert got == want, seed


def test_policy_invariants():
    differ = 0
    for seed in range(1500):
        t = tg.random_tiny(seed)
        s = oracle.races_dict(t, 0)
        r = oracle.races_dict(t, RELAXED)
        assert set(r) <= set(s), seed
        kinds = set((t.events["meta"] & 3).tolist())
        if R not in kinds or not (kinds & {AB, AG}):
            assert r == s, seed
        differ += r != s
    assert differ > 50   # the policies are genuinely different on these inputs


def _simulate(acc, order, bt, ws, policy):
    shadow = {}
    for i in order:
        a = acc[i]
        shadow[a["key"]], _ = h.fsm_step(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"], a["b"], a["w"],
                                         bt, ws, policy=policy)
    return {k: (v & 31) - 19 for k, v in shadow.items() if (v & 31) >= 20}, shadow


@pytest.mark.parametrize("probs", [None, (.4, .0, .3, .3), (.3, .1, .3, .3)], ids=["mix", "no_write", "atomic_heavy"])
def test_relaxed_fsm_bisimulation(probs):
    rng = np.random.default_rng(77)
    reached = set()
    for seed in range(1200):
        t = tg.random_tiny(seed, probs=probs)
        want = {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size, RELAXED).items()}
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        for _ in range(3):
            got, shadow = _simulate(acc, _random_linear_extension(acc, rng), t.block_threads, t.warp_size, RELAXED)
            assert got == want, (seed, got, want)
            reached |= {v & 31 for v in shadow.values()}
    assert len(reached) >= 10


def test_relaxed_all_states_reachable():
    rng = np.random.default_rng(9)
    reached = set()
    for seed in range(4000):
        t = tg.random_tiny(seed, probs=(.35, .15, .25, .25))
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        shadow = {}
        for i in _random_linear_extension(acc, rng):
            a = acc[i]
            shadow[a["key"]], _ = h.fsm_step(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"], a["b"], a["w"],
                                             t.block_threads, t.warp_size, policy=RELAXED)
            reached.add(shadow[a["key"]] & 31)
    assert reached == set(range(1, 23))


def test_relaxed_table_structure():
    t = h.fsm_table(RELAXED)
    assert (t != h.fsm_table(0)).any()
    assert (t[: 23 * 64] & 31).max() < 23
    for s in range(20, 23):
        row = t[s * 64:(s + 1) * 64]
        assert ((row & 31) >= s).all() and (row & 32).all()
    for s in range(0, 20):
        row = t[s * 64:(s + 1) * 64]
        assert ((row & 64) != 0).tolist() == ((row & 31) >= 20).tolist()
    # with no writes the relaxed automaton only races on AB across blocks: read labels never race
    for s in range(0, 20):
        for lab in range(16):   # kind R
            nxt = t[s * 64 + lab] & 31
            assert nxt < 20 or s in (4, 5, 6, 10, 11, 15), (s, lab)   # states holding a write
