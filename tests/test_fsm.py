"""The product's FSM (table + step function, via the C-ABI verification hooks) checked on CPU.

* the paper's worked state sequences (tests/golden/scenarios.json);
* the Murphi-style bisimulation property ("the analysis model transitions to
  the RACE state if and only if the driver model witnesses a data race"), strengthened to the
  race CLASS, over random tiny traces x random linear extensions of happens-before, against
  the literal brute-force enumerator (oracle/brute.py);
* structural properties of the 2048-entry table.
No GPU needed: hirace_fsm_step runs the same inline step function the kernels run.
"""
import numpy as np
import pytest

import tracegen as tg
from oracle import brute
from tests.helpers import load_golden, scenario_trace

h = pytest.importorskip("paper_conf_sc_jacobsonbg24_b200")

PAPER_STATE = {"READ": {1}, "GREAD": {18}, "BREAD": {14}, "WRITE": {4}, "RACE": {20, 21, 22}}
RACE0 = 20


def _unpack(ev, bt, ws):
    out = []
    for e in ev:
        addr, tid, meta = int(e["addr"]), int(e["tid"]), int(e["meta"])
        kind, size = meta & 3, 1 << ((meta >> 2) & 7)
        w, b, g = (meta >> 5) & 511, (meta >> 14) & 1023, (meta >> 24) & 255
        block = tid // bt
        word0 = (addr & ~(1 << 63)) >> 2
        for k in range(1 if size <= 4 else size // 4):
            key = ((1 << 63) | (block << 32) | (word0 + k)) if addr >> 63 else word0 + k
            out.append(dict(key=key, tid=tid, kind=kind, g=g, b=b, w=w, block=block, warp=(tid % bt) // ws))
    return out


def _hb(a, c):
    """a happens-before c (barrier hierarchy)."""
    if a["g"] != c["g"]:
        return a["g"] < c["g"]
    if a["block"] != c["block"]:
        return False
    if a["b"] != c["b"]:
        return a["b"] < c["b"]
    return a["warp"] == c["warp"] and a["w"] < c["w"]


def _random_linear_extension(acc, rng):
    n = len(acc)
    preds = [sum(1 for j in range(n) if _hb(acc[j], acc[i])) for i in range(n)]
    done = [False] * n
    order = []
    for _ in range(n):
        ready = [i for i in range(n) if not done[i] and preds[i] == 0]
        i = ready[rng.integers(len(ready))]
        done[i] = True
        order.append(i)
        for j in range(n):
            if not done[j] and _hb(acc[i], acc[j]):
                preds[j] -= 1
    return order


def _simulate(acc, order, bt, ws):
    shadow = {}
    for i in order:
        a = acc[i]
        o = shadow.get(a["key"], 0)
        n, _ = h.fsm_step(o, a["tid"], a["kind"], a["g"], a["b"], a["w"], bt, ws)
        shadow[a["key"]] = n
    out = {}
    for k, v in shadow.items():
        st = v & 31
        if st >= RACE0:
            out[k] = st - RACE0 + 1
    return out, shadow


@pytest.mark.parametrize("sc", load_golden("scenarios.json")["scenarios"], ids=lambda s: s["name"])
def test_paper_state_sequences(sc):
    geom = load_golden("scenarios.json")["geometry"]
    t = scenario_trace(geom, sc["steps"])
    o = 0
    for e, want in zip(t.events, sc["paper_states"]):
        meta = int(e["meta"])
        o, _ = h.fsm_step(o, int(e["tid"]), meta & 3, meta >> 24, (meta >> 14) & 1023, (meta >> 5) & 511,
                          geom["block_threads"], geom["warp_size"])
        assert (o & 31) in PAPER_STATE[want], (sc["cite"], o & 31, want)


def test_listing5_read_history_not_lost():
    # thread 1 reads data[1], thread 0 reads data[1] (evicting thread 1 in a
    # one-reader scheme), thread 0 writes data[1] -> RACE.
    o = 0
    for tid, kind in ((1, 0), (0, 0), (0, 1)):
        o, _ = h.fsm_step(o, tid, kind, 0, 0, 0, 32, 32)
    assert o & 31 == 20


@pytest.mark.parametrize("chunk", range(6))
def test_bisimulation_random_linear_extensions(chunk):
    rng = np.random.default_rng(1000 + chunk)
    reached = set()
    for seed in range(chunk * 350, (chunk + 1) * 350):
        t = tg.random_tiny(seed)
        want = {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size).items()}
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        for _ in range(4):
            order = _random_linear_extension(acc, rng)
            got, shadow = _simulate(acc, order, t.block_threads, t.warp_size)
            assert got == want, (seed, order, got, want)
            reached |= {v & 31 for v in shadow.values()}
    assert len(reached) >= 10


def test_all_states_reachable():
    rng = np.random.default_rng(5)
    reached = set()
    for seed in range(3000):
        t = tg.random_tiny(seed)
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        order = _random_linear_extension(acc, rng)
        shadow = {}
        for i in order:
            a = acc[i]
            n, _ = h.fsm_step(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"], a["b"], a["w"],
                              t.block_threads, t.warp_size)
            shadow[a["key"]] = n
            reached.add(n & 31)
    assert reached == set(range(1, 23))


def test_table_structure():
    t = h.fsm_table()
    assert t.shape == (2048,)
    nxt = t & 31
    assert nxt[: 23 * 64].max() < 23
    # INIT: every label starts a single-thread record, never keeps the (empty) record
    init = t[0:64]
    assert set((init & 31).tolist()) <= {1, 4, 5, 6} and not (init & 32).any()
    # RACE is absorbing; class never decreases; entries into RACE report
    for s in range(20, 23):
        row = t[s * 64:(s + 1) * 64]
        assert ((row & 31) >= s).all() and (row & 32).all()
    for s in range(0, 20):
        row = t[s * 64:(s + 1) * 64]
        into_race = (row & 31) >= 20
        assert ((row & 64) != 0).tolist() == into_race.tolist()
    # read-only labels (kind R) never lead to RACE from read-only states
    for s in (1, 8, 14, 18):
        for lab in range(16):   # kind R = labels 0..15
            assert t[s * 64 + lab] & 31 < 20


def test_step_keeps_frozen_race_record():
    o = 0
    o, _ = h.fsm_step(o, 0, 1, 0, 0, 0, 64, 32)      # W by t0
    o, r = h.fsm_step(o, 1, 0, 0, 0, 0, 64, 32)      # R by t1 same warp -> RACE_W
    assert o & 31 == 20 and r == 1
    frozen = o >> 5
    o, r = h.fsm_step(o, 40, 0, 0, 0, 0, 64, 32)     # other warp, same b -> RACE_B upgrade
    assert o & 31 == 21 and r == 1 and o >> 5 == frozen
    o, r = h.fsm_step(o, 33, 0, 0, 1, 0, 64, 32)     # later block epoch: no change
    assert o & 31 == 21 and r == 0
    o, r = h.fsm_step(o, 64, 0, 0, 0, 0, 64, 32)     # other block, same g -> RACE_G
    assert o & 31 == 22 and r == 1
    o, r = h.fsm_step(o, 64, 1, 1, 0, 0, 64, 32)     # next grid epoch: sticky, unchanged
    assert o & 31 == 22 and r == 0
