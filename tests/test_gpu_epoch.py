"""GPU parity of the epoch reset (include/hirace.h HIRACE_RESET_EPOCH; reading R19).

In epoch mode hirace_shadow_reset clears only the RACE records named in the report buffer and
moves the replay's grid-epoch offset past every epoch used so far: a record left by an earlier
check then has another g and the FSM restarts it as if INIT (reading R4).  The race set, the
classes and the reported g must equal a fresh shadow's - across many checks (the offset wraps:
rebase sweeps), report-buffer overflow (full sweep), replay calls of one check that push the
offset past 254 mid-check, and switches to paths that need the shadow at offset 0.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402


def oracle_full(t):
    """{key: (class, g*)} - the g a report carries is the trace's g of the first racing epoch."""
    k, c, g = oracle.races_of(t)
    return {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}


def got_full(r):
    return {int(k): (int(v) & 0xFF, (int(v) >> 8) & 0xFF) for k, v in zip(r["key"], r["cls_and_epoch"])}


def run(c, t, chunks=1):
    c.reset()
    d = hr.events_to_device(t.events)
    bounds = np.linspace(0, t.n, chunks + 1).astype(np.int64)
    for lo, hi in zip(bounds[:-1], bounds[1:]):
        if hi > lo:
            c.replay_ptr(d.data_ptr() + 16 * int(lo), int(hi - lo))
    return got_full(c.collect())


def _random_trace(rng, nb=3, bs=8, ws=4, words=6):
    n = int(rng.integers(1, 60))
    ev = np.empty(n, dtype=tg.EVENT_DTYPE)
    ev["tid"] = rng.integers(0, nb * bs, n)
    word = rng.integers(0, words, n).astype(np.uint64)
    sh = rng.random(n) < 0.3
    ev["addr"] = (word << np.uint64(2)) | np.where(sh, tg.SHARED_BIT, np.uint64(0))
    ev["meta"] = tg.pack_meta(rng.choice(4, n, p=[.4, .3, .15, .15]), 2, rng.integers(0, 2, n),
                              rng.integers(0, 3, n), rng.integers(0, 4, n))
    return tg.Trace("rnd", tg.sort_by_batch(ev), nb, bs, ws, words, words)


def test_epoch_reset_many_checks_vs_oracle():
    # one context, 600 checks of random traces with up to 4 grid epochs each: the offset crosses
    # 254 many times (rebase sweeps) and records of every earlier check are still around
    rng = np.random.default_rng(7)
    c = hr.Checker(3, 8, 4, 6, 6)
    c.set_reset_mode(hr.RESET_EPOCH)
    for it in range(600):
        t = _random_trace(rng)
        assert run(c, t) == oracle_full(t), it
    c.close()


def test_epoch_reset_same_results_as_full_reset_on_configs():
    for make in (lambda: tg.cfg2(True, n=128, steps=4), lambda: tg.cfg4("B", 6, 128, 34),
                 lambda: tg.cfg3("bfs", True, scale=12, edge_factor=16), lambda: tg.cfg1("post_init")):
        t = make()
        want = oracle_full(t)
        full = hr.Checker.for_trace(t)
        ep = hr.Checker.for_trace(t)
        ep.set_reset_mode(hr.RESET_EPOCH)
        for _ in range(12):               # 12 checks in a row: offsets 0, G, 2G, ... then rebases
            assert run(ep, t) == want
        assert run(full, t) == want
        full.close()
        ep.close()


def test_epoch_reset_report_overflow_falls_back_to_a_full_sweep():
    racy, clean = tg.cfg2(True, n=64, steps=2), tg.cfg2(False, n=64, steps=2)
    c = hr.Checker.for_trace(racy, report_capacity=16)   # far fewer than the flagged words
    c.set_reset_mode(hr.RESET_EPOCH)
    for _ in range(3):
        assert run(c, racy) == oracle_full(racy)
        assert run(c, clean) == {}
    c.close()


def test_epoch_reset_mid_check_rebase_keeps_the_check():
    # a trace split over replay calls whose g grows: once the offset is high, a later call of
    # the same check must rebase without losing the earlier calls' records
    t = tg.cfg4("G", 6, 128, 40)           # 40 grid epochs per check
    want = oracle_full(t)
    c = hr.Checker.for_trace(t)
    c.set_reset_mode(hr.RESET_EPOCH)
    for it in range(15):                    # offsets 0, 40, ..., past 254 several times
        assert run(c, t, chunks=5) == want, it
    c.close()


def test_epoch_reset_then_inline_and_host_paths():
    # paths that do not add the offset normalise the shadow first (inline hooks, hirace_barrier)
    t = tg.listing2(1, 64)
    c = hr.Checker.for_trace(t)
    c.set_reset_mode(hr.RESET_EPOCH)
    for _ in range(5):
        assert run(c, t) == oracle_full(t)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    for _ in range(300):                    # grid-epoch wraps with rebase sweeps
        c.barrier()
    assert {k: v[0] for k, v in got_full(c.collect()).items()} == {0: 2}
    c.close()


def test_epoch_reset_rejected_for_compact_and_window_contexts():
    t = tg.cfg2(True, n=64, steps=2)
    cc = hr.Checker.for_trace(t, compact=True)
    with pytest.raises(hr.HiraceError):
        cc.set_reset_mode(hr.RESET_EPOCH)
    cc.close()
    w = hr.Checker.for_trace(t)
    w.set_replay_mode(hr.REPLAY_WINDOW, 6)
    with pytest.raises(hr.HiraceError):
        w.set_reset_mode(hr.RESET_EPOCH)
    w.close()


def test_epoch_reset_fused_check_device_cfg5_medium():
    t = tg.cfg5(grid_blocks=1024, words_log2=26)
    want = {w: {"WARP": 1, "BLOCK": 2, "GRID": 3}[c] for w, c in t.info["expected"].items()}
    c = hr.Checker.for_trace(t)
    c.set_reset_mode(hr.RESET_EPOCH)
    d = hr.events_to_device(t.events)
    cap = 1 << 16
    out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
    tot = torch.zeros(1, dtype=torch.int64, device="cuda")
    for _ in range(70):                      # 4 epochs per check: crosses 254 once
        c.reset()
        c.check_device(d, out, cap, tot)
    torch.cuda.synchronize()
    assert c.sync() == 0
    n = int(tot.item())
    recs = out.cpu().numpy().view(hr.RACE_DTYPE)[:n]
    assert {int(k): int(v) & 0xFF for k, v in zip(recs["key"], recs["cls_and_epoch"])} == want
    assert c.stats()["checked"] == t.n
    c.close()
