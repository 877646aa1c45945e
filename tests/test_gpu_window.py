"""GPU parity of the window-major path (csrc/window.cu; include/hirace.h HIRACE_REPLAY_WINDOW).

The window path regroups the element accesses by shadow window (one or two counting-sort
passes that keep batch order inside every window) and replays each window in shared memory,
heavy windows through the global shadow.  The bar is the one of the batch-major path: the
flagged (key, class) set equals the oracle's bit for bit.  Small window sizes (2^5..2^10
records) make small traces span many windows, so both partition layouts (one pass when the
window id fits 9 bits, two passes otherwise), ragged windows and the heavy path
(HIRACE_WIN_HEAVY forces a small threshold) run here at test sizes.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from tests.helpers import CLS, expand_expected, listing_trace, load_golden

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402


def as_dict(r):
    return {int(k): int(c) & 0xFF for k, c in zip(r["key"], r["cls_and_epoch"])}


def oracle_dict(trace, policy=0):
    k, c, _ = oracle.races_of(trace, policy)
    return {int(a): int(b) for a, b in zip(k, c)}


def win_checker(trace, wl, **kw):
    c = hr.Checker.for_trace(trace, **kw)
    c.set_replay_mode(hr.REPLAY_WINDOW, wl)
    assert c.window_active
    return c


def run(c, trace, chunks=1):
    c.reset()
    if trace.n:
        d = hr.events_to_device(trace.events)
        bounds = np.linspace(0, trace.n, chunks + 1).astype(np.int64)
        for lo, hi in zip(bounds[:-1], bounds[1:]):
            if hi > lo:
                c.replay_ptr(d.data_ptr() + 16 * int(lo), int(hi - lo))
    r = c.collect()
    return as_dict(r), c.stats()


def shuffled(t, seed):
    return tg.Trace(t.name, tg._shuffle_within_batches(t.events, seed), t.grid_blocks, t.block_threads,
                    t.warp_size, t.global_words, t.smem_words)


@pytest.mark.parametrize("wl", [5, 7])
@pytest.mark.parametrize("chunk", range(2))
def test_window_random_tiny_vs_oracle(wl, chunk):
    c = None
    for seed in range(chunk * 200, (chunk + 1) * 200):
        t = tg.random_tiny(seed, max_events=40)
        c = win_checker(t, wl)
        for s in (None, seed):
            ts = t if s is None else shuffled(t, s)
            got, st = run(c, ts)
            assert got == oracle_dict(ts), seed
            assert st["checked"] == ts.n
        c.close()


@pytest.mark.parametrize("wl", [5, 9])
def test_window_dense_contention_vs_oracle(wl):
    rng = np.random.default_rng(11)
    for it in range(20):
        nb, bs, ws = int(rng.integers(1, 6)), 64, 32
        n = int(rng.integers(500, 20000))
        ev = np.empty(n, dtype=tg.EVENT_DTYPE)
        nkeys = int(rng.integers(1, 200))
        ev["tid"] = rng.integers(0, nb * bs, n)
        word = rng.integers(0, nkeys, n).astype(np.uint64)
        sh = rng.random(n) < 0.3
        ev["addr"] = (word << np.uint64(2)) | np.where(sh, np.uint64(1) << np.uint64(63), np.uint64(0))
        kinds = rng.choice(4, n, p=[0.7, 0.05, 0.1, 0.15])
        ev["meta"] = tg.pack_meta(kinds, 2, rng.integers(0, 3, n), rng.integers(0, 3, n), rng.integers(0, 3, n))
        t = tg.Trace("dense", tg.sort_by_batch(ev), nb, bs, ws, nkeys, nkeys)
        c = win_checker(t, wl)
        got, st = run(c, t)
        assert got == oracle_dict(t), it
        assert st["checked"] == n
        c.close()


@pytest.mark.parametrize("entry", load_golden("listings.json")["cases"],
                         ids=lambda e: e["case"] + "-" + "-".join(f"{k}{v}" for k, v in e["params"].items()))
def test_window_listings(entry):
    t = listing_trace(entry["case"], entry["params"], shuffle_seed=0)
    c = win_checker(t, 5)
    got, _ = run(c, t)
    assert got == expand_expected(entry["expected"]), entry["cite"]
    c.close()


@pytest.mark.parametrize("wl", [5, 8, 14])
@pytest.mark.parametrize("racy", [False, True])
def test_window_cfg2_small_one_and_two_passes(wl, racy):
    t = tg.cfg2(racy, n=128, steps=3)
    want = oracle_dict(t)
    c = win_checker(t, wl)
    for seed in (None, 0, 1):
        got, _ = run(c, t if seed is None else shuffled(t, seed))
        assert got == want, seed
    c.close()


@pytest.mark.parametrize("racy", [None, "G", "B"])
def test_window_cfg4_small_many_batches(racy):
    t = tg.cfg4(racy, 6, 128, 34)
    c = win_checker(t, 6)
    got, _ = run(c, t)
    assert got == oracle_dict(t)
    c.close()


@pytest.mark.parametrize("kind", ["bfs", "cc"])
@pytest.mark.parametrize("racy", [False, True])
def test_window_cfg3_graph_kernels(kind, racy):
    t = tg.cfg3(kind, racy, scale=14, edge_factor=16)
    want = oracle_dict(t)
    c = win_checker(t, 8)
    for seed in (None, 0):
        got, st = run(c, t if seed is None else shuffled(t, seed))
        assert got == want
        assert st["checked"] == t.n
    c.close()


@pytest.mark.parametrize("heavy", ["64", "1000"])
def test_window_heavy_path(heavy, monkeypatch):
    # a small heavy threshold sends the busiest windows through the global-shadow kernel
    monkeypatch.setenv("HIRACE_WIN_HEAVY", heavy)
    for make in (lambda: tg.cfg3("bfs", True, scale=14, edge_factor=16), lambda: tg.cfg2(True, n=128, steps=3),
                 lambda: tg.cfg4("B", 6, 128, 34)):
        t = make()
        c = win_checker(t, 7)
        got, st = run(c, t)
        assert got == oracle_dict(t)
        assert st["checked"] == t.n
        c.close()


def test_window_split_calls_and_lazy_reset():
    # replay calls accumulate (windows written by one call are loaded by the next); a reset
    # between traces leaves nothing behind (lazy reset: stale windows read as INIT)
    racy = tg.cfg2(True, n=128, steps=4)
    clean = tg.cfg2(False, n=128, steps=4)       # same geometry, no races
    c = win_checker(racy, 6)
    for chunks in (2, 7):
        got, _ = run(c, racy, chunks=chunks)
        assert got == oracle_dict(racy)
        got, _ = run(c, clean, chunks=chunks)
        assert got == {}
    c.close()


def test_window_then_direct_shadow_paths():
    # after a lazy reset, paths that touch the shadow directly make stale windows INIT first:
    # grid-epoch rebase (barrier) and the shadow-scan collect
    t = tg.listing2(1, 64)
    c = win_checker(t, 5)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    for _ in range(300):
        c.barrier()
    assert as_dict(c.collect()) == {0: CLS["BLOCK"]}
    c.close()


@pytest.mark.parametrize("collect", ["scan", "reports"])
def test_window_fused_check_device(collect, monkeypatch):
    monkeypatch.setenv("HIRACE_COLLECT", collect)
    for make in (lambda: tg.cfg2(True, n=128, steps=3), lambda: tg.cfg1("post_init"),
                 lambda: tg.cfg2(False, n=64, steps=2)):
        t = make()
        c = win_checker(t, 6)
        c.reset()
        d = hr.events_to_device(t.events)
        cap = 1 << 16
        out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        c.check_device(d, out, cap, tot)
        torch.cuda.synchronize()
        assert c.sync() == 0
        n = int(tot.item())
        recs = out.cpu().numpy().view(hr.RACE_DTYPE)[:n]
        want = oracle_dict(t)
        assert n == len(want) and as_dict(recs) == want
        assert bool(np.all(recs["key"][1:] > recs["key"][:-1]))
        c.close()


def test_window_host_entry_point():
    t = tg.cfg2(True, n=128, steps=3)
    c = win_checker(t, 7)
    c.reset()
    assert as_dict(c.check_host(t.events)) == oracle_dict(t)
    c.close()


def test_window_multiword_and_bad_trace():
    ev = np.empty(3, dtype=tg.EVENT_DTYPE)
    ev[0] = (8, 0, tg.pack_meta(tg.WRITE, 3, 0, 0, 0))
    ev[1] = (0, 1, tg.pack_meta(tg.READ, 4, 0, 0, 0))
    ev[2] = (16, 40, tg.pack_meta(tg.READ, 0, 0, 0, 0))
    t = tg.Trace("mw", ev, 1, 64, 32, 64, 0)
    c = win_checker(t, 5)
    got, st = run(c, t)
    assert got == oracle_dict(t) == {2: 1, 3: 1}
    assert st["checked"] == 7
    bad = t.events.copy()
    bad["tid"][1] = 1000
    c.reset()
    c.replay(hr.events_to_device(bad))
    with pytest.raises(hr.HiraceError) as e:
        c.collect()
    assert e.value.status == -6
    c.close()


def test_window_capacity_overflow_is_an_error():
    # every event a 16-byte access (4 elements): more element accesses than the window path holds
    n = 200_000
    ev = np.empty(n, dtype=tg.EVENT_DTYPE)
    ev["tid"] = np.arange(n) % 256
    ev["addr"] = (np.arange(n, dtype=np.uint64) % np.uint64(4096)) << np.uint64(4)
    ev["meta"] = tg.pack_meta(np.zeros(n, np.int64), 4, 0, 0, 0)
    t = tg.Trace("wide", ev, 1, 256, 32, 4 * 4096, 0)
    c = win_checker(t, 8)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    with pytest.raises(hr.HiraceError) as e:
        c.collect()
    assert e.value.status == -2
    c.set_replay_mode(hr.REPLAY_BATCH)
    got, _ = run(c, t)
    assert got == oracle_dict(t)
    c.close()


def test_window_relaxed_policy():
    t = tg.cfg3("cc", True, scale=14, edge_factor=16)
    c = win_checker(t, 8)
    c.set_policy(hr.POLICY_RELAXED_READ_ATOMIC)
    got, _ = run(c, t)
    assert got == oracle_dict(t, hr.POLICY_RELAXED_READ_ATOMIC)
    c.close()


def test_window_filter_selected_accesses():
    t = tg.cfg2(True, n=128, steps=3)
    c = win_checker(t, 6)
    c.set_filter(tid_mask=1, tid_match=0)
    sel = (t.events["tid"] & 1) == 0
    sub = tg.Trace("even", t.events[sel], t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    got, st = run(c, t)
    assert got == oracle_dict(sub)
    assert st["checked"] == sub.n
    c.close()


def test_auto_mode_is_batch_unless_enabled(monkeypatch):
    big = hr.Checker(64, 256, 32, 1 << 28, 0)       # 2 GiB of records
    assert not big.window_active
    big.close()
    monkeypatch.setenv("HIRACE_WINDOW_AUTO_BYTES", str(1 << 30))
    big = hr.Checker(64, 256, 32, 1 << 28, 0)
    small = hr.Checker(64, 256, 32, 1 << 20, 0)
    assert big.window_active and not small.window_active
    big.close()
    small.close()


def test_window_vs_batch_cfg5_reduced():
    t = tg.cfg5(grid_blocks=256, words_log2=22, npatterns=512)
    want = {w: CLS[c] for w, c in t.info["expected"].items()}
    assert oracle_dict(t) == want
    for mode, wl in ((hr.REPLAY_WINDOW, 8), (hr.REPLAY_WINDOW, 14), (hr.REPLAY_BATCH, 0)):
        c = hr.Checker.for_trace(t)
        c.set_replay_mode(mode, wl)
        got, st = run(c, t)
        assert got == want, (mode, wl)
        assert st["checked"] == t.n
        c.close()
