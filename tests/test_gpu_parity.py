"""GPU parity: the CUDA replay (through the C-ABI) vs the oracle and the paper's closed forms.

The bar (BASELINE.json north_star): the set of flagged (key, race class) pairs is bit-exact;
internal shadow words and detecting thread ids legitimately depend on the interleaving and are
not compared.  Every config runs in natural order and under seeded within-batch shuffles.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from tests.helpers import CLS, expand_expected, listing_trace, load_golden, scenario_trace, skey

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402


def gpu_races(trace, checker=None, chunks=1, report_capacity=0):
    c = checker or hr.Checker.for_trace(trace, report_capacity=report_capacity)
    c.reset()
    if trace.n:
        d = hr.events_to_device(trace.events)
        bounds = np.linspace(0, trace.n, chunks + 1).astype(np.int64)
        for lo, hi in zip(bounds[:-1], bounds[1:]):
            if hi > lo:
                c.replay_ptr(d.data_ptr() + 16 * int(lo), int(hi - lo))
    r = c.collect()
    st = c.stats()
    if checker is None:
        c.close()
    return r, st


def as_dict(r):
    return {int(k): int(c) & 0xFF for k, c in zip(r["key"], r["cls_and_epoch"])}


def oracle_dict(trace):
    k, c, _ = oracle.races_of(trace)
    return {int(a): int(b) for a, b in zip(k, c)}


def word_accesses(trace):
    sz = 1 << ((trace.events["meta"] >> 2) & 7).astype(np.int64)
    return int(np.where(sz <= 4, 1, sz // 4).sum())


@pytest.mark.parametrize("entry", load_golden("listings.json")["cases"],
                         ids=lambda e: e["case"] + "-" + "-".join(f"{k}{v}" for k, v in e["params"].items()))
@pytest.mark.parametrize("seed", [None, 0, 1, 2, 3, 4])
def test_listings(entry, seed):
    t = listing_trace(entry["case"], entry["params"], shuffle_seed=seed)
    r, st = gpu_races(t)
    assert as_dict(r) == expand_expected(entry["expected"]), entry["cite"]
    assert st["checked"] == word_accesses(t)
    assert bool(np.all(r["key"][1:] > r["key"][:-1]))


@pytest.mark.parametrize("sc", load_golden("scenarios.json")["scenarios"], ids=lambda s: s["name"])
def test_paper_scenarios(sc):
    geom = load_golden("scenarios.json")["geometry"]
    t = scenario_trace(geom, sc["steps"])
    t.events = tg.sort_by_batch(t.events)
    r, _ = gpu_races(t)
    want = {} if sc["race"] is None else {0: CLS[sc["race"]]}
    assert as_dict(r) == want


@pytest.mark.parametrize("chunk", range(4))
def test_random_tiny_vs_oracle(chunk):
    for seed in range(chunk * 250, (chunk + 1) * 250):
        t = tg.random_tiny(seed, max_events=40)
        for s in (None, seed):
            ts = t if s is None else tg.Trace(t.name, tg._shuffle_within_batches(t.events, s), t.grid_blocks,
                                               t.block_threads, t.warp_size, t.global_words, t.smem_words)
            r, _ = gpu_races(ts)
            assert as_dict(r) == oracle_dict(ts), seed


def test_random_dense_traces_vs_oracle():
    # many events on few words from many threads: exercises warp aggregation and CAS retries
    rng = np.random.default_rng(11)
    for it in range(40):
        nb, bs, ws = int(rng.integers(1, 6)), 64, 32
        n = int(rng.integers(500, 20000))
        ev = np.empty(n, dtype=tg.EVENT_DTYPE)
        nkeys = int(rng.integers(1, 50))
        ev["tid"] = rng.integers(0, nb * bs, n)
        word = rng.integers(0, nkeys, n).astype(np.uint64)
        sh = rng.random(n) < 0.3
        ev["addr"] = (word << np.uint64(2)) | np.where(sh, np.uint64(1) << np.uint64(63), np.uint64(0))
        kinds = rng.choice(4, n, p=[0.7, 0.05, 0.1, 0.15])
        ev["meta"] = tg.pack_meta(kinds, 2, rng.integers(0, 3, n), rng.integers(0, 3, n), rng.integers(0, 3, n))
        t = tg.Trace("dense", tg.sort_by_batch(ev), nb, bs, ws, nkeys, nkeys)
        r, st = gpu_races(t)
        assert as_dict(r) == oracle_dict(t), it
        assert st["checked"] == n


@pytest.mark.parametrize("racy", [None, "post_init", "level"])
@pytest.mark.parametrize("bs", [32, 64])
def test_cfg1(racy, bs):
    for seed in (None, 0, 1, 2, 3, 4):
        t = tg.cfg1(racy, block_threads=bs, shuffle_seed=seed)
        r, _ = gpu_races(t)
        assert as_dict(r) == oracle_dict(t)


@pytest.mark.parametrize("racy", [False, True])
def test_cfg2_small(racy):
    for seed in (None, 0, 1, 2, 3, 4):
        t = tg.cfg2(racy, n=128, steps=3, shuffle_seed=seed)
        r, _ = gpu_races(t)
        assert as_dict(r) == oracle_dict(t)


def test_cfg2_full_bench_config():
    # the bench workload, natural order and one shuffled interleaving, vs the oracle and the
    # closed form 32,768 WARP + 229,376 BLOCK
    t = tg.cfg2(True)
    want = oracle_dict(t)
    assert sorted(np.bincount(list(want.values()), minlength=4).tolist()) == sorted([0, 32768, 229376, 0])
    c = hr.Checker.for_trace(t)
    r, st = gpu_races(t, checker=c)
    assert as_dict(r) == want
    assert st["checked"] == t.n
    t2 = tg.cfg2(True, shuffle_seed=0)
    r2, _ = gpu_races(t2, checker=c)
    assert as_dict(r2) == want
    c.close()


@pytest.mark.parametrize("racy", [None, "G", "B"])
def test_cfg4_small(racy):
    for seed in (None, 0, 1):
        t = tg.cfg4(racy, 6, 128, 34, shuffle_seed=seed)
        r, _ = gpu_races(t)
        assert as_dict(r) == oracle_dict(t)


@pytest.mark.parametrize("racy", ["G", "B"])
def test_cfg4_full_closed_form(racy):
    # full size (592 x 256, 64 phases, ~9.7e7 events): closed forms of SURVEY §8(c) C3
    t = tg.cfg4(racy)
    r, st = gpu_races(t)
    d = as_dict(r)
    nb, bs = 592, 256
    if racy == "G":
        assert len(d) == 2 * 1182 and set(d.values()) == {CLS["GRID"]}
        total = nb * bs
        for k in range(1, nb):
            for base in (0, 2 * total):
                assert d[base + 2 * k * bs - 1] == 3 and d[base + 2 * k * bs] == 3
    else:
        assert len(d) == 301_920
        assert sum(v == CLS["BLOCK"] for v in d.values()) == 8_288
        assert d[skey(0, 64)] == CLS["BLOCK"] and d[skey(591, 65)] == CLS["BLOCK"] and d[skey(3, 5)] == CLS["WARP"]
    assert st["checked"] == t.n


def test_split_replay_calls_continue_the_linearisation():
    t = tg.cfg2(True, n=128, steps=4)
    want = oracle_dict(t)
    for chunks in (2, 7, 33):
        r, _ = gpu_races(t, chunks=chunks)
        assert as_dict(r) == want


def test_many_batches():
    # > 1000 tiny batches with ragged sizes: batch discovery at every position class
    rng = np.random.default_rng(3)
    parts = []
    for g in range(3):
        for b in range(40):
            for w in range(12):
                m = int(rng.integers(1, 70))
                e = np.empty(m, dtype=tg.EVENT_DTYPE)
                e["tid"] = rng.integers(0, 256, m)
                e["addr"] = rng.integers(0, 64, m).astype(np.uint64) << np.uint64(2)
                e["meta"] = tg.pack_meta(rng.choice(4, m, p=[.85, .05, .05, .05]), 2, w, b, g)
                parts.append(e)
    ev = np.concatenate(parts)
    t = tg.Trace("many", ev, 2, 128, 32, 64, 0)
    assert t.batch_count() == 3 * 40 * 12
    r, _ = gpu_races(t)
    assert as_dict(r) == oracle_dict(t)


def test_host_entry_point_matches_device_path():
    t = tg.cfg2(True, n=128, steps=3)
    c = hr.Checker.for_trace(t)
    c.reset()
    r = c.check_host(t.events)
    assert as_dict(r) == oracle_dict(t)
    c.close()


def test_multiword_accesses():
    ev = np.empty(3, dtype=tg.EVENT_DTYPE)
    ev[0] = (8, 0, tg.pack_meta(tg.WRITE, 3, 0, 0, 0))          # words 2,3
    ev[1] = (0, 1, tg.pack_meta(tg.READ, 4, 0, 0, 0))           # words 0..3
    ev[2] = (16, 40, tg.pack_meta(tg.READ, 0, 0, 0, 0))         # byte access -> word 4
    t = tg.Trace("mw", ev, 1, 64, 32, 8, 0)
    r, st = gpu_races(t)
    assert as_dict(r) == oracle_dict(t) == {2: 1, 3: 1}
    assert st["checked"] == 2 + 4 + 1


@pytest.mark.parametrize("bad", ["unsorted", "tid", "addr", "shared_addr", "size", "g255"])
def test_bad_trace_is_reported_and_sticky(bad):
    t = tg.cfg1("post_init")
    ev = t.events.copy()
    if bad == "unsorted":
        ev = ev[::-1].copy()
    elif bad == "tid":
        ev["tid"][5] = 10_000
    elif bad == "addr":
        ev["addr"][7] = 4 * 1000
    elif bad == "shared_addr":
        ev["addr"][3] = (np.uint64(1) << np.uint64(63)) | np.uint64(4 * 40)
    elif bad == "size":
        ev["meta"][9] |= np.uint32(5 << 2)
    elif bad == "g255":
        ev["meta"][-1] = (ev["meta"][-1] & np.uint32(0x00FFFFFF)) | np.uint32(255 << 24)
    tb = tg.Trace("bad", ev, t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    c = hr.Checker.for_trace(tb)
    d = hr.events_to_device(tb.events)
    c.replay(d)
    with pytest.raises(hr.HiraceError) as e:
        c.collect()
    assert e.value.status == -6
    with pytest.raises(hr.HiraceError):
        c.replay(d)                      # sticky
    c.reset()                            # reset clears it
    good = hr.events_to_device(t.events)
    c.replay(good)
    assert as_dict(c.collect()) == oracle_dict(t)
    c.close()


def test_grid_epoch_rebase_keeps_races():
    t = tg.listing2(1, 64)
    c = hr.Checker.for_trace(t)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    for _ in range(600):                 # wraps the 8-bit grid epoch twice -> rebase sweeps
        c.barrier()
    r = c.collect()
    assert as_dict(r) == {0: CLS["BLOCK"]}
    c.close()


def test_report_buffer_counts_every_class_transition():
    t = tg.cfg2(True, n=64, steps=2)
    c = hr.Checker.for_trace(t, report_capacity=16)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    r = c.collect()
    assert as_dict(r) == oracle_dict(t)      # collection is lossless even past capacity
    st = c.stats()
    assert st["dropped_reports"] >= len(r) - 16
    c.close()


def _fused(trace, cap=1 << 20):
    c = hr.Checker.for_trace(trace)
    c.reset()
    d = hr.events_to_device(trace.events)
    out = torch.zeros(max(cap, 1) * 16, dtype=torch.uint8, device="cuda")
    tot = torch.zeros(1, dtype=torch.int64, device="cuda")
    c.check_device(d, out, cap, tot)
    torch.cuda.synchronize()
    assert c.sync() == 0
    n = int(tot.item())
    recs = out.cpu().numpy().view(hr.RACE_DTYPE)[: min(n, cap)]
    c.close()
    return n, recs


@pytest.mark.parametrize("make", [lambda: tg.cfg1("post_init"), lambda: tg.cfg2(True, n=128, steps=3),
                                  lambda: tg.cfg4("B", 6, 128, 34), lambda: tg.listing5(40, 1, 64),
                                  lambda: tg.cfg2(False, n=64, steps=2)])
def test_fused_check_device_matches_oracle(make):
    t = make()
    n, recs = _fused(t)
    want = oracle_dict(t)
    assert n == len(want)
    assert as_dict(recs) == want
    assert bool(np.all(recs["key"][1:] > recs["key"][:-1]))


def test_collect_with_small_capacity_reports_total():
    t = tg.cfg2(True, n=128, steps=2)
    want = oracle_dict(t)
    n, recs = _fused(t, cap=100)
    assert n == len(want) and len(recs) == 100
    keys = sorted(want)[:100]
    assert recs["key"].tolist() == keys
    c = hr.Checker.for_trace(t)
    c.replay(hr.events_to_device(t.events))
    r = c.collect(cap=10)           # grows the buffer and retries
    assert as_dict(r) == want
    c.close()


@pytest.mark.parametrize("kind", ["bfs", "cc"])
@pytest.mark.parametrize("racy", [False, True])
def test_cfg3_graph_kernels_vs_oracle(kind, racy):
    # RMAT scale 14 (16K vertices, hubs of degree ~1e3): hot words, atomics, plain R/W races
    t = tg.cfg3(kind, racy, scale=14, edge_factor=16)
    want = oracle_dict(t)
    assert bool(want) == racy
    for seed in (None, 0, 1):
        ts = t if seed is None else tg.Trace(t.name, tg._shuffle_within_batches(t.events, seed), t.grid_blocks,
                                              t.block_threads, t.warp_size, t.global_words, t.smem_words)
        r, st = gpu_races(ts)
        assert as_dict(r) == want
        assert st["checked"] == t.n


@pytest.mark.slow
@pytest.mark.parametrize("racy", [False, True])
def test_cfg3_full_rmat20_bfs_vs_oracle(racy):
    # BASELINE configs[2]: RMAT-20 (1,048,576 vertices, ~3.1e7 CSR entries), BFS, ~7e7-1e8 events
    t = tg.cfg3("bfs", racy)
    assert t.n > 6e7
    want = oracle_dict(t)
    n, recs = _fused(t, cap=max(1, len(want)) + 16)
    assert n == len(want)
    assert as_dict(recs) == want
    _both_modes(t, want)


def _oracle_all_cores(t):
    k, c, _ = oracle.races_parallel(t.events, t.block_threads, t.warp_size)
    return {int(a): int(b) for a, b in zip(k, c)}


def _both_modes(t, want):
    """The check in both replay strategies (include/hirace.h hirace_replay_mode) == want."""
    for mode in (hr.REPLAY_WINDOW, hr.REPLAY_BATCH):
        c = hr.Checker.for_trace(t)
        c.set_replay_mode(mode)
        c.reset()
        d = hr.events_to_device(t.events)
        cap = len(want) + 1024
        out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        c.check_device(d, out, cap, tot)
        torch.cuda.synchronize()
        assert c.sync() == 0
        n = int(tot.item())
        recs = out.cpu().numpy().view(hr.RACE_DTYPE)[:n]
        assert n == len(want), mode
        assert as_dict(recs) == want, mode
        assert c.stats()["checked"] == word_accesses(t)
        del d, out
        c.close()
        torch.cuda.empty_cache()


def test_cfg5_medium_vs_oracle_both_modes():
    # 2^28 tracked words, 8192 blocks x 256 threads, 32 batches: ~1.3e8 events; the whole trace
    # through the all-core oracle (oracle/oracle_par.c), and the construction
    t = tg.cfg5(grid_blocks=8192, words_log2=28)
    assert t.n > 1e8
    want = _oracle_all_cores(t)
    assert want == {w: CLS[c] for w, c in t.info["expected"].items()}
    _both_modes(t, want)


@pytest.mark.slow
def test_cfg5_full_1e9_vs_oracle_both_modes():
    # BASELINE configs[4] on one GPU: 2^32 tracked words (32 GiB shadow), 1.07e9 events (17 GB);
    # GPU race set == the oracle's on the WHOLE trace (all host cores, address-sharded)
    t = tg.cfg5()
    assert t.n > 1.07e9
    want = _oracle_all_cores(t)
    assert want == {w: CLS[c] for w, c in t.info["expected"].items()}
    _both_modes(t, want)


@pytest.mark.slow
@pytest.mark.parametrize("racy", [False, True])
def test_cfg3_full_rmat20_cc_vs_oracle(racy):
    # BASELINE configs[2], connected components (2 label-propagation kernels) on RMAT-20
    t = tg.cfg3("cc", racy)
    want = _oracle_all_cores(t)
    assert bool(want) == racy
    _both_modes(t, want)


# ---- relaxed read-vs-atomic policy (reading R2b) ----------------

def _relaxed(t, seeds=(None, 0, 1)):
    want = {int(a): int(b) for a, b in zip(*oracle.races_of(t, hr.POLICY_RELAXED_READ_ATOMIC)[:2])}
    c = hr.Checker.for_trace(t, policy=hr.POLICY_RELAXED_READ_ATOMIC)
    for seed in seeds:
        ts = t if seed is None else tg.Trace(t.name, tg._shuffle_within_batches(t.events, seed), t.grid_blocks,
                                              t.block_threads, t.warp_size, t.global_words, t.smem_words)
        r, _ = gpu_races(ts, checker=c)
        assert as_dict(r) == want, seed
    c.close()
    return want


@pytest.mark.parametrize("chunk", range(2))
def test_relaxed_policy_random_tiny_vs_oracle(chunk):
    for seed in range(chunk * 250, (chunk + 1) * 250):
        _relaxed(tg.random_tiny(seed, max_events=40, probs=(.35, .15, .25, .25)), seeds=(None, seed))


def test_relaxed_policy_dense_atomics_vs_oracle():
    rng = np.random.default_rng(12)
    differ = 0
    for it in range(20):
        nb, bs, ws = int(rng.integers(1, 6)), 64, 32
        n = int(rng.integers(500, 20000))
        ev = np.empty(n, dtype=tg.EVENT_DTYPE)
        nkeys = int(rng.integers(1, 50))
        ev["tid"] = rng.integers(0, nb * bs, n)
        ev["addr"] = rng.integers(0, nkeys, n).astype(np.uint64) << np.uint64(2)
        kinds = rng.choice(4, n, p=[0.6, 0.002, 0.15, 0.248])
        ev["meta"] = tg.pack_meta(kinds, 2, rng.integers(0, 3, n), rng.integers(0, 3, n), rng.integers(0, 3, n))
        t = tg.Trace("dense", tg.sort_by_batch(ev), nb, bs, ws, nkeys, nkeys)
        differ += _relaxed(t, seeds=(None,)) != oracle_dict(t)
    assert differ > 0


@pytest.mark.parametrize("kind", ["bfs", "cc"])
def test_relaxed_policy_cfg3_graph_kernels(kind):
    # graph kernels mix plain reads of dist/labels with atomicMin: the policy changes the verdict
    t = tg.cfg3(kind, True, scale=14, edge_factor=16)
    _relaxed(t)


def test_relaxed_policy_cfg5_small_and_switch_on_one_context():
    # config-5 mix (App. C): its injected GRID patterns are half AB/AB, half R vs AG; under the
    # relaxed policy the R-vs-AG half is not a race (oracle: 129 flagged strict, 107 relaxed)
    t = tg.cfg5(grid_blocks=64, words_log2=20, npatterns=256)
    c = hr.Checker.for_trace(t)
    got = []
    for pol in (0, 1, 0, 1):
        c.set_policy(pol)
        r, _ = gpu_races(t, checker=c)
        want = {int(a): int(b) for a, b in zip(*oracle.races_of(t, pol)[:2])}
        assert as_dict(r) == want, pol
        got.append(len(want))
    c.close()
    assert got[0] > got[1]
