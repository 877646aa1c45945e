"""GPU parity of the compact 4-byte shadow (hirace_shadow_alloc_compact) with
the oracle: the same bar as tests/test_gpu_parity.py (flagged (key, class) set bit-exact, any
interleaving), through the same C-ABI entry points, on compact contexts.  Also: the epoch-limit
contract (a batch beyond the declared limits raises CLOCK_OVERFLOW and is not checked), the
halved footprint, and that the 8-byte-only entry points refuse a compact context.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg
from tests.helpers import expand_expected, listing_trace, load_golden

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


def compact_races(trace, fused=False, policy=0, chunks=1):
    c = hr.Checker.for_trace(trace, compact=True, policy=policy)
    assert c.rec_bytes == 4
    c.reset()
    d = hr.events_to_device(trace.events)
    if fused:
        cap = 1 << 20
        out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        c.check_device(d, out, cap, tot)
        torch.cuda.synchronize()
        assert c.sync() == 0
        n = int(tot.item())
        r = out.cpu().numpy().view(hr.RACE_DTYPE)[:n]
    else:
        bounds = np.linspace(0, trace.n, chunks + 1).astype(np.int64)
        for lo, hi in zip(bounds[:-1], bounds[1:]):
            if hi > lo:
                c.replay_ptr(d.data_ptr() + 16 * int(lo), int(hi - lo))
        r = c.collect()
    st = c.stats()
    c.close()
    return r, st


def _shuffled(t, seed):
    if seed is None:
        return t
    return tg.Trace(t.name, tg._shuffle_within_batches(t.events, seed), t.grid_blocks, t.block_threads, t.warp_size,
                    t.global_words, t.smem_words)


@pytest.mark.parametrize("entry", load_golden("listings.json")["cases"],
                         ids=lambda e: e["case"] + "-" + "-".join(f"{k}{v}" for k, v in e["params"].items()))
def test_compact_listings(entry):
    for seed in (None, 0, 1):
        t = listing_trace(entry["case"], entry["params"], shuffle_seed=seed)
        r, _ = compact_races(t)
        assert as_dict(r) == expand_expected(entry["expected"]), entry["cite"]


@pytest.mark.parametrize("chunk", range(4))
def test_compact_random_tiny_vs_oracle(chunk):
    for seed in range(chunk * 100, (chunk + 1) * 100):
        t = tg.random_tiny(seed)
        r, st = compact_races(t)
        assert as_dict(r) == oracle_dict(t), seed


@pytest.mark.parametrize("make", [
    lambda: tg.cfg1("post_init"), lambda: tg.cfg1(None), lambda: tg.cfg1("post_init", block_threads=64),
    lambda: tg.cfg2(True, n=128, steps=3), lambda: tg.cfg2(False, n=128, steps=3),
    lambda: tg.cfg4("G", 8, 128, 34), lambda: tg.cfg4("B", 8, 128, 34), lambda: tg.cfg4(None, 8, 128, 34),
    lambda: tg.cfg3("bfs", True, scale=14), lambda: tg.cfg3("bfs", False, scale=14),
    lambda: tg.cfg3("cc", True, scale=14),
])
def test_compact_configs_vs_oracle(make):
    t = make()
    want = oracle_dict(t)
    for seed in (None, 0):
        r, st = compact_races(_shuffled(t, seed))
        assert as_dict(r) == want
        assert st["checked"] >= t.n


def test_compact_fused_and_split_calls():
    t = tg.cfg2(True, n=256, steps=4)
    want = oracle_dict(t)
    r, _ = compact_races(t, fused=True)
    assert as_dict(r) == want
    assert bool(np.all(r["key"][1:] > r["key"][:-1]))
    r, _ = compact_races(t, chunks=5)
    assert as_dict(r) == want


def test_compact_relaxed_policy():
    t = tg.cfg3("bfs", True, scale=12)
    r, _ = compact_races(t, policy=hr.POLICY_RELAXED_READ_ATOMIC)
    assert as_dict(r) == oracle_dict(t, policy=1)


def test_compact_full_bench_config2():
    # BASELINE configs[1] at full size: 17.8M events, 32,768 WARP + 229,376 BLOCK shared keys
    t = tg.cfg2(True)
    r, st = compact_races(t, fused=True)
    d = as_dict(r)
    assert sum(1 for v in d.values() if v == 1) == 32768 and sum(1 for v in d.values() if v == 2) == 229376
    assert len(d) == 262144


@pytest.mark.slow
def test_compact_full_rmat20_bfs_vs_oracle():
    t = tg.cfg3("bfs", True)
    want = oracle_dict(t)
    r, _ = compact_races(t, fused=True)
    assert as_dict(r) == want


def test_compact_limits_contract():
    t = tg.cfg2(True, n=64, steps=4)           # g = 0..3, b = 0..1
    lim = hr.trace_epoch_limits(t.events)
    assert lim[0] == 3
    # declared limits one grid epoch short: batches of g = 3 are not checked and raise
    # CLOCK_OVERFLOW; races of the earlier epochs stay valid (PAPER.md L227 fn. 3)
    early = t.events[(t.events["meta"] >> 24) < 3]
    te = tg.Trace(t.name, early, t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    want = oracle_dict(te)
    assert want
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words,
                   compact=(2, lim[1], lim[2]))
    c.reset()
    cap = 1 << 16
    out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
    tot = torch.zeros(1, dtype=torch.int64, device="cuda")
    c.check_device(hr.events_to_device(t.events), out, cap, tot)
    torch.cuda.synchronize()
    assert c.sync() == -4
    n = int(tot.item())
    assert as_dict(out.cpu().numpy().view(hr.RACE_DTYPE)[:n]) == want
    with pytest.raises(hr.HiraceError):       # the error is sticky
        c.collect()
    c.close()


def test_compact_footprint_and_refusals():
    c8 = hr.Checker(1024, 256, 32, 1 << 20, 324)
    c4 = hr.Checker(1024, 256, 32, 1 << 20, 324, compact=(7, 1, 0))
    assert c4.shadow_bytes * 2 == c8.shadow_bytes
    with pytest.raises(hr.HiraceError):       # inline hooks need the 8-byte record
        c4.dev_ctx()
    with pytest.raises(hr.HiraceError):       # host grid barrier (inline mode) likewise
        c4.barrier()
    c8.close()
    c4.close()
    with pytest.raises(hr.HiraceError):       # 2^24 threads + 4/4/2 epochs: 34 bits
        hr.Checker(65536, 256, 32, 1 << 20, 0, compact=(3, 3, 1))
    with pytest.raises(hr.HiraceError):       # beyond the event fields
        hr.Checker(4, 32, 32, 64, 0, compact=(255, 0, 0))


# ---- report-buffer collection (sort + unique of the reports; scan fallback) ----

@pytest.mark.parametrize("compact", [False, True])
@pytest.mark.parametrize("make", [
    lambda: tg.cfg1("post_init"), lambda: tg.cfg1("post_init", block_threads=64),
    lambda: tg.cfg3("bfs", True, scale=14), lambda: tg.cfg4("G", 8, 128, 34), lambda: tg.cfg4("B", 8, 128, 34),
    lambda: tg.cfg2(True, n=128, steps=3),   # 16K flagged words + upgrades: > sort cap -> scan fallback
    lambda: tg.cfg2(False, n=64, steps=2),   # no race: empty report buffer
])
def test_report_collect_matches_oracle(monkeypatch, make, compact):
    monkeypatch.setenv("HIRACE_COLLECT", "reports")
    t = make()
    want = oracle_dict(t)
    for seed in (None, 1):
        ts = _shuffled(t, seed)
        c = hr.Checker.for_trace(ts, compact=compact)
        c.reset()
        d = hr.events_to_device(ts.events)
        c.replay(d)
        got = c.collect()                    # standalone: k_collect_reports, then the scan stands down
        assert as_dict(got) == want
        assert bool(np.all(got["key"][1:] > got["key"][:-1]))
        c.reset()
        cap = 1 << 20
        out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        c.check_device(d, out, cap, tot)     # fused: the replay kernel skips its scan
        torch.cuda.synchronize()
        assert c.sync() == 0
        n = int(tot.item())
        recs = out.cpu().numpy().view(hr.RACE_DTYPE)[:n]
        assert as_dict(recs) == want
        # the same records (class, g*) as the shadow scan
        monkeypatch.setenv("HIRACE_COLLECT", "scan")
        scan = c.collect()
        monkeypatch.setenv("HIRACE_COLLECT", "reports")
        assert np.array_equal(scan["key"], recs["key"]) and np.array_equal(scan["cls_and_epoch"], recs["cls_and_epoch"])
        c.close()


def test_report_collect_overflow_falls_back_to_scan(monkeypatch):
    monkeypatch.setenv("HIRACE_COLLECT", "reports")
    t = tg.cfg3("bfs", True, scale=12)
    want = oracle_dict(t)
    assert len(want) > 8
    c = hr.Checker.for_trace(t, report_capacity=4)   # the buffer overflows: reports do not cover
    c.reset()
    c.replay(hr.events_to_device(t.events))
    assert as_dict(c.collect()) == want
    assert c.stats()["dropped_reports"] > 0
    c.close()


def test_compact_cfg5_medium_by_construction():
    """Config 5 shape at 2^28 words and 2^21 threads fits the compact record (5 + 2 + 2 + 1 + 21
    bits): 1.3e8 events, report-buffer collect on a 1 GiB compact shadow; the flagged set is known
    by construction (tracegen; pinned against the oracle at reduced scale in the CPU suite)."""
    from tests.helpers import CLS
    t = tg.cfg5(grid_blocks=8192, words_log2=28)
    want = {w: CLS[c] for w, c in t.info["expected"].items()}
    r, st = compact_races(t, fused=True)
    assert as_dict(r) == want
    assert st["dropped_reports"] == 0


def test_compact_host_entry_point():
    t = tg.cfg4("B", 8, 128, 34)
    c = hr.Checker.for_trace(t, compact=True)
    c.reset()
    got = as_dict(c.check_host(t.events))
    c.close()
    assert got == oracle_dict(t)
