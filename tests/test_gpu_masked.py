"""GPU parity of the partial-mask __syncwarp(mask) replay (hirace_set_warp_syncs; SURVEY §8(f)
f3, reading R20) against the masked oracle (oracle.races_masked),
element by element: random programs with random masks (both policies, both record layouts,
shuffled batches, split calls), the hand cases of tests/golden/masked.json, tiled reductions
from small to 1M threads, resets, the epoch reset, and the error paths."""
import numpy as np
import pytest

import oracle
import tracegen as tg
from tests.helpers import CLS, SHARED, load_golden
from tests.test_masked_oracle import _golden_trace

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402


def _gpu(t, policy=0, compact=False, chunks=1, checker=None, history_slots=0, reset=True):
    c = checker or hr.Checker.for_trace(t, policy=policy, compact=compact, history_slots=history_slots)
    try:
        if reset:
            c.reset()
        if t.n:
            d = hr.events_to_device(t.events)
            bounds = np.linspace(0, t.n, chunks + 1).astype(np.int64)
            for lo, hi in zip(bounds[:-1], bounds[1:]):
                if hi > lo:
                    c.replay_ptr(d.data_ptr() + 16 * int(lo), int(hi - lo))
        r = c.collect()
        return {int(k): (int(x) & 255, int(x) >> 8) for k, x in zip(r["key"], r["cls_and_epoch"])}, c.stats()
    finally:
        if checker is None:
            c.close()


def _want(t, policy=0):
    k, c, g = oracle.races_masked(t.events, t.block_threads, t.warp_size, t.warp_syncs, policy)
    return {int(a): (int(b), int(x)) for a, b, x in zip(k, c, g)}


def _with(t, events):
    return tg.Trace(t.name, events, t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words,
                    dict(t.info), warp_syncs=t.warp_syncs)


@pytest.mark.parametrize("chunk", range(4))
def test_random_masked_programs(chunk):
    for seed in range(chunk * 150, (chunk + 1) * 150):
        t = tg.random_tiny_masked(seed)
        want = _want(t)
        got, st = _gpu(t)
        assert got == want, t.name
        assert st["checked"] == t.n
        ts = _with(t, tg._shuffle_within_batches(t.events, seed))
        assert _gpu(ts)[0] == want, t.name


def test_random_masked_programs_relaxed_policy():
    for seed in range(200):
        t = tg.random_tiny_masked(seed)
        assert _gpu(t, policy=hr.POLICY_RELAXED_READ_ATOMIC)[0] == _want(t, 1), t.name


def test_random_masked_programs_compact_and_split_calls():
    for seed in range(200):
        t = tg.random_tiny_masked(seed)
        want = _want(t)
        assert _gpu(t, compact=True)[0] == want, t.name
        assert _gpu(t, chunks=3)[0] == want, t.name


def test_partial_masks_change_verdicts_on_gpu():
    """the GPU sees what the plain (full-mask) reading cannot"""
    differ = 0
    for seed in range(150):
        t = tg.random_tiny_masked(seed)
        got = _gpu(t)[0]
        plain = {int(a): int(b) for a, b in zip(*oracle.races_of(t)[:2])}
        differ += {k: v[0] for k, v in got.items()} != plain
    assert differ >= 10


@pytest.mark.parametrize("case", [c for c in load_golden("masked.json")["cases"] if c["expected"] is not None],
                         ids=lambda c: c["name"])
def test_golden_cases(case):
    t = _golden_trace(case)
    got = {k: v[0] for k, v in _gpu(t)[0].items()}
    assert got == {int(k): CLS[v] for k, v in case["expected"].items()}


def test_access_outside_its_sync_mask_is_bad_trace():
    case = [c for c in load_golden("masked.json")["cases"] if c["expected"] is None][0]
    t = _golden_trace(case)
    with pytest.raises(hr.HiraceError) as e:
        _gpu(t)
    assert e.value.status == -6


@pytest.mark.parametrize("nb,bs,tile", [(2, 64, 4), (8, 128, 8), (16, 256, 16), (4, 64, 32)])
@pytest.mark.parametrize("racy", [None, "half_mask", "pair"])
@pytest.mark.parametrize("shuffle", [None, 3])
def test_tiled_reductions(nb, bs, tile, racy, shuffle):
    t = tg.tiled_reduce(nb, bs, tile, 3, racy, shuffle_seed=shuffle)
    want = _want(t)
    got, st = _gpu(t)
    assert got == want
    assert st["checked"] == t.n
    assert (len(want) == 0) == (racy is None)


@pytest.mark.parametrize("racy", [None, "half_mask", "pair"])
def test_tiled_reduction_million_threads(racy):
    """4096 blocks x 256 threads, tile 8, 2 rounds: ~2.4e7 events, 5e5 log records"""
    t = tg.tiled_reduce(4096, 256, 8, 2, racy)
    want = oracle.races_masked(t.events, t.block_threads, t.warp_size, t.warp_syncs)
    got, st = _gpu(t, history_slots=1 << 22)
    assert {k: v[0] for k, v in got.items()} == {int(a): int(b) for a, b in zip(want[0], want[1])}
    assert st["checked"] == t.n
    if racy == "half_mask":
        assert len(got) == 4096 * 128


def test_reset_clears_the_history():
    """a second check of the same trace on the same context gives the same verdict (stale
    history from the first check must not leak into it)"""
    for seed in range(40):
        t = tg.random_tiny_masked(seed)
        c = hr.Checker.for_trace(t)
        try:
            a = _gpu(t, checker=c)[0]
            b = _gpu(t, checker=c)[0]
        finally:
            c.close()
        assert a == b == _want(t), t.name


def test_epoch_reset_mode():
    for seed in range(60):
        t = tg.random_tiny_masked(seed)
        c = hr.Checker.for_trace(t)
        c.set_reset_mode(hr.RESET_EPOCH)
        c.set_warp_syncs(t.warp_syncs)
        try:
            for _ in range(3):
                assert _gpu(t, checker=c)[0] == _want(t), t.name
        finally:
            c.close()


def test_removing_the_log_restores_the_plain_reading():
    t = tg.tiled_reduce(4, 64, 8, 2, "half_mask")
    c = hr.Checker.for_trace(t)
    try:
        assert len(_gpu(t, checker=c)[0]) == 4 * 32
        c.set_warp_syncs(None)
        assert _gpu(t, checker=c)[0] == {}
    finally:
        c.close()


def test_history_overflow_is_reported():
    t = tg.tiled_reduce(64, 256, 8, 1, None)
    c = hr.Checker.for_trace(t, history_slots=64)
    try:
        with pytest.raises(hr.HiraceError) as e:
            _gpu(t, checker=c)
        assert e.value.status == -8
    finally:
        c.close()


@pytest.mark.parametrize("bad", ["unsorted", "zero_w", "zero_mask", "wide_mask", "warp"])
def test_bad_logs_are_rejected(bad):
    t = tg.tiled_reduce(2, 64, 8, 1, "half_mask")
    sy = t.warp_syncs.copy()
    if bad == "unsorted":
        sy = sy[::-1].copy()
    elif bad == "zero_w":
        sy["meta"][0] = 0
    elif bad == "zero_mask":
        sy["mask"][0] = 0
    elif bad == "wide_mask":
        t = tg.tiled_reduce(2, 16, 4, 1, "half_mask", warp_size=8)
        sy = t.warp_syncs.copy()
        sy["mask"][0] = 1 << 8
    else:
        sy["warp"][-1] = 10 ** 6
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    try:
        with pytest.raises(hr.HiraceError) as e:
            c.set_warp_syncs(sy)
        assert e.value.status == -6
    finally:
        c.close()


def test_sharded_and_inline_entry_points_refuse_a_log():
    t = tg.tiled_reduce(2, 64, 8, 1, "half_mask")
    c = hr.Checker.for_trace(t)
    try:
        with pytest.raises(hr.HiraceError) as e:
            c.dev_ctx()
        assert e.value.status == -1
        d = hr.events_to_device(t.events)
        with pytest.raises(hr.HiraceError):
            c.bucket(d, t.n, 2, 0, torch.empty_like(d))
    finally:
        c.close()


def test_window_mode_replays_batch_major_with_a_log():
    t = tg.tiled_reduce(8, 128, 8, 2, "pair")
    c = hr.Checker.for_trace(t)
    try:
        c.set_replay_mode(hr.REPLAY_WINDOW, 6)
        c.set_warp_syncs(t.warp_syncs)
        assert not c.window_active
        assert _gpu(t, checker=c)[0] == _want(t)
    finally:
        c.close()


def _broadcast_trace(nwords, lanes_mask, writer_lane):
    """one warp of 32 lanes: every lane reads words 0..nwords-1 (w = 0); a partial sync of
    lanes_mask; writer_lane writes every word (w = 1).  Readers outside the mask race with the
    write; the 32 (lane, read) pairs per word overflow a slot's five entries into a spill block."""
    import numpy as np
    rows = [(wd, False, ln, tg.READ, 0, 0, 0) for wd in range(nwords) for ln in range(32)]
    rows += [(wd, False, writer_lane, tg.WRITE, 1, 0, 0) for wd in range(nwords)]
    ev = np.empty(len(rows), dtype=tg.EVENT_DTYPE)
    a = np.array(rows, dtype=np.int64)
    ev["addr"] = a[:, 0].astype(np.uint64) << np.uint64(2)
    ev["tid"] = a[:, 2]
    ev["meta"] = tg.pack_meta(a[:, 3], 2, a[:, 4], a[:, 5], a[:, 6])
    sy = tg.make_syncs([0], [lanes_mask], [1], [0], [0])
    return tg.Trace("bcast", tg.sort_by_batch(ev), 1, 32, 32, nwords, 0, warp_syncs=sy)


@pytest.mark.parametrize("mask,writer,expect_race", [(0x0000FFFF, 0, True), (0xFFFFFFFE, 31, True),
                                                     (0xFFFFFFFF, 0, False)])
def test_spilled_history_is_exact(mask, writer, expect_race):
    """32 readers per word exceed the slot's five (lane, class) entries: the spill block keeps the
    history exact (the writer after a sync of `mask`; a race iff some reader is outside it)"""
    t = _broadcast_trace(64, mask, writer)
    want = _want(t)
    assert bool(want) == expect_race
    for shuffle in (None, 1, 2):
        ts = t if shuffle is None else _with(t, tg._shuffle_within_batches(t.events, shuffle))
        assert _gpu(ts)[0] == want


def test_spill_pool_overflow_is_reported():
    t = _broadcast_trace(256, 0x0000FFFF, 0)
    c = hr.Checker.for_trace(t, history_slots=64)  # 64 slots -> 8 spill blocks for 256 words
    try:
        with pytest.raises(hr.HiraceError) as e:
            _gpu(t, checker=c)
        assert e.value.status == -8
    finally:
        c.close()


def test_random_masked_programs_with_wide_accesses():
    """8/16-byte accesses: the masked replay checks every covered word (k_replay_masked's word loop)"""
    for seed in range(300):
        t = tg.random_tiny_masked(seed, wide=True)
        assert _gpu(t)[0] == _want(t), t.name
        assert _gpu(t, compact=True)[0] == _want(t), t.name


def test_masked_replay_with_selective_tracking():
    """hirace_set_filter (f4) on the masked path: with shared memory deselected the verdict equals
    the oracle's on the global accesses alone (the partial syncs still order them)"""
    import numpy as np
    for seed in range(200):
        t = tg.random_tiny_masked(seed)
        c = hr.Checker.for_trace(t)
        try:
            c.set_filter(0, 0, 1)  # global memory only
            got = _gpu(t, checker=c)[0]
        finally:
            c.close()
        glob = (t.events["addr"] >> np.uint64(63)) == 0
        assert got == _want(_with(t, t.events[glob])), t.name
