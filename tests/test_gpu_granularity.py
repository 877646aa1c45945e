"""GPU parity at element granularity 1 and 2 bytes (hirace_config.granularity_log2 0 / 1; one
shadow record per element, "for each element"; reading R8) against the
oracle at the same granularity (itself pinned by brute force and closed forms in
tests/test_oracle_pins.py), for the 8-byte and the compact record.
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


def as_dict(r):
    return {int(k): int(c) & 0xFF for k, c in zip(r["key"], r["cls_and_epoch"])}


def gpu(t, compact=False):
    c = hr.Checker.for_trace(t, compact=compact)
    c.reset()
    if t.n:
        c.replay(hr.events_to_device(t.events))
    r = c.collect()
    st = c.stats()
    c.close()
    return as_dict(r), st


@pytest.mark.parametrize("compact", [False, True])
@pytest.mark.parametrize("gran", [0, 1, 2])
def test_random_byte_accesses_vs_oracle(gran, compact):
    for seed in range(150):
        t = tg.random_tiny_bytes(seed, gran)
        want = oracle.races_dict(t)
        got, st = gpu(t, compact)
        assert got == want, (gran, seed)
        szl = (t.events["meta"] >> 2) & 7
        assert st["checked"] == int(np.where(szl <= gran, 1, 1 << np.maximum(szl.astype(np.int64) - gran, 0)).sum())


def _char_rows(gran, racy):
    """One block of 64 threads writes a 64-byte char row (thread t -> byte t), then (after a
    __syncthreads unless racy) reads its right neighbour's byte."""
    n = 64
    ev = np.empty(2 * n, dtype=tg.EVENT_DTYPE)
    t = np.arange(n)
    ev["addr"][:n] = t.astype(np.uint64) | tg.SHARED_BIT
    ev["addr"][n:] = ((t + 1) % n).astype(np.uint64) | tg.SHARED_BIT
    ev["tid"][:n] = t
    ev["tid"][n:] = t
    ev["meta"][:n] = tg.pack_meta(1, 0, 0, 0, 0)
    ev["meta"][n:] = tg.pack_meta(0, 0, 0, 0 if racy else 1, 0)
    return tg.Trace("chars", tg.sort_by_batch(ev), 1, n, 32, 0, 16, granularity_log2=gran)


@pytest.mark.parametrize("racy", [False, True])
def test_char_array_false_sharing(racy):
    """Per-byte writes by different threads: at byte granularity only the racy read pattern is
    flagged (one race per byte); at word granularity four writers share every word, so every
    word is flagged even with the barrier."""
    for gran in (0, 1, 2):
        t = _char_rows(gran, racy)
        want = oracle.races_dict(t)
        got, _ = gpu(t)
        assert got == want
        if gran == 0:
            assert len(got) == (64 if racy else 0)
        if gran == 2:
            assert len(got) == 16


def test_wide_access_at_byte_granularity():
    # a 16-byte write covers 16 elements at byte granularity; another warp's byte read of one
    ev = np.empty(2, dtype=tg.EVENT_DTYPE)
    ev["addr"] = np.array([16, 21], np.uint64)
    ev["tid"] = [0, 40]
    ev["meta"] = tg.pack_meta(np.array([1, 0]), np.array([4, 0]), 0, 0, 0)
    t = tg.Trace("wide", ev, 1, 64, 32, 16, 0, granularity_log2=0)
    got, st = gpu(t)
    assert got == {21: 2} == oracle.races_dict(t)
    assert st["checked"] == 17


def test_sharded_entry_points_need_word_granularity():
    c = hr.Checker(4, 64, 32, 64, 16, granularity_log2=0)
    ev = torch.zeros(2, dtype=torch.int64, device="cuda")
    with pytest.raises(hr.HiraceError):
        c.bucket_wire(ev.view(1, 2), np.array([0, 1], np.uint32), 2, 0)
    c.close()
    with pytest.raises(hr.HiraceError):
        hr.Checker(4, 64, 32, 64, 16, granularity_log2=3)


def test_inline_hook_granularity_must_match_its_build():
    # the examples are built with the default inline element size (4-byte words): a context at
    # byte granularity disables their tracking and reports BAD_TRACE instead of mis-keying
    from paper_conf_sc_jacobsonbg24_b200 import examples as ex
    n, steps = 64, 2
    t = tg.cfg2(True, n=n, steps=steps)
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, granularity_log2=0)
    c.reset()
    buf = torch.rand(2 * n * n, device="cuda")
    ex.stencil(c, buf, n, steps, True)
    assert c.sync() == -6
    c.close()
