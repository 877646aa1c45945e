"""Degenerate and boundary inputs of the replay path (GPU, through the C-ABI): empty traces,
one event, the batch-count limit (HIRACE_MAX_BATCHES) and one beyond it, ragged chunk tails
at every length 1..65, and a single-thread grid."""
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


@pytest.mark.parametrize("compact", [False, True])
def test_empty_trace(compact):
    c = hr.Checker(4, 64, 32, 64, 16, compact=(0, 0, 0) if compact else None)
    c.reset()
    ev = torch.zeros(0, dtype=torch.uint8, device="cuda")
    c.replay(ev, 0)
    assert len(c.collect()) == 0
    out = torch.zeros(16, dtype=torch.uint8, device="cuda")
    tot = torch.full((1,), 7, dtype=torch.int64, device="cuda")
    c.check_device(ev, out, 1, tot, n=0)
    torch.cuda.synchronize()
    assert int(tot.item()) == 0 and c.sync() == 0
    assert len(c.check_host(np.empty(0, tg.EVENT_DTYPE))) == 0
    assert c.stats()["checked"] == 0
    c.close()


def test_single_event_and_single_thread_grid():
    ev = np.empty(1, dtype=tg.EVENT_DTYPE)
    ev[0] = (4, 0, tg.pack_meta(tg.WRITE, 2, 0, 0, 0))
    t = tg.Trace("one", ev, 1, 1, 1, 4, 0)
    c = hr.Checker.for_trace(t)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    assert len(c.collect()) == 0 and c.stats()["checked"] == 1
    c.close()


def test_ragged_chunk_tails():
    # batches of every length 1..65 (partial last chunk of 32 lanes, one and two chunks)
    rng = np.random.default_rng(9)
    parts = []
    for m in range(1, 66):
        e = np.empty(m, dtype=tg.EVENT_DTYPE)
        e["tid"] = rng.integers(0, 128, m)
        e["addr"] = rng.integers(0, 16, m).astype(np.uint64) << np.uint64(2)
        e["meta"] = tg.pack_meta(rng.choice(4, m), 2, m % 3, 0, m)
        parts.append(e)
    t = tg.Trace("ragged", tg.sort_by_batch(np.concatenate(parts)), 2, 64, 32, 16, 0)
    for compact in (False, True):
        c = hr.Checker.for_trace(t, compact=compact)
        c.reset()
        c.replay(hr.events_to_device(t.events))
        assert as_dict(c.collect()) == oracle.races_dict(t)
        assert c.stats()["checked"] == t.n
        c.close()


def _batches(nb):
    ev = np.empty(nb, dtype=tg.EVENT_DTYPE)
    k = np.arange(nb)
    ev["tid"] = k % 64
    ev["addr"] = ((k % 8) << 2).astype(np.uint64)
    # nb distinct increasing (g, b, w): w fastest (9 bits), then b (10 bits)
    ev["meta"] = tg.pack_meta(tg.WRITE, 2, k % 512, (k // 512) % 1024, k // (512 * 1024))
    return tg.Trace("nb", ev, 1, 64, 32, 8, 0)


def test_batch_count_limit():
    t = _batches(hr.hirace.MAX_BATCHES)          # exactly the limit: accepted
    c = hr.Checker.for_trace(t)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    assert as_dict(c.collect()) == oracle.races_dict(t)
    c.close()
    t = _batches(hr.hirace.MAX_BATCHES + 1)      # one more: BAD_TRACE, sticky
    c = hr.Checker.for_trace(t)
    c.reset()
    c.replay(hr.events_to_device(t.events))
    with pytest.raises(hr.HiraceError) as e:
        c.collect()
    assert e.value.status == -6
    c.close()
