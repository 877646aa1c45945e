"""Selective tracking (include/hirace.h hirace_set_filter; PAPER.md L245
"Individual threads or test data addresses may have their instrumentation enabled or disabled
dynamically ... tracking only representative threads").  The GPU result under a filter must
equal the oracle on exactly the selected accesses (selected in numpy here, by the documented
predicate), in replay and in inline mode.
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
from paper_conf_sc_jacobsonbg24_b200 import examples as ex  # noqa: E402


def as_dict(r):
    return {int(k): int(c) & 0xFF for k, c in zip(r["key"], r["cls_and_epoch"])}


def selected(t, mask, match, spaces, lo, hi):
    ev = t.events
    sh = (ev["addr"] & tg.SHARED_BIT) != 0
    elem = (ev["addr"] & ~tg.SHARED_BIT) >> np.uint64(t.granularity_log2)
    keep = ((ev["tid"] & np.uint32(mask)) == match) & np.where(
        sh, (spaces & 2) != 0, ((spaces & 1) != 0) & (elem >= np.uint64(lo)) & (elem < np.uint64(hi)))
    return tg.Trace(t.name, ev[keep], t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words,
                    granularity_log2=t.granularity_log2)


FILTERS = [(0, 0, 3, 0, 2**64 - 1), (31, 0, 3, 0, 2**64 - 1), (1, 1, 3, 0, 2**64 - 1), (0, 0, 1, 0, 2**64 - 1),
           (0, 0, 2, 0, 2**64 - 1), (0, 0, 3, 2, 6), (3, 2, 1, 1, 5)]


@pytest.mark.parametrize("flt", FILTERS)
@pytest.mark.parametrize("compact", [False, True])
def test_filter_random_tiny_vs_oracle_on_selection(flt, compact):
    for seed in range(120):
        t = tg.random_tiny(seed) if seed % 2 else tg.random_tiny_bytes(seed, seed % 3)
        c = hr.Checker.for_trace(t, compact=compact)
        c.reset()
        c.set_filter(*flt)
        c.replay(hr.events_to_device(t.events))
        got = as_dict(c.collect())
        st = c.stats()
        c.close()
        s = selected(t, *flt)
        assert got == oracle.races_dict(s), (flt, seed)
        szl = (s.events["meta"] >> 2) & 7
        g = t.granularity_log2
        assert st["checked"] == int(np.where(szl <= g, 1, 1 << np.maximum(szl.astype(np.int64) - g, 0)).sum())


def test_filter_representative_lanes_on_config2():
    # lane 0 of every warp only: one representative per warp (a "symmetric group")
    t = tg.cfg2(True, n=128, steps=3)
    c = hr.Checker.for_trace(t)
    c.reset()
    c.set_filter(31, 0)
    c.replay(hr.events_to_device(t.events))
    got = as_dict(c.collect())
    c.close()
    assert got == oracle.races_dict(selected(t, 31, 0, 3, 0, 2**64 - 1))
    assert len(got) < len(oracle.races_dict(t))


def test_filter_inline_stencil_spaces():
    # the racy stencil's races are all in shared memory: tracking only global memory finds none,
    # tracking only shared memory finds all of them
    n, steps = 128, 3
    t = tg.cfg2(True, n=n, steps=steps)
    want = oracle.races_dict(t)
    buf = torch.rand(2 * n * n, device="cuda")
    for spaces, expect in ((1, {}), (2, want)):
        c = hr.Checker.for_trace(t)
        c.reset()
        c.set_filter(0, 0, spaces)
        ex.stencil(c, buf, n, steps, True)
        assert as_dict(c.collect()) == expect
        c.close()


def test_filter_rejects_bad_arguments():
    c = hr.Checker(4, 64, 32, 64, 16)
    for bad in ((1, 2, 3, 0, 10), (0, 0, 4, 0, 10), (0, 0, 3, 5, 4)):
        with pytest.raises(hr.HiraceError):
            c.set_filter(*bad)
    c.close()
