"""Partial-mask __syncwarp(mask) in the INLINE hooks (
DESIGN.md R20): a native cooperative-groups tiled_partition<T> reduction with real
__syncwarp(tile mask) calls, checked by hirace::ws::on_access_ws / syncwarp / barrier_ws, against
the masked oracle on the trace of the same program (tracegen.tiled_reduce).  The inline sync
numbering is the order the warp reaches its syncs, not the generator's; the happens-before
relation, hence the race set, is the same."""
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
from paper_conf_sc_jacobsonbg24_b200 import examples as ex  # noqa: E402


def _run(t, tile, rounds, racy, history_slots=0, smem_tracking=True):
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    try:
        out = torch.zeros(t.global_words, dtype=torch.float32, device="cuda")
        ex.tiled(c, out, t.grid_blocks, t.block_threads, tile, rounds, racy,
                 history_slots or t.info.get("history_slots", 0), smem_tracking)
        torch.cuda.synchronize()
        return hr.races_to_dict(c.collect())
    finally:
        c.close()


@pytest.mark.parametrize("smem_tracking", [True, False])
@pytest.mark.parametrize("racy", [None, "half_mask", "pair"])
@pytest.mark.parametrize("nb,bs,tile,rounds", [(2, 64, 4, 2), (8, 128, 8, 3), (16, 256, 16, 2), (4, 64, 32, 2),
                                               (64, 256, 8, 2)])
def test_inline_tiled_reduction(racy, nb, bs, tile, rounds, smem_tracking):
    t = tg.tiled_reduce(nb, bs, tile, rounds, racy)
    want = oracle.races_masked_dict(t)
    assert _run(t, tile, rounds, racy, smem_tracking=smem_tracking) == want
    assert (len(want) == 0) == (racy is None)


def test_inline_without_the_sub_warp_hooks_misses_the_half_mask_race():
    """the plain inline hooks (full-mask reading) see no race in the half-mask program: the
    partial masks are what expose it (the replay and the oracle agree)"""
    t = tg.tiled_reduce(4, 64, 8, 2, "half_mask")
    assert oracle.races_dict(t) == {} and len(oracle.races_masked_dict(t)) == 4 * 32


def test_inline_history_overflow_is_reported():
    t = tg.tiled_reduce(64, 256, 8, 1, None)
    c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
    try:
        out = torch.zeros(t.global_words, dtype=torch.float32, device="cuda")
        ex.tiled(c, out, t.grid_blocks, t.block_threads, 8, 1, None, history_slots=64, smem_tracking=False)
        torch.cuda.synchronize()
        with pytest.raises(hr.HiraceError) as e:
            c.collect()
        assert e.value.status == -8
    finally:
        c.close()
