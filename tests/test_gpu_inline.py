"""Inline mode: native CUDA programs checked by the device hooks while they run
(hirace::on_access / hirace::barrier).  The race set of a data race is a
property of the program, not of the schedule, so the inline result must equal the oracle on
the trace generator's model of the same program (configs 1-4) and the closed forms."""
import numpy as np
import pytest

import oracle
import tracegen as tg
from tests.helpers import CLS, skey

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
from paper_conf_sc_jacobsonbg24_b200 import examples as ex  # noqa: E402


@pytest.fixture(autouse=True, params=[False, True], ids=["thread_hooks", "warp_hooks"])
def hooks(request):
    """Every inline test runs with the per-thread hooks and with the warp-aggregated ones
    (hirace::on_access_warp, libhirace_examples_agg.so)."""
    ex.use_aggregated_hooks(request.param)
    yield request.param
    ex.use_aggregated_hooks(False)


def odict(t):
    k, c, _ = oracle.races_of(t)
    return {int(a): int(b) for a, b in zip(k, c)}


def rdict(r):
    return {int(k): int(c) & 0xFF for k, c in zip(r["key"], r["cls_and_epoch"])}


@pytest.mark.parametrize("smem", [True, False])
@pytest.mark.parametrize("racy", [False, True])
@pytest.mark.parametrize("n,steps", [(128, 3), (512, 8)])
def test_inline_stencil(racy, n, steps, smem):
    t = tg.cfg2(racy, n=n, steps=steps)
    c = hr.Checker.for_trace(t)
    buf = torch.rand(2 * n * n, device="cuda")
    ex.stencil(c, buf, n, steps, racy, smem_shadow=smem)
    got = rdict(c.collect())
    want = odict(t)
    assert got == want
    if n == 512 and racy:
        assert sorted(np.bincount(list(got.values()), minlength=4).tolist()) == [0, 0, 32768, 229376]
    st = c.stats()
    c.close()
    assert st["dropped_reports"] == 0


@pytest.mark.parametrize("smem", [True, False])
@pytest.mark.parametrize("bs", [32, 64])
@pytest.mark.parametrize("racy", [0, 1, 2])
def test_inline_reduction(bs, racy, smem):
    t = tg.cfg1([None, "post_init", "level"][racy], block_threads=bs)
    c = hr.Checker.for_trace(t)
    out = torch.zeros(8, device="cuda")
    ex.reduce(c, out, bs, 8, racy, smem_shadow=smem)
    assert rdict(c.collect()) == odict(t)
    c.close()


@pytest.mark.parametrize("smem", [True, False])
@pytest.mark.parametrize("racy", [0, 1, 2])
def test_inline_multiphase_small(racy, smem):
    nb, phases = 6, 34
    t = tg.cfg4([None, "G", "B"][racy], nb, 256, phases)
    c = hr.Checker.for_trace(t)
    AB = torch.rand(4 * nb * 256, device="cuda")
    bar = torch.zeros(1, dtype=torch.int32, device="cuda")
    ex.multiphase(c, AB, nb, phases, racy, bar, smem_shadow=smem)
    assert rdict(c.collect()) == odict(t)
    c.close()


@pytest.mark.parametrize("racy", [1, 2])
def test_inline_multiphase_full_closed_form(racy):  # shared-variable shadows in shared memory
    nb, phases = 592, 64
    t_geom = dict(grid_blocks=nb, block_threads=256, warp_size=32, global_words=4 * nb * 256, smem_words=514)
    c = hr.Checker(**t_geom)
    AB = torch.rand(4 * nb * 256, device="cuda")
    bar = torch.zeros(1, dtype=torch.int32, device="cuda")
    ex.multiphase(c, AB, nb, phases, racy, bar)
    d = rdict(c.collect())
    c.close()
    if racy == 1:
        assert len(d) == 2 * 1182 and set(d.values()) == {CLS["GRID"]}
    else:
        assert len(d) == 301_920 and sum(v == CLS["BLOCK"] for v in d.values()) == 8_288
        assert d[skey(0, 64)] == CLS["BLOCK"] and d[skey(3, 5)] == CLS["WARP"]


@pytest.mark.parametrize("racy", [False, True])
def test_inline_bfs(racy):
    nindex, nlist = tg.rmat_graph(12, 8)
    t = tg.cfg3("bfs", racy, graph=(nindex, nlist))
    V, E = nindex.shape[0] - 1, nlist.shape[0]
    buf = torch.empty(V + 1 + E + V, dtype=torch.int32, device="cuda")
    buf[:V + 1] = torch.from_numpy(nindex.astype(np.int32))
    buf[V + 1:V + 1 + E] = torch.from_numpy(nlist.astype(np.int32))
    dist = buf[V + 1 + E:]
    dist.fill_(2**31 - 1)
    dist[int(np.argmax(nindex[1:] - nindex[:-1]))] = 0
    c = hr.Checker.for_trace(t)
    levels = ex.bfs(c, buf.data_ptr(), buf[:V + 1], buf[V + 1:V + 1 + E], dist, V, racy)
    assert levels == t.batch_count()
    assert rdict(c.collect()) == odict(t)
    c.close()


def test_inline_sticky_race_across_launches_with_smem_shadow():
    # a shared word that raced in launch g=0 stays RACE (class from g*) after clean launches:
    # the shared-memory shadow is loaded from and written back to the context every launch
    t = tg.cfg1("post_init")
    c = hr.Checker.for_trace(t)
    out = torch.zeros(8, device="cuda")
    ex.reduce(c, out, 32, 1, 1, g0=0)            # racy pass
    ex.reduce(c, out, 32, 3, 0, g0=1)            # clean passes
    got = rdict(c.collect())
    assert got == {skey(0, w): CLS["WARP"] for w in range(16, 32)}
    c.close()


def test_inline_cooperative_kernels_in_sequence_with_epoch_advance():
    # a cooperative kernel whose threads pass k device grid syncs ends k epochs past
    # the host's g.  hirace_advance_grid_epochs(k + 1) before the next kernel moves the host g
    # past every epoch the kernel used, so the next launch starts in a fresh epoch: two clean
    # multiphase launches in a row (each starting at the host context's g) report nothing.
    nb, phases = 6, 34
    AB = torch.rand(4 * nb * 256, device="cuda")
    bar = torch.zeros(1, dtype=torch.int32, device="cuda")
    c = hr.Checker(nb, 256, 32, 4 * nb * 256, 514)
    c.reset()
    g_first = c.dev_ctx().g
    ex.multiphase(c, AB, nb, phases, 0, bar, g0=g_first)
    torch.cuda.synchronize()
    c.advance_grid_epochs(phases)          # (phases - 1) device grid syncs + the kernel boundary
    assert c.dev_ctx().g == g_first + phases
    ex.multiphase(c, AB, nb, phases, 0, bar, g0=c.dev_ctx().g)
    assert rdict(c.collect()) == {}
    while c.dev_ctx().g + 2 * phases <= 254:   # more launches while their epochs fit the 8-bit g
        c.advance_grid_epochs(phases)
        ex.multiphase(c, AB, nb, phases, 0, bar, g0=c.dev_ctx().g)
    assert rdict(c.collect()) == {}
    c.close()
