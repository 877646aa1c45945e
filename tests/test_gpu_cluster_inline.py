"""Cluster scope in the inline hooks (reading R16; the paper's
wrapper): native cluster kernels with real DSMEM accesses
(cluster.map_shared_rank) and cluster.sync(), checked inline by hirace::cluster::on_access /
barrier, against the cluster oracle on the trace of the same program (tracegen.cluster_halo /
cluster_histogram)."""
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
from paper_conf_sc_jacobsonbg24_b200 import examples as ex  # noqa: E402


def _got(c):
    r = c.collect()
    return {int(k): int(x) & 255 for k, x in zip(r["key"], r["cls_and_epoch"])}


@pytest.mark.parametrize("sync", ["cluster", "block", "none"])
@pytest.mark.parametrize("nclusters,cb,bs", [(2, 4, 64), (16, 2, 128), (64, 8, 256), (37, 4, 96)])
def test_inline_dsmem_halo(sync, nclusters, cb, bs):
    t = tg.cluster_halo(nclusters, cb, bs, sync)
    c = hr.ClusterChecker.for_trace(t)
    try:
        out = torch.zeros(nclusters * cb * bs, dtype=torch.float32, device="cuda")
        ex.cluster_halo(c, out, nclusters, cb, bs, sync)
        torch.cuda.synchronize()
        got = _got(c)
    finally:
        c.close()
    assert got == oracle.races_cluster_dict(t)
    assert (len(got) == 0) == (sync == "cluster")


@pytest.mark.parametrize("atomic,drop", [(tg.ATOMIC_GRID, None), (tg.ATOMIC_GRID, 1), (tg.ATOMIC_GRID, 2),
                                         (tg.ATOMIC_BLOCK, None)])
@pytest.mark.parametrize("nclusters,cb,bs,bins", [(2, 4, 64, 16), (32, 8, 256, 64)])
def test_inline_dsmem_histogram(atomic, drop, nclusters, cb, bs, bins):
    t = tg.cluster_histogram(nclusters, cb, bs, bins, atomic, drop)
    c = hr.ClusterChecker.for_trace(t)
    try:
        out = torch.zeros(nclusters * bins, dtype=torch.int32, device="cuda")
        ex.cluster_hist(c, out, nclusters, cb, bs, bins, atomic == tg.ATOMIC_BLOCK, drop)
        torch.cuda.synchronize()
        got = _got(c)
        if drop is None:  # the program itself is correct whatever the checker says
            assert bool((out == cb * bs // bins).all())
    finally:
        c.close()
    assert got == oracle.races_cluster_dict(t)
    assert (len(got) == 0) == (atomic == tg.ATOMIC_GRID and drop is None)


def test_inline_cluster_checks_agree_with_replay():
    """the inline hooks and the cluster replay of the same program's trace give one verdict"""
    t = tg.cluster_halo(8, 4, 64, "block")
    c = hr.ClusterChecker.for_trace(t)
    try:
        out = torch.zeros(8 * 4 * 64, dtype=torch.float32, device="cuda")
        ex.cluster_halo(c, out, 8, 4, 64, "block")
        torch.cuda.synchronize()
        inline = _got(c)
        c.reset()
        c.replay(hr.events_to_device(t.events, "cuda:0"))
        replay = _got(c)
    finally:
        c.close()
    assert inline == replay and inline
