"""Barrier arrival spread per batch (diagnostics build with -DHIRACE_BARRIER_TRACE)."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["HIRACE_LIB"] = os.path.abspath("build/variants/bartrace.so")
import torch  # noqa: E402

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
import tracegen as tg  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
t = tg.cfg2(True) if cfg == 2 else tg.cfg4("B")
c = hr.Checker.for_trace(t)
d = hr.events_to_device(t.events)
for _ in range(3):
    c.reset()
    c.replay(d)
torch.cuda.synchronize()
lib = hr.load()
lib.hirace_debug_barrier_trace.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
buf = np.zeros(128 * 2048 * 2, np.uint64)
lib.hirace_debug_barrier_trace(buf.ctypes.data, buf.size)
buf = buf.reshape(128, 2048, 2).astype(np.int64)
grid = int((buf[0, :, 0] != 0).sum())
nb = t.batch_count()
prev_rel = None
for b in range(min(nb - 1, 12)):
    arr, rel = buf[b, :grid, 0], buf[b, :grid, 1]
    a0, a1, r1 = arr.min(), arr.max(), rel.max()
    start = prev_rel if prev_rel is not None else a0
    print(f"batch {b}: work {(a0 - start) / 1e3:7.2f}..{(a1 - start) / 1e3:7.2f} us (first..last CTA arrival), "
          f"spread {(a1 - a0) / 1e3:6.2f} us, p50 {(np.median(arr) - start) / 1e3:7.2f}, release {(r1 - a1) / 1e3:5.2f} us")
    prev_rel = rel.min()

# persistence of lateness: rank correlation of per-CTA arrival order between batches, and the
# arrival spread by SM die half (CTA i runs on SM ~ i mod #SMs for a 2-CTA/SM persistent grid)
ranks = []
for b in range(min(nb - 1, 12)):
    arr = buf[b, :grid, 0]
    ranks.append(np.argsort(np.argsort(arr)))
ranks = np.array(ranks, dtype=np.float64)
if len(ranks) > 2:
    cc = np.corrcoef(ranks)
    off = cc[np.triu_indices(len(ranks), 1)]
    print(f"rank correlation of CTA arrival order across batches: mean {off.mean():.3f} "
          f"(min {off.min():.3f}, max {off.max():.3f})")
    mean_rank = ranks.mean(axis=0)
    print("latest 10 CTAs on average:", np.argsort(-mean_rank)[:10].tolist())

# per-SM view: an SM's arrival = its last CTA's; is the spread between SMs or inside an SM?
lib.hirace_debug_barrier_smid.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
smid = np.zeros(2048, np.uint32)
lib.hirace_debug_barrier_smid(smid.ctypes.data, smid.size)
smid = smid[:grid]
for b in range(min(nb - 1, 12)):
    arr = buf[b, :grid, 0]
    per_sm = {}
    for i in range(grid):
        per_sm.setdefault(int(smid[i]), []).append(int(arr[i]))
    last = np.array([max(v) for v in per_sm.values()], dtype=np.int64)
    first = np.array([min(v) for v in per_sm.values()], dtype=np.int64)
    print(f"batch {b}: {len(per_sm)} SMs; SM finish spread {(last.max() - last.min()) / 1e3:6.2f} us "
          f"(p50 {(np.median(last) - last.min()) / 1e3:5.2f}); intra-SM CTA gap p50 {np.median(last - first) / 1e3:5.2f} us")
