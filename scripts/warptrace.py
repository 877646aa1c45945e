"""Per-warp share completion times per batch (diagnostics build with -DHIRACE_WARP_TRACE
-DHIRACE_BARRIER_TRACE): is the batch tail intra-CTA (warp) variance or per-SM?"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["HIRACE_LIB"] = os.path.abspath(os.environ.get("TRACE_SO", "build/variants/trace.so"))
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
lib.hirace_debug_warp_trace.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
bt = np.zeros(128 * 2048 * 2, np.uint64)
lib.hirace_debug_barrier_trace(bt.ctypes.data, bt.size)
bt = bt.reshape(128, 2048, 2).astype(np.int64)
wt = np.zeros(16 * 8192 * 4, np.uint64)
lib.hirace_debug_warp_trace(wt.ctypes.data, wt.size)
wt = wt.reshape(16, 8192, 4).astype(np.int64)
grid = int((bt[0, :, 0] != 0).sum())
nw = grid * 16
for b in range(1, min(t.batch_count() - 1, 8)):
    start = bt[b - 1, :grid, 1].min()
    done = (wt[b, :nw, 0] - start) / 1e3
    sm = wt[b, :nw, 1]
    cta = done.reshape(grid, 16)
    ctamax, ctamean = cta.max(1), cta.mean(1)
    smmean = np.array([done[sm == s].mean() for s in np.unique(sm)])
    print(f"batch {b}: warp done p10 {np.percentile(done, 10):6.2f} p50 {np.median(done):6.2f} "
          f"p90 {np.percentile(done, 90):6.2f} max {done.max():6.2f} us | CTA max-mean avg "
          f"{(ctamax - ctamean).mean():5.2f} | CTA mean p10/p50/p90/max {np.percentile(ctamean, 10):6.2f} "
          f"{np.median(ctamean):6.2f} {np.percentile(ctamean, 90):6.2f} {ctamean.max():6.2f} | SM mean "
          f"min/max {smmean.min():6.2f}/{smmean.max():6.2f}")
    if b == 1:
        order = np.argsort(-done)[:10]
        print("  slowest warps (us, sm, cta):", [(round(done[i], 2), int(sm[i]), int(i // 16)) for i in order])
lib.hirace_debug_chunk_detail.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
cd = np.zeros(8192 * 4, np.uint64)
lib.hirace_debug_chunk_detail(cd.ctypes.data, cd.size)
cd = cd.reshape(8192, 4)[:nw].astype(np.int64)
print("per warp max chunk time (us) without CAS failure p50/p99/max", np.percentile(cd[:, 0], [50, 99, 100]) / 1e3,
      "| with failure", np.percentile(cd[:, 1], [50, 99, 100]) / 1e3, "| chunks with failure per warp", np.percentile(cd[:, 2], [50, 99, 100]),
      "| load wait max", np.percentile(cd[:, 3], [50, 99, 100]) / 1e3)
np.savez(os.path.join("gpurun_out", f"warptrace_cfg{cfg}_{os.path.basename(os.environ['HIRACE_LIB'])}.npz"), bt=bt, wt=wt,
         grid=grid)
