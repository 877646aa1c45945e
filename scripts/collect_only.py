"""Replay config 2 once, then the standalone collect kernel (for an ncu capture of k_collect)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
import tracegen as tg  # noqa: E402

t = tg.cfg2(True)
c = hr.Checker.for_trace(t)
d = hr.events_to_device(t.events)
cap = 1 << 20
out = torch.empty(cap * 16, dtype=torch.uint8, device="cuda")
tot = torch.zeros(1, dtype=torch.int64, device="cuda")
for _ in range(3):
    c.reset()
    c.replay(d)
    c.collect_device(out, cap, tot)
torch.cuda.synchronize()
print("flagged", int(tot.item()))
