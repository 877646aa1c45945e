"""One window-major check of a medium config-5 trace (2^28 words, 8192 x 256 threads, 1.3e8
events) for ncu captures of the window kernels (scripts/gpu_r2_prof.sh)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_jacobsonbg24_b200 as hr  # noqa: E402
import tracegen as tg  # noqa: E402

wl = int(os.environ.get("WL", "14"))
t = tg.cfg5(grid_blocks=int(os.environ.get("BLOCKS", "8192")), words_log2=int(os.environ.get("WORDS_LOG2", "28")))
c = hr.Checker.for_trace(t)
c.set_replay_mode(hr.REPLAY_WINDOW, wl)
d = hr.events_to_device(t.events)
cap = 1 << 16
out = torch.zeros(cap * 16, dtype=torch.uint8, device="cuda")
tot = torch.zeros(1, dtype=torch.int64, device="cuda")
for _ in range(int(os.environ.get("REPS", "2"))):
    c.reset()
    c.check_device(d, out, cap, tot)
torch.cuda.synchronize()
print("flagged", int(tot.item()), "expected", len(t.info["expected"]), c.stats())
