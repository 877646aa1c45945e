"""Measured ceilings: 64-bit atomic / coherent-load rates and the grid-barrier cost (B200)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_jacobsonbg24_b200 import hirace as h  # noqa: E402

torch.cuda.set_device(0)
out = {f"grid_sync_mode{m}_us": h.microbench_grid_sync(400, m) for m in (0, 1, 2)}
ops = {0: "cas", 1: "add", 2: "load", 3: "load+cas"}
for label, nwords in (("l2_4MiB", 1 << 19), ("l2_32MiB", 1 << 22), ("hbm_4GiB", 1 << 29)):
    for rnd in (0, 1):
        for op, name in ops.items():
            r = h.microbench_atomics(nwords, rnd, op, 1 << 28)
            out[f"{label}_{'random' if rnd else 'coalesced'}_{name}_ops_per_s"] = r
print(json.dumps(out, indent=1))
