"""Random 8-byte load+CAS rate vs footprint (B200): is the random-RMW rate of config 5 bounded by
DRAM, or by address translation as the footprint outgrows the TLB reach?"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_jacobsonbg24_b200 import hirace as h  # noqa: E402

torch.cuda.set_device(0)
out = {}
for log2 in (22, 24, 26, 27, 28, 29, 30, 31, 32):   # 32 MiB .. 32 GiB of 8-byte words
    for op, name in ((2, "load"), (3, "load+cas")):
        out[f"{8 << log2 >> 20}MiB_random_{name}_ops_per_s"] = h.microbench_atomics(1 << log2, 1, op, 1 << 27)
    print(log2, out, flush=True)
print(json.dumps(out, indent=1))
