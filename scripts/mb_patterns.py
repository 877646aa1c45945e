"""DRAM access-pattern microbenchmark for config 5's random shadow traffic (B200).

Config 5 spends most of its replay on first-touch random 8-byte load+CAS pairs into a 32 GiB
shadow.  Which orderings of the same set of words make DRAM cheaper?
  random          uniform random order (what the batch-ordered replay does today)
  sorted          the same words in ascending order (a full sort by address)
  sorted_perbatch ascending inside each 1e7-access slice (a per-batch address sort)
  win2^k          window-major: windows of 2^k words in ascending order, random inside
  dense           consecutive words (coalesced streaming, the sector-efficient limit)
Every pass starts cold (256 MiB written to flush L2).  Rates = accesses / kernel time.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_jacobsonbg24_b200 import hirace as h  # noqa: E402

torch.cuda.set_device(0)
dev = "cuda:0"
LOG2W = 30                                    # 8 GiB of 8-byte words (config 5's gather region)
words = torch.zeros(1 << LOG2W, dtype=torch.int64, device=dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
g = torch.Generator(device=dev)
g.manual_seed(20241117)
out = {"words": 1 << LOG2W}


def run(name, idx, ops=(2, 3)):
    for op in ops:
        flush.fill_(1)
        torch.cuda.synchronize()
        ms = h.microbench_indexed(words.data_ptr(), idx.data_ptr(), idx.numel(), op, 8)
        key = f"{name}_{'load' if op == 2 else 'loadcas'}"
        out[key] = idx.numel() / (ms * 1e-3)
        print(f"{key:40s} n={idx.numel():.3g} {ms:8.3f} ms {out[key]:.3e}/s", flush=True)


for n in (32 * 10**6, 320 * 10**6):
    tag = f"n{n // 10**6}M"
    r = torch.randint(0, 1 << LOG2W, (n,), generator=g, device=dev, dtype=torch.int64)
    run(f"{tag}_random", r)
    s, _ = torch.sort(r)
    run(f"{tag}_sorted", s)
    del s
    sl = 10**7
    pb = torch.cat([torch.sort(r[i:i + sl])[0] for i in range(0, n, sl)])
    run(f"{tag}_sorted_perbatch", pb)
    del pb
    for k in (14, 17, 20, 23):
        key = ((r >> k) << 32) | torch.randint(0, 1 << 31, (n,), generator=g, device=dev, dtype=torch.int64)
        order = torch.argsort(key)
        run(f"{tag}_win2^{k}", r[order])
        del key, order
    del r
    d = torch.arange(n, device=dev, dtype=torch.int64)
    run(f"{tag}_dense", d)
    run(f"{tag}_sector_stride", (d * 4) % (1 << LOG2W))
    del d
    torch.cuda.empty_cache()
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
with open("gpurun_out/mb_patterns.json", "w") as f:
    json.dump(out, f, indent=1)
