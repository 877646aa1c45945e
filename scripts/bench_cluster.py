"""Cluster-level replay rate on a DSMEM halo exchange: checked accesses/s with
the inputs resident in HBM, CUDA events on the launching stream, and the HBM roofline fraction at
32 algorithmic bytes per checked access (16 B event + 8 B record read + 8 B record write)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_jacobsonbg24_b200 as h  # noqa: E402
import tracegen as tg  # noqa: E402


def main():
    peak = 6540.5
    try:
        mp = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                         "MEASURED_PEAKS.json")))
        peak = float(mp["hbm_gbs"])
    except Exception:
        pass
    out = []
    for name, t in (("halo_none_8192x4x256", tg.cluster_halo(8192, 4, 256, "none")),
                    ("halo_cluster_8192x4x256", tg.cluster_halo(8192, 4, 256, "cluster")),
                    ("hist_AG_1024x8x256", tg.cluster_histogram(1024, 8, 256, 64, tg.ATOMIC_GRID))):
        c = h.ClusterChecker.for_trace(t)
        ev = h.events_to_device(t.events, "cuda:0")
        s = torch.cuda.Stream()
        flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
        times = []
        with torch.cuda.stream(s):
            for i in range(13):
                c.reset(s)
                flush.fill_(i)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                c.replay(ev, stream=s)
                e1.record(s)
                e1.synchronize()
                if i >= 3:
                    times.append(e0.elapsed_time(e1))
        checked, retries = c.stats()
        nraces = c.collect().shape[0]
        ms = float(np.median(times))
        rate = t.n / (ms * 1e-3)
        out.append(dict(workload=name, events=t.n, checked=checked, ms=ms, accesses_per_s=rate,
            roofline=dict(bound="hbm", achieved=rate * 32 / 1e9, peak=peak, unit="GB/s", frac=rate * 32 / 1e9 / peak),
            cas_retries=retries, flagged=nraces, l2="256 MB buffer written before every timed replay"))
        c.close()
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/bench_cluster.json", "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
