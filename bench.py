"""bench.py — checked accesses/s of the B200 HiRace hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl hirace|reference] [--config 2]

One step = one pass of the whole hot path over the workload: shadow reset (a11), replay of
the full trace through the FSM with CAS updates and race reports (a1-a9), and the device-side
collection of flagged words (a7).  The step's launches are captured once as a CUDA graph and
the graph is replayed for the timed steps (`--no-graph`: eager launches); the replay kernel's
own time comes from CUDA events around it in an eager pass.  Default workload = BASELINE.json configs[1] (config 2:
tiled shared-memory stencil, 1024 blocks x 256 threads, racy-A variant, 17,825,792 events);
inputs are resident in HBM when timing starts and are larger than L2 (285 MB of events).

`value` = word-level accesses checked per second (whole job, all ranks).  `e2e` = the same
metric through the C-ABI host entry point (hirace_check_trace_host: pinned host events ->
H2D -> replay -> collect -> D2H).  `roofline` = the replay kernel against the measured HBM
copy bandwidth at 32 algorithmic bytes per access.  `cpu_baseline` = the oracle (C, one core).
`--impl reference` times that oracle as the reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "checked accesses/sec"
UNIT = "accesses/s"
BYTES_PER_ACCESS = 32  # 16-B event + 8-B shadow read + 8-B shadow write


def bytes_per_access(rec_bytes: int) -> int:
    """16-B event + shadow read + shadow write of one record (8 B, or 4 B compact)."""
    return 16 + 2 * rec_bytes


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def make_trace(config: int, variant: str, nranks: int = 1, rank: int = 0):
    import tracegen as tg
    if config == 1:
        return tg.cfg1("post_init" if variant == "racy" else None)
    if config == 2:
        return tg.cfg2(variant == "racy")
    if config == 3:
        return tg.cfg3("bfs", variant == "racy")
    if config == 4:
        return tg.cfg4("B" if variant == "racy" else None)
    if config == 5:
        return tg.cfg5(nranks=nranks, rank=rank)
    raise SystemExit(f"unknown config {config}")


def word_accesses(events) -> int:
    sz = 1 << ((events["meta"] >> 2) & 7).astype(np.int64)
    return int(np.where(sz <= 4, 1, sz // 4).sum())


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled while the timed region runs."""

    Q = ("timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.windows = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (FileNotFoundError, OSError):
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append((time.time(), [x.strip() for x in line.split(",")]))

    def mark(self, t0, t1):
        self.windows.append((t0, t1))

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        inside = [r for t, r in self.rows if any(a - 0.06 <= t <= b + 0.06 for a, b in self.windows)]
        rows = inside or [r for _, r in self.rows]
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in rows for n, v in zip(names, r[5:9]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows), "samples_in_timed_region": len(inside)}


def load_traffic(config: int, variant: str, compact: bool = False):
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(f"cfg{config}_{variant}" + ("_compact" if compact else ""))
    return None


def time_oracle(trace, budget_s: float):
    """Oracle-D as it stands on a bounded sample: the events of the first m blocks."""
    import oracle
    import tracegen as tg
    ev = trace.events
    blk = ev["tid"] // trace.block_threads
    # calibrate on 1/64 of the blocks
    m0 = max(1, trace.grid_blocks // 64)
    s0 = ev[blk < m0]
    t = time.perf_counter()
    oracle.races(s0, trace.block_threads, trace.warp_size)
    rate = max(len(s0), 1) / max(time.perf_counter() - t, 1e-6)
    m = int(min(trace.grid_blocks, max(m0, trace.grid_blocks * min(1.0, budget_s * rate / max(len(ev), 1)))))
    sample = ev[blk < m]
    sub = tg.Trace(trace.name, sample, trace.grid_blocks, trace.block_threads, trace.warp_size,
                   trace.global_words, trace.smem_words)
    return sub, m


def run_reference(args, trace, world):
    import oracle
    if int(os.environ.get("RANK", "0")) != 0:
        return
    budget = max(0.05, 150.0 / max(args.steps + args.warmup, 1))
    sub, m = time_oracle(trace, budget)
    n_acc = word_accesses(sub.events)
    for _ in range(args.warmup):
        oracle.races(sub.events, sub.block_threads, sub.warp_size)
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.races(sub.events, sub.block_threads, sub.warp_size)
    dt = (time.perf_counter() - t) / max(args.steps, 1)
    v = n_acc / dt
    sample = f"events of blocks [0,{m}) of {trace.name} ({n_acc} word accesses) per step"
    out = {"metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "u64", "data": "synthetic", "impl": "reference",
           "config": config_block(args, trace, world),
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample, **host_cpu()},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def config_block(args, trace, world):
    return {"workload": f"config {args.config} ({trace.name}): {BASELINE_CFG.get(args.config, '')}",
            "events_per_rank": int(trace.n), "grid_blocks": trace.grid_blocks,
            "block_threads": trace.block_threads, "batches": trace.batch_count(),
            "shadow_bytes": (4 if getattr(args, "compact", False) else 8) * (trace.global_words + trace.grid_blocks * trace.smem_words),
            "shadow_record_bytes": 4 if getattr(args, "compact", False) else 8,
            "l2": "inputs larger than L2 (events %.0f MB > 126 MB L2)" % (trace.n * 16 / 1e6),
            "parallelism": f"replicas{world}" if world > 1 else "single"}


BASELINE_CFG = {
    1: "tiny shared-mem reduction, 1 block x 32 threads, missing __syncthreads",
    2: "tiled shared-memory stencil, 1024 blocks x 256 threads, racy-A (load->compute barrier dropped)",
    3: "Indigo-style BFS on RMAT-20 (1M vertices, edge factor 16), atomicBug racy variant",
    4: "cooperative multi-phase kernel, 592 x 256, 64 grid phases, racy-B",
    5: "1.07e9 accesses over 2^32 tracked words (16 GiB tracked, 32 GiB shadow), 65536 x 256 threads, 32 batches",
}


def host_cpu() -> dict:
    """The box's host CPU (report the oracle's core count, nproc and CPU model)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


def l2_roofline(st: dict, n_acc: int, kern_ms: float, rec_bytes: int, dev: int) -> dict:
    """the L2-atomic roofline of this workload, from microbenchmarks run in the same
    process on L2-resident words (coalesced, the replay's access shape): every access is one
    coherent load, the ones that change their record add a CAS.  t = loads / load_rate +
    CASes / cas_rate; the binding roofline is the lower of this and the HBM one."""
    from paper_conf_sc_jacobsonbg24_b200 import hirace as h
    nwords = 1 << 22  # 32 MiB of 8-byte words: L2-resident
    load_rate = h.microbench_atomics(nwords, False, 2, 1 << 27, device=dev)
    cas_rate = h.microbench_atomics(nwords, False, 0, 1 << 27, device=dev)
    t = n_acc / load_rate + st["cas_ops"] / cas_rate
    return {"bound": "l2_atomic", "accesses_per_s_peak": n_acc / t, "achieved": n_acc / (kern_ms / 1e3),
            "frac": (n_acc / (kern_ms / 1e3)) / (n_acc / t), "coalesced_load_ops_per_s": load_rate,
            "coalesced_cas_ops_per_s": cas_rate, "cas_ops": st["cas_ops"], "loads": n_acc,
            "note": "64-bit microbenchmark rates; min(HBM, this) binds (SURVEY 8(d))"}


def measure_slowdown(dev: int, reps: int = 5) -> dict:
    """Instrumented slowdown (BASELINE.json metric): native CUDA programs timed uninstrumented
    and with every tracked access / barrier checked inline by the HiRace device hooks
    (examples.cu).  Shadow resets are outside the timed regions."""
    import torch

    import paper_conf_sc_jacobsonbg24_b200 as hr
    import tracegen as tg
    from paper_conf_sc_jacobsonbg24_b200 import examples as ex

    def timed(fn, prep=None):
        fn()
        torch.cuda.synchronize()
        tot = 0.0
        for _ in range(reps):
            if prep:
                prep()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            tot += a.elapsed_time(b)
        return tot / reps

    out = {}
    n, steps = 512, 8
    c = hr.Checker(1024, 256, 32, 2 * n * n, 324, device=dev)
    buf = torch.rand(2 * n * n, device=f"cuda:{dev}")
    nat = timed(lambda: ex.stencil(None, buf, n, steps, True))
    ins = timed(lambda: ex.stencil(c, buf, n, steps, True), c.reset)
    ins_g = timed(lambda: ex.stencil(c, buf, n, steps, True, smem_shadow=False), c.reset)
    out["cfg2_stencil_racy"] = {"native_ms": nat, "instrumented_ms": ins, "slowdown": ins / nat,
                                "slowdown_global_shadow": ins_g / nat}
    c.close()
    nb, phases = 592, 64
    c = hr.Checker(nb, 256, 32, 4 * nb * 256, 514, device=dev)
    AB = torch.rand(4 * nb * 256, device=f"cuda:{dev}")
    bar = torch.zeros(1, dtype=torch.int32, device=f"cuda:{dev}")
    nat = timed(lambda: ex.multiphase(None, AB, nb, phases, 0, bar))
    ins = timed(lambda: ex.multiphase(c, AB, nb, phases, 0, bar), c.reset)
    ins_g = timed(lambda: ex.multiphase(c, AB, nb, phases, 0, bar, smem_shadow=False), c.reset)
    out["cfg4_multiphase_clean"] = {"native_ms": nat, "instrumented_ms": ins, "slowdown": ins / nat,
                                    "slowdown_global_shadow": ins_g / nat}
    c.close()
    c = hr.Checker(1, 32, 32, 8, 32, device=dev)
    o = torch.zeros(8, device=f"cuda:{dev}")
    nat = timed(lambda: ex.reduce(None, o, 32, 8, 1))
    ins = timed(lambda: ex.reduce(c, o, 32, 8, 1), c.reset)
    out["cfg1_reduction_racy"] = {"native_ms": nat, "instrumented_ms": ins, "slowdown": ins / nat}
    c.close()
    nindex, nlist = tg.rmat_graph(18, 16)
    V, E = nindex.shape[0] - 1, nlist.shape[0]
    gb = torch.empty(V + 1 + E + V, dtype=torch.int32, device=f"cuda:{dev}")
    gb[:V + 1] = torch.from_numpy(nindex.astype(np.int32))
    gb[V + 1:V + 1 + E] = torch.from_numpy(nlist.astype(np.int32))
    dist = gb[V + 1 + E:]
    src = int(np.argmax(nindex[1:] - nindex[:-1]))

    def reset_dist():
        dist.fill_(2**31 - 1)
        dist[src] = 0

    c = hr.Checker(-(-V // 256), 256, 32, V + 1 + E + V + V + 1, 0, device=dev)
    nat = timed(lambda: ex.bfs(None, gb.data_ptr(), gb[:V + 1], gb[V + 1:V + 1 + E], dist, V, False), reset_dist)
    ins = timed(lambda: ex.bfs(c, gb.data_ptr(), gb[:V + 1], gb[V + 1:V + 1 + E], dist, V, False),
                lambda: (reset_dist(), c.reset()))
    out["cfg3_bfs_rmat18_clean"] = {"native_ms": nat, "instrumented_ms": ins, "slowdown": ins / nat}
    c.close()
    return out


def run_sharded_bench(args, world, rank, local_rank):
    """Config 5 across `world` GPUs: each rank generates its blocks' events; they are bucketed by
    owner (64 KiB chunks of the 2^32-word space) into 8-byte wire records on the GPU, exchanged
    per batch with NCCL all_to_all_single (all batches in flight, overlapped with the replays),
    and replayed on the owner's shard (strong scaling: fixed trace)."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_jacobsonbg24_b200 import sharded
    dev = local_rank % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    shared_gpu = world > torch.cuda.device_count()  # several ranks per GPU: NCCL cannot run there
    if args.transport == "nccl" or (args.transport == "p2p" and not shared_gpu):
        dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        ex = sharded.NcclExchange(None, f"cuda:{dev}") if args.transport == "nccl" else \
            sharded.PeerExchange(None, dist, device=dev)
    elif args.transport == "p2p":  # control plane over gloo; the records still go peer to peer
        dist.init_process_group("gloo")
        ex = sharded.PeerExchange(None, dist, device=dev)
    else:
        dist.init_process_group("gloo")
        ex = sharded.HostExchange(None, device=f"cuda:{dev}")
    t = make_trace(5, args.variant, world, rank)
    n_local = word_accesses(t.events)
    nccl = dist.get_backend() == "nccl"
    tot = torch.tensor([n_local], dtype=torch.int64, device=f"cuda:{dev}" if nccl else "cpu")
    dist.all_reduce(tot)
    n_total = int(tot.item())
    ops = sharded.GpuOps(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words, world, rank,
                         device=dev)
    ev = torch.from_numpy(t.events.view(np.int64).reshape(-1, 2)).to(f"cuda:{dev}")
    cap = 1 << 20
    d_out = torch.empty(cap * 16, dtype=torch.uint8, device=f"cuda:{dev}")
    d_total = torch.zeros(1, dtype=torch.int64, device=f"cuda:{dev}")

    wire = sharded.wire_fits(t.grid_blocks * t.block_threads, t.global_words, t.smem_words, world)
    if args.transport == "p2p" and not wire:
        raise SystemExit("p2p transport needs the 8-byte wire format")
    run = (sharded.run_sharded_p2p if args.transport == "p2p" else sharded.run_sharded_wire) if wire else \
        sharded.run_sharded

    def step():
        ops.ctx.reset()
        run(ev, ops, ex, None, dist)
        ops.ctx.collect_device(d_out, cap, d_total)

    clocks = ClockSampler(dev)
    clocks.start()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    flagged = int(d_total.item())
    dist.barrier()
    torch.cuda.synchronize()
    w0 = time.time()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        step()
    e1.record()
    torch.cuda.synchronize()
    w1 = time.time()
    dist.barrier()
    clocks.mark(w0, w1)
    clocks.stop()
    ms = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64)
    fl = torch.tensor([flagged], dtype=torch.int64)
    if nccl:
        ms, fl = ms.cuda(), fl.cuda()
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    dist.all_reduce(fl)
    ms, flagged = float(ms.item()), int(fl.item())
    if rank == 0:
        peak, peak_kind = peaks()
        per_step = ms / args.steps
        out = {"metric": METRIC, "value": n_total * args.steps / (ms / 1e3), "unit": UNIT, "n_gpus": world,
               "steps": args.steps, "warmup": args.warmup, "ms_per_step": per_step, "higher_is_better": True,
               "scaling": "strong", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
               "config": {"workload": f"config 5: {BASELINE_CFG[5]}", "events_total": n_total,
                          "parallelism": (f"address-sharded x{world} (" + (
                              "peer dispatch: bucketing kernel stores 8-byte wire records into the owners' "
                              "IPC-mapped buffers over NVLink)" if args.transport == "p2p" else
                              f"{args.transport} all_to_all per batch, "
                              + ("8-byte wire records, async exchange overlapped with replay)" if wire
                                 else "16-byte events)"))),
                          "l2": "inputs larger than L2",
                          "ranks_per_gpu": -(-world // torch.cuda.device_count())},
               "roofline": {"bound": "hbm", "achieved": BYTES_PER_ACCESS * n_total / world / (per_step / 1e3) / 1e9,
                            "peak": peak, "unit": "GB/s",
                            "frac": BYTES_PER_ACCESS * n_total / world / (per_step / 1e3) / 1e9 / peak,
                            "traffic": None, "kernel": "whole sharded step per GPU", "peak_kind": peak_kind},
               "cpu_baseline": None, "e2e": None, "gpu_launches": None, "clocks": clocks.summary(),
               "check": {"flagged_words": flagged, "expected": len(t.info["expected"])}}
        print(json.dumps(out), flush=True)
    if isinstance(ex, sharded.PeerExchange):
        ex.close()
    dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="hirace", choices=["hirace", "reference"])
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--variant", default="racy", choices=["racy", "clean"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-slowdown", action="store_true")
    ap.add_argument("--no-graph", action="store_true", help="time the eager step instead of its CUDA graph")
    ap.add_argument("--compact", action="store_true",
                    help="compact 4-byte shadow records (hirace_shadow_alloc_compact, SURVEY §8(f) f1)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p", "host"],
                    help="config-5 shard exchange: NCCL device all_to_all, peer-memory dispatch (CUDA IPC / "
                         "NVLink stores from the bucketing kernel), or gloo host staging")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.config == 5 and world > 1 and args.impl != "reference":
        run_sharded_bench(args, world, rank, local_rank)
        return
    trace = make_trace(args.config, args.variant)

    if args.impl == "reference":
        run_reference(args, trace, world)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_sc_jacobsonbg24_b200 as hr
    ngpu = torch.cuda.device_count()
    local_rank = local_rank % ngpu  # several ranks per GPU only in single-GPU functional runs
    torch.cuda.set_device(local_rank)
    red_dev = "cuda"
    if world > 1:
        if world <= ngpu:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:  # ranks share a GPU: NCCL cannot run there; timing reductions go through gloo
            dist.init_process_group("gloo")
            red_dev = "cpu"

    n_acc = word_accesses(trace.events)
    c = hr.Checker.for_trace(trace, device=local_rank, compact=args.compact)
    bpa = bytes_per_access(c.rec_bytes)
    d_ev = hr.events_to_device(trace.events, f"cuda:{local_rank}")
    cap = 1 << 20
    d_out = torch.empty(cap * 16, dtype=torch.uint8, device="cuda")
    d_total = torch.zeros(1, dtype=torch.int64, device="cuda")
    stream = torch.cuda.current_stream()
    K, W = args.steps, args.warmup
    ks = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    ke = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    for e in ks + ke:
        e.record(stream)

    def step(i=None):
        c.reset(stream)
        if i is not None:
            c.set_kernel_timing(ks[i], ke[i])
        else:
            c.set_kernel_timing(None, None)
        c.check_device(d_ev, d_out, cap, d_total, stream=stream)  # replay + fused collect

    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    for _ in range(W):
        step()
    torch.cuda.synchronize()
    flagged = int(d_total.item())

    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    w0 = time.time()
    t0.record(stream)
    for i in range(K):
        step(i)
    t1.record(stream)
    torch.cuda.synchronize()
    w1 = time.time()
    if world > 1:
        dist.barrier()
    clocks.mark(w0, w1)
    ms = t0.elapsed_time(t1)
    eager_ms = ms
    kern_ms = sum(a.elapsed_time(b) for a, b in zip(ks, ke)) / K
    c.set_kernel_timing(None, None)
    # the same step captured once as a CUDA graph (reset + batch discovery + persistent replay
    # with fused collect) and replayed K times: the launch gaps between the step's kernels go
    # away; this is the timed `value`.  The kernel-only time above comes from the eager pass.
    step_mode = "eager"
    if not args.no_graph:
        try:
            gs = torch.cuda.Stream()
            gs.wait_stream(stream)
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph, stream=gs):
                c.reset(gs)
                c.check_device(d_ev, d_out, cap, d_total, stream=gs)
            d_total.zero_()
            with torch.cuda.stream(gs):
                for _ in range(W):
                    graph.replay()
            torch.cuda.synchronize()
            if int(d_total.item()) != flagged:
                raise RuntimeError("graph replay disagrees with the eager step")
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            w0 = time.time()
            t0.record(gs)
            with torch.cuda.stream(gs):
                for _ in range(K):
                    graph.replay()
            t1.record(gs)
            torch.cuda.synchronize()
            w1 = time.time()
            if world > 1:
                dist.barrier()
            clocks.mark(w0, w1)
            ms = t0.elapsed_time(t1)
            step_mode = "cuda_graph"
        except Exception as exc:  # capture unsupported: the eager timing stands
            print(f"bench: CUDA graph step unavailable ({exc}); eager timing", file=sys.stderr)
            ms = eager_ms
    if world > 1:
        tt = torch.tensor([ms, kern_ms], dtype=torch.float64, device=red_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms, kern_ms = float(tt[0]), float(tt[1])
    ms_per_step = ms / K
    value = n_acc * world * K / (ms / 1e3)
    st = c.stats()

    # e2e through the C-ABI host entry point: pinned host events -> H2D -> replay -> D2H
    e2e = None
    if not args.no_e2e:
        small = trace.n * 16 <= (4 << 30)
        pin = torch.empty(trace.n * 16, dtype=torch.uint8, pin_memory=small)
        pin.numpy()[:] = trace.events.view(np.uint8)
        hout = torch.empty(cap * 16, dtype=torch.uint8, pin_memory=True)
        ke2 = max(3, min(K, 10))
        for _ in range(2):
            c.reset(stream)
            c.check_host_ptr(pin.data_ptr(), trace.n, hout.data_ptr(), cap, stream=stream)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        we0 = time.perf_counter()
        for _ in range(ke2):
            c.reset(stream)
            tot = c.check_host_ptr(pin.data_ptr(), trace.n, hout.data_ptr(), cap, stream=stream)
        torch.cuda.synchronize()
        e2e_s = (time.perf_counter() - we0) / ke2
        if world > 1:
            tt = torch.tensor([e2e_s], dtype=torch.float64, device=red_dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            e2e_s = float(tt[0])
        e2e = {"value": n_acc * world / e2e_s, "unit": UNIT, "h2d_bytes_per_step": int(trace.n * 16),
               "host_memory": "pinned" if small else "pageable",
               "d2h_bytes_per_step": int(min(tot, cap) * 16 + 8), "ms_per_step": e2e_s * 1e3}
    clocks.stop()

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    peak, peak_kind = peaks()
    achieved = bpa * n_acc / (kern_ms / 1e3) / 1e9
    try:
        l2 = l2_roofline(st, n_acc, kern_ms, c.rec_bytes, local_rank)
        l2["hbm_accesses_per_s_peak"] = peak * 1e9 / bpa
        l2["binding"] = "hbm" if peak * 1e9 / bpa <= l2["accesses_per_s_peak"] else "l2_atomic"
    except Exception as exc:  # diagnostics only; never fails the bench line
        l2 = {"error": str(exc)}
    slow = None if args.no_slowdown else measure_slowdown(local_rank)
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        import oracle
        sub, m = time_oracle(trace, 20.0)
        t = time.perf_counter()
        oracle.races(sub.events, sub.block_threads, sub.warp_size)
        dt = time.perf_counter() - t
        na = word_accesses(sub.events)
        cpu = {"value": na / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"events of blocks [0,{m}) of {trace.name} ({na} word accesses), one run, 1 thread",
               **host_cpu()}
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": W,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u64" if c.rec_bytes == 8 else "u32", "data": "synthetic", "config": config_block(args, trace, world),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": load_traffic(args.config, args.variant, args.compact),
                     "kernel": "k_replay (incl. fused collect)", "kernel_ms": kern_ms, "kernel_share": kern_ms / ms_per_step,
                     "bytes_per_access": bpa, "peak_kind": peak_kind},
        "roofline_l2": l2,
        "cpu_baseline": cpu,
        "e2e": e2e,
        # per step: k_reset, k_batches, k_replay (fused collect) [+ k_collect_reports in report mode]
        "gpu_launches": (4 if c.shadow_bytes >= (64 << 20) else 3) * K,
        "step_mode": step_mode, "eager_ms_per_step": eager_ms / K,
        "clocks": clocks.summary(),
        "check": {"flagged_words": flagged, "per_step": st},  # stats are per step (reset clears them)
        "instrumented_slowdown": slow,
        "shadow_overhead": {"bytes_per_tracked_word": c.rec_bytes, "ratio_to_tracked_bytes": c.rec_bytes / 4,
                            "iguard_ratio_context": 4.0},
    }
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
