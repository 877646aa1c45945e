"""bench.py — checked accesses/s of the B200 HiRace hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl hirace|reference] [--config 2]

One step = one pass of the whole hot path over the workload: shadow reset (a11), replay of
the full trace through the FSM with CAS updates and race reports (a1-a9), and the device-side
collection of flagged words (a7).  The step's launches are captured once as a CUDA graph and
the graph is replayed for the timed steps (`--no-graph`: eager launches); per-kernel times come
from CUDA events around each kernel in an eager pass.

Default workload = config 5 (BASELINE.json configs[4], the config the metric is quoted on at
1/2/4/8 GPUs): 1.07e9 accesses over 2^32 tracked words, 65,536 x 256 threads, 32 batches.
N=1 replays the whole trace on one GPU; N>1 (torchrun) shards it by address (strong scaling,
owner = 64 KiB chunk mod N) with the exchange over NCCL (`--transport nccl`, default) or peer
stores (`--transport p2p`).  Configs 2, 3 and 4 are measured after it at N=1 and reported under
`per_config` (`--no-per-config` skips them).  Inputs are resident in HBM when timing starts
and are larger than L2 (17 GB of events for config 5).

`value` = word-level accesses checked per second (whole job, all ranks).  `e2e` = the same
metric through the C-ABI host entry point (hirace_check_trace_host: pinned host events ->
H2D -> replay -> collect -> D2H; N>1: per rank host -> device, then the sharded step).
`roofline` = the dominant kernel against the measured HBM copy bandwidth at its algorithmic
bytes; `roofline_step` = the whole step at 32 algorithmic bytes per access.  `cpu_baseline` =
Oracle-D on all host cores (address-sharded, oracle/oracle_par.c) on a bounded sample, with the
one-thread rate beside it.  `--impl reference` times that oracle as the reference arm.
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
    if config == 6:  # partial-mask __syncwarp: tiled_partition<8> reduction, 1M threads
        return tg.tiled_reduce(4096, 256, 8, 4, "half_mask" if variant == "racy" else None)
    raise SystemExit(f"unknown config {config}")


def word_accesses(events, chunk: int = 1 << 26) -> int:
    """Word-level accesses (8/16-byte accesses count 2/4 words), chunked for 1e9-event traces."""
    tot = 0
    for lo in range(0, events.shape[0], chunk):
        szl = (events["meta"][lo:lo + chunk] >> 2) & 7
        tot += int(np.where(szl <= 2, 1, 1 << np.maximum(szl.astype(np.int64) - 2, 0)).sum())
    return tot


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


def load_traffic(key: str):
    """DRAM bytes per launch of the dominant kernel for this workload, from the committed ncu
    captures (profiles/traffic.json, one key per config/variant/record layout)."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        v = d.get(key)
        return v.get("bytes") if isinstance(v, dict) else v
    return None


def sample_blocks(trace, m: int):
    """The events of blocks [0, m) of a trace (a bounded sample of the same workload)."""
    import tracegen as tg
    ev = trace.events
    if m >= trace.grid_blocks:
        return trace
    sel = ev["tid"] < np.uint32(m * trace.block_threads)
    return tg.Trace(trace.name, ev[sel], trace.grid_blocks, trace.block_threads, trace.warp_size,
                    trace.global_words, trace.smem_words)


def oracle_sample(trace, budget_s: float, threads: int):
    """Blocks [0, m) with m sized (from a calibration run on 1/256 of the blocks) so that the
    oracle on `threads` cores takes about budget_s."""
    import oracle
    m0 = max(1, trace.grid_blocks // 256)
    s0 = sample_blocks(trace, m0)
    t = time.perf_counter()
    oracle.races_parallel(s0.events, s0.block_threads, s0.warp_size, threads=threads)
    dt = max(time.perf_counter() - t, 1e-6)
    m = int(min(trace.grid_blocks, max(m0, m0 * budget_s / dt)))
    return sample_blocks(trace, m), m


def cpu_baseline(trace, budget_s: float = 20.0) -> dict:
    """Oracle-D as it stands on the box's host cores (SURVEY §8(d) "Oracle timing"): all cores
    (hardware_concurrency threads over address shards) on a ~budget_s sample, and one core on a
    smaller sample."""
    import oracle
    cores = oracle.hardware_threads()
    sub, m = oracle_sample(trace, budget_s, cores)
    na = word_accesses(sub.events)
    t = time.perf_counter()
    oracle.races_parallel(sub.events, sub.block_threads, sub.warp_size, threads=cores)
    dt = time.perf_counter() - t
    sub1 = sample_blocks(trace, max(1, m // (4 * cores)))
    na1 = word_accesses(sub1.events)
    t = time.perf_counter()
    oracle.races(sub1.events, sub1.block_threads, sub1.warp_size)
    dt1 = time.perf_counter() - t
    return {"value": na / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"events of blocks [0,{m}) of {trace.name} ({na} word accesses), one run, {cores} threads "
                      f"over address shards (oracle/oracle_par.c)",
            "one_thread": {"value": na1 / dt1, "unit": UNIT,
                           "sample": f"events of blocks [0,{max(1, m // (4 * cores))}) ({na1} word accesses)"},
            **host_cpu()}


def run_reference(args, world):
    """Reference arm: the oracle (all host cores) as it stands, on a bounded sample of the
    workload per step.  Rank 0 only; other ranks exit without work."""
    import oracle
    if int(os.environ.get("RANK", "0")) != 0:
        return
    trace = make_trace(args.config, args.variant)
    cores = oracle.hardware_threads()
    budget = max(0.05, 150.0 / max(args.steps + args.warmup, 1))
    sub, m = oracle_sample(trace, budget, cores)
    if args.config == 5:
        trace.info.pop("buffer", None)
    n_acc = word_accesses(sub.events)
    for _ in range(args.warmup):
        oracle.races_parallel(sub.events, sub.block_threads, sub.warp_size, threads=cores)
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.races_parallel(sub.events, sub.block_threads, sub.warp_size, threads=cores)
    dt = (time.perf_counter() - t) / max(args.steps, 1)
    v = n_acc / dt
    sample = (f"events of blocks [0,{m}) of {trace.name} ({n_acc} word accesses) per step, {cores} threads over "
              "address shards")
    out = {"metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
           "scaling": "strong" if args.config == 5 else "weak",
           "vs_baseline": None, "dtype": "u64", "data": "synthetic", "impl": "reference",
           "config": config_block(args, trace, world),
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                            **host_cpu()},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def config_block(args, trace, world, config=None):
    config = args.config if config is None else config
    rb = 4 if getattr(args, "compact", False) else 8
    return {"workload": f"config {config} ({trace.name}): {BASELINE_CFG.get(config, '')}",
            "events_per_rank": int(trace.n), "grid_blocks": trace.grid_blocks,
            "block_threads": trace.block_threads, "batches": trace.batch_count(),
            "shadow_bytes": rb * (trace.global_words + trace.grid_blocks * trace.smem_words),
            "shadow_record_bytes": rb,
            "l2": "inputs larger than L2 (events %.0f MB > 126 MB L2)" % (trace.n * 16 / 1e6),
            "parallelism": "single" if world == 1 else f"replicas{world}"}


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


def random_rmw_count(trace, d_ev) -> int:
    """Config 5: accesses to its two randomly addressed regions (the uniform gather over 2^30
    words and the one-word-per-thread fillers; tracegen.cfg5 regions), counted on the device."""
    import torch
    reg = trace.info["regions"]
    T = trace.grid_blocks * trace.block_threads
    lo1, hi1 = reg["gather"], reg["hot"]          # [W/2, 3W/4)
    lo2, hi2 = reg["inj"], reg["inj"] + T
    addr = d_ev.view(torch.int64).view(-1, 2)[:, 0]
    n = 0
    for a in range(0, addr.numel(), 1 << 27):
        w = (addr[a:a + (1 << 27)] & ((1 << 62) - 1)) >> 2
        n += int(((w >= lo1) & (w < hi1)).sum()) + int(((w >= lo2) & (w < hi2)).sum())
    return n


def random_roofline(n_random: int, kern_ms: float, dev: int) -> dict:
    """The resource config 5 is bound by: scattered first-touch load+CAS pairs into an HBM-sized
    shadow.  Peak = the same-process microbenchmark rate of random 8-byte
    load+CAS pairs over an 8 GiB word array (config 5's gather region), cold L2; achieved = the
    replay's random-region accesses per second of k_replay (which moves the streaming 2/3 of the
    trace at the same time)."""
    import torch

    from paper_conf_sc_jacobsonbg24_b200 import hirace as h
    dv = f"cuda:{dev}"
    words = torch.zeros(1 << 30, dtype=torch.int64, device=dv)
    gen = torch.Generator(device=dv)
    gen.manual_seed(20241117)
    m = min(n_random, 320 * 10**6)
    idx = torch.randint(0, 1 << 30, (m,), generator=gen, device=dv, dtype=torch.int64)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dv)
    best = 0.0
    for _ in range(2):
        flush.fill_(1)
        torch.cuda.synchronize()
        ms = h.microbench_indexed(words.data_ptr(), idx.data_ptr(), m, 3, 8, device=dev)
        best = max(best, m / (ms * 1e-3))
    del words, idx, flush
    torch.cuda.empty_cache()
    ach = n_random / (kern_ms / 1e3)
    return {"bound": "dram_random_rmw", "achieved": ach, "peak": best, "unit": "load+CAS pairs/s", "frac": ach / best,
            "random_accesses": n_random,
            "peak_kind": "measured (hirace_microbench_indexed op 3, 3.2e8 random words of 8 GiB, 8 CTAs/SM)",
            "note": "achieved counts only the gather + filler accesses; the kernel moves the coalesced "
                    "private accesses, the hot atomics and the 16-B events in the same time"}


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
    for agg in (False, True):  # per-thread hooks, then warp-aggregated hooks (HIRACE_INLINE_AGGREGATE)
        ex.use_aggregated_hooks(agg)
        r = _slowdown_programs(dev, reps, timed)
        if not agg:
            out.update(r)
        else:
            for k, v in r.items():
                out[k]["slowdown_warp_aggregated"] = v["slowdown"]
    ex.use_aggregated_hooks(False)
    return out


def _slowdown_programs(dev: int, reps: int, timed) -> dict:
    import torch

    import paper_conf_sc_jacobsonbg24_b200 as hr
    import tracegen as tg
    from paper_conf_sc_jacobsonbg24_b200 import examples as ex
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
    # partial-mask syncs (config 6's program, inline sub-warp hooks): tiled_partition<8> reduction
    nb, bs, tile = 4096, 256, 8
    c = hr.Checker(nb, bs, 32, nb * bs // tile, bs, device=dev)
    o = torch.zeros(nb * bs // tile, device=f"cuda:{dev}")
    c.inline_ws(2 * nb * bs)
    nat = timed(lambda: ex.tiled(None, o, nb, bs, tile, 4, "half_mask"))
    ins = timed(lambda: ex.tiled(c, o, nb, bs, tile, 4, "half_mask"), c.reset)
    ins_g = timed(lambda: ex.tiled(c, o, nb, bs, tile, 4, "half_mask", smem_tracking=False), c.reset)
    out["cfg6_tiled_masked_racy"] = {"native_ms": nat, "instrumented_ms": ins, "slowdown": ins / nat,
                                     "slowdown_global_history": ins_g / nat,
                                     "hooks": "hirace::ws (partial-mask syncs), shared-word history in smem"}
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
    # communicator-init lines (rank / nranks / transport) for the driver's rank check
    os.environ.setdefault("NCCL_DEBUG", "INFO")
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    dev = local_rank % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    shared_gpu = world > torch.cuda.device_count()  # several ranks per GPU: NCCL cannot run there
    if shared_gpu and args.transport == "nccl":
        # NCCL needs one GPU per rank; ranks sharing a GPU (functional runs on a 1-GPU pool) take
        # the peer-dispatch path, its control plane over gloo (the records still go peer to peer)
        args.transport = "p2p"
        print("bench: ranks share a GPU, NCCL unavailable: --transport p2p over gloo", file=sys.stderr)
    if args.transport == "nccl" or (args.transport == "p2p" and not shared_gpu):
        dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        ex = sharded.NcclExchange(None, f"cuda:{dev}") if args.transport == "nccl" else \
            sharded.PeerExchange(None, dist, device=dev)
    elif args.transport == "p2p":  # control plane over gloo; the records still go peer to peer
        dist.init_process_group("gloo")
        ex = sharded.PeerExchange(None, dist, device=dev, per_batch=False)
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
    from paper_conf_sc_jacobsonbg24_b200 import hirace as _hb
    l0 = _hb.launch_count()
    w0 = time.time()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        step()
    e1.record()
    torch.cuda.synchronize()
    w1 = time.time()
    launches = _hb.launch_count() - l0
    dist.barrier()
    clocks.mark(w0, w1)
    clocks.stop()
    ms = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64)
    fl = torch.tensor([flagged], dtype=torch.int64)
    if nccl:
        ms, fl = ms.cuda(), fl.cuda()
    nl = torch.tensor([launches], dtype=torch.int64)
    if nccl:
        nl = nl.cuda()
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    dist.all_reduce(fl)
    dist.all_reduce(nl)  # the library's kernels launched in the timed region, all ranks
    ms, flagged, launches = float(ms.item()), int(fl.item()), int(nl.item())
    # e2e: every step copies this rank's events from pinned host memory to the device, runs the
    # sharded step and reads the flagged words back (D2H); max over ranks of the wall time
    e2e = None
    if not args.no_e2e:
        host = torch.from_numpy(t.events.view(np.int64).reshape(-1, 2))
        try:
            host = host.pin_memory()
            pinned = True
        except RuntimeError:
            pinned = False
        h_out = torch.empty(cap * 16, dtype=torch.uint8, pin_memory=True)
        h_tot = torch.zeros(1, dtype=torch.int64, pin_memory=True)
        ke2 = max(3, min(args.steps, 5))

        def e2e_step():
            ev.copy_(host, non_blocking=True)
            step()
            h_tot.copy_(d_total, non_blocking=True)
            torch.cuda.synchronize()
            h_out[: min(int(h_tot.item()), cap) * 16].copy_(d_out[: min(int(h_tot.item()), cap) * 16])

        e2e_step()
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(ke2):
            e2e_step()
        dt = torch.tensor([(time.perf_counter() - t0) / ke2], dtype=torch.float64)
        if nccl:
            dt = dt.cuda()
        dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        dt = float(dt.item())
        e2e = {"value": n_total / dt, "unit": UNIT, "h2d_bytes_per_step": int(t.n * 16) * world,
               "d2h_bytes_per_step": int(min(flagged, cap) * 16 + 8), "ms_per_step": dt * 1e3,
               "host_memory": "pinned" if pinned else "pageable", "steps": ke2,
               "path": "per rank: H2D of its events, sharded step, collect, D2H"}
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
               "cpu_baseline": None,  # the oracle is timed on rank 0 at N=1 only
               "e2e": e2e, "gpu_launches": launches, "clocks": clocks.summary(),
               "check": {"flagged_words": flagged, "expected": len(t.info["expected"])}}
    if isinstance(ex, sharded.PeerExchange):
        ex.close()
    dist.destroy_process_group()
    if rank == 0:  # last, after NCCL's teardown log lines
        print(json.dumps(out), flush=True)


def measure_single(args, config: int, variant: str, K: int, W: int, dev: int, clocks=None, keep=False):
    """Times the full step (reset + check_device: batch discovery, replay with fused collect)
    of one workload on one GPU: an eager pass with CUDA events around the replay kernel, then the
    same step captured as a CUDA graph and replayed K times (the timed `value`)."""
    import torch

    import paper_conf_sc_jacobsonbg24_b200 as hr
    trace = make_trace(config, variant)
    n_acc = word_accesses(trace.events)
    c = hr.Checker.for_trace(trace, device=dev, compact=args.compact)
    if args.replay_mode != "auto":
        c.set_replay_mode({"batch": hr.REPLAY_BATCH, "window": hr.REPLAY_WINDOW}[args.replay_mode], args.window_log2)
    window = c.window_active
    epoch = args.reset_mode == "epoch" and not window and c.rec_bytes == 8
    if epoch:
        c.set_reset_mode(hr.RESET_EPOCH)
    d_ev = hr.events_to_device(trace.events, f"cuda:{dev}")
    cap = 1 << 20
    d_out = torch.empty(cap * 16, dtype=torch.uint8, device=f"cuda:{dev}")
    d_total = torch.zeros(1, dtype=torch.int64, device=f"cuda:{dev}")
    stream = torch.cuda.current_stream()
    ks = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    ke = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    for e in ks + ke:
        e.record(stream)

    def step(i=None):
        c.reset(stream)
        c.set_kernel_timing(ks[i], ke[i]) if i is not None else c.set_kernel_timing(None, None)
        c.check_device(d_ev, d_out, cap, d_total, stream=stream)  # replay + fused collect

    for _ in range(W):
        step()
    torch.cuda.synchronize()
    flagged = int(d_total.item())
    l0 = c.launches()
    step()
    torch.cuda.synchronize()
    launches_per_step = c.launches() - l0
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    w0 = time.time()
    t0.record(stream)
    for i in range(K):
        step(i)
    t1.record(stream)
    torch.cuda.synchronize()
    w1 = time.time()
    if clocks:
        clocks.mark(w0, w1)
    eager_ms = t0.elapsed_time(t1)
    kern_ms = sum(a.elapsed_time(b) for a, b in zip(ks, ke)) / K
    c.set_kernel_timing(None, None)
    ms, step_mode = eager_ms, "eager"
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
            torch.cuda.synchronize()
            w0 = time.time()
            t0.record(gs)
            with torch.cuda.stream(gs):
                for _ in range(K):
                    graph.replay()
            t1.record(gs)
            torch.cuda.synchronize()
            w1 = time.time()
            if clocks:
                clocks.mark(w0, w1)
            ms, step_mode = t0.elapsed_time(t1), "cuda_graph"
            del graph
        except Exception as exc:  # capture unsupported: the eager timing stands
            print(f"bench: CUDA graph step unavailable ({exc}); eager timing", file=sys.stderr)
    st = c.stats()
    reset = {"mode": "window-lazy" if window else ("epoch" if epoch else "full")}
    if epoch:
        # epoch reset: a rebase sweep of the whole shadow every floor(255 / epochs per check)
        # checks; its cost, amortised, is added to the measured step (reading R19)
        gmax = int((trace.events["meta"][-1] >> 24) & 255) if trace.n else 0
        per_sweep = max(1, 255 // (gmax + 1))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        c.barrier(stream=stream)         # normalises the shadow: one forced rebase sweep
        e1.record(stream)
        torch.cuda.synchronize()
        sweep_ms = e0.elapsed_time(e1)
        ms += K * sweep_ms / per_sweep
        reset.update(sweep_ms=sweep_ms, checks_per_sweep=per_sweep, amortized_ms_per_step=sweep_ms / per_sweep,
                     note="amortised sweep added to ms_per_step")
    peak, peak_kind = peaks()
    bpa = bytes_per_access(c.rec_bytes)
    ms_per_step = ms / K
    achieved = bpa * n_acc / (kern_ms / 1e3) / 1e9
    key = f"cfg{config}_{variant}" + ("_compact" if args.compact else "")
    res = {"config": config, "variant": variant, "trace": trace.name, "events": int(trace.n), "accesses": n_acc,
           "replay": "window-major" if window else "batch-major", "reset": reset,
           "value": n_acc * K / (ms / 1e3), "ms_per_step": ms_per_step, "step_mode": step_mode,
           "eager_ms_per_step": eager_ms / K, "launches_per_step": launches_per_step,
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                        "traffic": load_traffic(key), "traffic_key": key,
                        "kernel": ("k_replay_masked + collect" if trace.warp_syncs is not None
                                   else "k_replay (incl. fused collect)"), "kernel_ms": kern_ms,
                        "kernel_share": kern_ms / ms_per_step, "bytes_per_access": bpa, "peak_kind": peak_kind},
           "roofline_step": {"bound": "hbm", "achieved": bpa * n_acc / (ms_per_step / 1e3) / 1e9, "peak": peak,
                             "unit": "GB/s", "frac": bpa * n_acc / (ms_per_step / 1e3) / 1e9 / peak,
                             "bytes_per_access": bpa, "what": "whole step (reset + batches + replay + collect)"},
           "flagged_words": flagged, "stats_per_step": st,
           "expected_flagged": len(trace.info["expected"]) if "expected" in trace.info else None}
    if keep:
        return res, dict(trace=trace, checker=c, n_acc=n_acc, cap=cap, d_ev=d_ev)
    c.close()
    del d_ev, d_out, d_total
    torch.cuda.empty_cache()
    return res, None


def measure_e2e(ctx, K: int, dev: int) -> dict:
    """The same metric through the C-ABI host entry point: pinned host events -> H2D (chunked,
    overlapped) -> replay -> collect -> D2H of the flagged words, every step."""
    import torch
    trace, c, n_acc, cap = ctx["trace"], ctx["checker"], ctx["n_acc"], ctx["cap"]
    ev = trace.events
    nbytes = ev.shape[0] * 16
    registered = False
    try:  # page-lock the generator's buffer in place (no 17 GB copy)
        rc = torch.cuda.cudart().cudaHostRegister(ev.ctypes.data, nbytes, 0)
        registered = int(rc) == 0 if not isinstance(rc, tuple) else int(rc[0]) == 0
    except Exception:
        registered = False
    hout = torch.empty(cap * 16, dtype=torch.uint8, pin_memory=True)
    stream = torch.cuda.current_stream()
    for _ in range(2):
        c.reset(stream)
        c.check_host_ptr(ev.ctypes.data, ev.shape[0], hout.data_ptr(), cap, stream=stream)
    torch.cuda.synchronize()
    k = max(3, min(K, 10))
    t = time.perf_counter()
    tot = 0
    for _ in range(k):
        c.reset(stream)
        tot = c.check_host_ptr(ev.ctypes.data, ev.shape[0], hout.data_ptr(), cap, stream=stream)
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t) / k
    if registered:
        torch.cuda.cudart().cudaHostUnregister(ev.ctypes.data)
    return {"value": n_acc / dt, "unit": UNIT, "h2d_bytes_per_step": int(nbytes),
            "host_memory": "pinned" if registered else "pageable",
            "d2h_bytes_per_step": int(min(tot, cap) * 16 + 8), "ms_per_step": dt * 1e3, "steps": k,
            "path": "hirace_check_trace_host"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="hirace", choices=["hirace", "reference"])
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--variant", default="racy", choices=["racy", "clean"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-slowdown", action="store_true")
    ap.add_argument("--no-per-config", action="store_true", help="skip the config 2/3/4 secondary measurements")
    ap.add_argument("--no-graph", action="store_true", help="time the eager step instead of its CUDA graph")
    ap.add_argument("--replay-mode", default="auto", choices=["auto", "batch", "window"],
                    help="hirace_set_replay_mode: batch-major k_replay or window-major (auto: window for >= 1 GiB)")
    ap.add_argument("--window-log2", type=int, default=0, help="records per window (log2; 0 = 12)")
    ap.add_argument("--reset-mode", default="epoch", choices=["epoch", "full"],
                    help="hirace_set_reset_mode: epoch (O(flagged) reset, amortised sweeps counted) or full memset")
    ap.add_argument("--compact", action="store_true",
                    help="compact 4-byte shadow records (hirace_shadow_alloc_compact, SURVEY §8(f) f1)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p", "host"],
                    help="config-5 shard exchange (N>1): NCCL device all_to_all, peer-memory dispatch (CUDA IPC / "
                         "NVLink stores from the bucketing kernel), or gloo host staging")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, world)
        return
    if args.config == 5 and world > 1:
        run_sharded_bench(args, world, rank, local_rank)
        return

    import torch
    import torch.distributed as dist
    ngpu = torch.cuda.device_count()
    dev = local_rank % ngpu  # several ranks per GPU only in single-GPU functional runs
    torch.cuda.set_device(dev)
    red_dev = "cuda"
    if world > 1:  # configs 1-4 at N>1: independent replicas (weak scaling, no collective)
        if world <= ngpu:
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group("gloo")
            red_dev = "cpu"
        dist.barrier()
    K, W = args.steps, args.warmup
    clocks = ClockSampler(dev)
    clocks.start()
    time.sleep(0.3)
    res, ctx = measure_single(args, args.config, args.variant, K, W, dev, clocks, keep=True)
    ms, kern_ms = res["ms_per_step"] * K, res["roofline"]["kernel_ms"]
    if world > 1:
        tt = torch.tensor([ms, kern_ms], dtype=torch.float64, device=red_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms, kern_ms = float(tt[0]), float(tt[1])
    ms_per_step = ms / K
    trace, c, n_acc = ctx["trace"], ctx["checker"], ctx["n_acc"]
    cb = config_block(args, trace, world)
    e2e = None if args.no_e2e else measure_e2e(ctx, K, dev)
    if e2e and world > 1:
        tt = torch.tensor([e2e["ms_per_step"]], dtype=torch.float64, device=red_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e["ms_per_step"] = float(tt[0])
        e2e["value"] = n_acc * world / (e2e["ms_per_step"] / 1e3)
    st = res["stats_per_step"]
    l2 = None
    if rank == 0:
        try:
            l2 = l2_roofline(st, n_acc, kern_ms, c.rec_bytes, dev)
            bpa = bytes_per_access(c.rec_bytes)
            l2["hbm_accesses_per_s_peak"] = peaks()[0] * 1e9 / bpa
            l2["binding"] = "hbm" if l2["hbm_accesses_per_s_peak"] <= l2["accesses_per_s_peak"] else "l2_atomic"
        except Exception as exc:  # diagnostics only; never fails the bench line
            l2 = {"error": str(exc)}
    rec_bytes = c.rec_bytes
    n_random = None
    if rank == 0 and args.config == 5 and "regions" in trace.info:
        try:
            n_random = random_rmw_count(trace, ctx["d_ev"])
        except Exception as exc:  # diagnostics only
            print(f"bench: random-region count failed ({exc})", file=sys.stderr)
    c.close()
    ctx["d_ev"] = None
    torch.cuda.empty_cache()
    rnd = None
    if n_random:
        try:
            rnd = random_roofline(n_random, kern_ms, dev)
        except Exception as exc:  # diagnostics only
            rnd = {"error": str(exc)}
    cpu = None
    if not args.no_cpu_baseline and world == 1 and rank == 0:
        cpu = cpu_baseline(trace, 20.0)
    trace.info.pop("buffer", None)
    del trace, ctx
    per_config = {}
    if not args.no_per_config and world == 1:
        for cfg in (2, 3, 4, 6):
            if cfg == args.config:
                continue
            r, _ = measure_single(args, cfg, "racy", min(K, 20), W, dev, None)
            per_config[f"config{cfg}"] = {k: r[k] for k in ("trace", "events", "value", "ms_per_step", "step_mode",
                                                            "roofline", "roofline_step", "flagged_words",
                                                            "launches_per_step", "replay", "reset")}
    slow = None if (args.no_slowdown or rank != 0) else measure_slowdown(dev)
    clocks.stop()
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    roof = dict(res["roofline"])
    roof["kernel_ms"] = kern_ms
    roof["achieved"] = roof["bytes_per_access"] * n_acc / (kern_ms / 1e3) / 1e9
    roof["frac"] = roof["achieved"] / roof["peak"]
    roof["kernel_share"] = kern_ms / ms_per_step
    out = {
        "metric": METRIC, "value": n_acc * world * K / (ms / 1e3), "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": W, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong" if args.config == 5 else "weak", "vs_baseline": None,
        "dtype": "u64" if rec_bytes == 8 else "u32", "data": "synthetic", "config": cb,
        "roofline": roof, "roofline_step": res["roofline_step"], "roofline_l2": l2,
        "roofline_dram_random": rnd,
        "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": res["launches_per_step"] * K,
        "step_mode": res["step_mode"], "eager_ms_per_step": res["eager_ms_per_step"],
        "replay": res["replay"], "reset": res["reset"],
        "clocks": clocks.summary(),
        "check": {"flagged_words": res["flagged_words"], "expected_flagged": res["expected_flagged"],
                  "per_step": st},  # stats are per step (reset clears them)
        "per_config": per_config or None,
        "instrumented_slowdown": slow,
        "shadow_overhead": {"bytes_per_tracked_word": rec_bytes, "ratio_to_tracked_bytes": rec_bytes / 4,
                            "iguard_ratio_context": 4.0},
    }
    if world > 1:
        dist.destroy_process_group()
    print(json.dumps(out), flush=True)  # last, after any NCCL teardown log lines


if __name__ == "__main__":
    main()
