#!/usr/bin/env python
"""Benchmark: malloc+free calls/s of the B200-native allocator vs CUDA device malloc.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` prints ONE JSON
line on rank 0.  One "step" = one pass of the whole hot path over one batch: the
mixed-size churn trace d4 (BASELINE.json configs[3]) at full B200
occupancy -- 303,104 threads x 16 rounds of {free previous block; malloc 16 B..64 KiB}
plus the final free-all, on a 4 GiB heap ("pressure": ~71 % of the heap live after
rounding) -- run as ONE kernel (timing mode, ga_trace_timed).  ``value`` = malloc
calls (failed ones included) + frees, per second, summed over ranks.

N > 1: one process per GPU, each with its own heap (replicas, no data-path
collective); timing is the max over ranks.

``--impl reference``: the reference arm is the sequential CPU oracle (oracle/),
timed on this host on the same trace (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import tracegen  # noqa: E402

METRIC = "malloc+free calls/s on 1 B200 vs CUDA device malloc; fragmentation ratio"
UNIT = "calls/s"
L2_FLUSH_BYTES = 512 << 20


# ----------------------------------------------------------------------------- helpers
def algorithmic_atomics(sizes: np.ndarray) -> int:
    """Minimum L2 atomics the method must issue for one pass of a D=1 trace with
    every call succeeding: per warp-round and size class,
    a group of N lanes needs 1 semaphore op + ceil(N / slots-per-bitmap-word)
    tracking ops (bins: min(64, 4096/class); tree: 64 nodes per level word), for
    the mallocs and again for the frees of the same blocks."""
    R, T = sizes.shape
    n = sizes.astype(np.int64)
    lg = np.ceil(np.log2(np.maximum(n, 16))).astype(np.int64)           # class log2
    key = lg - 4                                                        # 0..7 bins, 8.. tree
    W = T // 32
    k = key[:, : W * 32].reshape(R, W, 32)
    total = 0
    for c in range(int(key.max()) + 1):
        N = (k == c).sum(axis=2)
        per_word = min(64, 4096 >> (c + 4)) if c < 8 else 64
        total += int(((N > 0) * (1 + (N + per_word - 1) // per_word)).sum())
    return 2 * total


class Clocks:
    """SM clock and throttle-reason sampling DURING the timed region (the
    B200_PROFILING.md clocks line).  NVML polled from a thread every ~2 ms
    between mark() and stop(): the timed region of this bench is tens of
    milliseconds, shorter than nvidia-smi's sampling period."""

    NAMES = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
             ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
             ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
             ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
             ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, index: int):
        import threading
        self.samples, self.reasons, self.max_mhz, self.err = [], set(), None, None
        self.run = threading.Event()
        self.done = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            phys = int(vis.split(",")[index]) if vis and vis.split(",")[index].strip().isdigit() else index
            self.nv, self.h = pynvml, pynvml.nvmlDeviceGetHandleByIndex(phys)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception as e:                                # noqa: BLE001
            self.nv, self.err = None, repr(e)
            return
        self.t = threading.Thread(target=self._loop, daemon=True)
        self.t.start()

    def _loop(self):
        nv = self.nv
        while not self.done.is_set():
            if self.run.is_set():
                try:
                    self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                    for name, const in self.NAMES:
                        if r & getattr(nv, const, 0):
                            self.reasons.add(name)
                except Exception:                              # noqa: BLE001
                    pass
            time.sleep(0.002)

    def mark(self):
        """Start of the timed region."""
        self.run.set()

    def stop(self) -> dict:
        if self.nv is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [f"nvml unavailable: {self.err}"], "samples": 0}
        self.done.set()
        self.t.join(timeout=2)
        sm = self.samples
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(sm), "source": "nvml, ~2 ms period"}


def cpu_cores() -> int:
    return len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()


def oracle_leg(trace, budget_s: float = 10.0) -> dict:
    """The oracle as it stands, on this host, 1 thread: the whole trace, repeated
    until ~budget_s of CPU work (bounded sample)."""
    import oracle
    oracle.build()
    runs, calls, t_total, st = 0, 0, 0.0, None
    while t_total < budget_s or runs == 0:
        t0 = time.perf_counter()
        r = oracle.run_trace(trace.sizes, trace.heap_bytes, trace.D, want_ok=False)
        t_total += time.perf_counter() - t0
        st = r.stats
        calls += st["calls"]
        runs += 1
        if runs >= 64:
            break
    return {"value": calls / t_total, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{trace.name}: whole trace ({trace.R} rounds x {trace.T} threads, "
                      f"{st['calls']} calls) x {runs} runs, sequential C oracle, {t_total:.1f} s",
            "seconds": t_total, "stats": st}


def _oracle_shard(arg):
    sizes, heap_bytes, D, budget_s = arg
    import oracle
    calls, t_total, runs = 0, 0.0, 0
    while t_total < budget_s or runs == 0:
        t0 = time.perf_counter()
        r = oracle.run_trace(sizes, heap_bytes, D, want_ok=False)
        t_total += time.perf_counter() - t0
        calls += r.stats["calls"]
        runs += 1
    return calls, t_total


def oracle_leg_parallel(trace, budget_s: float = 6.0) -> dict:
    """SURVEY.md 8(d) "P cores": P = usable host cores independent oracle instances,
    instance j on the threads tid = j mod P with a heap/P heap (rounded down to a
    chunk multiple); the aggregate of their calls/s."""
    import multiprocessing as mp
    import oracle
    oracle.build()
    P = max(1, min(cpu_cores(), 64))
    hb = max(256 << 10, (trace.heap_bytes // P) & ~((256 << 10) - 1))
    shards = [(np.ascontiguousarray(trace.sizes[:, j::P]), hb, trace.D, budget_s) for j in range(P)]
    with mp.get_context("fork").Pool(P) as pool:
        out = pool.map(_oracle_shard, shards)
    value = sum(c / t for c, t in out)
    return {"value": value, "unit": UNIT, "cores": P, "kind": "oracle",
            "sample": f"{trace.name}: {P} independent sequential C oracles, shard j = threads tid = j mod {P}, "
                      f"heap {hb} B each, each repeated for ~{budget_s:.0f} s"}


# ----------------------------------------------------------------------------- reference arm
def run_reference(args, trace):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    for _ in range(args.warmup):
        oracle.run_trace(trace.sizes, trace.heap_bytes, trace.D, want_ok=False)
    times, calls = [], 0
    for _ in range(args.steps):
        t0 = time.perf_counter()
        r = oracle.run_trace(trace.sizes, trace.heap_bytes, trace.D, want_ok=False)
        times.append(time.perf_counter() - t0)
        calls = r.stats["calls"]
    ms = 1e3 * sum(times) / len(times)
    value = calls / (ms / 1e3)
    out = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
           "config": config_of(trace, args),
           "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": f"{trace.name}: the whole trace per step ({calls} calls), sequential C oracle"},
           "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "fragmentation": {"oracle": r.stats["peak_reserved_bytes"] / max(1, r.stats["peak_live_bytes"])}}
    print(json.dumps(out), flush=True)
    return 0


def config_of(trace, args):
    return {"workload": trace.name, "threads": trace.T, "rounds": trace.R, "free_depth": trace.D,
            "heap_bytes": trace.heap_bytes, "sizes": "n = 2^k + U[1,2^k], k~U{3..15} (16 B - 64 KiB classes)",
            "block": args.block, "l2": "flushed between steps (512 MiB write)", "seed": hex(trace.seed)}


def d3_sweep(ga, heap, stream, dev, T, args, sizes=(16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 8192), R=16):
    import torch
    res = {}
    cc = torch.zeros(8, dtype=torch.int64, device=dev)
    for sz in sizes:
        d = torch.full((R * T,), sz, dtype=torch.int32, device=dev)
        heap.reset()
        times = []
        for rep in range(4):
            cc.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_trace_timed(heap.h, stream.cuda_stream, d.data_ptr(), R, T, 0, cc.data_ptr(), args.block)
            a1.record(stream)
            a1.synchronize()
            if rep:
                times.append(a0.elapsed_time(a1) / 1e3)
        c = cc.cpu().numpy()
        ours = float(c[0] + c[2]) / (sum(times) / len(times))
        fails = int(c[1])
        cc.zero_()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        ga.ga_cuda_trace_timed(stream.cuda_stream, d.data_ptr(), 1, T, 0, cc.data_ptr(), args.block)
        a1.record(stream)
        a1.synchronize()
        c = cc.cpu().numpy()
        cuda = float(c[0] + c[2]) / (a0.elapsed_time(a1) / 1e3)
        res[str(sz)] = {"ours": ours, "cuda_malloc": cuda, "speedup": ours / cuda, "ours_failed": fails,
                        "cuda_failed": int(c[1]), "ours_rounds": R, "cuda_rounds": 1}
    vals = [v["speedup"] for v in res.values()]
    res["min_speedup"] = min(vals)
    res["geomean_speedup"] = float(np.exp(np.mean(np.log(vals))))
    return res


def d4_levels(ga, stream, dev, args, flush, levels=("fit", "exhaust", "overcommit"), reps=3):
    """d4 at the other two pressure levels: the same mixed trace on
    a 16 GiB heap (fit: every malloc succeeds), a 3 GiB heap (exhaust: the peak
    reserved reaches ~99 % of the heap) and a 2.75 GiB heap (overcommit: below
    the oracle's own peak reserved, so both sides fail mallocs and reclaim under
    real exhaustion).  calls/s from the timed
    kernel; failures and fragmentation from correctness mode, beside the oracle's."""
    import torch
    import oracle
    from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness
    oracle.build()
    res = {}
    cc = torch.zeros(8, dtype=torch.int64, device=dev)
    for lv in levels:
        t = tracegen.d4_mixed(lv)
        heap = GpuHeap(t.heap_bytes, device=dev.index or 0, stream=stream)
        d = torch.from_numpy(t.sizes.view(np.int32)).to(dev)
        times, fails = [], 0
        for rep in range(reps + 1):
            flush.fill_(rep)
            cc.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_trace_timed(heap.h, stream.cuda_stream, d.data_ptr(), t.R, t.T, t.D, cc.data_ptr(), args.block)
            a1.record(stream)
            a1.synchronize()
            if rep:
                times.append(a0.elapsed_time(a1) / 1e3)
                fails = max(fails, int(cc[1].item()))
        calls = int(cc[0].item() + cc[2].item())
        heap.reset()
        run = run_correctness(heap, t.sizes, t.D, log=False, tag=False, reserved=True)
        ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_ok=False).stats
        fg = run.peak_reserved_bytes / run.peak_live_bytes if run.peak_live_bytes else None
        fo = ref["peak_reserved_bytes"] / ref["peak_live_bytes"]
        st = heap.stats()
        res[lv] = {"heap_bytes": t.heap_bytes, "calls_per_s": calls / (sum(times) / len(times)),
                   "ms": 1e3 * sum(times) / len(times), "timed_failed_mallocs": fails,
                   "correctness_failed_mallocs": run.counts["n_fail"], "oracle_failed_mallocs": ref["n_malloc_fail"],
                   "fragmentation": {"gpu": fg, "oracle": fo, "ratio": fg / fo if fg else None},
                   "stats": {k: int(v) for k, v in st.items() if isinstance(v, (int, np.integer))}}
        heap.close()
        del d
    return res


def d2_bsem(ga, stream, dev, grid=148 * 8, block=256, iters=32):
    """wait(k)/signal(k) per thread per iteration on a full grid; ops = wait+signal pairs."""
    import torch
    names = {0: "warp_aggregated_bulk", 1: "per_thread_bulk", 2: "per_thread_counting", 3: "plain_atomics"}
    res = {}
    sems = torch.zeros(148 * 4 + 8, dtype=torch.int64, device=dev)
    out = torch.zeros(8, dtype=torch.int64, device=dev)
    for n_sems in (1, 148):
        for k in (1, 32, 0):
            for v in (0, 1, 2, 3):
                if v == 2 and k != 1:
                    continue
                cfg = ga.BsemCfg(variant=v, k=k, B=512, n_sems=n_sems, iters=iters, acquire_only=0, grid=grid,
                                 block=block, seed=tracegen.BASE_SEED + 2)
                best = None
                for rep in range(3):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    ga.ga_bsem_bench(stream.cuda_stream, cfg, sems.data_ptr(), out.data_ptr())
                    e1.record(stream)
                    e1.synchronize()
                    t = e0.elapsed_time(e1) / 1e3
                    best = t if best is None else min(best, t)
                o = out.cpu().numpy()
                res[f"{names[v]}/k={k or 'rand'}/sems={n_sems}"] = {
                    "pairs_per_s": grid * block * iters / best, "units_per_s": float(o[0]) / best,
                    "quiescent_C_equals_produced": bool(o[4] == o[3]), "max_abs_D": int(o[5])}
    return res


# ----------------------------------------------------------------------------- multi-GPU (replicas)
def rank_trace(trace, rank: int):
    """Replicas: rank r runs the same recipe with seed + r;
    rank 0 runs the canonical bench trace."""
    if rank == 0:
        return trace
    return tracegen.Trace(trace.name, tracegen.mixed_sizes(trace.seed + rank, trace.R, trace.T), trace.D,
                          trace.heap_bytes, trace.seed + rank)


def reduce_over_ranks(dist, ms: float, calls: float, device):
    """Whole-job numbers: the slowest rank's time and the calls of all ranks."""
    import torch
    t = torch.tensor([ms], device=device, dtype=torch.float64)
    c = torch.tensor([calls], device=device, dtype=torch.float64)
    if dist is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(c, op=dist.ReduceOp.SUM)
    return float(t.item()), float(c.item())


# ----------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--block", type=int, default=256)
    ap.add_argument("--no-extras", action="store_true", help="skip CUDA-malloc, sweep, frag, cpu legs")
    ap.add_argument("--cuda-budget-s", type=float, default=20.0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    trace = tracegen.d4_mixed("pressure")
    if args.impl == "reference":
        return run_reference(args, trace)

    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)

    # per-rank trace (replicas: seed + rank); rank 0 uses the canonical trace
    trace = rank_trace(trace, rank)
    R, T, D = trace.R, trace.T, trace.D
    if not args.no_extras:
        ga.ga_cuda_set_heap_limit(trace.heap_bytes)       # before any kernel that uses malloc
    heap = GpuHeap(trace.heap_bytes, device=local, stream=stream)
    d_sizes = torch.from_numpy(trace.sizes.view(np.int32)).to(dev)
    counts = torch.zeros(8, dtype=torch.int64, device=dev)
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=dev)

    def step():
        ga.ga_trace_timed(heap.h, stream.cuda_stream, d_sizes.data_ptr(), R, T, D, counts.data_ptr(), args.block)

    def timed_steps(n, cold):
        """n steps, each bracketed by CUDA events on the heap's stream.  cold: the
        heap is reset (ga_heap_reset, untimed) before every step, SURVEY 8(d)."""
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        for i, (s, e) in enumerate(ev):
            if cold:
                heap.reset()                                # untimed, outside the events
            flush.fill_(i & 7)                              # L2 flush (512 MiB write), outside the events
            s.record(stream)
            step()
            e.record(stream)
        return ev

    for _ in range(args.warmup):
        heap.reset()
        flush.fill_(1)
        step()
    torch.cuda.synchronize()
    counts.zero_()
    clocks = Clocks(local)
    clocks.mark()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    t_wall = time.perf_counter()
    ev = timed_steps(args.steps, cold=True)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    wall = time.perf_counter() - t_wall
    clk = clocks.stop()
    kern_ms = [s.elapsed_time(e) for s, e in ev]
    ms = sum(kern_ms) / len(kern_ms)
    c = counts.cpu().numpy()
    # the same steps on a warm heap (no reset: bins and chunks of the previous step reused)
    counts.zero_()
    ev_w = timed_steps(args.steps, cold=False)
    torch.cuda.synchronize()
    warm_ms = sum(s.elapsed_time(e) for s, e in ev_w) / args.steps
    calls_step = int(c[0] + c[2]) // args.steps
    fails_step = int(c[1]) // args.steps
    ms_max, tot = reduce_over_ranks(dist, ms, calls_step, dev)
    value = tot / (ms_max / 1e3)

    # ---- e2e: host buffers through the C ABI (H2D of the trace, kernel, D2H of counts)
    h_sizes = torch.from_numpy(trace.sizes.view(np.int32)).pin_memory()
    h_counts = np.zeros(4, dtype=np.uint64)
    from paper_conf_ppopp_geladog19_b200.runner import run_timed_host
    e2e_ms = []
    for i in range(args.warmup + args.steps):
        heap.reset()
        flush.fill_(2)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        run_timed_host(heap, h_sizes, R, T, D, h_counts, args.block, stream)
        s1.record(stream)
        s1.synchronize()
        if i >= args.warmup:
            e2e_ms.append(s0.elapsed_time(s1))
    e2e_calls = int(h_counts[0] + h_counts[2])
    e2e_ms_max, e2e_tot = reduce_over_ranks(dist, sum(e2e_ms) / len(e2e_ms), e2e_calls, dev)
    e2e = {"value": e2e_tot / (e2e_ms_max / 1e3), "unit": UNIT,
           "h2d_bytes_per_step": int(trace.sizes.nbytes), "d2h_bytes_per_step": 32,
           "ms_per_step": e2e_ms_max}

    if rank != 0:
        if dist:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    # ---- roofline: L2 atomics, peak from the committed microbenchmark, measured live
    buf = torch.zeros(148 * 8 * 256 * 4 + 8192, dtype=torch.int64, device=dev)
    sink = torch.zeros(8, dtype=torch.int64, device=dev)
    peaks = {}
    grid, blk, iters = 148 * 8, 256, 64
    for pat in (0, 1, 3):
        for rep in range(3):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_l2_atomic_bench(stream.cuda_stream, pat, buf.data_ptr(), buf.numel(), iters, grid, blk,
                                  sink.data_ptr())
            a1.record(stream)
            a1.synchronize()
            if rep:
                rate = grid * blk * iters / (a0.elapsed_time(a1) / 1e3) / 1e9
                peaks[pat] = max(peaks.get(pat, 0.0), rate)
    p_atom = max(peaks[0], peaks[1])
    a_min = algorithmic_atomics(trace.sizes)
    achieved = a_min / (ms / 1e3) / 1e9
    kinfo = ga.ga_kernel_info(0, args.block)
    traffic = None                                          # DRAM bytes per launch, from the committed ncu capture
    tf = os.path.join(ROOT, "profiles", "r01_ncu_traffic.json")
    if os.path.exists(tf):
        traffic = json.load(open(tf)).get("traffic_bytes")
    roofline = {"bound": "l2_atomic", "achieved": achieved, "peak": p_atom, "unit": "Gatom/s",
                "frac": achieved / p_atom, "traffic": traffic, "traffic_unit": "DRAM bytes per launch (ncu)",
                "per_launch_algorithmic_atomics": a_min,
                "peak_source": "measured live: ga_l2_atomic_bench distinct-word ATOMG/REDG (max)",
                "peak_patterns_gatom_s": {"atomg_distinct": peaks[0], "redg_distinct": peaks[1],
                                          "atomg_1184_words": peaks[3]},
                "kernel": {"regs": kinfo["regs"], "blocks_per_sm": kinfo["blocks_per_sm"],
                           "stack_bytes": kinfo["local_bytes"]}}

    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms_max, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "u64", "data": "synthetic",
           "config": config_of(trace, args), "e2e": e2e, "gpu_launches": args.steps,
           "clocks": clk, "roofline": roofline,
           "calls_per_step": calls_step, "failed_mallocs_per_step": fails_step,
           "kernel_ms": {"min": min(kern_ms), "max": max(kern_ms)},
           "heap": "cold: ga_heap_reset (untimed) before every step",
           "warm": {"ms_per_step": warm_ms, "value": calls_step / (warm_ms / 1e3)}, "wall_s_timed_region": wall}

    if not args.no_extras:
        # ---- fragmentation (correctness mode: one kernel per round, reserved at boundaries)
        heap.reset()
        run = run_correctness(heap, trace.sizes, D, log=False, tag=False, reserved=True)
        live_peak = run.peak_live_bytes                    # the GPU's own successful requests
        cpu = oracle_leg(trace, budget_s=10.0)
        frag_ora = cpu["stats"]["peak_reserved_bytes"] / cpu["stats"]["peak_live_bytes"]
        frag_gpu = run.peak_reserved_bytes / live_peak if live_peak else None
        out["fragmentation"] = {"gpu": frag_gpu, "oracle": frag_ora,
                                "ratio": frag_gpu / frag_ora if frag_gpu else None,
                                "gpu_peak_reserved_bytes": run.peak_reserved_bytes,
                                "peak_live_bytes": live_peak,
                                "oracle_peak_reserved_bytes": cpu["stats"]["peak_reserved_bytes"],
                                "gpu_failed_mallocs": run.counts["n_fail"]}
        cpu.pop("stats")
        cpu.pop("seconds")
        out["cpu_baseline"] = cpu
        out["cpu_baseline_all_cores"] = oracle_leg_parallel(trace)

        # ---- CUDA device malloc on the same trace (bounded prefix of rounds)
        heap.reset()
        torch.cuda.synchronize()
        cc = torch.zeros(8, dtype=torch.int64, device=dev)
        rr, t_cuda = 1, None
        while True:
            cc.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_cuda_trace_timed(stream.cuda_stream, d_sizes.data_ptr(), rr, T, D, cc.data_ptr(), args.block)
            a1.record(stream)
            a1.synchronize()
            t_cuda = a0.elapsed_time(a1) / 1e3
            if t_cuda * 2 > args.cuda_budget_s or rr >= R:
                break
            rr = min(R, rr * 2)
        ccn = cc.cpu().numpy()
        cuda_rate = float(ccn[0] + ccn[2]) / t_cuda
        out["cuda_malloc"] = {"value": cuda_rate, "unit": UNIT, "rounds": rr,
                              "failed_mallocs": int(ccn[1]), "seconds": t_cuda,
                              "heap_limit_bytes": trace.heap_bytes}
        out["speedup_vs_cuda_malloc"] = value / cuda_rate

        # ---- d3: warp-uniform sizes 16 B - 8 KiB (BASELINE configs[2]), malloc+free per
        # thread and round (D = 0), full grid; CUDA malloc on a bounded prefix of rounds
        out["d3_sweep"] = d3_sweep(ga, heap, stream, dev, T, args)

        # ---- d4 at the fit and exhaust pressure levels
        out["d4_levels"] = d4_levels(ga, stream, dev, args, flush)

        # ---- d2: bulk-semaphore microbenchmark (BASELINE configs[1], Sec. 5.1)
        out["d2_bsem"] = d2_bsem(ga, stream, dev)

    print(json.dumps(out), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()
    heap.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
