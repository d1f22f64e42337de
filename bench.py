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
_T0 = time.time()


def _progress(what: str):
    """Elapsed wall time of each bench leg on stderr (the JSON line stays on stdout)."""
    print(f"[bench] {time.time() - _T0:7.1f} s  {what}", file=sys.stderr, flush=True)


def algorithmic_atomics(sizes: np.ndarray, group: int = 32) -> int:
    """Minimum L2 atomics the method must issue for one pass of a D=1 trace with
    every call succeeding: per warp-round and size class,
    a group of N lanes needs 1 semaphore op + ceil(N / slots-per-bitmap-word)
    tracking ops (bins: min(64, 4096/class); tree: 64 nodes per level word), for
    the mallocs and again for the frees of the same blocks.  `group`: threads
    that call together (32 warp calls; the block or cluster size for the
    collective calls, whose class groups are whole CTAs / clusters)."""
    R, T = sizes.shape
    n = sizes.astype(np.int64)
    lg = np.ceil(np.log2(np.maximum(n, 16))).astype(np.int64)           # class log2
    key = lg - 4                                                        # 0..7 bins, 8.. tree
    W = T // group
    k = key[:, : W * group].reshape(R, W, group)
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
            "block": args.block, "l2": "flushed between steps (512 MiB write)", "heap_state": "cold (reset per step)",
            "seed": hex(trace.seed)}


def d3_sweep(ga, heap, stream, dev, T, args, sizes=(16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 8192), R=16):
    """d3 (BASELINE configs[2]): warp-uniform size s, every thread R rounds of
    malloc(s) + free on a 4 GiB heap at full occupancy, heap reset (untimed)
    before every rep; CUDA malloc on one round of the same trace; fragmentation
    of one malloc-only phase (correctness mode) beside the oracle's."""
    import torch
    import oracle
    from paper_conf_ppopp_geladog19_b200.runner import run_correctness
    res = {}
    cc = torch.zeros(8, dtype=torch.int64, device=dev)
    for sz in sizes:
        d = torch.full((R * T,), sz, dtype=torch.int32, device=dev)
        times, fails = [], 0
        for rep in range(4):
            heap.reset()
            cc.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_trace_timed(heap.h, stream.cuda_stream, d.data_ptr(), R, T, 0, cc.data_ptr(), args.block)
            a1.record(stream)
            a1.synchronize()
            if rep:
                times.append(a0.elapsed_time(a1) / 1e3)
                fails += int(cc[1].item())
        times.sort()
        ours = float(R * T * 2) / times[len(times) // 2]
        cc.zero_()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        ga.ga_cuda_trace_timed(stream.cuda_stream, d.data_ptr(), 1, T, 0, cc.data_ptr(), args.block)
        a1.record(stream)
        a1.synchronize()
        c = cc.cpu().numpy()
        cuda = float(c[0] + c[2]) / (a0.elapsed_time(a1) / 1e3)
        one = np.full((1, T), sz, dtype=np.uint32)
        heap.reset()
        run = run_correctness(heap, one, 0, log=False, tag=False, reserved=True)
        ref = oracle.run_trace(one, heap.heap_bytes, 0, want_ok=False).stats
        fg = run.peak_reserved_bytes / run.peak_live_bytes
        fo = ref["peak_reserved_bytes"] / ref["peak_live_bytes"]
        _progress(f"d3 {sz} B")
        res[str(sz)] = {"Gcalls_s": ours / 1e9, "cuda_Mcalls_s": cuda / 1e6, "x_cuda": ours / cuda,
                        "failed": fails + int(c[1]) + run.counts["n_fail"],
                        "frag": {"gpu": round(fg, 4), "oracle": round(fo, 4), "ratio": round(fg / fo, 4)}}
    vals = [v["x_cuda"] for v in res.values()]
    res["min_x_cuda"] = min(vals)
    res["geomean_x_cuda"] = float(np.exp(np.mean(np.log(vals))))
    res["max_frag_ratio"] = max(v["frag"]["ratio"] for k, v in res.items() if isinstance(v, dict))
    return res


def d4_levels(ga, stream, dev, args, flush, levels=("fit", "exhaust", "overcommit"), reps=3):
    """d4 at the other pressure levels: the same mixed trace on
    a 16 GiB heap (fit: every malloc succeeds), a 3 GiB heap (exhaust: the peak
    reserved reaches ~99 % of the heap) and a 2.75 GiB heap (overcommit: below
    the oracle's own peak reserved, so both sides fail mallocs).  calls/s from
    the timed kernel on a cold heap; failures and fragmentation from correctness
    mode, beside the oracle's."""
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
            heap.reset()
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
        st = heap.stats()
        ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_ok=False).stats
        fg = run.peak_reserved_bytes / run.peak_live_bytes if run.peak_live_bytes else None
        fo = ref["peak_reserved_bytes"] / ref["peak_live_bytes"]
        res[lv] = {"heap_GiB": t.heap_bytes / 2 ** 30, "ms": 1e3 * sum(times) / len(times),
                   "Gcalls_s": calls / (sum(times) / len(times)) / 1e9, "failed_timed": fails,
                   "failed": {"gpu": run.counts["n_fail"], "oracle": ref["n_malloc_fail"]},
                   "frag": {"gpu": fg, "oracle": fo, "ratio": fg / fo if fg else None},
                   "reclaims": {"bins": int(st["n_bin_reclaim"]), "by_waiters": int(st["n_waiter_reclaim"])}}
        heap.close()
        del d
        _progress(f"d4 level {lv}")
    return res


def d2_bsem(ga, stream, dev, grid=148 * 8, block=256, iters=32):
    """A summary of d2 (the full k x B x variant matrix is tools/d2_matrix.py):
    wait(k)/signal(k) per thread per iteration on a full grid, B = 512 (the
    paper's); G wait+signal pairs per second."""
    import torch
    names = {0: "warp_bulk", 1: "thread_bulk", 2: "thread_counting", 3: "plain_atomics"}
    res = {}
    sems = torch.zeros(148 * 4 + 8, dtype=torch.int64, device=dev)
    out = torch.zeros(8, dtype=torch.int64, device=dev)
    for n_sems in (1, 148):
        for k in (1, 32, 0):
            for v in (0, 1, 2, 3):
                if v == 2 and k != 1:
                    continue
                # per-thread forms on ONE hot word run ~1e5 pairs/s (the collapse d2
                # exists to show): a bounded sample of them (one block per SM, 4
                # iterations, one rep) keeps the leg to seconds
                slow = v in (1, 2) and n_sems == 1
                g = 148 if slow else grid
                cfg = ga.BsemCfg(variant=v, k=k, B=512, n_sems=n_sems, iters=4 if (slow or v == 2) else iters,
                                 acquire_only=0, grid=g, block=block, seed=tracegen.BASE_SEED + 2)
                best = None
                for rep in range(1 if slow else 3):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    ga.ga_bsem_bench(stream.cuda_stream, cfg, sems.data_ptr(), out.data_ptr())
                    e1.record(stream)
                    e1.synchronize()
                    t = e0.elapsed_time(e1) / 1e3
                    best = t if best is None else min(best, t)
                o = out.cpu().numpy()
                ok = bool(o[4] == o[3]) and int(o[5]) == 0
                res[f"{names[v]}/k={k or 'rand'}/sems={n_sems}"] = round(g * block * cfg.iters / best / 1e9, 4) \
                    if ok else "accounting mismatch"
    res["unit"] = "G wait+signal pairs/s"
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


def launch_or_refuse(args, argv) -> int | None:
    """--gpus N: one process per GPU.  Without a torchrun environment and N > 1,
    relaunch this command under torch.distributed.run on N local GPUs; inside
    one, refuse a WORLD_SIZE that is not N (a silent 1-GPU run would mislabel
    n_gpus).  None = go on in this process."""
    world = os.environ.get("WORLD_SIZE")
    if world is None:
        if args.gpus <= 1:
            return None
        import socket
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *argv]
        return subprocess.call(cmd)
    if int(world) != args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; refusing\n")
        return 2
    return None


def parse_args(argv):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--block", type=int, default=256)
    ap.add_argument("--no-extras", action="store_true", help="skip CUDA-malloc, sweep, frag, cpu legs")
    ap.add_argument("--cuda-budget-s", type=float, default=20.0)
    args = ap.parse_args(argv)
    args.warmup = max(args.warmup, 3)
    return args


# ----------------------------------------------------------------------------- our arm (one rank, one GPU)
class GpuArm:
    """The device work of one rank: its own heap and trace (replicas), W warm-up
    and K timed steps of the d4 trace in ONE kernel each, CUDA events on the
    heap's stream, the heap reset (one kernel, untimed) and L2 flushed before
    every step; then the same through the C ABI with host buffers (e2e)."""
    backend = "nccl"

    def __init__(self, args, rank, local):
        import torch
        import paper_conf_ppopp_geladog19_b200 as ga
        from paper_conf_ppopp_geladog19_b200.runner import GpuHeap
        self.torch, self.ga, self.args, self.rank = torch, ga, args, rank
        torch.cuda.set_device(local)
        self.dev = torch.device("cuda", local)
        self.reduce_device = self.dev
        self.local = local
        self.stream = torch.cuda.current_stream(self.dev)
        self.trace = rank_trace(tracegen.d4_mixed("pressure"), rank)
        if not args.no_extras:
            ga.ga_cuda_set_heap_limit(self.trace.heap_bytes)   # before any kernel that uses malloc
        self.heap = GpuHeap(self.trace.heap_bytes, device=local, stream=self.stream)
        self.d_sizes = torch.from_numpy(self.trace.sizes.view(np.int32)).to(self.dev)
        self.counts = torch.zeros(8, dtype=torch.int64, device=self.dev)
        self.flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=self.dev)

    def _step(self):
        t = self.trace
        self.ga.ga_trace_timed(self.heap.h, self.stream.cuda_stream, self.d_sizes.data_ptr(), t.R, t.T, t.D,
                               self.counts.data_ptr(), self.args.block)

    def _timed_steps(self, n, cold):
        torch = self.torch
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        for i, (s, e) in enumerate(ev):
            if cold:
                self.heap.reset()                           # one kernel, untimed (outside the events)
            self.flush.fill_(i & 7)                         # L2 flush (512 MiB write), outside the events
            s.record(self.stream)
            self._step()
            e.record(self.stream)
        return ev

    def measure(self, barrier):
        torch, args, t = self.torch, self.args, self.trace
        for _ in range(args.warmup):
            self.heap.reset()
            self.flush.fill_(1)
            self._step()
        torch.cuda.synchronize()
        self.counts.zero_()
        clocks = Clocks(self.local)
        clocks.mark()
        barrier()
        torch.cuda.synchronize()
        t_wall = time.perf_counter()
        ev = self._timed_steps(args.steps, cold=True)
        torch.cuda.synchronize()
        barrier()
        wall = time.perf_counter() - t_wall
        clk = clocks.stop()
        kern_ms = [s.elapsed_time(e) for s, e in ev]
        c = self.counts.cpu().numpy()
        self.counts.zero_()
        ev_w = self._timed_steps(args.steps, cold=False)         # warm heap: the previous step's bins reused
        torch.cuda.synchronize()
        warm_ms = sum(s.elapsed_time(e) for s, e in ev_w) / args.steps
        # e2e through the C ABI: H2D of the step's trace from pinned memory, the
        # kernel, D2H of the counts, all inside the events
        from paper_conf_ppopp_geladog19_b200.runner import run_timed_host
        h_sizes = torch.from_numpy(t.sizes.view(np.int32)).pin_memory()
        h_counts = np.zeros(4, dtype=np.uint64)
        e2e_ms = []
        for i in range(args.warmup + args.steps):
            self.heap.reset()
            self.flush.fill_(2)
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s0.record(self.stream)
            run_timed_host(self.heap, h_sizes, t.R, t.T, t.D, h_counts, args.block, self.stream)
            s1.record(self.stream)
            s1.synchronize()
            if i >= args.warmup:
                e2e_ms.append(s0.elapsed_time(s1))
        calls = int(c[0] + c[2]) // args.steps
        return {"ms": sum(kern_ms) / len(kern_ms), "calls": calls, "fails": int(c[1]) // args.steps,
                "kern_ms": kern_ms, "warm_ms": warm_ms, "wall": wall, "clocks": clk,
                "e2e_ms": sum(e2e_ms) / len(e2e_ms), "e2e_calls": int(h_counts[0] + h_counts[2]),
                "h2d": int(t.sizes.nbytes), "d2h": 32,
                # per step: the timed kernel; between the events: 1 reset kernel + 1 torch fill (L2 flush)
                "launches": args.steps * 2, "launch_note": "per step: k_timed (timed) + k_reset (untimed, between events)"}

    def roofline(self, ms):
        ga, torch = self.ga, self.torch
        peak = l2_peak(ga, torch, self.dev, self.stream)
        a_min = algorithmic_atomics(self.trace.sizes)
        achieved = a_min / (ms / 1e3) / 1e9
        kinfo = ga.ga_kernel_info(0, self.args.block)
        traffic = None                                       # DRAM bytes per launch, from the committed ncu capture
        for name in ("r02_ncu_traffic.json", "r01_ncu_traffic.json"):
            tf = os.path.join(ROOT, "profiles", name)
            if os.path.exists(tf):
                traffic = json.load(open(tf)).get("traffic_bytes")
                break
        return {"bound": "l2_atomic", "achieved": achieved, "peak": peak["peak"], "unit": "Gatom/s",
                "frac": achieved / peak["peak"], "traffic": traffic, "traffic_unit": "DRAM bytes per launch (ncu)",
                "per_launch_algorithmic_atomics": a_min, "peak_source": peak["source"], "live_peak": peak["live"],
                "kernel": {"regs": kinfo["regs"], "blocks_per_sm": kinfo["blocks_per_sm"],
                           "stack_bytes": kinfo["local_bytes"]}}

    def extras(self, out, value):
        """Rank 0 only: CUDA malloc, fragmentation, CPU baselines, d3 / d4 / d2."""
        from paper_conf_ppopp_geladog19_b200.runner import run_correctness
        torch, ga, args, t, heap = self.torch, self.ga, self.args, self.trace, self.heap
        stream, dev = self.stream, self.dev
        # CUDA device malloc on the same trace (bounded prefix of rounds)
        heap.reset()
        torch.cuda.synchronize()
        cc = torch.zeros(8, dtype=torch.int64, device=dev)
        rr, t_cuda = 1, None
        while True:
            cc.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_cuda_trace_timed(stream.cuda_stream, self.d_sizes.data_ptr(), rr, t.T, t.D, cc.data_ptr(),
                                   args.block)
            a1.record(stream)
            a1.synchronize()
            t_cuda = a0.elapsed_time(a1) / 1e3
            if t_cuda * 2 > args.cuda_budget_s or rr >= t.R:
                break
            rr = min(t.R, rr * 2)
        ccn = cc.cpu().numpy()
        cuda_rate = float(ccn[0] + ccn[2]) / t_cuda
        out["cuda_malloc"] = {"value": cuda_rate, "unit": UNIT, "speedup": value / cuda_rate, "rounds": rr,
                              "failed_mallocs": int(ccn[1]), "seconds": round(t_cuda, 3)}
        # fragmentation: correctness mode, one kernel per round
        heap.reset()
        run = run_correctness(heap, t.sizes, t.D, log=False, tag=False, reserved=True)
        st = heap.stats()
        cpu = oracle_leg(t, budget_s=10.0)
        frag_ora = cpu["stats"]["peak_reserved_bytes"] / cpu["stats"]["peak_live_bytes"]
        frag_gpu = run.peak_reserved_bytes / run.peak_live_bytes if run.peak_live_bytes else None
        out["fragmentation"] = {"gpu": frag_gpu, "oracle": frag_ora,
                                "ratio": frag_gpu / frag_ora if frag_gpu else None,
                                "gpu_failed_mallocs": run.counts["n_fail"],
                                "device_peak_reserved_bytes": st["peak_reserved_bytes"],
                                "boundary_peak_reserved_bytes": run.peak_reserved_bytes}
        cpu.pop("stats")
        cpu.pop("seconds")
        out["cpu_baseline"] = cpu
        _progress("cuda_malloc + fragmentation + cpu_baseline")
        out["d4_levels"] = d4_levels(ga, stream, dev, args, self.flush)
        _progress("d4_levels")
        out["d3"] = d3_sweep(ga, heap, stream, dev, t.T, args)
        _progress("d3")
        out["d2"] = d2_bsem(ga, stream, dev)
        _progress("d2")
        out["cpu_baseline_all_cores"] = oracle_leg_parallel(t)
        _progress("cpu_baseline_all_cores")


def l2_peak(ga, torch, dev, stream):
    """The roofline denominator: the committed, ncu-checked L2-atomic peak
    (profiles/l2_atomic_peak.json, tools/l2_peak.py) if present, and the same
    microbenchmark measured live beside it."""
    buf = torch.zeros(148 * 8 * 256 * 4 + 8192, dtype=torch.int64, device=dev)
    sink = torch.zeros(8, dtype=torch.int64, device=dev)
    live = {}
    grid, blk, iters = 148 * 8, 256, 64
    for pat, name in ((0, "atomg_distinct"), (1, "redg_distinct"), (3, "atomg_1184_words")):
        for rep in range(3):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ga.ga_l2_atomic_bench(stream.cuda_stream, pat, buf.data_ptr(), buf.numel(), iters, grid, blk,
                                  sink.data_ptr())
            a1.record(stream)
            a1.synchronize()
            if rep:
                live[name] = max(live.get(name, 0.0), grid * blk * iters / (a0.elapsed_time(a1) / 1e3) / 1e9)
    pf = os.path.join(ROOT, "profiles", "l2_atomic_peak.json")
    if os.path.exists(pf):
        p = json.load(open(pf))
        return {"peak": p["peak_gatom_s"], "source": p["source"], "live": live}
    return {"peak": max(live["atomg_distinct"], live["redg_distinct"]), "live": live,
            "source": "measured live: ga_l2_atomic_bench distinct-word ATOMG/REDG (max)"}


def main(argv=None, arm_factory=GpuArm):
    argv = sys.argv[1:] if argv is None else list(argv)
    args = parse_args(argv)
    if args.impl == "reference":
        return run_reference(args, tracegen.d4_mixed("pressure"))
    rc = launch_or_refuse(args, argv)
    if rc is not None:
        return rc
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    dist = None
    arm = arm_factory(args, rank, local)
    if world > 1:
        import torch
        import torch.distributed as dist
        kw = {"device_id": torch.device("cuda", local)} if arm.backend == "nccl" else {}
        dist.init_process_group(arm.backend, **kw)
    barrier = dist.barrier if dist else (lambda: None)
    m = arm.measure(barrier)
    ms_max, tot = reduce_over_ranks(dist, m["ms"], m["calls"], arm.reduce_device)
    e2e_ms, e2e_tot = reduce_over_ranks(dist, m["e2e_ms"], m["e2e_calls"], arm.reduce_device)
    if rank != 0:
        if dist:
            dist.barrier()
            dist.destroy_process_group()
        return 0
    value = tot / (ms_max / 1e3)
    t = arm.trace
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms_max, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "u64", "data": "synthetic", "config": config_of(t, args),
           "e2e": {"value": e2e_tot / (e2e_ms / 1e3), "unit": UNIT, "h2d_bytes_per_step": m["h2d"],
                   "d2h_bytes_per_step": m["d2h"], "ms_per_step": e2e_ms},
           "gpu_launches": m["launches"] * world, "gpu_launches_note": m["launch_note"],
           "clocks": m["clocks"], "roofline": arm.roofline(m["ms"])}
    tail = {"calls_per_step": m["calls"], "failed_mallocs_per_step": m["fails"],
            "kernel_ms": {"min": min(m["kern_ms"]), "max": max(m["kern_ms"])},
            "heap": "cold: ga_heap_reset (one kernel, untimed) before every step",
            "warm": {"ms_per_step": m["warm_ms"], "value": m["calls"] / (m["warm_ms"] / 1e3)},
            "wall_s_timed_region": m["wall"]}
    if not args.no_extras:
        arm.extras(out, value)
    out.update(tail)
    # the driver shows the END of the line: the comparator, fragmentation and
    # the headline's own numbers go last, after the bulky sweeps
    for k in ("cuda_malloc", "fragmentation", "roofline", "e2e"):
        if k in out:
            out[k] = out.pop(k)
    out["headline"] = {"value": value, "ms_per_step": ms_max, "unit": UNIT}
    print(json.dumps(out), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
