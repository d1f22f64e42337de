"""The N > 1 bench path on CPU: world_size 2 over gloo (replicas, no data-path
collective).  Each rank runs its own trace (seed + rank,
rank 0 the canonical one) and the job's numbers are the slowest rank's time and
the sum of all ranks' calls."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import bench
import tracegen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        _work(rank, world, port, q)
    except Exception as e:                      # report instead of leaving the parent waiting
        q.put((rank, repr(e), 0, 0.0, 0.0, 0.0))
        raise


def _work(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    base = tracegen.d4_mixed("pressure", T=4096, R=2)
    tr = bench.rank_trace(base, rank)
    ms = 10.0 + 5.0 * rank
    calls = float(tr.calls())
    ms_max, tot = bench.reduce_over_ranks(dist, ms, calls, torch.device("cpu"))
    q.put((rank, int(tr.seed), int(tr.sizes.sum()), ms_max, tot, calls))
    dist.barrier()
    dist.destroy_process_group()


def test_two_ranks_replicas_and_reduction():
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, seed0, sum0, ms0, tot0, c0), (r1, seed1, sum1, ms1, tot1, c1) = out
    base = tracegen.d4_mixed("pressure", T=4096, R=2)
    assert seed0 == base.seed and seed1 == base.seed + 1          # rank 0 canonical, rank 1 seed + 1
    assert sum0 == int(base.sizes.sum()) and sum1 != sum0         # independent traces
    assert ms0 == ms1 == 15.0                                     # max over ranks
    assert tot0 == tot1 == c0 + c1                                # sum over ranks


class FakeArm:
    """A CPU stand-in for bench.GpuArm: the device work of one rank is faked
    (rank-dependent time and call count), everything else -- argument handling,
    process group, barriers, max/sum reduction over ranks, rank 0's single JSON
    line -- is bench.main() itself."""
    backend = "gloo"

    def __init__(self, args, rank, local):
        self.args, self.rank = args, rank
        self.reduce_device = torch.device("cpu")
        self.trace = bench.rank_trace(tracegen.d4_mixed("pressure", T=1024, R=2), rank)
        self.barriers = 0

    def measure(self, barrier):
        barrier()
        self.barriers += 1
        barrier()
        return {"ms": 10.0 + 5.0 * self.rank, "calls": 1000 * (self.rank + 1), "fails": 0, "kern_ms": [1.0],
                "warm_ms": 1.0, "wall": 0.1, "clocks": {}, "e2e_ms": 20.0 + self.rank, "e2e_calls": 100,
                "h2d": 8, "d2h": 32, "launches": 2 * self.args.steps, "launch_note": "fake"}

    def roofline(self, ms):
        return {"bound": "fake"}

    def extras(self, out, value):
        out["extras_rank"] = self.rank


def _main_worker(rank, world, port, q):
    import contextlib
    import io
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    buf = io.StringIO()
    with contextlib.redirect_stdout(buf):
        rc = bench.main(["--gpus", str(world), "--steps", "4", "--warmup", "3"], arm_factory=FakeArm)
    q.put((rank, rc, buf.getvalue()))


def test_bench_main_two_ranks_gloo():
    """bench.main() at world size 2 over gloo: only rank 0 prints, exactly one
    JSON line; value = the calls of both ranks / the slowest rank's time;
    n_gpus = 2; the extras run on rank 0 only."""
    import json
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_main_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=180) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, rc0, s0), (r1, rc1, s1) = out
    assert rc0 == rc1 == 0 and s1 == ""
    lines = [ln for ln in s0.splitlines() if ln.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["ms_per_step"] == 15.0
    assert d["value"] == (1000 + 2000) / 0.015
    assert d["e2e"]["value"] == 200 / 0.021
    assert d["extras_rank"] == 0 and d["gpu_launches"] == 2 * 4 * 2


def test_bench_refuses_mismatched_world(monkeypatch):
    """--gpus N inside a torchrun environment of another size is refused
    (no silently mislabelled 1-GPU run)."""
    monkeypatch.setenv("WORLD_SIZE", "1")
    assert bench.main(["--gpus", "2"], arm_factory=FakeArm) == 2
