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
