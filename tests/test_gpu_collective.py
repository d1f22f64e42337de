"""GPU parity of the block- and cluster-collective calls (the
paper's collective synchronization primitives at thread-block scope, Sec.
4.2.2; cluster scope through distributed shared memory).

The same seeded traces as tests/test_gpu_parity.py, with every allocator call
made by the whole CTA (scope 1) or the whole cluster (scope 2..8) together,
compared with the oracle on what is unique (counts when demand <= capacity,
the oracle's log checker, the empty-heap snapshot after free-all + quiesce).
Partial blocks (T % block != 0) keep their idle threads in every call.
"""
import numpy as np
import pytest
import torch

import oracle
import tracegen
from oracle import snapshot as S

pytestmark = pytest.mark.gpu

ga = pytest.importorskip("paper_conf_ppopp_geladog19_b200")
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness, run_timed  # noqa: E402

SCOPES = [1, 2, 4, 8]


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def _empty_parity(heap: GpuHeap):
    st = heap.stats()
    assert st["n_repair_nonfull"] == 0 and st["n_repair_summary"] == 0, st
    heap.quiesce()
    snap = heap.snapshot()
    errs = S.check(S.parse(snap), require_reclaimed=True)
    assert not errs, errs[:5]
    assert snap == oracle.snapshot_of_fresh(heap.heap_bytes), "post-free snapshot differs from the empty heap"


def _check_log(run, sizes, D, heap_bytes):
    R, T = sizes.shape
    err, cs = oracle.check_log(run.log, R, T, D, heap_bytes)
    assert err == 0, (err, cs)
    assert run.counts["tag_errors"] == 0
    return cs


@pytest.mark.parametrize("scope", SCOPES)
def test_d1_tiny_collective(scope):
    t = tracegen.d1_tiny()
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D, scope=scope)
    assert run.counts["n_malloc"] == ref.stats["n_malloc"] == 1024
    assert run.counts["n_fail"] == ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_free"] == ref.stats["n_free"]
    _check_log(run, t.sizes, t.D, t.heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("scope", SCOPES)
@pytest.mark.parametrize("size", [16, 100, 256, 2048, 4096, 65536])
def test_d3_uniform_collective(scope, size):
    """Warp-uniform sizes, every block live at once: one semaphore operation
    per class per CTA / cluster; counts equal the oracle's."""
    T = 16384 + 77                                   # ragged last block
    heap_bytes = 2 << 30 if size >= 65536 else 256 << 20
    sizes = np.full((3, T), size, dtype=np.uint32)
    ref = oracle.run_trace(sizes, heap_bytes, 0)
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 0, scope=scope)
    assert run.counts["n_fail"] == ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_malloc"] == ref.stats["n_malloc"]
    _check_log(run, sizes, 0, heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("scope", SCOPES)
@pytest.mark.parametrize("size", [16, 256, 4096])
def test_single_class_exhaust_collective(scope, size):
    """Threads = capacity + 64: exactly capacity succeed."""
    heap_bytes = 8 << 20
    cap = heap_bytes // size
    sizes = np.full((1, cap + 64), size, dtype=np.uint32)
    ref = oracle.run_trace(sizes, heap_bytes, 0)
    assert ref.stats["n_malloc_fail"] == 64
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 0, scope=scope)
    assert run.counts["n_malloc"] - run.counts["n_fail"] == cap
    _check_log(run, sizes, 0, heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("scope", SCOPES)
def test_d4_small_fit_collective(scope):
    """Mixed 16 B - 64 KiB churn (D = 1) at fit: counts equal the oracle's."""
    t = tracegen.d4_small(T=8192 + 33, R=8, heap_bytes=256 << 20)
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D, scope=scope)
    assert ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_fail"] == 0 and run.counts["n_malloc"] == ref.stats["n_malloc"]
    assert run.counts["n_free"] == ref.stats["n_free"]
    _check_log(run, t.sizes, t.D, t.heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("scope", [1, 2])
def test_mixed_churn_with_tree_sizes_collective(scope):
    """Classes 16 B - 1 MiB: the TBuddy lanes take the warp path inside the
    collective call; counts equal the oracle's, the log passes."""
    T, R = 4096, 6
    sizes = tracegen.mixed_sizes(tracegen.BASE_SEED + 41, R, T, 3, 19)
    heap_bytes = 4 << 30
    ref = oracle.run_trace(sizes, heap_bytes, 1)
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 1, scope=scope)
    assert run.counts["n_fail"] == 0 and run.counts["n_malloc"] == ref.stats["n_malloc"]
    _check_log(run, sizes, 1, heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("scope", SCOPES)
def test_timed_full_d4_collective(scope):
    """The full d4 bench trace (303,104 threads x 16 rounds, 4 GiB) through the
    timed kernel at each scope: every call succeeds (the oracle fails none at
    this level), every block is freed, the heap returns to empty."""
    t = tracegen.d4_mixed("fit")
    ref_fail = 0
    heap = GpuHeap(t.heap_bytes)
    d_sizes = torch.from_numpy(t.sizes.view(np.int32)).cuda()
    counts = torch.zeros(8, dtype=torch.int64, device="cuda")
    run_timed(heap, d_sizes, t.R, t.T, t.D, counts, scope=scope)
    torch.cuda.synchronize()
    c = counts.cpu().numpy()
    assert c[0] == t.R * t.T and c[1] == ref_fail and c[2] == c[0]
    st = heap.stats()                                # T = 1184 x 256: no idle threads, no padding
    assert st["n_malloc"] == t.R * t.T and st["n_free"] == t.R * t.T, st
    _empty_parity(heap)


def test_invalid_scope_rejected():
    heap = GpuHeap(1 << 20)
    d = torch.zeros(64, dtype=torch.int32, device="cuda")
    c = torch.zeros(8, dtype=torch.int64, device="cuda")
    with pytest.raises(ga.GaError):
        run_timed(heap, d, 1, 64, 0, c, scope=9)
    with pytest.raises(ga.GaError):
        run_timed(heap, d, 1, 64, 0, c, block=512, scope=8)          # 4096 threads > 2048
    heap.close()
