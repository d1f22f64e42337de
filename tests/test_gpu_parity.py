"""GPU parity: the CUDA path (through the C ABI) against the oracle, on the same
seeded traces.  Addresses are never compared -- several
placements are correct -- only what is unique:

* success / failure counts when demand <= capacity (bit-exact);
* the GPU allocation log passes the oracle's checker (bounds, alignment,
  class, frees, pairwise disjointness at every phase boundary), and no block's
  lifetime tags were overwritten while it was live;
* after freeing everything and quiesce, the GPU's canonical snapshot equals the
  oracle's empty-heap snapshot byte for byte;
* quiescent GPU snapshots satisfy the oracle's invariants (semaphore counts ==
  free resources, buddy properties).
"""
import os

import numpy as np
import pytest
import torch

import oracle
import tracegen
from oracle import snapshot as S

pytestmark = pytest.mark.gpu

ga = pytest.importorskip("paper_conf_ppopp_geladog19_b200")
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness, run_timed  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def test_loaded_build():
    """The library under test is the one the run asked for (GA_LIB variants,
    tests/test_gpu_variants.py): its span classes match GA_EXPECT_NSPAN."""
    want = os.environ.get("GA_EXPECT_NSPAN")
    lay = ga.ga_layout()
    assert lay["n_span_classes"] == (int(want) if want is not None else 5)


def _empty_parity(heap: GpuHeap):
    st = heap.stats()                                   # the safety net never ran (ga.h: expected 0)
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


def test_fresh_heap_snapshot_equals_oracle():
    for nbytes in (1 << 20, 3 * (256 << 10), 37 << 20):
        heap = GpuHeap(nbytes)
        snap = heap.snapshot()
        assert snap == oracle.snapshot_of_fresh(nbytes)
        heap.close()


def test_d1_tiny():
    """config d1: 1,024 threads malloc(16) + free on a 1 MiB heap."""
    t = tracegen.d1_tiny()
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_log=True)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D)
    assert run.counts["n_malloc"] == ref.stats["n_malloc"] == 1024
    assert run.counts["n_fail"] == ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_free"] == ref.stats["n_free"]
    _check_log(run, t.sizes, t.D, t.heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("size", [16, 32, 48, 64, 100, 128, 256, 512, 1000, 1024, 2048, 3000, 4096, 8192])
def test_d3_uniform_phase_split(size):
    """config d3 (reduced): warp-uniform sizes, every block live at once, 3 rounds."""
    T = 16384
    heap_bytes = 256 << 20
    sizes = np.full((3, T), size, dtype=np.uint32)
    ref = oracle.run_trace(sizes, heap_bytes, 0)
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 0)
    assert run.counts["n_fail"] == ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_malloc"] == ref.stats["n_malloc"]
    _check_log(run, sizes, 0, heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("size", [16, 64, 256, 2048, 4096, 8192])
def test_single_class_exhaust_exact(size):
    """P-6 / Fig. 7 methodology: threads = capacity; every call must succeed
    (no fragmentation -> no failures), one more must fail."""
    heap_bytes = 8 << 20
    cap = heap_bytes // size
    sizes = np.full((1, cap + 64), size, dtype=np.uint32)
    ref = oracle.run_trace(sizes, heap_bytes, 0)
    assert ref.stats["n_malloc_fail"] == 64
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 0)
    assert run.counts["n_malloc"] - run.counts["n_fail"] == cap
    _check_log(run, sizes, 0, heap_bytes)
    _empty_parity(heap)


@pytest.mark.parametrize("size", [65536, 131072, 524288, 2 << 20])
def test_single_class_exhaust_exact_tree_sizes(size):
    """The same for spans' largest class and TBuddy orders above it (Fig. 7's
    64 KiB - 512 KiB points and beyond): counts equal capacity exactly."""
    heap_bytes = 64 << 20
    cap = heap_bytes // size
    sizes = np.full((1, cap + 32), size, dtype=np.uint32)
    ref = oracle.run_trace(sizes, heap_bytes, 0)
    assert ref.stats["n_malloc_fail"] == 32
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 0)
    assert run.counts["n_malloc"] - run.counts["n_fail"] == cap
    _check_log(run, sizes, 0, heap_bytes)
    _empty_parity(heap)


def test_mixed_churn_up_to_1mib():
    """Mixed churn with classes 16 B - 1 MiB (octaves 3..19): bins, spans and
    TBuddy orders 5-8 in one warp; fit-level heap, so counts equal the
    oracle's; the log passes and the heap empties."""
    T, R = 4096, 6
    sizes = tracegen.mixed_sizes(tracegen.BASE_SEED + 41, R, T, 3, 19)
    heap_bytes = 4 << 30
    ref = oracle.run_trace(sizes, heap_bytes, 1)
    assert ref.stats["n_malloc_fail"] == 0
    heap = GpuHeap(heap_bytes)
    run = run_correctness(heap, sizes, 1)
    assert run.counts["n_fail"] == 0 and run.counts["n_malloc"] == ref.stats["n_malloc"]
    _check_log(run, sizes, 1, heap_bytes)
    _empty_parity(heap)


def test_d4_small_fit_churn():
    """config d4 (reduced, fit): mixed 16 B - 64 KiB churn, D = 1; counts equal."""
    t = tracegen.d4_small(T=8192, R=8, heap_bytes=256 << 20)
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D)
    assert ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_fail"] == 0 and run.counts["n_malloc"] == ref.stats["n_malloc"]
    assert run.counts["n_free"] == ref.stats["n_free"]
    _check_log(run, t.sizes, t.D, t.heap_bytes)
    _empty_parity(heap)


def test_d4_small_pressure_valid_and_fragmentation():
    """Near exhaustion: failures differ legitimately; the log must stay valid,
    the heap must return to empty, fragmentation <= 1.3x the oracle's."""
    t = tracegen.d4_small(T=8192, R=8, heap_bytes=96 << 20)
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D)
    cs = _check_log(run, t.sizes, t.D, t.heap_bytes)
    _empty_parity(heap)
    frag_gpu = run.peak_reserved_bytes / cs["peak_live_bytes"]
    frag_ora = ref.stats["peak_reserved_bytes"] / ref.stats["peak_live_bytes"]
    assert frag_gpu <= 1.3 * frag_ora, (frag_gpu, frag_ora)


def test_quiescent_invariants_each_round():
    """Between rounds (no kernel running) the GPU metadata satisfies the oracle's
    invariants: semaphore values equal free resources, buddy properties hold."""
    t = tracegen.d4_small(T=4096, R=4, heap_bytes=64 << 20)
    heap = GpuHeap(t.heap_bytes)
    import paper_conf_ppopp_geladog19_b200.runner as rn
    for r in range(1, t.R + 1):
        sub = t.sizes[:r]
        heap.reset()
        run = rn.run_correctness(heap, sub, 1, log=False)
        # run_correctness ends with the free-all round; check the empty state too
        errs = S.check(S.parse(heap.snapshot()))
        assert not errs, errs[:5]
    heap.close()


def test_timed_kernel_counts_and_empty():
    t = tracegen.d4_small(T=16384, R=8, heap_bytes=512 << 20)
    heap = GpuHeap(t.heap_bytes)
    d_sizes = torch.from_numpy(t.sizes.view(np.int32)).cuda()
    counts = torch.zeros(8, dtype=torch.int64, device="cuda")
    run_timed(heap, d_sizes, t.R, t.T, t.D, counts)
    torch.cuda.synchronize()
    c = counts.cpu().numpy()
    assert c[0] == t.R * t.T and c[1] == 0 and c[2] == c[0]
    _empty_parity(heap)


def test_cuda_malloc_baseline_runs():
    ga.ga_cuda_set_heap_limit(64 << 20)
    sizes = np.full((1, 4096), 64, dtype=np.uint32)
    run = run_correctness(None, sizes, 0, log=False)
    assert run.counts["n_malloc"] == 4096 and run.counts["tag_errors"] == 0
    assert run.counts["n_free"] == 4096 - run.counts["n_fail"]
