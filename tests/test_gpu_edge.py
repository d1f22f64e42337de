"""GPU checks of the device API's edge cases, the device counters (SURVEY 8(a)
a10) and the failure path, through the C ABI:

* ga_malloc(0) and sizes above the heap return NULL and are not failures
  (reading R-15); ga_free(NULL) is a no-op (R-16); a partial last warp
  (T % 32 != 0) allocates, frees and empties the heap like full warps;
* ga_stats' device counters equal what the trace kernels counted: n_malloc,
  n_free, n_fail; the device reserved-page counter equals the reserved pages
  derived from the tree bitmaps at every phase boundary, and its atomicMax peak
  is the phase maximum (failures are the fragmentation proxy);
* deferred reclamation is delegated to threads blocked in a semaphore wait
  (P:L1206-1244): under exhaustion some bins are reclaimed by waiters before
  any quiesce;
* a malloc fails only when nothing could serve it (no false
  resource starvation; reading R-26): after a malloc-only phase every class
  that saw a NULL has no free slot, no free arena page and no tree block left.
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

NULL = (1 << 64) - 1
PAGE = 4096


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


def _quiet(heap):
    """No safety-net repair ran (ga.h: expected 0)."""
    st = heap.stats()
    assert st["n_repair_nonfull"] == 0 and st["n_repair_summary"] == 0, st
    return st


def _empty(heap):
    heap.quiesce()
    snap = heap.snapshot()
    assert not S.check(S.parse(snap), require_reclaimed=True)
    assert snap == oracle.snapshot_of_fresh(heap.heap_bytes)


def _edge(heap, sizes, free=False, block=256):
    d = torch.from_numpy(np.asarray(sizes, dtype=np.uint64).view(np.int64)).cuda()
    offs = torch.empty_like(d)
    ga.ga_edge_calls(heap.h, torch.cuda.current_stream().cuda_stream, d.data_ptr(), len(sizes), offs.data_ptr(),
                     1 if free else 0, block)
    torch.cuda.synchronize()
    return offs.cpu().numpy().view(np.uint64)


def _cls_align(n):
    c = max(16, 1 << (int(n) - 1).bit_length())
    return min(c, 2 << 20)


def _valid_blocks(offs, sizes, heap_bytes):
    ok = offs != NULL
    o, n = offs[ok].astype(np.int64), np.asarray(sizes, dtype=np.uint64)[ok].astype(np.int64)
    cls = np.array([max(16, 1 << (int(x) - 1).bit_length()) for x in n], dtype=np.int64)
    assert np.all(o + n <= heap_bytes) and np.all(o >= 0)
    assert all(int(a) % _cls_align(b) == 0 for a, b in zip(o, n))          # class / block alignment (R-31)
    idx = np.argsort(o)
    assert np.all(o[idx][1:] >= o[idx][:-1] + cls[idx][:-1]), "overlapping blocks"
    return ok


def test_null_requests_and_free_null():
    """R-15 / R-16 on the device: 0, heap + 1 and 2^63 give NULL without counting
    as failures; every thread also calls ga_free(NULL)."""
    heap = GpuHeap(16 << 20)
    hb = heap.heap_bytes
    sizes = [0, hb + 1, 1 << 63, (1 << 64) - 1, 16, 0, 4096, hb + PAGE] * 40       # T = 320
    offs = _edge(heap, sizes)
    for n, o in zip(sizes, offs):
        assert (o == NULL) == (n == 0 or n > hb), (n, o)
    st = _quiet(heap)
    assert st["n_malloc"] == len(sizes) and st["n_fail"] == 0 and st["n_free"] == 0
    _valid_blocks(offs, sizes, hb)


@pytest.mark.parametrize("T", [1, 31, 33, 1000, 4099])
def test_partial_warps_edge_kernel(T):
    """T % 32 != 0: the last warp runs partial.  Mixed sizes 1 B - 256 KiB; every
    call succeeds (the heap fits them), blocks are valid, frees restore the heap."""
    heap = GpuHeap(512 << 20)
    rng = np.random.default_rng(T)
    sizes = (1 << rng.integers(0, 18, T)) + rng.integers(0, 7, T)
    offs = _edge(heap, sizes)
    assert np.all(offs != NULL)
    _valid_blocks(offs, sizes, heap.heap_bytes)
    st = _quiet(heap)
    assert st["n_malloc"] == T and st["n_fail"] == 0
    heap.reset()
    offs = _edge(heap, sizes, free=True)
    st = _quiet(heap)
    assert st["n_malloc"] == T and st["n_free"] == T and st["n_fail"] == 0
    _empty(heap)


def test_whole_heap_request():
    """A single request for the whole (power-of-two) heap succeeds at offset 0;
    raced against a 16 B request exactly one of the two fails (the heap cannot
    hold both)."""
    heap = GpuHeap(16 << 20)
    hb = heap.heap_bytes
    assert _edge(heap, [hb])[0] == 0
    heap.reset()
    offs = _edge(heap, [hb, 16])
    assert (offs == NULL).sum() == 1
    assert _quiet(heap)["n_fail"] == 1


@pytest.mark.parametrize("T", [1000, 4097])
def test_partial_warps_trace_parity(T):
    """The trace kernels with T % 32 != 0: counts equal the oracle's, the log
    passes the oracle's checker, the heap empties; the timed kernel (which
    skips its warp reconvergence when T % 32 != 0) too."""
    t = tracegen.d4_small(T=T, R=4, heap_bytes=128 << 20)
    ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, t.sizes, t.D)
    assert run.counts["n_fail"] == ref.stats["n_malloc_fail"] == 0
    assert run.counts["n_malloc"] == ref.stats["n_malloc"] and run.counts["n_free"] == ref.stats["n_free"]
    err, _ = oracle.check_log(run.log, t.R, t.T, t.D, t.heap_bytes)
    assert err == 0
    _empty(heap)
    heap.reset()
    d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
    c = torch.zeros(8, dtype=torch.int64, device="cuda")
    run_timed(heap, d, t.R, t.T, t.D, c)
    torch.cuda.synchronize()
    cc = c.cpu().numpy()
    assert cc[0] == ref.stats["n_malloc"] and cc[1] == 0 and cc[2] == cc[0]
    _empty(heap)


@pytest.mark.parametrize("D", [0, 1])
def test_stats_equal_trace_counts_and_reserved(D):
    """ga_stats' device counters against the trace kernel's own counts, and the
    device reserved-page counter against the tree bitmaps at every boundary."""
    t = tracegen.d4_small(T=8192, R=6, heap_bytes=160 << 20)
    sizes = t.sizes
    heap = GpuHeap(t.heap_bytes)
    run = run_correctness(heap, sizes, D, log=False)
    st = _quiet(heap)
    assert st["n_malloc"] == run.counts["n_malloc"] and st["n_free"] == run.counts["n_free"]
    assert st["n_fail"] == run.counts["n_fail"]
    assert run.reserved_dev_per_round == run.reserved_per_round
    assert st["peak_reserved_bytes"] >= max(run.reserved_per_round)
    assert st["peak_reserved_bytes"] <= heap.heap_bytes
    _empty(heap)
    assert heap.stats()["reserved_bytes"] == heap.reserved_bytes() == 0


def test_peak_reserved_equals_malloc_phase_end():
    """One malloc-only phase: reserved only grows, so the device atomicMax peak
    equals the reserved pages at the phase boundary exactly."""
    sizes = tracegen.mixed_sizes(tracegen.BASE_SEED + 7, 1, 16384)
    heap = GpuHeap(1 << 30)
    run = run_correctness(heap, sizes, 0, log=False)
    st = _quiet(heap)
    assert st["peak_reserved_bytes"] == run.reserved_per_round[0] == max(run.reserved_per_round)
    assert st["reserved_bytes"] == heap.reserved_bytes()


def test_timed_kernel_stats():
    t = tracegen.d4_small(T=16384, R=8, heap_bytes=512 << 20)
    heap = GpuHeap(t.heap_bytes)
    d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
    c = torch.zeros(8, dtype=torch.int64, device="cuda")
    run_timed(heap, d, t.R, t.T, t.D, c)
    torch.cuda.synchronize()
    cc = c.cpu().numpy()
    st = _quiet(heap)
    assert st["n_malloc"] == cc[0] and st["n_free"] == cc[2] and st["n_fail"] == cc[1] == 0
    assert st["reserved_bytes"] == heap.reserved_bytes()


def test_delegated_reclamation_runs_under_exhaustion():
    """freed-empty bins are reclaimed by threads already blocked in
    an arena semaphore wait -- counted before any quiesce."""
    t = tracegen.d4_mixed("exhaust", R=4)
    heap = GpuHeap(t.heap_bytes)
    run_correctness(heap, t.sizes, t.D, log=False, tag=False, reserved=False)
    st = _quiet(heap)
    assert st["n_waiter_reclaim"] > 0 and st["n_bin_reclaim"] >= st["n_waiter_reclaim"], st
    _empty(heap)


# ---------------------------------------------------------------------------
# A failure must be justified by the heap's own state (no false starvation).
# ---------------------------------------------------------------------------
def serving_capacity(s: S.Snapshot, n: int, n_span: int) -> int:
    """Units in a snapshot that could serve a request of n bytes under the
    build's routing: free slots of its class, free arena pages (bins only) and
    Available tree nodes of the order it needs (a chunk for bins and spans)."""
    c = max(16, 1 << (int(n) - 1).bit_length())
    lg = c.bit_length() - 1
    free_nodes = lambda o: sum(int(b.sum()) for b in s.level_bits[o:])      # noqa: E731
    chunk_order = (s.chunk_pages).bit_length() - 1
    if c <= 2048:
        k = lg - 4
        slots = sum(int((~bits).sum()) for p, bits in s.bins.items() if s.kind[p] == (S.K_BIN | k))
        return slots + int((s.kind == S.K_CHUNK_FREE).sum()) + free_nodes(chunk_order)
    if n_span and c <= (PAGE << (n_span - 1)):
        k = lg - 12
        slots = sum(int((~bits).sum()) for p, bits in s.bins.items() if s.kind[p] == (S.K_SPAN | k))
        return slots + free_nodes(chunk_order)
    return free_nodes(lg - 12)


@pytest.mark.parametrize("heap_mib", [1536, 2304])
def test_failures_only_when_nothing_can_serve(heap_mib):
    """A full-grid malloc-only phase of the mixed 16 B - 64 KiB trace on a heap
    too small for it: after the phase (no frees ran, so resources only shrank),
    every size that got NULL finds zero serving capacity in the GPU's own
    snapshot.  This replaces round 1's fixed failure tolerances: the bound is
    derived from the state, not from the oracle's different placement."""
    sizes = tracegen.mixed_sizes(tracegen.BASE_SEED + 3, 1, 303104)
    heap = GpuHeap(heap_mib << 20)
    T = sizes.shape[1]
    s = torch.cuda.current_stream().cuda_stream
    d = torch.from_numpy(sizes.view(np.int32)).cuda()
    held = torch.empty(2 * T, dtype=torch.int64, device="cuda")
    held[0::2] = -1
    held[1::2] = 0
    counts = torch.zeros(8, dtype=torch.int64, device="cuda")
    log = torch.zeros(2 * T * 2, dtype=torch.int64, device="cuda")
    ga.ga_trace_phase(heap.h, s, d.data_ptr(), 1, T, 0, 0, 0, held.data_ptr(), log.data_ptr(), counts.data_ptr(),
                      ga.GA_TRACE_LOG, 256)
    torch.cuda.synchronize()
    n_fail = int(counts[1].item())
    assert n_fail > 0, "the heap is meant to be too small for the phase"
    snap = S.parse(heap.snapshot())
    assert not S.check(snap)
    n_span = ga.ga_layout()["n_span_classes"]
    rec = log.cpu().numpy().view(oracle.LOG_DTYPE)[0::2]
    failed_sizes = sorted({int(r["size"]) for r in rec if r["off"] == NULL and r["size"]})
    classes = {max(16, 1 << (n - 1).bit_length()): n for n in failed_sizes}
    bad = {c: serving_capacity(snap, n, n_span) for c, n in classes.items()}
    assert all(v == 0 for v in bad.values()), bad
    st = _quiet(heap)
    assert st["n_fail"] == n_fail
    ga.ga_trace_phase(heap.h, s, d.data_ptr(), 1, T, 0, 0, 1, held.data_ptr(), 0, counts.data_ptr(), 0, 256)
    _empty(heap)
