"""B200-native throughput-oriented device allocator (Gelado & Garland, PPoPP'19).

Thin ctypes binding over the C ABI in ``include/ga.h`` and ``include/ga_bench.h``
(``libga.so``, built in-tree for sm_100a by ``_build.py``).  Functions keep the C
names; arguments are plain ints (device pointers, sizes, stream handles).
There is no fallback: if the CUDA library cannot be built or loaded, importing
this package raises.  Every step of the hot path runs in the library's kernels.
"""
from __future__ import annotations

import ctypes
import os

from . import _build

__all__ = ["lib", "GaError", "Layout", "Stats", "DevHeap", "ga_heap_create", "ga_heap_destroy",
           "ga_heap_reset", "ga_stats", "ga_heap_device", "ga_heap_info", "ga_layout",
           "ga_heap_quiesce", "ga_heap_snapshot", "ga_reserved_pages", "ga_status_str",
           "ga_trace_phase", "ga_trace_timed", "ga_trace_timed_scope", "ga_trace_timed_host",
           "ga_cuda_set_heap_limit", "GA_TRACE_SCOPE",
           "ga_cuda_trace_phase", "ga_cuda_trace_timed", "ga_kernel_info", "ga_l2_atomic_bench",
           "ga_bsem_bench", "BsemCfg", "EXPORTED", "GA_TRACE_LOG", "GA_TRACE_TAG",
           "ga_rcu_workspace_bytes", "ga_rcu_list_removal", "ga_edge_calls"]

GA_TRACE_LOG = 1
GA_TRACE_TAG = 2


def GA_TRACE_SCOPE(scope: int) -> int:
    """flags bits 8..11: 0 warp calls, 1 block-collective, 2..8 cluster-collective (include/ga_bench.h)"""
    return scope << 8

# every symbol include/ga.h and include/ga_bench.h declare
EXPORTED = ["ga_heap_create", "ga_heap_destroy", "ga_heap_reset", "ga_stats", "ga_heap_device",
            "ga_heap_info", "ga_layout", "ga_heap_quiesce", "ga_heap_snapshot", "ga_reserved_pages",
            "ga_status_str", "ga_trace_phase", "ga_trace_timed", "ga_trace_timed_scope", "ga_trace_timed_host",
            "ga_cuda_set_heap_limit", "ga_cuda_trace_phase", "ga_cuda_trace_timed",
            "ga_kernel_info", "ga_l2_atomic_bench", "ga_bsem_bench", "ga_debug_attach", "ga_edge_calls",
            "ga_rcu_workspace_bytes", "ga_rcu_list_removal"]


class GaError(RuntimeError):
    pass


class Layout(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint32) for n in
                ("page", "chunk_pages", "min_class", "bin_max", "n_classes", "bitmap_bits",
                 "n_span_classes", "span_max")]


class Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "heap_bytes", "metadata_bytes", "reserved_bytes", "peak_reserved_bytes", "n_malloc", "n_free", "n_bin_grow",
        "n_chunk_grow", "n_bin_reclaim", "n_chunk_reclaim", "n_fallback", "n_fail",
        "n_pending_reclaim", "n_repair_nonfull", "n_repair_summary", "n_waiter_reclaim")] + [
        ("n_arenas", ctypes.c_uint32), ("pad", ctypes.c_uint32)]


class DevHeap(ctypes.Structure):
    """ga_dev_heap: the 16-byte handle kernels receive by value."""
    _fields_ = [("desc", ctypes.c_void_p), ("base", ctypes.c_void_p)]


class BsemCfg(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint32) for n in
                ("variant", "k", "B", "n_sems", "iters", "acquire_only", "grid", "block")] + [
                ("seed", ctypes.c_uint64)]


_lib = None


def lib():
    """Load libga.so (building it first if stale).  Raises if it cannot."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("GA_LIB")            # a tuning variant built by _build.build(out=...)
    if not path:
        path = _build.LIB
        if not os.path.exists(path) or _build._stale():
            path = _build.build()
    L = ctypes.CDLL(path)
    vp, u32, u64, i32, sz = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_size_t
    P = ctypes.POINTER
    sig = {
        "ga_heap_create": [i32, vp, vp, sz, u32, P(vp)],
        "ga_heap_destroy": [vp],
        "ga_heap_reset": [vp, vp],
        "ga_stats": [vp, vp, P(Stats)],
        "ga_heap_device": [vp, P(DevHeap)],
        "ga_heap_info": [vp, P(u64), P(vp), P(u64)],
        "ga_layout": [P(Layout)],
        "ga_heap_quiesce": [vp, vp],
        "ga_heap_snapshot": [vp, vp, vp, sz, P(sz)],
        "ga_reserved_pages": [vp, vp, P(u64)],
        "ga_trace_phase": [vp, vp, vp, u32, u32, u32, u32, u32, vp, vp, vp, u32, u32],
        "ga_trace_timed": [vp, vp, vp, u32, u32, u32, vp, u32],
        "ga_trace_timed_scope": [vp, vp, vp, u32, u32, u32, vp, u32, u32],
        "ga_trace_timed_host": [vp, vp, vp, u32, u32, u32, vp, u32],
        "ga_cuda_set_heap_limit": [sz],
        "ga_cuda_trace_phase": [vp, vp, u32, u32, u32, u32, u32, vp, vp, u32, u32],
        "ga_cuda_trace_timed": [vp, vp, u32, u32, u32, vp, u32],
        "ga_kernel_info": [i32, u32, P(i32), P(i32), P(i32)],
        "ga_l2_atomic_bench": [vp, i32, vp, u64, u32, u32, u32, vp],
        "ga_bsem_bench": [vp, P(BsemCfg), vp, vp],
        "ga_debug_attach": [vp, P(P(u64))],
        "ga_edge_calls": [vp, vp, vp, u32, vp, u32, u32],
        "ga_rcu_workspace_bytes": [u32, P(sz)],
        "ga_rcu_list_removal": [vp, u32, u32, vp, vp, sz, u32, u32, vp],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = i32
    L.ga_status_str.argtypes = [i32]
    L.ga_status_str.restype = ctypes.c_char_p
    _lib = L
    return L


def ga_status_str(code: int) -> str:
    return lib().ga_status_str(code).decode()


def _ok(code: int, what: str):
    if code != 0:
        raise GaError(f"{what}: {ga_status_str(code)} ({code})")


def ga_heap_create(device: int, stream: int, buf: int | None, nbytes: int, flags: int = 0) -> int:
    h = ctypes.c_void_p()
    _ok(lib().ga_heap_create(device, stream or None, buf or None, nbytes, flags, ctypes.byref(h)),
        "ga_heap_create")
    return h.value


def ga_heap_destroy(h: int):
    _ok(lib().ga_heap_destroy(h), "ga_heap_destroy")


def ga_heap_reset(h: int, stream: int):
    _ok(lib().ga_heap_reset(h, stream or None), "ga_heap_reset")


def ga_stats(h: int, stream: int) -> dict:
    s = Stats()
    _ok(lib().ga_stats(h, stream or None, ctypes.byref(s)), "ga_stats")
    return {n: getattr(s, n) for n, _ in Stats._fields_ if n != "pad"}


def ga_heap_device(h: int) -> DevHeap:
    d = DevHeap()
    _ok(lib().ga_heap_device(h, ctypes.byref(d)), "ga_heap_device")
    return d


def ga_heap_info(h: int) -> dict:
    hb, base, mb = ctypes.c_uint64(), ctypes.c_void_p(), ctypes.c_uint64()
    _ok(lib().ga_heap_info(h, ctypes.byref(hb), ctypes.byref(base), ctypes.byref(mb)), "ga_heap_info")
    return {"heap_bytes": hb.value, "base": base.value, "metadata_bytes": mb.value}


def ga_layout() -> dict:
    l = Layout()
    _ok(lib().ga_layout(ctypes.byref(l)), "ga_layout")
    return {n: getattr(l, n) for n, _ in Layout._fields_}


def ga_heap_quiesce(h: int, stream: int):
    _ok(lib().ga_heap_quiesce(h, stream or None), "ga_heap_quiesce")


def ga_heap_snapshot(h: int, stream: int) -> bytes:
    used = ctypes.c_size_t()
    _ok(lib().ga_heap_snapshot(h, stream or None, None, 0, ctypes.byref(used)), "ga_heap_snapshot")
    buf = ctypes.create_string_buffer(used.value)
    _ok(lib().ga_heap_snapshot(h, stream or None, buf, used.value, ctypes.byref(used)), "ga_heap_snapshot")
    return buf.raw


def ga_reserved_pages(h: int, stream: int) -> int:
    v = ctypes.c_uint64()
    _ok(lib().ga_reserved_pages(h, stream or None, ctypes.byref(v)), "ga_reserved_pages")
    return v.value


def ga_trace_phase(h, stream, sizes, R, T, D, rnd, phase, held, log, counts, flags, block=256):
    _ok(lib().ga_trace_phase(h, stream or None, sizes, R, T, D, rnd, phase, held, log or None, counts,
                             flags, block), "ga_trace_phase")


def ga_trace_timed(h, stream, sizes, R, T, D, counts, block=256):
    _ok(lib().ga_trace_timed(h, stream or None, sizes, R, T, D, counts, block), "ga_trace_timed")


def ga_trace_timed_scope(h, stream, sizes, R, T, D, counts, block=256, scope=0):
    _ok(lib().ga_trace_timed_scope(h, stream or None, sizes, R, T, D, counts, block, scope), "ga_trace_timed_scope")


def ga_trace_timed_host(h, stream, host_sizes, R, T, D, host_counts, block=256):
    _ok(lib().ga_trace_timed_host(h, stream or None, host_sizes, R, T, D, host_counts, block),
        "ga_trace_timed_host")


def ga_cuda_set_heap_limit(nbytes: int):
    _ok(lib().ga_cuda_set_heap_limit(nbytes), "ga_cuda_set_heap_limit")


def ga_cuda_trace_phase(stream, sizes, R, T, D, rnd, phase, held, counts, flags, block=256):
    _ok(lib().ga_cuda_trace_phase(stream or None, sizes, R, T, D, rnd, phase, held, counts, flags, block),
        "ga_cuda_trace_phase")


def ga_cuda_trace_timed(stream, sizes, R, T, D, counts, block=256):
    _ok(lib().ga_cuda_trace_timed(stream or None, sizes, R, T, D, counts, block), "ga_cuda_trace_timed")


def ga_kernel_info(which: int, block: int = 256) -> dict:
    r, b, l = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    _ok(lib().ga_kernel_info(which, block, ctypes.byref(r), ctypes.byref(b), ctypes.byref(l)),
        "ga_kernel_info")
    return {"regs": r.value, "blocks_per_sm": b.value, "local_bytes": l.value}


def ga_l2_atomic_bench(stream, pattern, buf, n_words, iters, grid, block, sink):
    _ok(lib().ga_l2_atomic_bench(stream or None, pattern, buf, n_words, iters, grid, block, sink),
        "ga_l2_atomic_bench")


def ga_rcu_workspace_bytes(n_nodes: int) -> int:
    out = ctypes.c_size_t()
    _ok(lib().ga_rcu_workspace_bytes(n_nodes, ctypes.byref(out)), "ga_rcu_workspace_bytes")
    return out.value


def ga_rcu_list_removal(stream, n_threads, n_nodes, tags, ws, ws_bytes, delegate, block, out):
    _ok(lib().ga_rcu_list_removal(stream or None, n_threads, n_nodes, tags, ws, ws_bytes, delegate, block, out),
        "ga_rcu_list_removal")


def ga_bsem_bench(stream, cfg: BsemCfg, sems, out):
    _ok(lib().ga_bsem_bench(stream or None, ctypes.byref(cfg), sems, out), "ga_bsem_bench")


def ga_edge_calls(h, stream, sizes, T, offs, flags=0, block=256):
    _ok(lib().ga_edge_calls(h, stream or None, sizes, T, offs, flags, block), "ga_edge_calls")
