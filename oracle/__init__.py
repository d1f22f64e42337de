"""Sequential CPU oracle for Gelado & Garland, PPoPP'19 -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with the
CUDA path (``paper_conf_ppopp_geladog19_b200``) and imports nothing from it.

* ``oracle/ga_oracle.c`` -- the allocator (Alg. 1/2 semaphores, TBuddy, UAlloc,
  front end), trace runner, log checker, snapshot and invariant checker.
* ``oracle/bsem.py``     -- a step-by-step bulk-semaphore model (Alg. 1/2) for
  the Fig. 1 golden traces and the exhaustive interleaving check.
* ``oracle/snapshot.py`` -- parser + invariant checker for canonical snapshots
  (applied to the oracle's own and to the GPU library's snapshots).

Parity pins live in ``tests/test_oracle_*.py``; see DESIGN.md "Oracle".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ga_oracle.c")
_SO = os.path.join(_HERE, "libga_oracle.so")
NULL = (1 << 64) - 1


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, -O2).  Building the checker is not using it."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-Wall", "-shared", "-fPIC",
                               "-o", _SO + ".tmp", _SRC])
        os.replace(_SO + ".tmp", _SO)
    return _SO


class Layout(ctypes.Structure):
    _fields_ = [("page", ctypes.c_uint32), ("chunk_pages", ctypes.c_uint32),
                ("min_class", ctypes.c_uint32), ("bin_max", ctypes.c_uint32),
                ("paper_layout", ctypes.c_uint32), ("snap_max_class", ctypes.c_uint32)]


# Build layout: 4 KiB pages (R-9), 64-page chunks (R-10),
# classes 16 B (R-13) .. 2 KiB in bins, >= 4 KiB on the tree (R-12).
# snap_max_class is snapshot FORMAT only (include/ga.h): the canonical snapshot
# has one class counter pair per power of two from 16 B to 64 KiB, the top of
# BASELINE.json's mixed range (configs[3]); the oracle routes sizes above 2 KiB
# to TBuddy, as the paper does, and writes zeros for those entries.
BUILD = dict(page=4096, chunk_pages=64, min_class=16, bin_max=2048, paper_layout=0, snap_max_class=65536)
# The paper's own layout: 8 B minimum, <= 1 KB in bins with an
# in-band 128 B header, 2 header bins + 62 tails per chunk, 2 KB -> a 4 KB page.
PAPER = dict(page=4096, chunk_pages=64, min_class=8, bin_max=1024, paper_layout=1)
# Tiny layout for brute force: 64 B pages, 4-page chunks,
# classes {16, 32} in bins, 64 / 128 B on the tree.
TINY = dict(page=64, chunk_pages=4, min_class=16, bin_max=32, paper_layout=0)


class TraceStats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "n_malloc", "n_malloc_fail", "n_free", "calls", "peak_live_bytes",
        "peak_reserved_bytes", "peak_reserved_any_bytes", "final_reserved_bytes",
        "n_bin_grow", "n_chunk_grow", "n_bin_reclaim", "n_chunk_reclaim")] + [
        ("invariant_error", ctypes.c_int64)]


class CheckStats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "n_malloc", "n_ok", "n_fail", "n_free", "peak_live_bytes", "bad_index")]


LOG_DTYPE = np.dtype([("off", "<u8"), ("size", "<u4"), ("meta", "<u4")])

_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        vp, u64, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int
        L.ora_heap_create.restype = vp
        L.ora_heap_create.argtypes = [ctypes.POINTER(Layout), u64]
        L.ora_heap_destroy.argtypes = [vp]
        L.ora_malloc.restype = u64
        L.ora_malloc.argtypes = [vp, u64]
        L.ora_free.restype = i32
        L.ora_free.argtypes = [vp, u64]
        L.ora_reserved_pages.restype = u64
        L.ora_reserved_pages.argtypes = [vp]
        L.ora_check_invariants.restype = i32
        L.ora_check_invariants.argtypes = [vp, ctypes.c_char_p, i32]
        L.ora_snapshot.restype = u64
        L.ora_snapshot.argtypes = [vp, vp, u64]
        L.ora_classify.restype = i32
        L.ora_classify.argtypes = [vp, u64, ctypes.POINTER(i32), ctypes.POINTER(i32)]
        L.ora_run_trace.restype = i32
        L.ora_run_trace.argtypes = [ctypes.POINTER(Layout), u64, vp, u64, u64, u64, vp, vp,
                                    ctypes.POINTER(TraceStats), i32]
        L.ora_check_log.restype = i32
        L.ora_check_log.argtypes = [ctypes.POINTER(Layout), u64, vp, u64, u64, u64,
                                    ctypes.POINTER(CheckStats)]
        _lib = L
    return _lib


def _layout(lay) -> Layout:
    return lay if isinstance(lay, Layout) else Layout(**lay)


class Heap:
    """One sequential oracle heap (single arena).  Offsets are relative to the base."""

    def __init__(self, bytes_: int, layout=BUILD):
        self._lay = _layout(layout)
        self._h = lib().ora_heap_create(ctypes.byref(self._lay), bytes_)
        if not self._h:
            raise ValueError("oracle: invalid layout / heap size")

    def close(self):
        if self._h:
            lib().ora_heap_destroy(self._h)
            self._h = None

    __del__ = close

    def malloc(self, n: int):
        off = lib().ora_malloc(self._h, n)
        return None if off == NULL else off

    def free(self, off) -> int:
        return lib().ora_free(self._h, NULL if off is None else off)

    def reserved_pages(self) -> int:
        return lib().ora_reserved_pages(self._h)

    def classify(self, n: int):
        c, o = ctypes.c_int(0), ctypes.c_int(0)
        r = lib().ora_classify(self._h, n, ctypes.byref(c), ctypes.byref(o))
        return ("null", None) if r == 0 else ("bin", c.value) if r == 1 else ("tree", o.value)

    def check(self) -> str | None:
        buf = ctypes.create_string_buffer(256)
        e = lib().ora_check_invariants(self._h, buf, 256)
        return None if e == 0 else f"{e}: {buf.value.decode()}"

    def snapshot(self) -> bytes:
        n = lib().ora_snapshot(self._h, None, 0)
        buf = ctypes.create_string_buffer(n)
        lib().ora_snapshot(self._h, buf, n)
        return buf.raw


def snapshot_of_fresh(bytes_: int, layout=BUILD) -> bytes:
    h = Heap(bytes_, layout)
    s = h.snapshot()
    h.close()
    return s


@dataclass
class TraceResult:
    stats: dict
    ok: np.ndarray | None
    log: np.ndarray | None


def run_trace(sizes: np.ndarray, heap_bytes: int, D: int, layout=BUILD, want_log=False,
              want_ok=True, check_each_round=False) -> TraceResult:
    """Run a trace (u32[R][T]) through the oracle in canonical order."""
    sizes = np.ascontiguousarray(sizes, dtype=np.uint32)
    R, T = sizes.shape
    lay = _layout(layout)
    rounds = R + 1 if D == 1 else R
    log = np.zeros(2 * rounds * T, dtype=LOG_DTYPE) if want_log else None
    ok = np.zeros((R, T), dtype=np.uint8) if want_ok else None
    st = TraceStats()
    rc = lib().ora_run_trace(ctypes.byref(lay), heap_bytes, sizes.ctypes.data, R, T, D,
                             log.ctypes.data if log is not None else None,
                             ok.ctypes.data if ok is not None else None,
                             ctypes.byref(st), int(check_each_round))
    if rc != 0:
        raise ValueError(f"oracle trace runner rejected the trace ({rc})")
    stats = {n: getattr(st, n) for n, _ in TraceStats._fields_}
    return TraceResult(stats, ok, log)


def check_log(log: np.ndarray, R: int, T: int, D: int, heap_bytes: int, layout=BUILD):
    """Validate an allocation log (the oracle's or the GPU's).  Returns (err, stats)."""
    log = np.ascontiguousarray(log, dtype=LOG_DTYPE)
    lay = _layout(layout)
    cs = CheckStats()
    err = lib().ora_check_log(ctypes.byref(lay), heap_bytes, log.ctypes.data, R, T, D,
                              ctypes.byref(cs))
    return err, {n: getattr(cs, n) for n, _ in CheckStats._fields_}
