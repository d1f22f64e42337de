"""Drive traces through the C ABI.  PyTorch is plumbing here: device buffers,
pinned host buffers and streams.  Every allocator step runs in libga.so."""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

from . import (GA_TRACE_LOG, GA_TRACE_SCOPE, GA_TRACE_TAG, ga_cuda_trace_phase, ga_cuda_trace_timed, ga_heap_create,
               ga_heap_destroy, ga_heap_quiesce, ga_heap_reset, ga_heap_snapshot, ga_heap_info,
               ga_reserved_pages, ga_stats, ga_trace_phase, ga_trace_timed, ga_trace_timed_host, ga_trace_timed_scope)

LOG_DTYPE = np.dtype([("off", "<u8"), ("size", "<u4"), ("meta", "<u4")])
PAGE = 4096


def _stream(s=None) -> int:
    return (s or torch.cuda.current_stream()).cuda_stream


class GpuHeap:
    """A device heap owned by libga (pool + metadata allocated by the library)."""

    def __init__(self, nbytes: int, device: int = 0, stream=None):
        self.device = device
        self.stream = stream or torch.cuda.current_stream(device)
        self.h = ga_heap_create(device, _stream(self.stream), None, nbytes)
        info = ga_heap_info(self.h)
        self.heap_bytes = info["heap_bytes"]
        self.metadata_bytes = info["metadata_bytes"]

    def close(self):
        if getattr(self, "h", None):
            ga_heap_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset(self):
        ga_heap_reset(self.h, _stream(self.stream))

    def quiesce(self):
        ga_heap_quiesce(self.h, _stream(self.stream))

    def snapshot(self) -> bytes:
        return ga_heap_snapshot(self.h, _stream(self.stream))

    def stats(self) -> dict:
        return ga_stats(self.h, _stream(self.stream))

    def reserved_bytes(self) -> int:
        return ga_reserved_pages(self.h, _stream(self.stream)) * PAGE


@dataclass
class TraceRun:
    counts: dict
    log: np.ndarray | None = None
    peak_reserved_bytes: int = 0
    reserved_per_round: list = field(default_factory=list)        # from the tree bitmaps (ga_reserved_pages)
    reserved_dev_per_round: list = field(default_factory=list)    # the device counter (ga_stats)
    live_per_round: list = field(default_factory=list)   # requested bytes held at each boundary

    @property
    def peak_live_bytes(self) -> int:
        return max(self.live_per_round) if self.live_per_round else 0


def _counts(t: torch.Tensor) -> dict:
    c = t.cpu().numpy()
    return {"n_malloc": int(c[0]), "n_fail": int(c[1]), "n_free": int(c[2]), "tag_errors": int(c[3])}


def run_correctness(heap: GpuHeap | None, sizes: np.ndarray, D: int, log: bool = True, tag: bool = True,
                    reserved: bool = True, block: int = 256, scope: int = 0) -> TraceRun:
    """Correctness mode: one kernel per phase, log + lifetime tags; reserved pages
    read at each phase boundary (after a round's mallocs).  heap=None runs CUDA malloc.
    scope: 0 warp calls, 1 block-collective, 2..8 cluster-collective (GA_TRACE_SCOPE)."""
    dev = torch.device("cuda", heap.device if heap else torch.cuda.current_device())
    R, T = sizes.shape
    st = heap.stream if heap else torch.cuda.current_stream()
    s = _stream(st)
    d_sizes = torch.from_numpy(np.ascontiguousarray(sizes, dtype=np.uint32).view(np.int32)).to(dev)
    held = torch.empty(2 * T, dtype=torch.int64, device=dev)
    held[0::2] = -1
    held[1::2] = 0
    counts = torch.zeros(8, dtype=torch.int64, device=dev)
    rounds = R + 1 if D == 1 else R
    d_log = torch.zeros(2 * rounds * T * 2, dtype=torch.int64, device=dev) if (log and heap) else None
    flags = (GA_TRACE_LOG if d_log is not None else 0) | (GA_TRACE_TAG if tag else 0) | GA_TRACE_SCOPE(scope)
    run = TraceRun({})
    lp = d_log.data_ptr() if d_log is not None else 0
    for r in range(rounds):
        if D == 1:
            if heap:
                ga_trace_phase(heap.h, s, d_sizes.data_ptr(), R, T, 1, r, 0, held.data_ptr(), lp,
                               counts.data_ptr(), flags, block)
            else:
                ga_cuda_trace_phase(s, d_sizes.data_ptr(), R, T, 1, r, 0, held.data_ptr(), counts.data_ptr(),
                                    flags, block)
            if heap and reserved and r < R:
                run.reserved_per_round.append(heap.reserved_bytes())
                run.reserved_dev_per_round.append(heap.stats()["reserved_bytes"])
                run.live_per_round.append(int(held[1::2].sum().item()))
        else:
            for ph in (0, 1):
                if heap:
                    ga_trace_phase(heap.h, s, d_sizes.data_ptr(), R, T, 0, r, ph, held.data_ptr(), lp,
                                   counts.data_ptr(), flags, block)
                else:
                    ga_cuda_trace_phase(s, d_sizes.data_ptr(), R, T, 0, r, ph, held.data_ptr(), counts.data_ptr(),
                                        flags, block)
                if heap and reserved and ph == 0:
                    run.reserved_per_round.append(heap.reserved_bytes())
                    run.reserved_dev_per_round.append(heap.stats()["reserved_bytes"])
                    run.live_per_round.append(int(held[1::2].sum().item()))
    st.synchronize()
    run.counts = _counts(counts)
    run.peak_reserved_bytes = max(run.reserved_per_round) if run.reserved_per_round else 0
    if d_log is not None:
        run.log = d_log.cpu().numpy().view(LOG_DTYPE)
    return run


def run_timed(heap: GpuHeap | None, d_sizes: torch.Tensor, R: int, T: int, D: int,
              counts: torch.Tensor, block: int = 256, stream=None, scope: int = 0):
    """Timing mode: one kernel, allocator calls only (heap=None: CUDA malloc).
    scope: 0 warp calls, 1 block-collective, 2..8 cluster-collective."""
    s = _stream(stream)
    if heap and scope:
        ga_trace_timed_scope(heap.h, s, d_sizes.data_ptr(), R, T, D, counts.data_ptr(), block, scope)
    elif heap:
        ga_trace_timed(heap.h, s, d_sizes.data_ptr(), R, T, D, counts.data_ptr(), block)
    else:
        ga_cuda_trace_timed(s, d_sizes.data_ptr(), R, T, D, counts.data_ptr(), block)


def run_timed_host(heap: GpuHeap, h_sizes: torch.Tensor, R: int, T: int, D: int, h_counts: np.ndarray,
                   block: int = 256, stream=None):
    """End-to-end: host sizes -> device, kernel, counts -> host, through one C-ABI call."""
    ga_trace_timed_host(heap.h, _stream(stream), h_sizes.data_ptr(), R, T, D, h_counts.ctypes.data, block)
