"""Canonical heap snapshot: parser + invariant checker -- TEST INFRASTRUCTURE ONLY.

The snapshot is a *logical* dump (format documented in include/ga.h, "Canonical
snapshot"), written independently by the oracle (ora_snapshot) and by the CUDA
library (ga_heap_snapshot).  This module parses either and checks the
quiescent-state invariants the paper fixes:

* buddy property 1 -- two sibling nodes are never both Available;
* buddy property 2 -- an Available node's sub-tree is all Busy,
  checked as "every page of an Available node is that node's head or a free
  interior page, and the nodes cover disjoint page ranges";
* each tree semaphore's value C equals the Available nodes of its order and
  D = E - R = 0 (two-stage accounting);
* each size-class semaphore's value (summed over arenas) equals the free slots
  of that class's bins, and D = 0;
* the page semaphore's value equals the free pages inside arena chunks;
* allocated tree blocks are aligned to their size (R-31);
* optionally (after quiesce): no empty bin and no empty chunk remains (R-22/23).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

MAGIC = 0x31304E5341534147  # "GASNAP01"

K_FREE_INTERIOR = 0x00
K_TREE_TAIL = 0x01
K_CHUNK_FREE = 0x02
K_CHUNK_HDR = 0x03
K_SPAN_TAIL = 0x04
K_BIN = 0x10      # | class index
K_SPAN = 0x20     # | span class index (first page of a span)
K_AVAIL = 0x40    # | order
K_ALLOC = 0x80    # | order


@dataclass
class Snapshot:
    heap_bytes: int
    pages: int
    page: int
    levels: int
    min_class: int
    ncls: int
    nspan: int
    chunk_pages: int
    kind: np.ndarray              # u8[pages]
    bins: dict                    # page -> np.ndarray(bool[slots]) (bin pages and span heads)
    level_bits: list              # list of bool arrays, level n has 2^(L-n) entries
    cls_C: np.ndarray             # i64[ncls + nspan]: bin classes, then span classes
    cls_absD: np.ndarray
    page_C: int
    page_absD: int
    tree_C: np.ndarray            # i64[levels]
    tree_D: np.ndarray
    pending: int

    def slots(self, c: int) -> int:
        """Slots of class c (0..ncls-1 bins, ncls.. spans)."""
        if c < self.ncls:
            return self.page // (self.min_class << c)
        return self.chunk_pages >> (c - self.ncls)

    def page_class(self, p: int) -> int:
        k = int(self.kind[p])
        return (k & 0x0F) + (self.ncls if (k & 0xF0) == K_SPAN else 0)

    def reserved_pages(self) -> int:
        return self.pages - sum(int(b.sum()) << n for n, b in enumerate(self.level_bits))


def parse(buf: bytes) -> Snapshot:
    b = np.frombuffer(buf, dtype=np.uint8)
    pos = 0

    def u64():
        nonlocal pos
        v = int(np.frombuffer(buf, dtype="<u8", count=1, offset=pos)[0])
        pos += 8
        return v

    def i64s(n):
        nonlocal pos
        v = np.frombuffer(buf, dtype="<i8", count=n, offset=pos).copy()
        pos += 8 * n
        return v

    if u64() != MAGIC:
        raise ValueError("not a GASNAP01 snapshot")
    heap_bytes, pages = u64(), u64()
    w = u64()
    page, levels = w & 0xFFFFFFFF, w >> 32
    w = u64()
    min_class, ncls, nspan, chunk_pages = w & 0xFFFFFFFF, (w >> 32) & 0xFF, (w >> 40) & 0xFF, w >> 48
    kind = b[pos:pos + pages].copy()
    pos += pages
    bins = {}
    for p in np.nonzero(((kind & 0xF0) == K_BIN) | ((kind & 0xF0) == K_SPAN))[0]:
        c = int(kind[p]) & 0x0F
        s = page // (min_class << c) if (kind[p] & 0xF0) == K_BIN else chunk_pages >> c
        nb = (s + 7) // 8
        bits = np.unpackbits(b[pos:pos + nb], bitorder="little")[:s].astype(bool)
        bins[int(p)] = bits
        pos += nb
    L = levels - 1
    level_bits = []
    for n in range(levels):
        cnt = 1 << (L - n)
        nb = (cnt + 7) // 8
        level_bits.append(np.unpackbits(b[pos:pos + nb], bitorder="little")[:cnt].astype(bool))
        pos += nb
    cls = i64s(2 * (ncls + nspan)).reshape(ncls + nspan, 2)
    pg = i64s(2)
    tr = i64s(2 * levels).reshape(levels, 2)
    pending = u64()
    if pos != len(buf):
        raise ValueError(f"snapshot length mismatch: parsed {pos} of {len(buf)} bytes")
    return Snapshot(heap_bytes, pages, page, levels, min_class, ncls, nspan, chunk_pages, kind, bins,
                    level_bits, cls[:, 0].copy(), cls[:, 1].copy(), int(pg[0]), int(pg[1]),
                    tr[:, 0].copy(), tr[:, 1].copy(), pending)


def check(s: Snapshot, require_reclaimed: bool = False) -> list:
    """Return a list of violated invariants (empty when all hold)."""
    errs = []
    L = s.levels - 1
    covered = np.zeros(s.pages, dtype=np.int32)
    for n, bits in enumerate(s.level_bits):
        idx = np.nonzero(bits)[0]
        if len(idx) and ((idx.astype(np.int64) + 1) << n).max() > s.pages:
            errs.append(f"level {n}: available node outside the heap")
            continue
        # property 1 (siblings both inside the heap never both available)
        if n < L:
            pair = bits[0::2] & bits[1::2]
            if pair.any():
                errs.append(f"level {n}: sibling nodes both available")
        if s.tree_C[n] != len(idx):
            errs.append(f"level {n}: tree semaphore C={s.tree_C[n]} but {len(idx)} available")
        if s.tree_D[n] != 0:
            errs.append(f"level {n}: tree semaphore D={s.tree_D[n]} != 0")
        for i in idx:
            lo, hi = int(i) << n, (int(i) + 1) << n
            covered[lo:hi] += 1
            if s.kind[lo] != (K_AVAIL | n):
                errs.append(f"level {n} node {i}: head page kind {s.kind[lo]:#x}")
            if hi - lo > 1 and (s.kind[lo + 1:hi] != K_FREE_INTERIOR).any():
                errs.append(f"level {n} node {i}: interior page not free")
    if (covered > 1).any():
        errs.append("property 2: available nodes overlap (an available node below another)")
    free_int = (s.kind == K_FREE_INTERIOR) | ((s.kind & 0xC0) == K_AVAIL)
    if ((covered == 1) != free_int).any():
        errs.append("page kinds disagree with the available nodes")
    # allocated tree blocks
    for p in np.nonzero((s.kind & 0xC0) == K_ALLOC)[0]:
        o = int(s.kind[p]) & 0x3F
        if p % (1 << o):
            errs.append(f"tree block at page {p} not aligned to its order {o}")
        elif (1 << o) > 1 and (s.kind[p + 1:p + (1 << o)] != K_TREE_TAIL).any():
            errs.append(f"tree block at page {p}: tail pages wrong")
    # chunks: aligned groups of chunk pages made only of free / bin / header pages
    cp = s.chunk_pages
    chunkish = (s.kind == K_CHUNK_FREE) | ((s.kind & 0xF0) == K_BIN) | (s.kind == K_CHUNK_HDR) | \
        (s.kind == K_SPAN_TAIL) | ((s.kind & 0xF0) == K_SPAN)
    ch = chunkish.reshape(-1, cp) if s.pages % cp == 0 else None
    # a span is a whole chunk: its head page first, then span tails only
    for p in np.nonzero((s.kind & 0xF0) == K_SPAN)[0]:
        if p % cp or (s.kind[p + 1:p + cp] != K_SPAN_TAIL).any():
            errs.append(f"span at page {p}: not a whole chunk (head + {cp - 1} tails)")
    tails = np.nonzero(s.kind == K_SPAN_TAIL)[0]
    if len(tails) and ((s.kind[tails - tails % cp] & 0xF0) != K_SPAN).any():
        errs.append("span tail page outside a span")
    if ch is None:
        errs.append("pages not a whole number of chunks")
    else:
        part = ch.any(axis=1) & ~ch.all(axis=1)
        if part.any():
            errs.append("a chunk is partly inside a tree block")
        if require_reclaimed:
            empty = ch.all(axis=1) & (s.kind.reshape(-1, cp) == K_CHUNK_FREE).all(axis=1)
            if empty.any():
                errs.append(f"{int(empty.sum())} empty chunk(s) not reclaimed")
    # class semaphores vs bin bitmaps
    free_slots = np.zeros(s.ncls + s.nspan, dtype=np.int64)
    for p, bits in s.bins.items():
        c = s.page_class(p)
        nfree = int((~bits).sum())
        free_slots[c] += nfree
        if require_reclaimed and nfree == len(bits):
            errs.append(f"empty bin at page {p} not reclaimed")
    for c in range(s.ncls + s.nspan):
        if s.cls_C[c] != free_slots[c]:
            errs.append(f"class {c}: semaphore C={s.cls_C[c]} but {free_slots[c]} free slots")
        if s.cls_absD[c] != 0:
            errs.append(f"class {c}: semaphore |D|={s.cls_absD[c]} != 0")
    nfreepages = int((s.kind == K_CHUNK_FREE).sum())
    if s.page_C != nfreepages:
        errs.append(f"page semaphore C={s.page_C} but {nfreepages} free chunk pages")
    if s.page_absD != 0:
        errs.append(f"page semaphore |D|={s.page_absD} != 0")
    if require_reclaimed and s.pending:
        errs.append(f"{s.pending} reclamation items pending")
    return errs
