"""Seeded synthetic request traces -- shared by the oracle tests and the CUDA path.

This module holds no allocator arithmetic: it only draws request sizes.  A trace
is ``u32 sizes[R][T]`` (round-major, so a GPU warp reads 32 consecutive u32;
0 = no malloc this round) plus a free depth ``D``:

* ``D == 1`` (churn): at round r each thread frees its round r-1 block, then
  mallocs ``sizes[r][t]``; a final free-all round follows the last round.
* ``D == 0`` (phase split): at round r every thread mallocs, then every
  round-r block is freed (correctness mode runs the two phases as two kernels).

Randomness is splitmix64 keyed by (seed, tid, round) -- counter based, so any
(round, tid) cell can be regenerated alone and both sides consume identical
bytes.  Recipes follow SURVEY.md 8(d) and DESIGN.md "Input recipe":

* d1 tiny     -- 1,024 threads, one round of malloc(16) + free, 1 MiB heap.
* d3 uniform  -- every thread requests the same size s (16 B .. 8 KiB), which
                 is the paper's Fig. 7 shape (one fixed size per run).
* d4 mixed    -- octave k ~ U{3..15}, n = 2^k + U[1, 2^k], so the class
                 2^(k+1) spans 16 B .. 64 KiB with 13 equiprobable classes and
                 lanes of a warp diverge; R = 16 churn rounds (D = 1).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

PHI = np.uint64(0x9E3779B97F4A7C15)
PSI = np.uint64(0xBF58476D1CE4E5B9)
BASE_SEED = 0x6A09E667F3BCC909
MASK64 = (1 << 64) - 1

FULL_GRID_THREADS = 148 * 2048      # 303,104: 148 SMs x 2,048 resident threads (B200)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)).astype(np.uint64)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def draws(seed: int, R: int, T: int) -> np.ndarray:
    """u64 random word for every (round, tid): splitmix64(seed ^ tid*PHI ^ round*PSI)."""
    with np.errstate(over="ignore"):
        tid = np.arange(T, dtype=np.uint64)[None, :]
        rnd = np.arange(R, dtype=np.uint64)[:, None]
        key = np.uint64(seed & MASK64) ^ (tid * PHI) ^ (rnd * PSI)
    return splitmix64(key)


@dataclass
class Trace:
    name: str
    sizes: np.ndarray       # u32[R][T]
    D: int                  # 0 phase split, 1 churn
    heap_bytes: int
    seed: int

    @property
    def R(self) -> int:
        return self.sizes.shape[0]

    @property
    def T(self) -> int:
        return self.sizes.shape[1]

    def calls(self) -> int:
        """malloc calls (failed ones included, R-17) + the frees of a full-success run."""
        return 2 * int(np.count_nonzero(self.sizes))


def d1_tiny(T: int = 1024, heap_bytes: int = 1 << 20) -> Trace:
    return Trace("d1_tiny", np.full((1, T), 16, dtype=np.uint32), 0, heap_bytes, BASE_SEED + 1)


def d3_uniform(size: int, T: int = FULL_GRID_THREADS, R: int = 1,
               heap_bytes: int = 4 << 30) -> Trace:
    return Trace(f"d3_uniform_{size}", np.full((R, T), size, dtype=np.uint32), 0, heap_bytes,
                 BASE_SEED + 3)


def d3_exhaust(size: int, heap_bytes: int, T: int | None = None) -> Trace:
    """Fig. 7 analogue: exactly enough threads to exhaust the pool."""
    if T is None:
        T = heap_bytes // size
    return Trace(f"d3_exhaust_{size}", np.full((1, T), size, dtype=np.uint32), 0, heap_bytes,
                 BASE_SEED + 3)


def mixed_sizes(seed: int, R: int, T: int, kmin: int = 3, kmax: int = 15) -> np.ndarray:
    """n = 2^k + U[1, 2^k], k ~ U{kmin..kmax}: class 2^(k+1)."""
    u = draws(seed, R, T)
    nk = np.uint64(kmax - kmin + 1)
    k = (u % nk).astype(np.int64) + kmin
    lo = (u >> np.uint64(32)).astype(np.uint64)
    span = (np.uint64(1) << k.astype(np.uint64))
    n = span + np.uint64(1) + (lo % span)
    return n.astype(np.uint32)


def d4_mixed(level: str = "pressure", T: int = FULL_GRID_THREADS, R: int = 16) -> Trace:
    # overcommit: 2.75 GiB, below the oracle's own peak reserved (3.07 GB), so
    # both sides fail some mallocs and reclaim under real exhaustion
    heap = {"fit": 16 << 30, "pressure": 4 << 30, "exhaust": 3 << 30, "overcommit": 11 << 28}[level]
    seed = BASE_SEED + 4
    return Trace(f"d4_mixed_{level}", mixed_sizes(seed, R, T), 1, heap, seed)


def d4_small(T: int = 4096, R: int = 8, heap_bytes: int = 64 << 20, seed: int = BASE_SEED + 40) -> Trace:
    """Reduced mixed trace for parity tests the oracle finishes in well under a second."""
    return Trace("d4_small", mixed_sizes(seed, R, T), 1, heap_bytes, seed)


def rcu_tags(T: int, W: int, seed: int = BASE_SEED + 6) -> np.ndarray:
    """Fig. 6 input: the W list tags 0..W-1 once each (writers)
    and T - W tags >= W that are not in the list (readers), in a seeded random
    order (splitmix64 keys, argsort)."""
    assert 0 < W <= T
    tags = np.concatenate([np.arange(W, dtype=np.uint32), W + np.arange(T - W, dtype=np.uint32)])
    keys = splitmix64(np.uint64(seed) ^ (np.arange(T, dtype=np.uint64) * np.uint64(0x9E3779B97F4A7C15)))
    return tags[np.argsort(keys, kind="stable")]
