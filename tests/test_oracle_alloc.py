"""Pins for the sequential allocator oracle (oracle/ga_oracle.c).

Each test pins the oracle to something other than itself:
closed-form capacities, the paper's printed failure rates, a
textbook buddy example, brute force over every short trace on tiny heaps
(P-4), the buddy properties, free-all == fresh snapshot (P-7),
and negative tests showing the log / snapshot checkers catch each plausible
mistake (overlap, misalignment, wrong free, wrong class, broken buddy state).
"""
import itertools
import os
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle
import tracegen
from oracle import BUILD, PAPER, TINY, snapshot as S

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# --------------------------------------------------------------------------- front end
@pytest.mark.parametrize("n,route,val", [
    (1, "bin", 0), (16, "bin", 0), (17, "bin", 1), (32, "bin", 1), (33, "bin", 2),
    (1000, "bin", 6), (1024, "bin", 6), (1025, "bin", 7), (2048, "bin", 7),
    (2049, "tree", 0), (4096, "tree", 0), (4097, "tree", 1), (65536, "tree", 4),
    (65537, "tree", 5), (0, "null", None)])
def test_classify_rounds_up_to_power_of_two(n, route, val):
    """round up to the closest power of two; R-12 threshold; R-15 malloc(0)."""
    h = oracle.Heap(8 << 20)
    assert h.classify(n) == (route, val)


def test_classify_rejects_larger_than_heap():
    h = oracle.Heap(1 << 20)
    assert h.classify((1 << 20) + 1) == ("null", None)
    assert h.malloc((1 << 20) + 1) is None
    assert h.malloc(0) is None
    assert h.free(None) == 1          # free(NULL) is a no-op (R-16)


# --------------------------------------------------------------------------- capacities
@pytest.mark.parametrize("size", [16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 8192, 65536])
def test_single_class_exhaust_equals_capacity(size):
    """P-6 / P:L1512-1520: without fragmentation there are no failures below
    capacity; build layout keeps metadata out of band (R-29) so cap = heap/size."""
    heap = 2 << 20
    h = oracle.Heap(heap)
    cap = heap // size
    offs = []
    for _ in range(cap):
        o = h.malloc(size)
        assert o is not None
        offs.append(o)
    assert h.malloc(size) is None
    assert len(set(offs)) == cap
    assert h.check() is None
    fresh = oracle.snapshot_of_fresh(heap)
    for o in offs:
        assert h.free(o) == 0
    assert h.check() is None and h.snapshot() == fresh


def _golden_rates():
    for line in open(os.path.join(GOLD, "paper_layout_failure_rates.txt")):
        if line.strip() and not line.startswith("#"):
            s, num, den, word = line.split()
            yield int(s), Fraction(int(num), int(den)), word


@pytest.mark.parametrize("size,rate,word", list(_golden_rates()))
def test_paper_layout_failure_rates(size, rate, word):
    """Fig. 7 methodology: just enough threads to exhaust the pool,
    one malloc each; the failure fraction must match the paper's words and the
    closed form of its layout (P-5)."""
    pool = 8 << 20 if size <= 512 else 32 << 20
    threads = pool // size
    t = np.full((1, threads), size, dtype=np.uint32)
    r = oracle.run_trace(t, pool, 0, layout=PAPER, want_ok=False)
    assert r.stats["invariant_error"] == 0
    got = Fraction(r.stats["n_malloc_fail"], threads)
    assert got == rate
    if word == "50%":
        assert got == Fraction(1, 2)
    if word == "never":
        assert got == 0
    if word == "small":
        assert got < Fraction(5, 100)
    if word == "moderate":
        assert Fraction(10, 100) < got < Fraction(30, 100)


# --------------------------------------------------------------------------- buddy
def test_textbook_buddy_example():
    """Lowest-address buddy allocation (Knuth's buddy system, the paper's [14]) on a
    16-page heap: every step is fixed by the textbook algorithm."""
    h = oracle.Heap(16 * 4096, dict(BUILD, chunk_pages=4))
    P = 4096
    a = h.malloc(P)          # splits 16 -> 8 -> 4 -> 2 -> 1: page 0
    b = h.malloc(2 * P)      # lowest order-1 block left: pages 2-3
    c = h.malloc(P)          # page 1 (the buddy of a)
    d = h.malloc(4 * P)      # pages 4-7
    e = h.malloc(8 * P)      # pages 8-15
    assert (a, b, c, d, e) == (0, 2 * P, P, 4 * P, 8 * P)
    assert h.malloc(P) is None
    assert h.free(c) == 0 and h.free(a) == 0      # a+c merge -> order-1 node [0,2)
    assert h.malloc(2 * P) == 0
    for o in (0, b, d, e):
        assert h.free(o) == 0
    assert h.check() is None
    assert h.malloc(16 * P) == 0                   # fully coalesced (R-19 cascade)


def test_forest_heap_not_power_of_two():
    """R-30: a 3-chunk heap is the forest {2 chunks, 1 chunk}."""
    h = oracle.Heap(3 * 64 * 4096)
    s = S.parse(h.snapshot())
    assert not S.check(s)
    roots = [(n, int(i)) for n, bits in enumerate(s.level_bits) for i in np.nonzero(bits)[0]]
    assert roots == [(6, 2), (7, 0)]
    assert h.malloc(128 * 4096) == 0
    assert h.malloc(64 * 4096) == 128 * 4096
    assert h.malloc(4096) is None


def test_random_ops_keep_invariants_and_free_all_restores():
    rng = random.Random(1)
    sizes = [16, 24, 100, 256, 700, 2048, 3000, 4096, 9000, 40000, 65536, 200000]
    for heap in (1 << 20, 3 << 20):
        fresh = oracle.snapshot_of_fresh(heap)
        h = oracle.Heap(heap)
        live = []
        for step in range(3000):
            if live and rng.random() < 0.45:
                o = live.pop(rng.randrange(len(live)))
                assert h.free(o) == 0
            else:
                o = h.malloc(rng.choice(sizes))
                if o is not None:
                    live.append(o)
            if step % 97 == 0:
                assert h.check() is None, step
                assert not S.check(S.parse(h.snapshot()))
        for o in live:
            assert h.free(o) == 0
        assert h.check() is None
        assert h.snapshot() == fresh
        assert h.reserved_pages() == 0


def test_double_and_foreign_free_rejected():
    h = oracle.Heap(1 << 20)
    o = h.malloc(64)
    assert h.free(o) == 0
    assert h.free(o) < 0            # double free
    assert h.free(12345) < 0        # not a block
    t = h.malloc(8192)
    assert h.free(t + 4096) < 0     # inside a tree block


# --------------------------------------------------------------------------- brute force
def _legal_exists(live, req, layout, pages):
    """Byte-occupancy model: does any legal placement exist?"""
    P, CP = layout["page"], layout["chunk_pages"]
    c = 1
    while c < max(req, layout["min_class"]):
        c <<= 1
    tree_pages = np.zeros(pages, bool)
    bin_cls = {}
    bin_used = {}
    for off, n in live:
        cc = 1
        while cc < max(n, layout["min_class"]):
            cc <<= 1
        if cc <= layout["bin_max"]:
            p = off // P
            bin_cls[p] = cc
            bin_used[p] = bin_used.get(p, 0) + 1
        else:
            ln = max(cc, P) // P
            tree_pages[off // P: off // P + ln] = True
    chunk_alloc = np.zeros(pages // CP, bool)
    for p in bin_cls:
        chunk_alloc[p // CP] = True
    free = ~tree_pages & ~np.repeat(chunk_alloc, CP)
    if c <= layout["bin_max"]:
        slots = P // c
        if any(cls == c and bin_used[p] < slots for p, cls in bin_cls.items()):
            return True
        for k in np.nonzero(chunk_alloc)[0]:
            if any(p not in bin_cls for p in range(k * CP, (k + 1) * CP)):
                return True
        return any(free[k * CP:(k + 1) * CP].all() for k in range(pages // CP))
    ln = max(c, P) // P
    return any(free[i:i + ln].all() for i in range(0, pages - ln + 1, ln))


def _brute(heap_pages, max_ops, sample=None, seed=0):
    layout = TINY
    P = layout["page"]
    alphabet = [16, 32, 64, 128]
    rng = random.Random(seed)
    checked = 0

    def run(seq):
        nonlocal checked
        h = oracle.Heap(heap_pages * P, layout)
        live = []
        for op in seq:
            if op[0] == "m":
                want = _legal_exists(live, op[1], layout, heap_pages)
                o = h.malloc(op[1])
                assert (o is not None) == want, (seq, op, live)
                if o is not None:
                    live.append((o, op[1]))
            else:
                if op[1] >= len(live):
                    return
                o, _ = live.pop(op[1])
                assert h.free(o) == 0
            checked += 1
        assert h.check() is None, seq

    ops = [("m", s) for s in alphabet] + [("f", i) for i in range(max_ops)]
    if sample is None:
        for L in range(1, max_ops + 1):
            for seq in itertools.product(ops, repeat=L):
                # skip frees of non-existent indices early
                nlive, okseq = 0, True
                for op in seq:
                    if op[0] == "m":
                        nlive += 1
                    elif op[1] >= nlive:
                        okseq = False
                        break
                    else:
                        nlive -= 1
                if okseq:
                    run(seq)
    else:
        for _ in range(sample):
            L = rng.randint(1, max_ops)
            seq, nlive = [], 0
            for _ in range(L):
                if nlive and rng.random() < 0.35:
                    seq.append(("f", rng.randrange(nlive)))
                    nlive -= 1
                else:
                    seq.append(("m", rng.choice(alphabet)))
                    nlive += 1
            run(seq)
    return checked


def test_brute_force_exhaustive_tiny_heap():
    """P-4: the oracle succeeds exactly when a legal placement exists (8-page heap,
    every trace of <= 5 ops over {malloc16/32/64/128, free(i-th live)})."""
    assert _brute(8, 5) > 10000


def test_brute_force_sampled_longer_traces():
    assert _brute(16, 14, sample=4000, seed=3) > 10000


# --------------------------------------------------------------------------- trace + log checker
def test_trace_runner_d1_and_log():
    t = tracegen.d1_tiny()
    r = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_log=True, check_each_round=True)
    st = r.stats
    assert st["n_malloc"] == 1024 and st["n_malloc_fail"] == 0 and st["n_free"] == 1024
    assert st["peak_reserved_bytes"] == 64 * 4096        # one chunk of 4 bins
    assert st["n_bin_grow"] == 4 and st["final_reserved_bytes"] == 0
    err, cs = oracle.check_log(r.log, t.R, t.T, t.D, t.heap_bytes)
    assert err == 0 and cs["n_ok"] == 1024


def test_trace_runner_churn_small():
    t = tracegen.d4_small()
    r = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_log=True, check_each_round=True)
    st = r.stats
    assert st["invariant_error"] == 0 and st["n_malloc_fail"] == 0
    assert st["n_free"] == st["n_malloc"] == t.R * t.T
    err, cs = oracle.check_log(r.log, t.R, t.T, t.D, t.heap_bytes)
    assert err == 0 and cs["peak_live_bytes"] == st["peak_live_bytes"]
    # fragmentation >= the rounding waste alone (requests are 2^k + U[1, 2^k])
    assert st["peak_reserved_bytes"] / st["peak_live_bytes"] > 1.2


def _valid_log():
    t = tracegen.d4_small(T=512, R=4, heap_bytes=16 << 20)
    r = oracle.run_trace(t.sizes, t.heap_bytes, t.D, want_log=True)
    assert oracle.check_log(r.log, t.R, t.T, t.D, t.heap_bytes)[0] == 0
    return t, r.log


def test_checker_catches_overlap():
    t, log = _valid_log()
    m = log[0::2]
    i, j = 3, 10            # round 0, tids 3 and 10: make j's block start inside i's
    log[2 * j]["off"] = log[2 * i]["off"]
    log[2 * (t.T + j) + 1]["off"] = log[2 * i]["off"]   # keep its free consistent
    assert oracle.check_log(log, t.R, t.T, t.D, t.heap_bytes)[0] in (3, 20)
    del m


def test_checker_catches_misalignment_and_bounds():
    t, log = _valid_log()
    bad = log.copy()
    bad[0]["off"] += 16 if bad[0]["size"] > 16 else 8
    bad[2 * t.T + 1]["off"] = bad[0]["off"]
    assert oracle.check_log(bad, t.R, t.T, t.D, t.heap_bytes)[0] in (2, 3)
    bad = log.copy()
    bad[0]["off"] = t.heap_bytes
    bad[2 * t.T + 1]["off"] = t.heap_bytes
    assert oracle.check_log(bad, t.R, t.T, t.D, t.heap_bytes)[0] == 1


def test_checker_catches_wrong_free_and_meta():
    t, log = _valid_log()
    bad = log.copy()
    bad[2 * t.T + 1]["off"] ^= 4096
    assert oracle.check_log(bad, t.R, t.T, t.D, t.heap_bytes)[0] == 11
    bad = log.copy()
    bad[0]["meta"] ^= 1
    assert oracle.check_log(bad, t.R, t.T, t.D, t.heap_bytes)[0] == 30


def test_checker_catches_wrong_class():
    """A block of a bigger request placed at a spacing valid only for a smaller class."""
    T = 64
    sizes = np.full((1, T), 16, dtype=np.uint32)
    r = oracle.run_trace(sizes, 1 << 20, 0, want_log=True)
    log = r.log.copy()
    log[0]["size"] = 32                 # tid 0 claims 32 B at a 16 B spacing
    log[1]["size"] = 32
    assert oracle.check_log(log, 1, T, 0, 1 << 20)[0] in (3, 20, 13)


# --------------------------------------------------------------------------- snapshot checker
def test_snapshot_checker_catches_broken_states():
    h = oracle.Heap(1 << 20)
    for _ in range(5):
        h.malloc(4096)
    buf = bytearray(h.snapshot())
    assert not S.check(S.parse(bytes(buf)))
    s = S.parse(bytes(buf))
    # make two siblings available at level 0: property 1
    lv = s.level_bits[0].copy()
    lv[4] = lv[5] = True
    s.level_bits[0] = lv
    assert any("sibling" in e or "semaphore" in e for e in S.check(s))
    s = S.parse(bytes(buf))
    s.tree_C[0] += 1
    assert any("tree semaphore" in e for e in S.check(s))
    s = S.parse(bytes(buf))
    s.kind[3] = S.K_FREE_INTERIOR
    assert S.check(s)


def _paper_fill(heap_bytes, sizes_cycle, seed):
    """Fill a paper-layout oracle heap with requests drawn from sizes_cycle
    until every size fails; returns [(offset, class_bytes)]."""
    h = oracle.Heap(heap_bytes, PAPER)
    rng = np.random.default_rng(seed)
    live, alive = [], set(sizes_cycle)
    while alive:
        n = int(rng.choice(sorted(alive)))
        off = h.malloc(n)
        if off is None:
            alive.discard(n)
            continue
        live.append((off, max(8, 1 << (n - 1).bit_length())))
    return h, live


@pytest.mark.parametrize("sizes", [(8, 16, 32, 64, 128), (8, 128), (16, 32, 256, 512, 1024), (8, 64, 1024, 2048, 4096)])
def test_paper_layout_slots_disjoint_and_outside_headers(sizes):
    """Reading R-11 (paper layout): every chunk keeps 128 B
    in-band headers at the start of each of its 64 pages (chunk header, the 62
    bin headers, the second header bin), bin bodies start at +128, and the 62
    128-byte tails live in the two header pages (tail t at chunk offset
    128 + 128t for t < 31, else 4096 + 128 + 128(t - 31)).  At full fill with
    mixed classes -- so every bin of every chunk uses its tail -- the slots are
    pairwise disjoint, aligned to min(class, 128) relative to their page, inside
    the heap, and none touches a header.  A tail off by one slot (or placed in
    the wrong header page) overlaps a neighbour or a header and fails here.
    Freeing everything restores the fresh heap."""
    heap_bytes = 4 * 256 << 10
    h, live = _paper_fill(heap_bytes, sizes, seed=len(sizes) * 7 + sizes[0])
    offs = np.array([o for o, _ in live], dtype=np.int64)
    lens = np.array([c for _, c in live], dtype=np.int64)
    assert offs.min() >= 0 and (offs + lens).max() <= heap_bytes
    idx = np.argsort(offs)
    assert np.all(offs[idx][1:] >= offs[idx][:-1] + lens[idx][:-1]), "overlapping slots"
    bins = lens <= 1024                                   # UAlloc slots (2 KB goes to a 4 KB page)
    in_page = offs[bins] % 4096
    assert np.all((in_page >= 128) | (lens[bins] > 4096)), "a slot inside a 128 B header"
    assert np.all((in_page % np.minimum(lens[bins], 128)) == 0)
    if 8 in sizes and 128 in sizes:                       # tails used: slots in pages 0/1 of chunks
        pg = (offs[bins] // 4096) % 64
        assert np.any(pg == 0) and np.any(pg == 1)
    fresh = oracle.snapshot_of_fresh(heap_bytes, PAPER)
    for o, _ in live:
        assert h.free(o) == 0
    assert h.snapshot() == fresh
    h.close()


def test_paper_layout_tail_capacity_per_chunk():
    """One chunk filled with 128 B requests: 62 bins x (3968/128 body slots + 1
    tail slot) = 62 x 32 = 1984 slots; the tails supply exactly
    62 of them, all inside the two header pages."""
    h, live = _paper_fill(256 << 10, (128,), seed=1)
    assert len(live) == 62 * 32
    pg = np.array([(o // 4096) % 64 for o, _ in live])
    assert int((pg <= 1).sum()) == 62
    h.close()
