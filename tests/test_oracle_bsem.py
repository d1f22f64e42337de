"""Pins for the bulk-semaphore model (oracle/bsem.py) -- Sec. 3.2-3.3 of the paper.

* Fig. 1(b) / Fig. 1(a) worked examples (tests/golden/*.txt, each citing P:L lines);
* special case: with E = infinity and B = 0 the bulk semaphore is a counting
  semaphore;
* exhaustive interleavings: no deadlock, no false resource
  starvation (successes = min(demand, supply)), no over-production
  (batches = min(pool, ceil(T/B))), terminal E = R = 0, C = leftover units;
  the (C, D = E - R) packing used by the CUDA path (R-6) gives the same terminals.
"""
import os
import random

import pytest

from oracle.bsem import (ACQUIRED, BLOCKED, GROW, BulkSemaphore, CountingSemaphore,
                         explore)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _rows(name):
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if line and not line.startswith("#"):
            yield line.split()


def test_fig1b_golden_trace():
    s = BulkSemaphore()
    for t, op, N, B, _, res, C, E, R in _rows("fig1b_bulk_semaphore.txt"):
        N, B = int(N), int(B)
        if op == "wait_enter":
            got = s.wait_enter(N, B)
            assert str(got) == res, (t, op)
        elif op == "signal":
            s.signal(N, B)
        elif op == "wait_retry":
            assert not s.spin_blocked(N), "waiter still blocked"
            s.wait_retry(N)
        assert s.state() == (int(C), int(E), int(R)), (t, op)
    # 5 units granted (T0..T4), two batches of four produced, 3 units left
    assert s.state() == (3, 0, 0)


def test_fig1b_waiters_block_until_signal():
    s = BulkSemaphore()
    assert s.wait_enter(1, 4) == GROW
    for _ in range(3):
        assert s.wait_enter(1, 4) == BLOCKED
    assert s.spin_blocked(1)               # covered by E, C still 0 -> keep waiting
    s.signal(3, 3)
    assert not s.spin_blocked(1)


def test_fig1a_counting_golden_trace():
    s = CountingSemaphore(0)
    for t, op, N, _, res, S in _rows("fig1a_counting_semaphore.txt"):
        N = int(N)
        if op == "wait":
            got = s.wait(N)
            assert (("blocked" if got is None else str(got)) == res), (t, op)
        else:
            s.signal(N)
        assert s.S == int(S), (t, op)


def test_bulk_with_infinite_expected_is_counting():
    """E = infinity, B = 0 -> counting-semaphore semantics."""
    rng = random.Random(7)
    INF = 1 << 40
    for _ in range(300):
        b = BulkSemaphore(C=0, E=INF, R=0)
        c = 0  # plain counting semaphore: wait(N) succeeds iff c >= N, else blocks
        for _ in range(40):
            N = rng.randint(1, 5)
            if rng.random() < 0.5:
                b.signal(N, 0)
                c += N
            else:
                r = b.wait_enter(N, 0)
                assert r != GROW
                if c >= N:
                    c -= N
                    assert r == ACQUIRED
                else:
                    assert r == BLOCKED and b.spin_blocked(N)
                    b.wait_retry(N)          # give up the reservation, state unchanged
            assert b.C == c and b.R == 0 and b.E == INF


@pytest.mark.parametrize("strict", [False, True])
@pytest.mark.parametrize("B", [2, 3, 4])
def test_exhaustive_interleavings_unit_demand(B, strict):
    """Every interleaving of T threads taking 1 unit each (Fig. 5 setting)."""
    for T in range(1, 6):
        for pool in range(0, 4):
            res = explore([1] * T, B, pool, strict=strict)
            assert res["deadlocks"] == 0, (T, B, pool)
            want_ok = min(T, pool * B)
            want_batches = min(pool, -(-T // B))
            for (C, E, R), used, ok in res["terminals"]:
                assert sum(ok) == want_ok, (T, B, pool, ok)       # no false starvation
                assert used == want_batches, (T, B, pool, used)   # no over-production
                assert E == 0 and R == 0
                assert C == used * B - sum(ok)


def test_cd_packing_matches_cer():
    """Reading R-6: Alg. 1/2 depend on E and R only through D = E - R."""
    for Ns, B, pool in [([1] * 5, 2, 2), ([1] * 5, 4, 1), ([2, 1, 3], 4, 2), ([1, 1, 1, 1], 3, 3)]:
        for strict in (False, True):
            a = explore(Ns, B, pool, strict=strict)
            b = explore(Ns, B, pool, strict=strict, cd_form=True)
            assert a["deadlocks"] == b["deadlocks"] == 0
            fa = {(C, E - R, used, ok) for (C, E, R), used, ok in a["terminals"]}
            fb = {(C, E - R, used, ok) for (C, E, R), used, ok in b["terminals"]}
            assert fa == fb


def test_group_demand_can_fail_with_units_left():
    """Reading R-27: warp groups (N > 1) can fail while C > 0, so the CUDA path
    degrades a failing group to per-lane N = 1 waits before returning NULL."""
    res = explore([3, 3, 3], 4, 2)
    assert res["deadlocks"] == 0
    assert any(C > 0 and not all(ok) for (C, E, R), used, ok in res["terminals"])


def test_group_demand_can_overproduce():
    res = explore([5, 1, 1], 4, 4)
    used = {u for _, u, _ in res["terminals"]}
    assert used >= {2} and max(used) <= 3


# ---------------------------------------------------------------------------
# The CUDA path's own semaphore protocols (oracle/bsem.py explore_gpu), checked
# against Alg. 1 on every interleaving of their atomic steps.
# ---------------------------------------------------------------------------
from oracle.bsem import explore_gpu  # noqa: E402


@pytest.mark.parametrize("form", ["fa", "arena"])
def test_gpu_forms_unit_demand_exact(form):
    """T <= 6 threads of demand 1 (the Fig. 5 setting): the form
    the CUDA path runs ("fa"; "arena" is a checked alternative) grants exactly min(T, pool*B) units (no false starvation,
    P:L488-506), use exactly min(pool, ceil(T/B)) batches (no over-production),
    never deadlock, never over-grant, end with D = 0, and are conservative in
    every reachable state (R-35)."""
    for T in range(1, 7):
        for B in (2, 3, 4):
            for pool in range(0, 4):
                r = explore_gpu([1] * T, B, pool, form)
                assert r["deadlocks"] == 0 and r["nonconservative"] == 0 and r["overgrant"] == 0, (T, B, pool)
                for (C, D), used, res in r["terminals"]:
                    ok = sum(o for _, o in res)
                    assert ok == min(T, pool * B), (T, B, pool, res)
                    assert used == min(pool, -(-T // B)), (T, B, pool, used)
                    assert D == 0 and C == used * B - ok


def _mixed_cases():
    import itertools
    for release in (False, True):
        for n in (2, 3):
            for Ns in itertools.combinations_with_replacement([1, 2, 3, 4], n):
                for B in (2, 4):
                    for C0 in (0, 1, 3, 4):
                        for pool in (1, 2, 3):
                            yield release, Ns, B, C0, pool


def test_gpu_forms_mixed_group_demand():
    """Warp groups (demand N > 1, reading R-8): on every interleaving the forms
    never deadlock, never over-grant, stay conservative, end with D = 0 and
    C = C0 + produced - held; they use at most ONE batch more than Alg. 1's
    worst interleaving (the over-production bound recorded in DESIGN.md R-35).
    Round 1's forms are checked too: they are not conservative."""
    worst = {"arena": 0, "fa": 0}
    for release, Ns, B, C0, pool in _mixed_cases():
        ref = explore_gpu(Ns, B, pool, "alg1", release=release, init_C=C0)
        ref_max = max(u for _, u, _ in ref["terminals"])
        for form in ("arena", "fa"):
            r = explore_gpu(Ns, B, pool, form, release=release, init_C=C0)
            assert r["deadlocks"] == 0 and r["nonconservative"] == 0 and r["overgrant"] == 0
            for (C, D), used, res in r["terminals"]:
                held = 0 if release else sum(N for N, o in res if o)
                assert D == 0 and C == C0 + used * B - held, (form, Ns, B, C0, pool, res)
            worst[form] = max(worst[form], max(u for _, u, _ in r["terminals"]) - ref_max)
    assert worst == {"arena": 1, "fa": 1}, worst


def test_round1_forms_are_caught():
    """Sensitivity of the checker: round 1's fast paths are flagged.
    * the unconditional fetch-add C -= N hid units from other deciders: states
      are not conservative, and a warp group fails while a batch is left that
      Alg. 1 would have used;
    * the optimistic TBuddy form starves a unit-demand thread (Alg. 1 never does)."""
    r = explore_gpu([1, 3], 2, 2, "arena_old", init_C=1)
    ref = explore_gpu([1, 3], 2, 2, "alg1", init_C=1)
    assert r["nonconservative"] > 0
    outcomes = {(u, res) for _, u, res in r["terminals"]}
    assert outcomes - {(u, res) for _, u, res in ref["terminals"]}
    assert any(not all(o for _, o in res) and u < 2 for u, res in outcomes)
    r = explore_gpu([1, 1], 2, 1, "tree_old")
    assert any(sum(o for _, o in res) < 2 for _, _, res in r["terminals"])
    assert r["nonconservative"] > 0
