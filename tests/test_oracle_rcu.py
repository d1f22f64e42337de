"""Pins for oracle/rcu.py -- SRCU and RCU delegation, the model
the f3 benchmark (Fig. 6) will be checked against.

What the paper fixes, checked over every schedule with a bounded number of
preemptions (context-bounded model checking) and over random schedules:
* grace periods: no callback releases a node while a reader that reached it
  is still inside its read-side critical section;
* RCU delegation loses nothing: a conditional barrier that returns at once
  leaves its callback to the pending barrier, so no callback is stranded
  (Fig. 4b);
* no deadlock.
Mutations that a plausible implementation mistake would make (no re-check on
reader entry, R-39; clearing the pending flag after taking the queue, R-40;
a barrier that does not wait for the old epoch to drain) must each be caught.
"""
import pytest

from oracle import rcu

pytestmark = pytest.mark.filterwarnings("ignore")


def _threads(delegate, readers=1, writers=2, nodes=(1, 2), **kw):
    def mk(S):
        ts = [rcu.reader(S, i, list(nodes), kw.get("recheck", True)) for i in range(readers)]
        ts += [rcu.writer(S, readers + j, nodes[j % len(nodes)] + 10 * (j // len(nodes)), delegate,
                          kw.get("clear_first", True)) for j in range(writers)]
        return ts
    return mk


@pytest.mark.parametrize("delegate", [False, True])
def test_grace_period_and_no_deadlock_bounded(delegate):
    runs, viol, stranded, dead = rcu.explore(_threads(delegate), preemptions=3)
    assert runs > 1000
    assert viol == 0 and dead == 0
    assert stranded == 0


@pytest.mark.parametrize("delegate", [False, True])
def test_two_readers_three_writers_random(delegate):
    runs, viol, stranded, dead = rcu.explore_random(_threads(delegate, readers=2, writers=3, nodes=(1, 2, 3)),
                                                    runs=3000, seed=7)
    assert viol == 0 and dead == 0 and stranded == 0


def test_delegation_actually_delegates():
    """Some schedules must take the conditional barrier's early return (else
    the model never exercises delegation)."""
    seen = []
    orig = rcu.conditional_barrier

    def spy(S, tid, clear_first=True):
        returned_early = S.pending
        seen.append(bool(returned_early))
        yield from orig(S, tid, clear_first)
    rcu.conditional_barrier = spy
    try:
        rcu.explore_random(_threads(True, readers=1, writers=3, nodes=(1, 2, 3)), runs=500, seed=3)
    finally:
        rcu.conditional_barrier = orig
    assert any(seen) and not all(seen)


def test_mutation_no_reader_recheck_is_caught():
    viol = 0
    for delegate in (False, True):
        viol += rcu.explore(_threads(delegate, recheck=False), preemptions=3)[1]
        viol += rcu.explore_random(_threads(delegate, readers=2, writers=3, nodes=(1, 2, 3), recheck=False),
                                   runs=3000, seed=11)[1]
    assert viol > 0


def test_mutation_clear_after_take_strands_callbacks():
    stranded = rcu.explore(_threads(True, writers=3, nodes=(1, 2, 3), clear_first=False), preemptions=3)[2]
    stranded += rcu.explore_random(_threads(True, writers=3, nodes=(1, 2, 3), clear_first=False),
                                   runs=3000, seed=5)[2]
    assert stranded > 0


def test_mutation_barrier_without_drain_is_caught(monkeypatch):
    def no_wait_barrier(S, tid):
        while S.mutex != -1:
            yield rcu.BLOCKED
        S.mutex = tid
        yield
        cbs, S.queue = S.queue, []
        S.epoch += 1
        yield
        rcu._release(S, cbs)               # no drain of the previous epoch
        S.mutex = -1
        yield
    monkeypatch.setattr(rcu, "full_barrier", no_wait_barrier)
    runs, viol, _, _ = rcu.explore_random(_threads(False), runs=2000, seed=2)
    assert viol > 0


def test_list_removal_outcome():
    """Fig. 6 benchmark outcome: every list tag present in the
    input is removed exactly once; the rest of the list stays."""
    removed, live = rcu.list_removal(range(8), [3, 9, 3, 0, 7, 12])
    assert removed == [3, 0, 7]
    assert live == [1, 2, 4, 5, 6]
    removed, live = rcu.list_removal(range(4), [0, 1, 2, 3] * 8)
    assert sorted(removed) == [0, 1, 2, 3] and live == []
