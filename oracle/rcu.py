"""SRCU with RCU delegation (conditional barrier) -- a step-by-step model.

TEST INFRASTRUCTURE (see oracle/__init__.py): only tests/, __graft_entry__ and
bench.py's CPU legs may use it.  It shares no code with the CUDA path.

Follows Sec. 4.2.1 of Gelado & Garland:

* SRCU: an epoch counter and a pair of reader counters.  A
  reader increments the counter of the current epoch on entering the read-side
  critical section and decrements it on exit.  A barrier acquires the RCU
  mutex, increments the epoch, waits for the previous epoch's counter to drain
  to zero, then releases the mutex.  A writer unlinks an element, queues a
  callback that releases it, and issues a barrier before the callbacks run
  (P:L1126-1134).
* Reading R-39 (reader entry, silent in the paper): the reader re-reads the
  epoch after incrementing its counter and retries on the new epoch if a flip
  raced with it; otherwise a reader could count itself into an epoch the
  barrier already finished draining.
* Conditional barrier / RCU delegation (Fig. 4b): a barrier
  issued while another barrier is waiting to increment the epoch counter
  returns at once; the waiting barrier runs its callbacks.  Reading R-40: "waiting to
  increment" = a barrier that has announced itself (a `pending` flag) and not
  yet taken the callback queue.  The pending barrier clears the flag, then
  takes the queue, then flips: a delegator enqueues first and tests the flag
  second, so its callback is taken by the barrier it delegated to (or, if the
  flag was already clear, it becomes the pending barrier itself).

Threads are generators that yield after every shared-memory step, so an
explorer can run them in any interleaving (sequential consistency).
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass, field


BLOCKED = "blocked"                    # yielded by a spin loop whose condition failed


@dataclass
class Shared:
    epoch: int = 0
    cnt: list = field(default_factory=lambda: [0, 0])
    mutex: int = -1                    # owner thread id, -1 = free
    pending: int = 0                   # a barrier waiting to increment the epoch (delegation)
    queue: list = field(default_factory=list)      # queued callbacks (node ids)
    unlinked: set = field(default_factory=set)     # nodes removed from the list, not yet released
    removed: set = field(default_factory=set)      # nodes ever removed from the list
    released: list = field(default_factory=list)   # node ids in release order
    holding: dict = field(default_factory=dict)    # reader id -> set of nodes it may still reach
    violations: list = field(default_factory=list)


def reader(S: Shared, tid: int, nodes, recheck: bool = True):
    """Enter the read-side critical section, traverse `nodes` (one step each),
    leave.  A node the reader reaches must not be released while it is inside."""
    while True:
        idx = S.epoch & 1
        yield
        S.cnt[idx] += 1
        yield
        if not recheck or (S.epoch & 1) == idx:   # R-39: re-check after counting in
            break
        S.cnt[idx] -= 1
        yield
    S.holding[tid] = set()
    for n in nodes:
        if n not in S.removed:             # still linked: the reader reaches it and may use it
            S.holding[tid].add(n)          # until it leaves the critical section
        yield
    del S.holding[tid]
    S.cnt[idx] -= 1
    yield


def _release(S: Shared, cbs):
    for n in cbs:
        for tid, held in S.holding.items():
            if n in held:
                S.violations.append(("released while a reader holds it", tid, n))
        S.released.append(n)
        S.unlinked.discard(n)


def full_barrier(S: Shared, tid: int):
    """Classical SRCU barrier: mutex, flip, drain the previous epoch, run callbacks."""
    while S.mutex != -1:
        yield BLOCKED
    S.mutex = tid
    yield
    cbs, S.queue = S.queue, []
    yield
    old = S.epoch & 1
    S.epoch += 1
    yield
    while S.cnt[old] != 0:
        yield BLOCKED
    _release(S, cbs)
    yield
    S.mutex = -1
    yield


def conditional_barrier(S: Shared, tid: int, clear_first: bool = True):
    """RCU delegation: return at once if a barrier is pending (its callbacks
    include ours), else become the pending barrier and run a full barrier."""
    if S.pending:
        yield
        return                             # delegated
    S.pending = 1
    yield
    while S.mutex != -1:
        yield BLOCKED
    S.mutex = tid
    yield
    if clear_first:
        S.pending = 0                      # R-40: clear the flag, then take the queue
        yield
    cbs, S.queue = S.queue, []
    yield
    if not clear_first:
        S.pending = 0
        yield
    old = S.epoch & 1
    S.epoch += 1
    yield
    while S.cnt[old] != 0:
        yield BLOCKED
    _release(S, cbs)
    yield
    S.mutex = -1
    yield


def writer(S: Shared, tid: int, node: int, delegate: bool, clear_first: bool = True):
    """Unlink `node`, queue its release, issue a (conditional) barrier."""
    S.unlinked.add(node)
    S.removed.add(node)
    yield
    S.queue.append(node)
    yield
    yield from (conditional_barrier(S, tid, clear_first) if delegate else full_barrier(S, tid))


def flush(S: Shared):
    """End of the kernel: one more full barrier releases what is still queued
    (delegated callbacks whose barrier had already taken the queue)."""
    for _ in full_barrier(S, -2):
        pass


def _sig(S: Shared):
    return (S.epoch, S.cnt[0], S.cnt[1], S.mutex, S.pending, len(S.queue), len(S.released), len(S.unlinked))


def _step(S, gens, last, done, t):
    """Run thread t one step; a blocked thread becomes runnable again only when
    some other thread's step changed the shared state."""
    before = _sig(S)
    try:
        last[t] = next(gens[t])
    except StopIteration:
        done[t] = True
    if _sig(S) != before:
        for u in range(len(gens)):
            if u != t and last[u] is BLOCKED:
                last[u] = "maybe"


def _run(make_threads, schedule):
    """Replay `schedule` (thread ids); return (S, gens, last yields, finished)."""
    S = Shared()
    gens = make_threads(S)
    last = [None] * len(gens)
    done = [False] * len(gens)
    for t in schedule:
        _step(S, gens, last, done, t)
    return S, gens, last, done


def _runnable(last, done):
    return [t for t in range(len(done)) if not done[t] and last[t] is not BLOCKED]


def explore(make_threads, preemptions: int = 2, max_steps: int = 300):
    """Every schedule with at most `preemptions` preemptive switches (a switch
    away from a thread that could continue; switching away from a blocked or
    finished thread is free), in the style of context-bounded model checking.
    Returns (schedules, violations, stranded, deadlocks): `stranded` counts
    schedules that end with queued callbacks no barrier took (they would wait
    for the end-of-kernel flush)."""
    n_runs = n_viol = n_leak = n_dead = 0
    stack = [([], -1, 0)]                 # (schedule, current thread, preemptions used)
    while stack:
        sched, cur, used = stack.pop()
        S, gens, last, done = _run(make_threads, sched)
        while True:
            run = _runnable(last, done)
            if not run:
                if not all(done):
                    n_dead += 1           # everyone left is blocked
                    break
                n_runs += 1
                n_leak += bool(S.queue)
                flush(S)
                n_viol += bool(S.violations)
                break
            if len(sched) > max_steps:
                n_dead += 1
                break
            cur_ok = cur in run
            for t in run:
                if t == cur or (not cur_ok and t == run[0]):
                    continue
                cost = 1 if cur_ok else 0
                if used + cost <= preemptions:
                    stack.append((sched + [t], t, used + cost))
            t = cur if cur_ok else run[0]
            sched = sched + [t]
            cur = t
            _step(S, gens, last, done, t)
    return n_runs, n_viol, n_leak, n_dead


def explore_random(make_threads, runs: int, seed: int = 1, max_steps: int = 2000):
    """Random schedules (uniform choice among runnable threads at every step)."""
    import random
    rng = random.Random(seed)
    n_viol = n_leak = n_dead = 0
    for _ in range(runs):
        S = Shared()
        gens = make_threads(S)
        last = [None] * len(gens)
        done = [False] * len(gens)
        steps = 0
        while True:
            run = _runnable(last, done)
            if not run:
                if not all(done):
                    n_dead += 1
                else:
                    n_leak += bool(S.queue)
                    flush(S)
                    n_viol += bool(S.violations)
                break
            steps += 1
            if steps > max_steps:
                n_dead += 1
                break
            t = rng.choice(run)
            _step(S, gens, last, done, t)
    return runs, n_viol, n_leak, n_dead


def list_removal(tags_in_list, input_tags):
    """The Fig. 6 benchmark's sequential outcome: each thread
    searches the list for its input tag and removes the element it finds.
    Returns (removed tags in input order, final list)."""
    live = list(tags_in_list)
    removed = []
    for t in input_tags:
        if t in live:
            live.remove(t)
            removed.append(t)
    return removed, live


if __name__ == "__main__":
    import time
    def mk(S):
        return [reader(S, 0, [1, 2]), writer(S, 1, 1, True), writer(S, 2, 2, True)]
    t0 = time.time()
    print(explore(mk, 2), time.time() - t0)
    print(explore_random(mk, 2000))
