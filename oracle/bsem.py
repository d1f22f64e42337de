"""Step-by-step bulk-semaphore model (Alg. 1 / Alg. 2) -- TEST INFRASTRUCTURE ONLY.

Paper: Gelado & Garland PPoPP'19, Sec. 3.2-3.3.

``BulkSemaphore`` holds the three counters of Sec. 3.3:
C (value), E (expected), R (reserved).  ``wait_enter`` is Alg. 1's first atomic
block, ``spin_blocked`` its while-test (reading R-2: keep
spinning while C < N and R <= C + E), ``wait_retry`` the second atomic block
(R -= N).  ``signal`` is Alg. 2 (reading R-3: C += N,
E -= B).  ``trywait`` is the TBuddy try-wait (reading R-7).

``CountingSemaphore`` is the growable counting semaphore of Sec. 3.2
 used by Fig. 1(a).

``explore`` runs an exhaustive depth-first search over every interleaving of
T logical threads doing two-stage allocation (wait -> grow-or-take) against a
pool of batches, the setting of Fig. 1 and Sec. 5.1.
"""
from __future__ import annotations

from dataclasses import dataclass

ACQUIRED, GROW, BLOCKED = 0, -1, 1


@dataclass
class BulkSemaphore:
    C: int = 0
    E: int = 0
    R: int = 0
    strict: bool = False   # R-2 alternative: spin while R < C + E (the garbled '<')

    def wait_enter(self, N: int, B: int) -> int:
        """Alg. 1, first atomic block.  Returns GROW (-1), ACQUIRED (0) or BLOCKED."""
        if self.C + self.E - self.R < N:
            self.E += B - N
            return GROW
        if self.C >= N:            # R-1: "Sem.C >= I" is "Sem.C >= N"
            self.C -= N
            return ACQUIRED
        self.R += N
        return BLOCKED

    def spin_blocked(self, N: int) -> bool:
        """Alg. 1 while-test: True while the waiter must keep yielding."""
        cover = (self.R < self.C + self.E) if self.strict else (self.R <= self.C + self.E)
        return self.C < N and cover

    def wait_retry(self, N: int) -> None:
        """Alg. 1, second atomic block: R <- R - N, then loop to the first block."""
        self.R -= N

    def signal(self, N: int, B: int) -> None:
        """Alg. 2."""
        self.C += N
        self.E -= B

    def trywait(self, N: int) -> bool:
        if self.C >= N:
            self.C -= N
            return True
        return False

    def state(self):
        return (self.C, self.E, self.R)


@dataclass
class CountingSemaphore:
    """Growable counting semaphore, Sec. 3.2."""
    S: int = 0

    def wait(self, N: int):
        """Returns N (acquired), the old S when the caller must grow, or None (blocked)."""
        if self.S >= N:
            self.S -= N
            return N
        if N > self.S >= 0:
            old = self.S
            self.S = -1
            return old
        return None

    def signal(self, N: int) -> None:
        self.S += N


# ---------------------------------------------------------------------------
# Exhaustive interleaving exploration (two-stage allocation).
# Thread program, per logical thread t with demand N[t] and batch B:
#   ENTER : Alg.1 block 1 -> ACQUIRED: DONE_OK | GROW: GROWING | BLOCKED: SPIN
#   SPIN  : enabled only once the while-test is false -> RETRY
#   RETRY : R -= N -> ENTER
#   GROWING: if a batch is left in the pool: pool -= 1, signal(B'-N, B'-N), DONE_OK
#            else signal(0, B'-N) (failure signal), DONE_FAIL
# ---------------------------------------------------------------------------
ENTER, SPIN, RETRY, GROWING, DONE_OK, DONE_FAIL = range(6)


def _bprime(N: int, B: int) -> int:
    return B * -(-N // B)   # R-8: B' = B * ceil(N / B)


def explore(Ns, B: int, pool: int, strict: bool = False, cd_form: bool = False):
    """Explore every interleaving.  Returns a summary of all terminal states.

    cd_form=True runs the same program on the (C, D = E - R) representation the
    CUDA path packs into one 64-bit word (reading R-6); its terminal summaries
    must equal the (C, E, R) ones.
    """
    Ns = tuple(Ns)
    T = len(Ns)
    start = ((0, 0, 0), pool, (ENTER,) * T)
    seen = set()
    terminals = set()
    deadlocks = 0
    stack = [start]
    while stack:
        st = stack.pop()
        if st in seen:
            continue
        seen.add(st)
        (C, E, R), pl, pcs = st
        succ = []
        for t in range(T):
            N, pc = Ns[t], pcs[t]
            Bp = _bprime(N, B)
            if cd_form:
                D = E - R
                if pc == ENTER:
                    if C + D < N:
                        succ.append(((C, E + Bp - N, R), pl, pcs[:t] + (GROWING,) + pcs[t + 1:]))
                    elif C >= N:
                        succ.append(((C - N, E, R), pl, pcs[:t] + (DONE_OK,) + pcs[t + 1:]))
                    else:
                        succ.append(((C, E, R + N), pl, pcs[:t] + (SPIN,) + pcs[t + 1:]))
                    continue
                if pc == SPIN:
                    cover = (C + D > 0) if strict else (C + D >= 0)
                    if not (C < N and cover):
                        succ.append(((C, E, R), pl, pcs[:t] + (RETRY,) + pcs[t + 1:]))
                    continue
            else:
                s = BulkSemaphore(C, E, R, strict)
                if pc == ENTER:
                    r = s.wait_enter(N, Bp)
                    npc = GROWING if r == GROW else DONE_OK if r == ACQUIRED else SPIN
                    succ.append((s.state(), pl, pcs[:t] + (npc,) + pcs[t + 1:]))
                    continue
                if pc == SPIN:
                    if not s.spin_blocked(N):
                        succ.append((s.state(), pl, pcs[:t] + (RETRY,) + pcs[t + 1:]))
                    continue
            if pc == RETRY:
                succ.append(((C, E, R - N), pl, pcs[:t] + (ENTER,) + pcs[t + 1:]))
            elif pc == GROWING:
                k = Bp // B                     # batches this grower needs
                if pl >= k:
                    succ.append(((C + Bp - N, E - (Bp - N), R), pl - k,
                                 pcs[:t] + (DONE_OK,) + pcs[t + 1:]))
                else:
                    succ.append(((C, E - (Bp - N), R), pl, pcs[:t] + (DONE_FAIL,) + pcs[t + 1:]))
        if not succ:
            if all(pc in (DONE_OK, DONE_FAIL) for pc in pcs):
                ok = tuple(pc == DONE_OK for pc in pcs)
                terminals.add(((C, E, R), pool - pl, ok))
            else:
                deadlocks += 1
        stack.extend(succ)
    return {"states": len(seen), "terminals": terminals, "deadlocks": deadlocks}


# ---------------------------------------------------------------------------
# The CUDA path's semaphore protocols as atomic-step programs (model only; no
# code is shared with the CUDA path).  The GPU keeps (C, D = E - R) in one
# 64-bit word (reading R-6) and replaces Alg. 1's single atomic block by
# fetch-adds where it pays (reading R-35).  Each program below is the sequence
# of atomic operations the CUDA code issues, one model step per atomic; a CAS
# works on a thread-local copy w of the word and fails if the word changed.
#
# forms:
#   "alg1"       Alg. 1 / Alg. 2 on (C, D): one atomic decision.
#   "arena_old"  round-1 arena fast path: fetch-add C -= N; on a short pre-image
#                add N back and run Alg. 1 as a CAS loop (what ADVICE r1 flagged:
#                the transient C - N hides N units from other deciders).
#   "arena"      (an intermediate round-2 form, kept as a checked alternative)
#                conservative fast path: fetch-add (C -= N, D += N) keeps C + D;
#                ACQUIRED iff the pre-image shows C >= N and C + D >= N, then a
#                repayment red D -= N; otherwise add (C += N, D -= N) back and
#                run the CAS loop.
#   "tree_old"   round-1 optimistic TBuddy form: fetch-add C -= N decides on the
#                pre-image; a second add converts to GROW (C += N, E += B' - N)
#                or to a reservation (C += N, R += N).
#   "fa"         the CUDA path's form for every semaphore (round 2): the first
#                fetch-add is (C -= N, D += B'); ACQUIRED repays D -= B', GROW
#                adds (C += N, D -= N), a reservation adds (C += N, D -= N + B').
# In the conservative forms every in-flight operation only lowers C and only
# raises C + D relative to the state with all decided operations applied, so no
# thread can take units that are not there (over-grant) or decide GROW when the
# decided state would not (over-production).  ``explore_gpu`` checks this in
# every reachable state ("conservative") besides the terminal properties.
# ---------------------------------------------------------------------------
(G_FAST, G_FIX, G_UNDO, G_CAS, G_SPIN, G_RETRY, G_TGROW, G_TRES, G_TSPIN, G_TRETRY,
 G_GROWING, G_REL, G_OK, G_FAIL) = range(14)
FORMS = ("alg1", "arena_old", "arena", "tree_old", "fa")


def _pending(form, pc, N, Bp):
    """(dC, dD) still to be applied by a thread at pc: the in-flight part of a
    decided operation (the 'decided state' is the word plus all of these)."""
    if form == "arena":
        return {G_FIX: (0, -N), G_UNDO: (N, -N)}.get(pc, (0, 0))
    if form == "arena_old":
        return {G_UNDO: (N, 0)}.get(pc, (0, 0))
    if form == "fa":
        return {G_FIX: (0, -Bp), G_TGROW: (N, -N), G_TRES: (N, -N - Bp)}.get(pc, (0, 0))
    if form == "tree_old":
        return {G_TGROW: (N, Bp - N), G_TRES: (N, -N)}.get(pc, (0, 0))
    return (0, 0)


def explore_gpu(Ns, B: int, pool: int, form: str, release: bool = False, init_C: int = 0,
                fast_needs_cover: bool = True):
    """Every interleaving of the CUDA path's atomic steps for threads with demands
    Ns (a demand N > 1 models a warp group), starting from C = init_C units.
    Growers take a batch from `pool` (Fig. 5's "resource");
    release=True adds each grant's signal(N, 0) (a free) after it.  Threads are
    sorted by (N, pc, w) in every state (symmetry reduction: threads with the
    same demand are interchangeable), so per-thread results are reported as the
    sorted tuple of (N, succeeded).  Returns states, terminal summaries
    ((C, D), batches used, results), deadlocks, and the number of reachable
    states where the word was NOT conservative w.r.t. the decided state (C above
    it, or C + D below it)."""
    assert form in FORMS
    first = {"alg1": G_CAS}.get(form, G_FAST)
    Ns = tuple(sorted(Ns))
    T = len(Ns)

    def canon(word, pl, pcs, ws):
        th = tuple(sorted(zip(Ns, pcs, ws), key=lambda x: (x[0], x[1], (-1 << 40,) if x[2] is None else x[2])))
        return (word, pl, tuple(x[1] for x in th), tuple(x[2] for x in th))

    start = canon((init_C, 0), pool, (first,) * T, (None,) * T)
    seen, terminals, stack = set(), set(), [start]
    deadlocks = nonconservative = overgrant = 0
    while stack:
        st = stack.pop()
        if st in seen:
            continue
        seen.add(st)
        (C, D), pl, pcs, ws = st
        pend = [_pending(form, pcs[t], Ns[t], _bprime(Ns[t], B)) for t in range(T)]
        dC = sum(p[0] for p in pend)
        dDC = sum(p[0] + p[1] for p in pend)
        if dC < 0 or dDC > 0:
            nonconservative += 1
        if C + dC < 0:                                       # the decided state granted units it did not have
            overgrant += 1
        succ = []

        def go(t, word, pc, w=None, pool_=pl):
            succ.append(canon(word, pool_, pcs[:t] + (pc,) + pcs[t + 1:], ws[:t] + (w,) + ws[t + 1:]))

        for t in range(T):
            N, pc, w = Ns[t], pcs[t], ws[t]
            Bp = _bprime(N, B)
            done = G_REL if release else G_OK
            if pc == G_CAS:                                   # Alg. 1 block 1 on w (alg1: on the word itself)
                cur = (C, D) if (form == "alg1" or w is None) else w
                if cur != (C, D):                             # CAS failed: it returns the current word
                    go(t, (C, D), G_CAS, (C, D))
                    continue
                if C + D < N:
                    go(t, (C, D + Bp - N), G_GROWING)
                elif C >= N:
                    go(t, (C - N, D), done)
                else:
                    go(t, (C, D - N), G_SPIN)
            elif pc == G_SPIN:                                # R-2: wait while C < N and C + D >= 0
                if not (C < N and C + D >= 0):
                    go(t, (C, D), G_RETRY)
            elif pc == G_RETRY:                               # R -= N, re-decide on the returned word
                go(t, (C, D + N), G_CAS, (C, D + N))
            elif pc == G_FAST:
                if form == "arena_old":
                    go(t, (C - N, D), done if C >= N else G_UNDO)
                elif form == "arena":
                    ok = C >= N and (C + D >= N or not fast_needs_cover)
                    go(t, (C - N, D + N), G_FIX if ok else G_UNDO)
                elif form == "tree_old":
                    go(t, (C - N, D), done if C >= N else (G_TGROW if C + D < N else G_TRES))
                else:                                         # fa
                    ok = C >= N and (C + D >= N or not fast_needs_cover)
                    go(t, (C - N, D + Bp), G_FIX if ok else (G_TGROW if C + D < N else G_TRES))
            elif pc == G_FIX:
                go(t, (C, D - (N if form == "arena" else Bp)), done)
            elif pc == G_UNDO:
                nw = (C + N, D - N) if form == "arena" else (C + N, D)
                go(t, nw, G_CAS, nw)
            elif pc == G_TGROW:
                go(t, (C + N, D - N) if form == "fa" else (C + N, D + Bp - N), G_GROWING)
            elif pc == G_TRES:
                go(t, (C + N, D - N - Bp) if form == "fa" else (C + N, D - N), G_TSPIN)
            elif pc == G_TSPIN:
                if not (C < N and C + D >= 0):
                    go(t, (C, D), G_TRETRY)
            elif pc == G_TRETRY:
                go(t, (C, D + N), G_FAST)
            elif pc == G_GROWING:
                k = Bp // B
                if pl >= k:
                    go(t, (C + Bp - N, D - (Bp - N)), done, None, pl - k)
                else:
                    go(t, (C, D - (Bp - N)), G_FAIL)
            elif pc == G_REL:
                go(t, (C + N, D), G_OK)
        if not succ:
            if all(pc in (G_OK, G_FAIL) for pc in pcs):
                terminals.add(((C, D), pool - pl, tuple(sorted(zip(Ns, (pc == G_OK for pc in pcs))))))
            else:
                deadlocks += 1
        stack.extend(succ)
    return {"states": len(seen), "terminals": terminals, "deadlocks": deadlocks,
            "nonconservative": nonconservative, "overgrant": overgrant}
