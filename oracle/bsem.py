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
