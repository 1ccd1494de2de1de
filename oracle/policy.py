"""Plain-Python oracle of the task manager's reservation + demand-aware preemption policy.

TEST INFRASTRUCTURE ONLY (same rules as the rest of oracle/): only tests/ may import it; it
shares no code with libswap's native scheduler (csrc/sched.cpp).

Follows PAPER.md step by step:
  * §3.3 (L136-138) / §3.4 (L142): swap-in requests become memory reservations kept in a priority
    queue; several can be granted at once when memory suffices; otherwise the request waits while
    backends are swapped out.
  * §3.5 (L146): candidates are the currently running backends, ranked by (1) shorter request queue,
    (2) oldest last-accessed time (LRU tie-breaker).
  * §3.5 (L148): victims are write-locked and evicted one at a time; after each eviction free memory
    is re-checked and the next best candidate is evicted only if still insufficient.
  * §6 (L230): each backend's GPU topology is fixed at init; reservations are per GPU and acquired /
    released together (scoped acquire-release).
Readings where the paper is silent (readings 20-23): a backend locked by an eviction in
progress is not a candidate; on several GPUs only backends occupying a GPU that is still short are
candidates; a final tie (equal queue and last-access) goes to the lower backend id; reservations are
served strictly in priority order (lower value first, then arrival order), a head that cannot be
satisfied even after evicting every candidate is reported infeasible and stays queued.
"""
from __future__ import annotations

from dataclasses import dataclass, field


@dataclass
class Backend:
    need: list  # bytes per GPU (0 = not placed on that GPU), fixed at init (§6)
    resident: bool = False
    locked: bool = False
    queue: int = 0  # request-queue length (§3.5 tier 1)
    last_access: float = 0.0  # §3.5 tier 2 (LRU)


@dataclass
class TaskManager:
    capacity: list  # bytes per GPU
    backends: dict = field(default_factory=dict)
    pending: list = field(default_factory=list)  # [(priority, seq, backend)]
    _seq: int = 0

    def used(self, g: int) -> int:
        return sum(b.need[g] for b in self.backends.values() if b.resident)

    def free(self, g: int) -> int:
        return self.capacity[g] - self.used(g)

    def plan(self, bid: int):
        """Victims in eviction order, [] if no eviction needed, None if infeasible."""
        req = self.backends[bid]
        if req.resident:
            return []
        free = [self.free(g) for g in range(len(self.capacity))]
        victims = []

        def short_gpus():
            return [g for g in range(len(self.capacity)) if req.need[g] > 0 and free[g] < req.need[g]]

        while short_gpus():
            short = short_gpus()
            cands = [i for i, b in self.backends.items()
                     if b.resident and not b.locked and i != bid and i not in victims
                     and any(b.need[g] > 0 for g in short)]
            if not cands:
                return None
            best = min(cands, key=lambda i: (self.backends[i].queue, self.backends[i].last_access, i))
            victims.append(best)
            for g in range(len(self.capacity)):
                free[g] += self.backends[best].need[g]
        return victims

    def reserve(self, bid: int, priority: float):
        self.pending.append((priority, self._seq, bid))
        self._seq += 1

    def grant(self):
        """Serve the highest-priority reservation: returns (backend, victims) or None if the
        queue is empty; raises RuntimeError if the head is infeasible."""
        if not self.pending:
            return None
        self.pending.sort()
        _, _, bid = self.pending[0]
        victims = self.plan(bid)
        if victims is None:
            raise RuntimeError("infeasible")
        self.pending.pop(0)
        for v in victims:
            self.backends[v].resident = False
        self.backends[bid].resident = True
        return bid, victims
