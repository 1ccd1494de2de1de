"""Task manager / demand-aware preemption (NEXT-1): libswap's native scheduler vs the plain-Python
oracle (oracle/policy.py), both pinned to the paper's worked example and policy statements
(tests/golden/paper_reservation.txt: PAPER.md L142, L146, L148)."""
import random

import pytest

from conftest import read_golden
from oracle.policy import Backend, TaskManager

GB = 10 ** 9


def scenarios():
    out, cur = [], None
    for row in read_golden("paper_reservation.txt"):
        words = row[0].split()
        if words[0] == "scenario":
            cur = {"name": words[1], "steps": []}
            out.append(cur)
        else:
            cur["steps"].append(words)
    return out


def run_scenario(sc, make):
    """Replays a fixture scenario on an implementation; returns the list of (granted, victims)."""
    names, impl, grants = {}, None, []
    for w in sc["steps"]:
        if w[0] == "gpus":
            impl = make([int(x) * GB for x in w[1].split(",")])
        elif w[0] == "backend":
            bid = len(names)
            names[w[1]] = bid
            opts = dict(x.split("=") for x in w[3:] if "=" in x)
            impl.add(bid, [int(x) * GB for x in w[2].split(",")], "resident" in w[3:], int(opts.get("queue", 0)),
                     float(opts.get("last", 0)))
        elif w[0] == "reserve":
            impl.reserve(names[w[1]], float(w[2]))
        elif w[0] == "grant":
            inv = {v: k for k, v in names.items()}
            bid, victims = impl.grant()
            want_victims = [] if w[3] == "-" else w[3:]
            assert inv[bid] == w[1], sc["name"]
            assert [inv[v] for v in victims] == want_victims, sc["name"]
            grants.append((bid, victims))
    return grants


class OracleImpl:
    def __init__(self, caps):
        self.tm = TaskManager(caps)

    def add(self, bid, need, resident, queue, last):
        self.tm.backends[bid] = Backend(need, resident, False, queue, last)

    def reserve(self, bid, prio):
        self.tm.reserve(bid, prio)

    def grant(self):
        return self.tm.grant()


class NativeImpl:
    def __init__(self, caps):
        from paper_conf_sc_stoyanovsracb25_b200.swap import Scheduler

        self.s = Scheduler(caps)

    def add(self, bid, need, resident, queue, last):
        self.s.add_backend(bid, need, resident)
        self.s.touch(bid, queue, last)

    def reserve(self, bid, prio):
        self.s.reserve(bid, prio)

    def grant(self):
        return self.s.grant()


@pytest.mark.parametrize("sc", scenarios(), ids=lambda s: s["name"])
def test_paper_scenarios_oracle(sc):
    run_scenario(sc, OracleImpl)


@pytest.mark.parametrize("sc", scenarios(), ids=lambda s: s["name"])
def test_paper_scenarios_native(sc):
    run_scenario(sc, NativeImpl)


def test_oracle_invariants_random():
    """Properties that hold for any correct policy: capacity never exceeded after a grant, the
    eviction stops as soon as memory suffices (dropping the last victim is not enough), and each
    victim had the best (queue, last-access, id) key among the useful candidates at its step."""
    rng = random.Random(7)
    for _ in range(300):
        G = rng.randint(1, 3)
        caps = [rng.randint(50, 100) for _ in range(G)]
        tm = TaskManager(caps)
        for bid in range(rng.randint(2, 7)):
            need = [rng.choice([0, rng.randint(5, 60)]) for _ in range(G)]
            if not any(need):
                need[0] = rng.randint(5, 40)
            need = [min(n, c) for n, c in zip(need, caps)]
            tm.backends[bid] = Backend(need, False, False, rng.randint(0, 3), rng.random())
            if all(tm.free(g) >= need[g] for g in range(G)) and rng.random() < 0.7:
                tm.backends[bid].resident = True
        for bid, b in tm.backends.items():
            v = tm.plan(bid)
            if b.resident:
                assert v == []
                continue
            if v is None:
                continue
            free = [tm.free(g) for g in range(G)]
            for x in v:
                free = [f + n for f, n in zip(free, tm.backends[x].need)]
            assert all(free[g] >= b.need[g] for g in range(G))
            if v:
                freed_minus_last = [f - n for f, n in zip(free, tm.backends[v[-1]].need)]
                assert any(freed_minus_last[g] < b.need[g] for g in range(G))


def test_native_matches_oracle_random():
    from paper_conf_sc_stoyanovsracb25_b200.swap import Scheduler

    rng = random.Random(11)
    for trial in range(200):
        G = rng.randint(1, 4)
        caps = [rng.randint(40, 160) * GB for _ in range(G)]
        tm, s = TaskManager(caps), Scheduler(caps)
        n = rng.randint(2, 9)
        for bid in range(n):
            need = [rng.choice([0, rng.randint(1, 80) * GB]) for _ in range(G)]
            if not any(need):
                need[rng.randrange(G)] = rng.randint(1, 30) * GB
            need = [min(x, c) for x, c in zip(need, caps)]
            resident = all(tm.free(g) >= need[g] for g in range(G)) and rng.random() < 0.6
            q, last = rng.randint(0, 2), float(rng.randint(0, 5))  # many ties on purpose
            tm.backends[bid] = Backend(need, resident, False, q, last)
            s.add_backend(bid, need, resident)
            s.touch(bid, q, last)
        for bid in range(n):
            if rng.random() < 0.2:
                tm.backends[bid].locked = True
                s.lock(bid, True)
        # plans agree for every backend
        for bid in range(n):
            assert s.plan(bid) == tm.plan(bid), (trial, bid)
        # a random reserve/grant/release sequence keeps both in lockstep
        for step in range(12):
            op = rng.random()
            bid = rng.randrange(n)
            if op < 0.4 and not tm.backends[bid].resident and all(p[2] != bid for p in tm.pending):
                prio = float(rng.randint(0, 3))
                tm.reserve(bid, prio)
                s.reserve(bid, prio)
            elif op < 0.8:
                try:
                    o = tm.grant()
                except RuntimeError:
                    o = ("blocked", tm.pending[0][2])
                assert s.grant() == o, (trial, step)
            elif tm.backends[bid].resident:
                tm.backends[bid].resident = False
                s.release(bid)
            for g in range(G):
                assert s.free(g) == tm.free(g)
        s.close()


def test_native_errors():
    from paper_conf_sc_stoyanovsracb25_b200.swap import Scheduler, SwapError

    s = Scheduler([80 * GB])
    s.add_backend(1, [50 * GB], resident=True)
    with pytest.raises(SwapError):
        s.add_backend(1, [10 * GB])  # duplicate id
    with pytest.raises(SwapError):
        s.add_backend(2, [90 * GB])  # larger than the GPU
    with pytest.raises(SwapError):
        s.add_backend(3, [40 * GB], resident=True)  # does not fit next to backend 1
    s.add_backend(4, [70 * GB])
    with pytest.raises(SwapError):
        s.reserve(1, 0)  # already resident
    s.lock(1)
    assert s.plan(4) is None  # the only candidate is write-locked
    s.reserve(4, 0)
    assert s.grant() == ("blocked", 4)
    s.lock(1, False)
    assert s.grant() == (4, [1])
    assert s.state(4) == {"resident": True, "queued": False} and s.free(0) == 10 * GB
    assert s.grant() is None
