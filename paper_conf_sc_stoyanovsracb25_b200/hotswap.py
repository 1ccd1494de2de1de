"""Hot-swap controller: the paper's swap-in / preemption workflow on top of libswap (NEXT-1).

PAPER.md §3.3-3.5 and §6, one step each:
  (4)-(5) a request for a non-resident backend becomes a reservation   -> Scheduler.reserve
  (6)-(8) the task manager grants it, choosing victims by the demand-aware policy
          (shorter queue first, then LRU)                               -> Scheduler.grant (native)
          each victim is write-locked and swapped out: checkpoint its shard on every GPU of its
          topology, then release the HBM                               -> Swapper.swap_out + Arena.release
  (9)     swap-in: re-acquire HBM at the recorded addresses, restore, verify on every rank
                                                                        -> Arena.reacquire + Swapper.swap_in
An Engine is one backend: one (Arena, Swapper) per GPU of its fixed topology. All data
movement and verification run in libswap; this module only sequences the calls.
"""
from __future__ import annotations

import time
from dataclasses import dataclass, field

from .swap import Arena, Scheduler, Swapper, exchange


@dataclass
class Shard:
    gpu: int  # logical GPU index in the scheduler's topology
    arena: Arena
    swapper: Swapper
    payload: int


@dataclass
class Engine:
    bid: int
    name: str
    shards: list = field(default_factory=list)

    @property
    def need(self) -> dict:
        return {s.gpu: s.arena.nbytes for s in self.shards}

    @property
    def payload(self) -> int:
        return sum(s.payload for s in self.shards)


class HotSwapController:
    """Serves swap-in requests for a fixed set of engines under per-GPU memory budgets."""

    def __init__(self, engines: list, budget_per_gpu: list, stream=None, duplex: bool = False, stream_in=None):
        self.engines = {e.bid: e for e in engines}
        self.n_gpus = len(budget_per_gpu)
        self.sched = Scheduler(budget_per_gpu)
        self.stream = stream
        self.duplex = duplex  # overlap victims' swap-out with the swap-in (swap_exchange), per GPU
        self.stream_in = stream_in if stream_in is not None else stream
        self.log = []  # (op, engine, seconds, bytes)
        for e in engines:
            need = [0] * self.n_gpus
            for g, b in e.need.items():
                need[g] += b
            resident = all(s.arena.resident for s in e.shards)
            self.sched.add_backend(e.bid, need, resident)

    def touch(self, bid: int, queue_len: int, last_access: float):
        self.sched.touch(bid, queue_len, last_access)

    def resident(self, bid: int) -> bool:
        return self.sched.state(bid)["resident"]

    def swap_out(self, bid: int) -> float:
        e = self.engines[bid]
        self.sched.lock(bid, True)  # no new requests reach it during the swap-out
        t0 = time.perf_counter()
        for s in e.shards:
            s.swapper.swap_out(s.arena, self.stream)
        dt = time.perf_counter() - t0
        self.sched.lock(bid, False)
        self.log.append(("out", e.name, dt, e.payload))
        return dt

    def swap_in(self, bid: int) -> float:
        e = self.engines[bid]
        t0 = time.perf_counter()
        for s in e.shards:
            res = s.swapper.swap_in(s.arena, self.stream, hbm_pass=True)
            if res["status"] != 0:
                raise RuntimeError(f"swap-in of {e.name} failed verification: {res}")
        dt = time.perf_counter() - t0
        self.log.append(("in", e.name, dt, e.payload))
        return dt

    def exchange(self, bid: int, victims: list, free_before: list) -> float:
        """Victims out and `bid` in, overlapped per GPU on the duplex link (swap_exchange). Each GPU's
        exchange may use that GPU's free budget before the grant as headroom."""
        e = self.engines[bid]
        t0 = time.perf_counter()
        for g in range(self.n_gpus):
            vs = [s.swapper for v in victims for s in self.engines[v].shards if s.gpu == g]
            ins = [s for s in e.shards if s.gpu == g]
            if not vs and not ins:
                continue
            for v in victims:
                self.sched.lock(v, True)
            exchange(vs, ins[0].swapper if ins else None, self.stream, self.stream_in, headroom=free_before[g])
            for v in victims:
                self.sched.lock(v, False)
            for s in ins:
                res = s.swapper.verify(self.stream_in, hbm_pass=True)
                if res["status"] != 0:
                    raise RuntimeError(f"swap-in of {e.name} failed verification: {res}")
        dt = time.perf_counter() - t0
        self.log.append(("exchange", e.name, dt, e.payload + sum(self.engines[v].payload for v in victims)))
        return dt

    def ensure_resident(self, bid: int, priority: float):
        """Steps (4)-(9) for one request. Returns (hit, victims, t_out, t_in) in seconds; with duplex
        exchanges t_out is 0 and t_in is the whole overlapped exchange."""
        if self.resident(bid):
            return True, [], 0.0, 0.0
        free_before = [self.sched.free(g) for g in range(self.n_gpus)]
        self.sched.reserve(bid, priority)
        g = self.sched.grant()
        if g is None or g[0] == "blocked" or g[0] != bid:
            self.sched.cancel(bid)
            raise RuntimeError(f"reservation for engine {bid} could not be granted: {g}")
        _, victims = g
        if self.duplex:
            return False, victims, 0.0, self.exchange(bid, victims, free_before)
        t_out = sum(self.swap_out(v) for v in victims)
        t_in = self.swap_in(bid)
        return False, victims, t_out, t_in

    def close(self):
        self.sched.close()
