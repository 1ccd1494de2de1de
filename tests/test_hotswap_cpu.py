"""Hot-swap controller host logic (paper §3.3-3.5 workflow) on CPU: the native scheduler decides, fake
shards record the data-path calls. Checks the config E topology (8B on GPU 0, 14B on GPU 1, 32B on both)
in sequential mode (victims out, then the engine in) and in full-duplex mode (one swap_exchange per GPU
with the GPU's free budget as headroom)."""
import pytest

GB = 10 ** 9


class FakeArena:
    def __init__(self, nbytes):
        self.nbytes = nbytes
        self.resident = False


class FakeSwapper:
    def __init__(self, name, log):
        self.name, self.log = name, log

    def swap_out(self, arena, stream=None):
        self.log.append(("out", self.name))
        arena.resident = False

    def swap_in(self, arena, stream=None, hbm_pass=True):
        self.log.append(("in", self.name))
        arena.resident = True
        return {"status": 0}

    def verify(self, stream=None, hbm_pass=True):
        self.log.append(("verify", self.name))
        return {"status": 0}


def build(log, duplex=False):
    from paper_conf_sc_stoyanovsracb25_b200 import hotswap as hs

    layout = [("8b", [(0, 27)]), ("14b", [(1, 45)]), ("32b", [(0, 44), (1, 44)])]
    engines = []
    for bid, (name, shards) in enumerate(layout):
        e = hs.Engine(bid, name)
        for rank, (g, gb) in enumerate(shards):
            e.shards.append(hs.Shard(g, FakeArena(gb * GB), FakeSwapper(f"{name}.r{rank}", log), gb * GB))
        engines.append(e)
    return hs, hs.HotSwapController(engines, [60 * GB, 60 * GB], duplex=duplex)


def test_sequential_workflow():
    log = []
    hs, ctl = build(log)
    assert ctl.ensure_resident(0, 0.0)[:2] == (False, [])   # 8B in, nothing to evict
    assert ctl.ensure_resident(1, 1.0)[:2] == (False, [])   # 14B co-resides (other GPU)
    assert ctl.ensure_resident(0, 2.0)[0] is True           # hit
    ctl.touch(0, 0, 5.0)                                     # 8B used more recently than 14B
    ctl.touch(1, 0, 3.0)
    hit, victims, _, _ = ctl.ensure_resident(2, 6.0)         # 32B needs both GPUs
    assert not hit and sorted(victims) == [0, 1]
    assert victims == [1, 0]                                 # equal queues -> oldest access first
    assert [x for x in log if x[0] == "out"] == [("out", "14b.r0"), ("out", "8b.r0")]
    assert log[-2:] == [("in", "32b.r0"), ("in", "32b.r1")]
    ctl.close()


def test_duplex_exchange_per_gpu(monkeypatch):
    log, calls = [], []
    hs, ctl = build(log, duplex=True)

    def fake_exchange(victims, incoming, s_out=None, s_in=None, headroom=0):
        calls.append(([v.name for v in victims], incoming.name if incoming else None, headroom))
        return 0

    monkeypatch.setattr(hs, "exchange", fake_exchange)
    ctl.ensure_resident(0, 0.0)  # 8B: GPU 0 only, nothing to evict
    ctl.ensure_resident(1, 1.0)  # 14B: GPU 1 only
    assert calls == [([], "8b.r0", 60 * GB), ([], "14b.r0", 60 * GB)]
    calls.clear()
    hit, victims, t_out, t_in = ctl.ensure_resident(2, 2.0)
    assert not hit and sorted(victims) == [0, 1] and t_out == 0.0
    # one exchange per GPU: the victims' shards on that GPU out, the 32B shard of that GPU in,
    # headroom = the GPU's free budget before the grant
    assert calls == [(["8b.r0"], "32b.r0", (60 - 27) * GB), (["14b.r0"], "32b.r1", (60 - 45) * GB)]
    assert ("verify", "32b.r0") in log and ("verify", "32b.r1") in log
    # then the 8B again: the 32B goes out on both GPUs, the 8B comes in on GPU 0 only
    calls.clear()
    ctl.ensure_resident(0, 3.0)
    assert calls == [(["32b.r0"], "8b.r0", (60 - 44) * GB), (["32b.r1"], None, (60 - 44) * GB)]
    ctl.close()
