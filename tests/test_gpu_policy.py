"""NEXT-3 engine-aware state reduction: per-region SAVE / SAVE_ONCE / DISCARD policies, bit-exact
against the oracle's definition of the captured bytes (oracle.policy_view)."""
import numpy as np
import pytest

import workloads as W
from gpu_util import device_case, poison

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def swp():
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


@pytest.mark.parametrize("mech", ["sm", "ce_pipe", "ce_region"])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_policies_weights_once_kv_discard(swp, orc, mech, kind):
    specs = W.scaled(W.config_b(), 48 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 31)
    pol = [orc.SAVE_ONCE if r.kind == W.KIND_WEIGHTS else orc.DISCARD if r.kind == W.KIND_KV else orc.SAVE
           for r in specs]
    C = 1 << 16
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=mech, pipe_mib=4) as sw, \
            torch.cuda.stream(s):
        for i, p in enumerate(pol):
            sw.set_region_policy(i, p)
        first = host.copy()
        sw.checkpoint(s)
        rc, ref1, moff = orc.checkpoint(or_regions, orc.policy_view(or_regions, pol, host, first, base), base, kind,
                                        C, 4096, threads=8)
        assert np.array_equal(sw.image(), ref1)
        with pytest.raises(swp.SwapError) as e:
            sw.set_region_policy(0, "save")
        assert e.value.status == swp.SWAP_ESTATE
        # the engine runs: weights are (wrongly) touched, workspace and KV change
        now = host.copy()
        rng = np.random.default_rng(3)
        for r, o in zip(specs, offs):
            if r.nbytes and r.kind in (W.KIND_WEIGHTS, W.KIND_WORKSPACE, W.KIND_KV) and rng.random() < 0.5:
                now[o:o + min(r.nbytes, 777)] ^= 0x3C
        arena.copy_(torch.from_numpy(now).cuda())
        sw.checkpoint(s)
        rc, ref2, _ = orc.checkpoint(or_regions, orc.policy_view(or_regions, pol, now, first, base), base, kind, C,
                                     4096, threads=8)
        assert np.array_equal(sw.image(), ref2)
        poison(arena, specs, offs)
        sw.restore(s)
        res = sw.verify(s)
        assert res["status"] == 0 and res["hbm_n_bad"] == 0
        want = orc.policy_view(or_regions, pol, now, first, base)  # weights as first saved, KV zeroed
        assert np.array_equal(arena.cpu().numpy(), want)
