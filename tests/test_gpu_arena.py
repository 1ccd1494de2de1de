"""Releasable HBM (NEXT-1): the VMM arena frees physical memory on swap-out and maps fresh memory
at the same virtual addresses on swap-in; a swap round trip through it is bit-exact vs the oracle."""
import numpy as np
import pytest

import workloads as W

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GiB = 1 << 30


@pytest.fixture(scope="module")
def swp():
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


def test_release_returns_hbm(swp):
    torch.cuda.synchronize()
    a = swp.Arena(4 * GiB + 12345)
    assert a.nbytes >= 4 * GiB + 12345 and a.resident
    free0, _ = torch.cuda.mem_get_info()
    a.release()
    free1, _ = torch.cuda.mem_get_info()
    assert not a.resident
    assert free1 - free0 >= 4 * GiB  # the physical memory went back to the device
    with pytest.raises(swp.SwapError) as e:
        a.release()
    assert e.value.status == swp.SWAP_ESTATE
    base = a.base
    a.reacquire()
    free2, _ = torch.cuda.mem_get_info()
    assert free1 - free2 >= 4 * GiB and a.base == base and a.resident
    t = a.tensor(0, 1 << 20)
    t.fill_(3)
    assert int(t.sum()) == 3 << 20
    a.close()


@pytest.mark.parametrize("mech", ["sm", "ce_pipe"])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_swap_out_in_through_arena(swp, orc, mech, kind):
    specs = W.config_a(1)
    host, offs = W.host_arena(specs, 1)
    arena = swp.Arena(host.size)
    base, view = arena.alloc(host.size)
    view.copy_(torch.from_numpy(host).cuda())
    regions = [(base + o, r.nbytes, r.kind, 100 + i) for i, (r, o) in enumerate(zip(specs, offs))]
    rc, ref, moff = orc.checkpoint([(i, a, n, k) for (a, n, k, i) in regions], host, base, kind, 1 << 16, 4096,
                                   threads=8)
    s = torch.cuda.Stream()
    with swp.Swapper(regions, chunk_bytes=1 << 16, checksum=kind, mechanism=mech, pipe_mib=16) as sw, \
            torch.cuda.stream(s):
        for _ in range(2):
            sw.swap_out(arena, s)
            assert np.array_equal(sw.image(), ref)
            assert not arena.resident
            junk = torch.full((host.size,), 0x77, dtype=torch.uint8, device="cuda")  # reuse the freed HBM
            del junk
            res = sw.swap_in(arena, s)
            assert res["status"] == 0 and res["hbm_n_bad"] == 0
            back = arena.tensor(0, host.size).cpu().numpy()
            # regions restored bit-exactly; guard gaps are not part of the image (undefined after re-map)
            for r, o in zip(specs, offs):
                assert np.array_equal(back[o:o + r.nbytes], host[o:o + r.nbytes])
    arena.close()


@pytest.mark.parametrize("mech", ["ce_pipe", "sm", "ce_region"])
def test_bound_arena_lazy_reacquire(swp, orc, mech):
    """With the arena bound to the ctx, restore re-acquires the HBM itself (CE_PIPE: group by group,
    overlapped with the copies); regions come back bit-exact, DISCARD regions as zeros."""
    specs = W.scaled(W.config_b(), 3 << 30)  # > 2 slabs of 1 GiB, several pipeline groups
    offs, total = W.place(specs)
    arena = swp.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=4)
    host = view.cpu().numpy()
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    s = torch.cuda.Stream()
    with swp.Swapper(regions, mechanism=mech, pipe_mib=64) as sw, torch.cuda.stream(s):
        kv = [i for i, r in enumerate(specs) if r.kind == W.KIND_KV]
        for i in kv:
            sw.set_region_policy(i, "discard")
        sw.bind_arena(arena)
        for _ in range(2):
            sw.swap_out(arena, s)
            assert not arena.resident
            res = sw.swap_in(arena, s)
            assert res["status"] == 0 and res["hbm_n_bad"] == 0
            assert arena.resident
            back = arena.tensor(0, total).cpu().numpy()
            for i, (r, o) in enumerate(zip(specs, offs)):
                want = np.zeros(r.nbytes, np.uint8) if i in kv else host[o:o + r.nbytes]
                assert np.array_equal(back[o:o + r.nbytes], want), (i, r.name)
        sw.bind_arena(None)
    arena.close()
