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


def _engine(swp, orc, seed, gib):
    specs = W.scaled(W.config_b(), int(gib * (1 << 30)))
    offs, total = W.place(specs)
    arena = swp.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=seed)
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    sw = swp.Swapper(regions, mechanism="ce_pipe", pipe_mib=128)
    sw.bind_arena(arena)
    return specs, offs, total, arena, view, sw, regions, base


def test_exchange_full_duplex(swp, orc):
    """Two victims out, one engine in, overlapped; the incoming maps HBM only as victims release it."""
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    ea = _engine(swp, orc, 1, 2.2)
    eb = _engine(swp, orc, 2, 1.5)
    ec = _engine(swp, orc, 3, 3.1)
    # C is parked: snapshot after init, HBM released
    c_specs, c_offs, c_total, c_arena, c_view, c_sw, c_regions, c_base = ec
    c_host = c_view.cpu().numpy()
    c_sw.swap_out(c_arena, s_in)
    # A and B run for a while: change some bytes, so their images must be re-gathered
    snaps = []
    for (specs, offs, total, arena, view, sw, regions, base) in (ea, eb):
        view[offs[3]:offs[3] + 999].fill_(0x42)
        torch.cuda.synchronize()
        snaps.append(view.cpu().numpy())
    headroom = 256 << 20
    peak = swp.exchange([ea[5], eb[5]], c_sw, s_out, s_in, headroom=headroom)
    assert peak <= headroom
    res = c_sw.verify(s_in)
    assert res["status"] == 0 and res["hbm_n_bad"] == 0 and c_arena.resident
    back = c_arena.tensor(0, c_total).cpu().numpy()
    for r, o in zip(c_specs, c_offs):
        assert np.array_equal(back[o:o + r.nbytes], c_host[o:o + r.nbytes])
    for (specs, offs, total, arena, view, sw, regions, base), host in zip((ea, eb), snaps):
        assert not arena.resident
        rc, ref, _ = orc.checkpoint([(i, a, n, k) for (a, n, k, i) in regions], host, base, 1, 1 << 20, 4096,
                                    threads=8)
        assert np.array_equal(sw.image(), ref)
        # and the victim comes back intact later
        res = sw.swap_in(arena, s_in)
        assert res["status"] == 0
        back = arena.tensor(0, total).cpu().numpy()
        for r, o in zip(specs, offs):
            assert np.array_equal(back[o:o + r.nbytes], host[o:o + r.nbytes])
    for e in (ea, eb, ec):
        e[5].close()
        e[3].close()
