"""NEXT-3 "move only touched KV blocks": per-chunk keep masks on SAVE regions (swap_set_chunk_mask,
DESIGN.md reading 25), bit-exact against the oracle's definition of the captured bytes
(oracle.policy_view with masks) through checkpoint -> restore -> verify sequences in which chunks
move between kept and masked (the image's stale bytes must be zeroed)."""
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


def _masks(rng, specs, C, frac):
    return {i: (rng.random(-(-r.nbytes // C)) < frac).astype(np.uint8)
            for i, r in enumerate(specs) if r.kind == W.KIND_KV and r.nbytes}


@pytest.mark.parametrize("mech", ["sm", "ce_pipe", "ce_region", "ce_chunk", "ce_batch"])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_masks_change_between_checkpoints(swp, orc, mech, kind):
    specs = W.scaled(W.config_b(), 48 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 41)
    pol = [orc.SAVE_ONCE if r.kind == W.KIND_WEIGHTS else orc.SAVE for r in specs]
    C = 1 << 16
    rng = np.random.default_rng(9)
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=mech, pipe_mib=4) as sw, \
            torch.cuda.stream(s):
        for i, p in enumerate(pol):
            sw.set_region_policy(i, p)
        first = host.copy()
        now = host
        masks = None
        for step, frac in enumerate([0.3, 0.6, None, 0.0, 0.5]):
            if step:  # the engine runs: KV and workspace change (weights must not, SAVE_ONCE)
                now = now.copy()
                for r, o in zip(specs, offs):
                    if r.nbytes and r.kind != W.KIND_WEIGHTS and rng.random() < 0.6:
                        lo = o + int(rng.integers(0, r.nbytes))
                        now[lo:lo + 4099] ^= 0x5C
                arena.copy_(torch.from_numpy(now).cuda())
            masks = _masks(rng, specs, C, frac) if frac is not None else None
            for i, r in enumerate(specs):
                if r.kind == W.KIND_KV and r.nbytes:
                    sw.set_chunk_mask(i, masks[i] if masks else None)
            sw.checkpoint(s)
            want = orc.policy_view(or_regions, pol, now, first, base, C, masks)
            rc, ref, _ = orc.checkpoint(or_regions, want, base, kind, C, 4096, threads=8)
            assert rc == 0
            assert np.array_equal(sw.image(), ref), f"step {step}: image differs from the oracle"
            poison(arena, specs, offs)
            sw.restore(s)
            res = sw.verify(s)
            assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0
            assert np.array_equal(arena.cpu().numpy(), want), f"step {step}: restored memory differs"
            now = want.copy()  # the engine resumes from what was restored


def test_mask_fault_in_kept_chunk(swp, orc):
    """A bit flip in a kept chunk's image bytes is reported as exactly that chunk."""
    specs = W.scaled(W.config_b(), 24 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 43)
    C = 1 << 16
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, mechanism="ce_pipe", pipe_mib=2) as sw, torch.cuda.stream(s):
        kv = next(i for i, r in enumerate(specs) if r.kind == W.KIND_KV and r.nbytes > 4 * C)
        n = -(-specs[kv].nbytes // C)
        keep = np.zeros(n, np.uint8)
        keep[1::3] = 1
        sw.set_chunk_mask(kv, keep)
        sw.checkpoint(s)
        img = sw.image()
        man = sw.manifest()
        reg_off = int(np.frombuffer(man[64 + 48 * kv + 24:64 + 48 * kv + 32].tobytes(), "<u8")[0])
        first = int(np.frombuffer(man[64 + 48 * kv + 32:64 + 48 * kv + 40].tobytes(), "<u8")[0])
        img[reg_off + 4 * C + 77] ^= 0x10  # chunk 4 of the region: kept (4 % 3 == 1)
        poison(arena, specs, offs)
        sw.restore(s)
        res = sw.verify(s, raise_on_corrupt=False)
        assert res["n_bad"] == 1 and res["first_bad_chunk"] == first + 4
        assert res["hbm_n_bad"] == 1 and res["hbm_first_bad"] == first + 4


def test_mask_through_released_arena(swp, orc):
    """Bound VMM arena released between swap-out and swap-in: masked chunks are re-mapped and zeroed,
    kept chunks restored group by group (CE_PIPE), everything verified."""
    specs = W.scaled(W.config_b(), 3 << 30)
    offs, total = W.place(specs)
    arena = swp.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=6)
    host = view.cpu().numpy()
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    or_regions = [(i, a, n, k) for (a, n, k, i) in regions]
    C = 1 << 20
    rng = np.random.default_rng(2)
    s = torch.cuda.Stream()
    with swp.Swapper(regions, chunk_bytes=C, mechanism="ce_pipe", pipe_mib=64) as sw, torch.cuda.stream(s):
        sw.bind_arena(arena)
        for frac in (0.25, 0.75):
            masks = _masks(rng, specs, C, frac)
            for i, m in masks.items():
                sw.set_chunk_mask(i, m)
            cur = arena.tensor(0, total).cpu().numpy()
            sw.swap_out(arena, s)
            assert not arena.resident
            res = sw.swap_in(arena, s)
            assert res["status"] == 0 and res["hbm_n_bad"] == 0 and arena.resident
            want = orc.policy_view(or_regions, [orc.SAVE] * len(regions), cur, cur, base, C, masks)
            back = arena.tensor(0, total).cpu().numpy()
            for r, o in zip(specs, offs):
                assert np.array_equal(back[o:o + r.nbytes], want[o:o + r.nbytes]), r.name
        sw.bind_arena(None)
    arena.close()
    del host


def test_mask_import_restores_whole_image(swp, orc):
    """After swap_import the restore moves the whole imported image; the pending mask is re-applied
    (with the image's masked chunks zeroed) at the next checkpoint."""
    specs = W.scaled(W.config_b(), 16 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 44)
    C = 1 << 15
    rng = np.random.default_rng(4)
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, mechanism="sm") as sw, torch.cuda.stream(s):
        rc, full, _ = orc.checkpoint(or_regions, host, base, 1, C, 4096, threads=8)
        masks = _masks(rng, specs, C, 0.4)
        for i, m in masks.items():
            sw.set_chunk_mask(i, m)
        sw.checkpoint(s)
        img = sw.image()
        img[:] = full  # an unmasked image from elsewhere
        sw.import_image()
        poison(arena, specs, offs)
        sw.restore(s)
        assert sw.verify(s)["status"] == 0
        assert np.array_equal(arena.cpu().numpy(), host)
        sw.checkpoint(s)
        want = orc.policy_view(or_regions, [orc.SAVE] * len(specs), host, host, base, C, masks)
        rc, ref, _ = orc.checkpoint(or_regions, want, base, 1, C, 4096, threads=8)
        assert np.array_equal(sw.image(), ref)


def test_mask_validation(swp, orc):
    specs = W.scaled(W.config_b(), 8 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 45)
    C = 1 << 16
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, mechanism="sm") as sw, torch.cuda.stream(s):
        kv = next(i for i, r in enumerate(specs) if r.kind == W.KIND_KV and r.nbytes)
        w = next(i for i, r in enumerate(specs) if r.kind == W.KIND_WEIGHTS and r.nbytes)
        n = -(-specs[kv].nbytes // C)
        with pytest.raises(swp.SwapError) as e:
            sw.set_chunk_mask(kv, np.ones(n + 1, np.uint8))
        assert e.value.status == swp.SWAP_EINVAL
        sw.set_region_policy(w, "save_once")
        with pytest.raises(swp.SwapError) as e:
            sw.set_chunk_mask(w, np.ones(-(-specs[w].nbytes // C), np.uint8))
        assert e.value.status == swp.SWAP_EINVAL
        sw.checkpoint(s, sync=False)
        with pytest.raises(swp.SwapError) as e:
            sw.set_chunk_mask(kv, np.zeros(n, np.uint8))
        assert e.value.status == swp.SWAP_ESTATE
        sw.sync(s)
        sw.set_chunk_mask(kv, np.zeros(n, np.uint8))


def _masked_engine(swp, seed, gib, rng, frac):
    specs = W.scaled(W.config_b(), int(gib * (1 << 30)))
    offs, total = W.place(specs)
    arena = swp.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=seed)
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    sw = swp.Swapper(regions, mechanism="ce_pipe", pipe_mib=128)
    sw.bind_arena(arena)
    masks = _masks(rng, specs, 1 << 20, frac)
    for i, m in masks.items():
        sw.set_chunk_mask(i, m)
    return dict(specs=specs, offs=offs, total=total, arena=arena, view=view, sw=sw, base=base, masks=masks,
                or_regions=[(i, a, n, k) for (a, n, k, i) in regions])


def test_mask_exchange_full_duplex(swp, orc):
    """swap_exchange with a masked victim (gathered under its new mask) and a masked incoming engine
    (only its kept chunks moved, the rest zero-filled), both bit-exact against the oracle."""
    rng = np.random.default_rng(12)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    inc = _masked_engine(swp, 21, 1.4, rng, 0.3)
    vic = _masked_engine(swp, 22, 2.2, rng, 0.5)
    inc_host = inc["view"].cpu().numpy()
    inc["sw"].swap_out(inc["arena"], s_in)
    vic["view"][vic["offs"][2]:vic["offs"][2] + 4321].fill_(0x17)
    torch.cuda.synchronize()
    vic_host = vic["view"].cpu().numpy()
    peak = swp.exchange([vic["sw"]], inc["sw"], s_out, s_in, headroom=256 << 20)
    assert peak <= 256 << 20
    res = inc["sw"].verify(s_in)
    assert res["status"] == 0 and res["hbm_n_bad"] == 0
    pol = [orc.SAVE] * len(inc["specs"])
    want = orc.policy_view(inc["or_regions"], pol, inc_host, inc_host, inc["base"], 1 << 20, inc["masks"])
    back = inc["arena"].tensor(0, inc["total"]).cpu().numpy()
    for r, o in zip(inc["specs"], inc["offs"]):
        assert np.array_equal(back[o:o + r.nbytes], want[o:o + r.nbytes]), r.name
    vwant = orc.policy_view(vic["or_regions"], [orc.SAVE] * len(vic["specs"]), vic_host, vic_host, vic["base"],
                            1 << 20, vic["masks"])
    rc, ref, _ = orc.checkpoint(vic["or_regions"], vwant, vic["base"], 1, 1 << 20, 4096, threads=8)
    assert np.array_equal(vic["sw"].image(), ref)
    for e in (inc, vic):
        e["sw"].close()
        e["arena"].close()
