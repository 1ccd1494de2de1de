"""NEXT-2 NVLink-assisted restore, degenerate one-GPU form: helper "peers" equal to the target device,
so every helper group goes host -> HBM staging -> regions, either pulled by the target's SM mover with the
fused check (default) or by peer copies + the HBM hash check (SWAP_ASSIST=copy). The striping, staging
offsets, cross-stream ordering and checks must give a bit-exact restore."""
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


@pytest.mark.parametrize("mode", ["fused", "copy"])
@pytest.mark.parametrize("n_helpers", [1, 2])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_assisted_restore_bit_exact(swp, orc, n_helpers, kind, mode, monkeypatch):
    if mode == "copy":
        monkeypatch.setenv("SWAP_ASSIST", "copy")
    else:
        monkeypatch.delenv("SWAP_ASSIST", raising=False)
    specs = W.scaled(W.config_b(), 160 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 41)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, 1 << 20, 4096, threads=8)
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, checksum=kind, mechanism="ce_pipe", pipe_mib=16) as sw, torch.cuda.stream(s):
        sw.set_helpers([0] * n_helpers)
        sw.checkpoint(s)
        assert np.array_equal(sw.image(), ref)
        for _ in range(2):
            poison(arena, specs, offs)
            sw.restore(s)
            res = sw.verify(s)
            assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0
            assert np.array_equal(arena.cpu().numpy(), host)
        # a corrupted image byte is still caught on a helper-moved group
        img = sw.image()
        img[len(img) // 3] ^= 0x01
        sw.restore(s)
        res = sw.verify(s, raise_on_corrupt=False)
        assert res["n_bad"] == 1 or (res["n_bad"] == 0 and img.size // 3 >= moff)
        img[len(img) // 3] ^= 0x01
        sw.set_helpers([])


def test_assisted_restore_with_bound_arena_and_policies(swp, orc):
    specs = W.scaled(W.config_b(), 2300 << 20)  # > 2 slabs: lazy mapping under helper groups
    offs, total = W.place(specs)
    arena = swp.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=8)
    host = view.cpu().numpy()
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    s = torch.cuda.Stream()
    kv = [i for i, r in enumerate(specs) if r.kind == W.KIND_KV]
    with swp.Swapper(regions, mechanism="ce_pipe", pipe_mib=64) as sw, torch.cuda.stream(s):
        sw.set_helpers([0, 0, 0])
        for i in kv:
            sw.set_region_policy(i, "discard")  # re-sizes the helpers' staging
        sw.bind_arena(arena)
        sw.swap_out(arena, s)
        res = sw.swap_in(arena, s)
        assert res["status"] == 0 and res["hbm_n_bad"] == 0
        back = arena.tensor(0, total).cpu().numpy()
        for i, (r, o) in enumerate(zip(specs, offs)):
            want = np.zeros(r.nbytes, np.uint8) if i in kv else host[o:o + r.nbytes]
            assert np.array_equal(back[o:o + r.nbytes], want)
        sw.bind_arena(None)
    arena.close()


def test_helpers_with_mask_and_import(swp, orc):
    """a chunk mask shrinks the restore groups (the helpers' staging is re-sized at the
    checkpoint); swap_import then rebuilds full groups, larger than that staging -- it must re-size the
    helpers again, and the CE_PIPE restore through the helpers stays bit-exact."""
    C = 1 << 20
    specs = W.scaled(W.config_b(), 300 << 20)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 17)
    big = max(range(len(specs)), key=lambda i: specs[i].nbytes)
    n = -(-specs[big].nbytes // C)
    keep = (np.arange(n) % 8 == 0).astype(np.uint8)
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, mechanism="ce_pipe", pipe_mib=16) as sw, torch.cuda.stream(s):
        sw.set_helpers([0])
        sw.set_chunk_mask(big, keep)
        sw.checkpoint(s)  # masked groups; helpers re-sized for them
        want = orc.policy_view(or_regions, [orc.SAVE] * len(specs), host, host, base, C, {big: keep})
        rc, ref, moff = orc.checkpoint(or_regions, want, base, 1, C, 4096, threads=8)
        assert np.array_equal(sw.image(), ref)
        sw.import_image()  # the image "came from elsewhere": full groups again
        poison(arena, specs, offs)
        sw.restore(s)
        res = sw.verify(s)
        assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0
        back = arena.cpu().numpy()
        for r, o in zip(specs, offs):
            assert np.array_equal(back[o:o + r.nbytes], want[o:o + r.nbytes]), r.name
        sw.set_helpers([])
