"""GPU parity: libswap's CUDA path vs the CPU oracle, bit-exact (SURVEY.md §4 parity row).

Every case goes through the C ABI (Swapper -> ctypes -> libswap.so). Compared element by
element with oracle/: the whole host image (payload, zero padding, manifest bytes including
every chunk checksum and the manifest CRC), the restored device arena (regions and the 0xA5
guard bands between them), and the verify counters.
"""
import numpy as np
import pytest

import workloads as W
from gpu_util import chunk_records, device_case, poison

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MECHS = ["sm", "ce_region", "ce_chunk", "ce_batch", "ce_pipe", "auto"]
U64_MAX = (1 << 64) - 1


@pytest.fixture(scope="module")
def swp():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


@pytest.fixture(scope="module")
def stream():
    return torch.cuda.Stream()


_oracle_cache = {}


def oracle_image(orc, key, or_regions, host, base, kind, C):
    if key not in _oracle_cache:
        rc, img, moff = orc.checkpoint(or_regions, host, base, kind, C, 4096, threads=8)
        assert rc == 0
        _oracle_cache.clear()
        _oracle_cache[key] = (img, moff)
    return _oracle_cache[key]


def roundtrip(swp, orc, stream, specs, seed, C, kind, mech, key=None, **kw):
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, seed)
    img_ref, moff = oracle_image(orc, (key or (id(specs), seed, C, kind)) + (base,), or_regions, host, base, kind, C)
    sw = swp.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=mech, **kw)
    try:
        with torch.cuda.stream(stream):
            sw.checkpoint(stream)
            img = sw.image()
            assert img.size == img_ref.size
            if mech == "sm_nocheck":
                payload = moff
                assert np.array_equal(img[:payload], img_ref[:payload])
            else:
                diff = np.flatnonzero(img != img_ref)
                assert diff.size == 0, f"image differs at {diff[:8]} (manifest starts at {moff})"
                assert orc.manifest_ok(sw.manifest())
            poison(arena, specs, offs)
            sw.restore(stream)
            # NOCHECK leaves c_g = 0 in the manifest, so only the data path can be compared
            res = sw.verify(stream, hbm_pass=(mech != "sm_nocheck"))
        torch.cuda.synchronize()
        assert res["status"] == 0
        assert (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"], res["manifest_ok"]) == (0, U64_MAX, 0, 1)
        back = arena.cpu().numpy()
        diff = np.flatnonzero(back != host)
        assert diff.size == 0, f"restored arena differs at {diff[:8]}"
        return sw.launch_count()
    finally:
        sw.close()


@pytest.mark.parametrize("mech", MECHS)
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
@pytest.mark.parametrize("C", [4096, 65536, 1 << 20, 16 << 20], ids=["4K", "64K", "1M", "16M"])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_config_a_bit_exact(swp, orc, stream, seed, C, kind, mech):
    specs = W.config_a(seed)
    n = roundtrip(swp, orc, stream, specs, seed, C, kind, mech, key=("A", seed, C, kind))
    assert n >= 2  # our kernels ran (hash/mover + HBM verify)


@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
@pytest.mark.parametrize("seed", range(3, 10))
def test_config_a_more_seeds(swp, orc, stream, seed, kind):
    roundtrip(swp, orc, stream, W.config_a(seed), seed, 1 << 20, kind, "sm", key=("A", seed, 1 << 20, kind))


def test_config_a_nocheck_payload(swp, orc, stream):
    roundtrip(swp, orc, stream, W.config_a(0), 0, 1 << 20, 1, "sm_nocheck", key=("A", 0, 1 << 20, 1))


@pytest.mark.parametrize("grid", [1, 3, 148])
@pytest.mark.parametrize("seg", [4096, 1 << 20])
def test_launch_shapes(swp, orc, stream, grid, seg):
    """Odd grids (rounds with partial descriptor batches) and segment splits of a chunk."""
    specs = W.config_a(4)
    roundtrip(swp, orc, stream, specs, 4, 1 << 20, 1, "sm", key=("A", 4, 1 << 20, 1), grid_ctas=grid, seg_bytes=seg)


@pytest.mark.parametrize("mech", ["ce_region", "ce_pipe"])
def test_xxh64_hash_kernels_many_and_few_chunks(swp, orc, stream, mech):
    """XXH64 HBM passes: 1 KiB chunks (65 K chunks -> lane-per-chunk kernel) and 16 MiB chunks
    (5 chunks -> TMA-ring kernel)."""
    for C in (1024, 16 << 20):
        roundtrip(swp, orc, stream, W.config_a(6), 6, C, 2, mech, key=("A", 6, C, 2))


@pytest.mark.parametrize("pipe_mib", [1, 3, 16])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_ce_pipe_groups(swp, orc, stream, pipe_mib, kind):
    """CE_PIPE with many groups: group boundaries cut regions; hash launches see descriptor offsets."""
    roundtrip(swp, orc, stream, W.config_a(2), 2, 1 << 16, kind, "ce_pipe", key=("A", 2, 1 << 16, kind),
              pipe_mib=pipe_mib, seg_bytes=16384)


@pytest.mark.parametrize("name", list(W.edge_tables(4096)))
@pytest.mark.parametrize("C", [16, 64, 4096])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_edge_tables(swp, orc, stream, name, C, kind):
    specs = W.edge_tables(C)[name]
    if sum(r.nbytes for r in specs) == 0:
        pytest.skip("nothing to move (covered by test_all_empty)")
    roundtrip(swp, orc, stream, specs, 11, C, kind, "sm", key=(name, C, kind))


def test_all_empty(swp, orc, stream):
    specs = W.edge_tables(64)["all_empty"]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 0)
    rc, img_ref, moff = orc.checkpoint(or_regions, host, base, 1, 64, 4096)
    with swp.Swapper(sw_regions, chunk_bytes=64) as sw:
        sw.checkpoint(stream)
        assert np.array_equal(sw.image(), img_ref)
        sw.restore(stream)
        assert sw.verify(stream)["status"] == 0


def test_scaled_engine_images(swp, orc, stream):
    """Config B's region mix (weights bf16 N(0,0.02), KV, workspace) scaled to 96 MiB."""
    specs = W.scaled(W.config_b(), 96 << 20)
    for kind in (1, 2):
        roundtrip(swp, orc, stream, specs, 21, 1 << 20, kind, "sm", key=("Bs", kind))


def test_restore_many_times_and_recheckpoint(swp, orc, stream):
    specs = W.config_a(5)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 5)
    rc, img_ref, moff = orc.checkpoint(or_regions, host, base, 1, 1 << 16, 4096, threads=8)
    with swp.Swapper(sw_regions, chunk_bytes=1 << 16) as sw, torch.cuda.stream(stream):
        sw.checkpoint(stream)
        for mech in ["sm", "ce_batch", "sm"]:
            sw.set_mechanism(mech)
            poison(arena, specs, offs)
            sw.restore(stream)
            assert sw.verify(stream)["status"] == 0
            assert np.array_equal(arena.cpu().numpy(), host)
        # modify the device state, re-snapshot, and the image follows
        arena[offs[0]:offs[0] + 100].fill_(7)
        host2 = host.copy()
        host2[offs[0]:offs[0] + 100] = 7
        sw.checkpoint(stream)
        rc, img2, _ = orc.checkpoint(or_regions, host2, base, 1, 1 << 16, 4096, threads=8)
        assert np.array_equal(sw.image(), img2)


def test_fault_injection(swp, orc, stream):
    C = 4096
    specs = W.edge_tables(C)["chunk_pm1"] + W.config_a(6)[:3]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 6)
    with swp.Swapper(sw_regions, chunk_bytes=C) as sw, torch.cuda.stream(stream):
        sw.checkpoint(stream)
        man = sw.manifest()
        n, m = len(specs), int(np.frombuffer(man[40:48].tobytes(), "<u8")[0])
        recs = chunk_records(man, n, m)
        img = sw.image()
        rng = np.random.default_rng(9)
        # (a) payload bit flips -> the restore's fused check names exactly that chunk,
        #     every byte is still written (the flipped one included), HBM pass agrees
        for g in sorted(rng.choice(m, 4, replace=False)):
            ri, _, lo, ln, _ = recs[g]
            region_off = int(np.frombuffer(man[64 + 48 * ri + 24:64 + 48 * ri + 32].tobytes(), "<u8")[0])
            pos = region_off + lo + int(rng.integers(0, ln))
            bit = np.uint8(1 << int(rng.integers(0, 8)))
            img[pos] ^= bit
            poison(arena, specs, offs)
            sw.restore(stream)
            res = sw.verify(stream, raise_on_corrupt=False)
            assert res["status"] == swp.SWAP_ECORRUPT
            assert (res["n_bad"], res["first_bad_chunk"]) == (1, g)
            assert (res["hbm_n_bad"], res["hbm_first_bad"]) == (1, g)
            want = host.copy()
            want[offs[ri] + lo + (pos - region_off - lo)] ^= bit
            assert np.array_equal(arena.cpu().numpy(), want)
            img[pos] ^= bit  # repair
        # (b) a manifest flip -> restore refuses before enqueueing anything
        poison(arena, specs, offs)
        before = arena.cpu().numpy()
        for pos in [moff := img.size - man.size, moff + 13, moff + 64 + 5, img.size - 3]:
            img[pos] ^= 0x20
            with pytest.raises(swp.SwapError) as e:
                sw.restore(stream)
            assert e.value.status == swp.SWAP_ECORRUPT
            img[pos] ^= 0x20
        torch.cuda.synchronize()
        assert np.array_equal(arena.cpu().numpy(), before)
        # (c) device corruption after a good restore -> only the HBM pass sees it
        sw.restore(stream)
        ri, _, lo, ln, _ = recs[2]
        torch.cuda.synchronize()
        arena[offs[ri] + lo + ln - 1] ^= 0x01
        res = sw.verify(stream, raise_on_corrupt=False)
        assert (res["n_bad"], res["hbm_n_bad"], res["hbm_first_bad"]) == (0, 1, 2)


def test_state_machine_and_validation(swp, stream):
    t = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    b = t.data_ptr()
    sw = swp.Swapper([(b, 1000, 0)], chunk_bytes=256)
    L = swp.load()
    assert swp.swap_restore(sw.ctx, stream.cuda_stream) == swp.SWAP_ESTATE  # restore before checkpoint
    assert swp.swap_verify(sw.ctx, stream.cuda_stream)[0] == swp.SWAP_ESTATE
    assert swp.swap_register_regions(sw.ctx, [(b + 4096, 16, 9, 0)]) == swp.SWAP_ESTATE  # twice
    assert swp.swap_checkpoint(sw.ctx, stream.cuda_stream) == 0
    assert swp.swap_checkpoint(sw.ctx, stream.cuda_stream) == swp.SWAP_ESTATE  # not synced
    assert swp.swap_sync(sw.ctx, stream.cuda_stream) == 0
    assert swp.swap_restore(sw.ctx, stream.cuda_stream) == 0
    assert L.swap_last_error(sw.ctx) is not None
    sw.close()
    for bad in ([(b + 8, 16, 0)], [(b, 256, 0, 1), (b + 128, 16, 0, 2)], [(b, 16, 0, 1), (b + 64, 16, 0, 1)],
                [(b, 16, 7)]):
        with pytest.raises(swp.SwapError) as e:
            swp.Swapper(bad)
        assert e.value.status == swp.SWAP_EINVAL
    for kw in ({"chunk_bytes": 48}, {"align": 8}, {"checksum": 3}, {"rank": 2, "world": 2}):
        with pytest.raises(swp.SwapError) as e:
            swp.Swapper([(b, 16, 0)], **kw)
        assert e.value.status == swp.SWAP_EINVAL


def test_summary_matches_oracle(swp, orc, stream):
    specs = W.config_a(8)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 8)
    rc, img_ref, moff = orc.checkpoint(or_regions, host, base, 2, 1 << 16, 4096, rank=1, world=2, threads=8)
    with swp.Swapper(sw_regions, chunk_bytes=1 << 16, checksum=2, rank=1, world=2) as sw:
        sw.checkpoint(stream)
        assert np.array_equal(sw.image(), img_ref)
        s = sw.summary()
        assert s == orc.summary(img_ref[moff:], img_ref.size)
        other = bytearray(s)
        other[0:4] = (0).to_bytes(4, "little")
        allb = bytes(other) + s
        assert sw.set_global(allb) == orc.global_digest(allb)
        with pytest.raises(swp.SwapError):
            sw.set_global(s + bytes(other))  # wrong order


def test_import_stored_image(swp, orc, stream):
    """An image written by the oracle and loaded into the library's buffer restores bit-exactly."""
    specs = W.config_a(7)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 7)
    rc, img_ref, moff = orc.checkpoint(or_regions, host, base, 1, 1 << 20, 4096, threads=8)
    with swp.Swapper(sw_regions, chunk_bytes=1 << 20) as sw, torch.cuda.stream(stream):
        sw.image()[:] = img_ref
        sw.import_image()
        poison(arena, specs, offs)
        sw.restore(stream)
        assert sw.verify(stream)["status"] == 0
        assert np.array_equal(arena.cpu().numpy(), host)
