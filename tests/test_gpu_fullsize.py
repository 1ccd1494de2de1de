"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

bench.py's N=1 workload is config B (Llama-3.1-8B engine image, 291 regions, 52.57 GB) in a
releasable VMM arena (swap_arena_*), chunk 1 MiB, CRC-32C, mechanism AUTO (-> CE_PIPE at this
size). The same setup is run here through the C ABI and checked against the CPU oracle:

* every chunk checksum of the GPU manifest is recomputed by the oracle (`oracle.verify`, all
  ~50 K chunks, OpenMP) over a host copy of the device bytes taken before the checkpoint;
* the manifest header, region records and chunk records (everything but c_g) equal the
  oracle's plan (`oracle.plan`) and SURVEY §8(c) step 3; the manifest CRC holds (oracle);
* the image payload equals the device bytes region by region; every padding byte is 0;
* the shard summary equals `oracle.summary` of that manifest;
* after poison -> restore -> HBM verify the whole arena (regions and 0xA5 guards) equals the
  pre-checkpoint copy, and a single flipped image bit is reported as exactly its chunk.

Config D (Llama-3.1-70B TP=8 shard, 30.5 GB, the N>1 bench workload) gets the same full
check with XXH64; config C (69.3 GB/rank, too large for two host copies) is checked on
sampled chunks (first and last chunk of every region plus random ones), hashed one by one
by the oracle.
"""
import os
import struct

import numpy as np
import pytest

import workloads as W

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]

C = 1 << 20
A = 4096
U64_MAX = (1 << 64) - 1
HDR = struct.Struct("<8sIIQQQQQII")
REG = struct.Struct("<IIQQQQQ")
THREADS = max(1, len(os.sched_getaffinity(0)))


@pytest.fixture(scope="module")
def swp():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


def host_free() -> int:
    with open("/proc/meminfo") as f:
        for line in f:
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) * 1024
    return 0


def check_records(man: np.ndarray, plan, specs, regions, kind: int, C: int = C):
    """Header, region records and chunk records (all but c_g) against oracle.plan + §8(c) step 3."""
    n, m = len(specs), plan.n_chunks
    magic, ver, k, c, a, nn, mm, payload, rank, world = HDR.unpack_from(man, 0)
    assert (magic, ver, k, c, a, nn, mm, payload, rank, world) == (
        b"SWAPMAN1", 1, kind, C, A, n, m, plan.payload_bytes, 0, 1)
    for i, (addr, nb, knd, rid) in enumerate(regions):
        assert REG.unpack_from(man, 64 + 48 * i) == (rid, knd, addr, nb, plan.off[i], plan.first[i], plan.nchunks[i])
    rec = man[64 + 48 * n: 64 + 48 * n + 32 * m].view(np.uint64).reshape(m, 4)
    region = np.repeat(np.arange(n, dtype=np.uint64), plan.nchunks)
    first = np.repeat(np.asarray(plan.first, dtype=np.uint64), plan.nchunks)
    j = np.arange(m, dtype=np.uint64) - first
    sizes = np.repeat(np.asarray([r.nbytes for r in specs], dtype=np.uint64), plan.nchunks)
    assert np.array_equal(rec[:, 0], region)  # u32 region index + u32 0 pad, little-endian
    assert np.array_equal(rec[:, 1], j * C)
    assert np.array_equal(rec[:, 2], np.minimum(C, sizes - j * C))
    return rec[:, 3]


def setup(swp, specs, seed):
    offs, arena_bytes = W.place(specs)
    vmm = swp.Arena(arena_bytes, device=0)
    base, arena = vmm.alloc(arena_bytes)
    W.fill_device_arena(arena, specs, offs, seed=seed)
    torch.cuda.synchronize()
    regions = [(base + o, r.nbytes, r.kind, 7 + i) for i, (r, o) in enumerate(zip(specs, offs))]
    return vmm, base, arena, offs, regions


def poison_restore_verify(sw, arena, specs, offs, stream):
    """a6 poison, a7 restore, a8 HBM verify: clean."""
    for r, o in zip(specs, offs):
        arena[o:o + r.nbytes].fill_(W.POISON_BYTE)
    sw.restore(stream)
    res = sw.verify(stream, hbm_pass=True)
    assert res["status"] == 0
    assert (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"], res["manifest_ok"]) == (0, U64_MAX, 0, 1)
    return res


def flip_check(swp, sw, plan, specs, stream, g, img, C: int = C):
    """One flipped image bit in chunk g is reported as exactly chunk g; then a clean restore."""
    i = int(np.searchsorted(np.asarray(plan.first), g, side="right") - 1)
    j = g - plan.first[i]
    pos = plan.off[i] + j * C + min(C, specs[i].nbytes - j * C) // 2
    img[pos] ^= 0x10
    try:
        sw.restore(stream)
        res = sw.verify(stream, hbm_pass=True, raise_on_corrupt=False)
        assert res["status"] == swp.SWAP_ECORRUPT
        assert (res["n_bad"], res["first_bad_chunk"]) == (1, g)
    finally:
        img[pos] ^= 0x10
    sw.restore(stream)
    assert sw.verify(stream, hbm_pass=True)["status"] == 0


@pytest.mark.parametrize("cfg,kind,C", [("B", 1, C), ("B", 2, C), ("D", 2, C), ("B", 2, 4 << 20), ("B", 2, 16 << 20)],
                         ids=["B-crc32c", "B-xxh64", "D-xxh64", "B-xxh64-4MiB", "B-xxh64-16MiB"])
def test_full_size_every_chunk(swp, orc, cfg, kind, C):
    """4 / 16 MiB XXH64 chunks: the round-2 quad-per-chunk kernels (2 x 3 KiB / 2 x 4 KiB rings) at full size;
    16 MiB restores take AUTO's coalesced copies + one hash pass (CE_BATCH)."""
    specs = W.config_b() if cfg == "B" else W.config_d(0)
    payload = sum(r.nbytes for r in specs)
    if host_free() < 2.3 * payload:
        pytest.skip(f"needs ~{2.3 * payload / 1e9:.0f} GB of free host RAM (pinned image + host copy)")
    vmm, base, arena, offs, regions = setup(swp, specs, seed=3)
    plan = orc.plan([(rid, a, nb, k) for (a, nb, k, rid) in regions], C, A)
    assert plan.rc == 0
    mem = arena.cpu().numpy()  # the device bytes before the checkpoint (regions + guards)
    stream = torch.cuda.Stream()
    sw = swp.Swapper(regions, chunk_bytes=C, checksum=kind, mechanism="auto")
    try:
        # the bench's launch configuration at this size (XXH64 with chunks > 4 MiB restores with CE_BATCH)
        assert sw.mechanism() == ("ce_batch" if C > (4 << 20) else "ce_pipe")
        assert sw.mechanism("checkpoint") == "ce_pipe"
        with torch.cuda.stream(stream):
            sw.checkpoint(stream)
            img, man = sw.image(), sw.manifest()
            assert img.size == plan.image_bytes and man.size == plan.image_bytes - plan.manifest_off
            cg = check_records(man, plan, specs, regions, kind, C)
            assert orc.manifest_ok(man)
            rc, nbad, fbad = orc.verify(man, mem, base, threads=THREADS)
            assert (rc, nbad, fbad) == (0, 0, U64_MAX), "GPU chunk checksums differ from the oracle"
            assert sw.summary() == orc.summary(man, plan.image_bytes)
            for i, (r, o) in enumerate(zip(specs, offs)):
                lo = plan.off[i]
                assert np.array_equal(img[lo:lo + r.nbytes], mem[o:o + r.nbytes]), f"image payload of region {i}"
                hi = plan.off[i + 1] if i + 1 < len(specs) else plan.manifest_off
                assert not img[lo + r.nbytes:hi].any(), f"padding after region {i}"
            poison_restore_verify(sw, arena, specs, offs, stream)
            torch.cuda.synchronize()
            step = 1 << 30
            for lo in range(0, mem.size, step):
                assert np.array_equal(arena[lo:lo + step].cpu().numpy(), mem[lo:lo + step]), f"arena at {lo}"
            rng = np.random.default_rng(5)
            g = int(rng.integers(0, plan.n_chunks))
            flip_check(swp, sw, plan, specs, stream, g, img, C)
    finally:
        sw.close()
        del arena
        vmm.close()
        torch.cuda.synchronize()


def test_full_size_config_c_sampled(swp, orc):
    specs = W.config_c(0)
    payload = sum(r.nbytes for r in specs)
    if host_free() < 1.15 * payload:
        pytest.skip(f"needs ~{1.15 * payload / 1e9:.0f} GB of free host RAM")
    kind = 1
    vmm, base, arena, offs, regions = setup(swp, specs, seed=4)
    plan = orc.plan([(rid, a, nb, k) for (a, nb, k, rid) in regions], C, A)
    rng = np.random.default_rng(11)
    sample = set()
    for i in range(len(specs)):
        if plan.nchunks[i]:
            sample.update({plan.first[i], plan.first[i] + plan.nchunks[i] - 1})
    sample.update(int(x) for x in rng.integers(0, plan.n_chunks, 256))
    sample = sorted(sample)
    owner = np.searchsorted(np.asarray(plan.first), sample, side="right") - 1

    def chunk_dev(g, i):
        j = g - plan.first[i]
        lo = offs[i] + j * C
        return arena[lo:lo + min(C, specs[i].nbytes - j * C)].cpu().numpy()

    before = [chunk_dev(g, i) for g, i in zip(sample, owner)]
    expect = [orc.chunk_hash(kind, b) for b in before]
    stream = torch.cuda.Stream()
    sw = swp.Swapper(regions, chunk_bytes=C, checksum=kind, mechanism="auto")
    try:
        with torch.cuda.stream(stream):
            sw.checkpoint(stream)
            img, man = sw.image(), sw.manifest()
            cg = check_records(man, plan, specs, regions, kind)
            assert orc.manifest_ok(man)
            for g, i, b, e in zip(sample, owner, before, expect):
                j = g - plan.first[i]
                assert int(cg[g]) == e, f"c_g of chunk {g}"
                lo = plan.off[i] + j * C
                assert np.array_equal(img[lo:lo + b.size], b), f"image bytes of chunk {g}"
            poison_restore_verify(sw, arena, specs, offs, stream)
            torch.cuda.synchronize()
            for g, i, b in zip(sample, owner, before):
                assert np.array_equal(chunk_dev(g, i), b), f"restored chunk {g}"
            for o in offs:  # guard bands in front of every region are untouched
                assert (arena[o - W.GUARD_BYTES:o].cpu().numpy() == W.GUARD_BYTE).all()
            flip_check(swp, sw, plan, specs, stream, sample[len(sample) // 2], img)
    finally:
        sw.close()
        del arena
        vmm.close()
        torch.cuda.synchronize()
