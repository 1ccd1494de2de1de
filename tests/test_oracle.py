"""Pins for the CPU oracle (oracle/): each test checks it against something other than itself.

SURVEY.md §8(c) "What pins each part": RFC 3720 CRC-32C vectors; xxHash spec vectors and
the `xxhash` library; three independent CRC implementations (bit-serial definition,
Sarwate table, SSE4.2 hardware instruction); the zlib combine algebra; a byte-at-a-time
layout builder (brute force over tiny tables); round-trip identity; single-bit detection.
"""
import itertools
import struct

import numpy as np
import pytest

import workloads as W
from conftest import decode_input, read_golden

HDR = struct.Struct("<8sIIQQQQQII")  # 64-B header
REG = struct.Struct("<IIQQQQQ")  # 48-B region record
CHK = struct.Struct("<IIQQQ")  # 32-B chunk record
SUM = struct.Struct("<IIIIQQQQQQ")  # 64-B shard summary
assert HDR.size == 64 and REG.size == 48 and CHK.size == 32 and SUM.size == 64


def parse_manifest(man: bytes):
    magic, ver, kind, C, A, n, m, payload, rank, world = HDR.unpack_from(man, 0)
    regs = [REG.unpack_from(man, 64 + 48 * i) for i in range(n)]
    chunks = [CHK.unpack_from(man, 64 + 48 * n + 32 * g) for g in range(m)]
    (crc,) = struct.unpack_from("<Q", man, 64 + 48 * n + 32 * m)
    return dict(magic=magic, ver=ver, kind=kind, C=C, A=A, n=n, m=m, payload=payload, rank=rank,
                world=world, regs=regs, chunks=chunks, crc=crc, size=64 + 48 * n + 32 * m + 8)


# ------------------------------------------------------------------ checksums
@pytest.mark.parametrize("row", read_golden("crc32c_rfc3720.txt"), ids=lambda r: r[0])
def test_crc32c_rfc3720_vectors(orc, row):
    name, inp, want = row
    data = decode_input(inp)
    want = int(want, 16)
    assert orc.crc32c_bitwise(data) == want
    assert orc.crc32c(data) == want
    assert orc.crc32c_sse42(data) == want


@pytest.mark.parametrize("row", read_golden("xxh64_spec.txt"), ids=lambda r: r[0])
def test_xxh64_spec_vectors(orc, row):
    name, inp, seed, want = row
    assert orc.xxh64(decode_input(inp), int(seed)) == int(want, 16)


def test_crc32c_three_implementations_agree(orc):
    assert orc.have_sse42()
    rng = np.random.default_rng(1)
    for n in list(range(0, 70)) + [255, 256, 257, 4095, 4096, 65537]:
        b = rng.integers(0, 256, n, dtype=np.uint8).tobytes()
        t = orc.crc32c(b)
        assert orc.crc32c_sse42(b) == t
        if n <= 4096:
            assert orc.crc32c_bitwise(b) == t
    big = rng.integers(0, 256, 3 << 20, dtype=np.uint8)
    assert orc.crc32c(big) == orc.crc32c_sse42(big)


def test_xxh64_matches_library(orc):
    xxhash = pytest.importorskip("xxhash")
    rng = np.random.default_rng(2)
    for n in list(range(0, 80)) + [127, 128, 129, 1000, 4096, 65536 + 7]:
        b = rng.integers(0, 256, n, dtype=np.uint8).tobytes()
        for seed in (0, 1, 2654435761, (1 << 64) - 1):
            assert orc.xxh64(b, seed) == xxhash.xxh64(b, seed=seed).intdigest()


def test_crc32c_combine_algebra(orc):
    rng = np.random.default_rng(3)
    for _ in range(200):
        a = rng.integers(0, 256, int(rng.integers(0, 300)), dtype=np.uint8).tobytes()
        b = rng.integers(0, 256, int(rng.integers(0, 300)), dtype=np.uint8).tobytes()
        assert orc.crc32c_combine(orc.crc32c(a), orc.crc32c(b), len(b)) == orc.crc32c(a + b)


def test_chunk_hash_kinds(orc):
    b = b"hello, swap image"
    assert orc.chunk_hash(orc.CRC32C, b) == orc.crc32c_sse42(b)
    xxhash = pytest.importorskip("xxhash")
    assert orc.chunk_hash(orc.XXH64, b) == xxhash.xxh64(b, seed=0).intdigest()


# ------------------------------------------------------------------ layout: brute force
def naive_image(sizes, contents, C, A):
    """Byte-at-a-time image builder written independently of the oracle's arithmetic."""
    img, offs, chunks = bytearray(), [], []
    for i, (size, data) in enumerate(zip(sizes, contents)):
        if i > 0:
            while len(img) % A:
                img.append(0)
        offs.append(len(img))
        for k in range(size):
            if k % C == 0:
                chunks.append([i, k, 0])
            img.append(data[k])
            chunks[-1][2] += 1
    return bytes(img), offs, chunks


SIZES = [0, 1, 15, 16, 17, 31, 32, 33, 48]


@pytest.mark.parametrize("C,A", [(16, 16), (16, 64), (32, 16), (32, 64), (64, 16), (64, 64)])
def test_layout_brute_force(orc, C, A):
    rng = np.random.default_rng(C * 100 + A)
    tables = [t for n in (1, 2, 3) for t in itertools.product(SIZES, repeat=n)]
    if len(tables) > 400:  # n=3 has 729 tuples; take every n<=2 and a seeded third of n=3
        keep = [t for t in tables if len(t) < 3]
        three = [t for t in tables if len(t) == 3]
        keep += [three[i] for i in rng.choice(len(three), 250, replace=False)]
        tables = keep
    for sizes in tables:
        n = len(sizes)
        mem = rng.integers(0, 256, 1024, dtype=np.uint8)
        addrs = [256 * i + 64 for i in range(n)]  # 16-aligned, disjoint
        regs = [(10 + i, 0x7000_0000 + a, s, i % 4) for i, (a, s) in enumerate(zip(addrs, sizes))]
        contents = [mem[a:a + s].tobytes() for a, s in zip(addrs, sizes)]
        for kind in (orc.CRC32C, orc.XXH64):
            rc, image, moff = orc.checkpoint(regs, mem, 0x7000_0000, kind, C, A)
            assert rc == 0
            want_img, want_offs, want_chunks = naive_image(sizes, contents, C, A)
            payload = len(want_img)
            assert moff == -(-payload // A) * A
            assert image[:payload].tobytes() == want_img
            assert not image[payload:moff].any()  # padding zero
            man = parse_manifest(image[moff:].tobytes())
            assert man["size"] == image.size - moff
            assert (man["C"], man["A"], man["n"], man["m"], man["payload"]) == (C, A, n, len(want_chunks), payload)
            assert [r[4] for r in man["regs"]] == want_offs
            # header constants and the region records' remaining fields, from the naive chunk list:
            # first_i = how many chunks the regions before i produced, n_i = how many region i produced
            assert (man["magic"], man["ver"], man["kind"], man["rank"], man["world"]) == (b"SWAPMAN1", 1, kind, 0, 1)
            firsts = [sum(1 for c in want_chunks if c[0] < i) for i in range(n)]
            counts = [sum(1 for c in want_chunks if c[0] == i) for i in range(n)]
            assert [r[:4] for r in man["regs"]] == [(rid, k, a, s) for (rid, a, s, k) in regs]
            assert [r[5] for r in man["regs"]] == firsts
            assert [r[6] for r in man["regs"]] == counts
            assert all(c[1] == 0 for c in man["chunks"])  # chunk-record pad
            assert [list(c[:1]) + list(c[2:4]) for c in man["chunks"]] == want_chunks
            for (ri, _, lo, ln, c) in man["chunks"]:
                piece = contents[ri][lo:lo + ln]
                want = orc.crc32c_sse42(piece) if kind == orc.CRC32C else orc.xxh64(piece)
                assert c == want


def test_region_crc_is_fold_of_chunk_crcs(orc):
    """Chunk boundaries pinned by the combine algebra: folding a region's chunk CRCs
    (each combined with the next chunk's length) must equal one CRC over the region."""
    rng = np.random.default_rng(4)
    C = 4096
    sizes = [1, 4095, 4096, 4097, 3 * 4096 + 5, 40000]
    mem = rng.integers(0, 256, sum(sizes) + 256 * len(sizes), dtype=np.uint8)
    regs, pos = [], 0
    for i, s in enumerate(sizes):
        regs.append((i, pos, s, 0))
        pos += (s + 255) // 256 * 256
    rc, image, moff = orc.checkpoint(regs, mem, 0, orc.CRC32C, C, 4096)
    assert rc == 0
    man = parse_manifest(image[moff:].tobytes())
    for i, (rid, addr, s, _) in enumerate(regs):
        cs = [c for c in man["chunks"] if c[0] == i]
        acc = cs[0][4]
        for c in cs[1:]:
            acc = orc.crc32c_combine(acc, c[4], c[3])
        assert acc == orc.crc32c_sse42(mem[addr:addr + s])


# ------------------------------------------------------------------ validation
def test_validation_rejects(orc):
    ok = [(0, 0x1000, 100, 0), (1, 0x2000, 100, 1)]
    assert orc.plan(ok, 64, 64).rc == 0
    bad = {
        "empty_table": [],
        "misaligned": [(0, 0x1008, 10, 0)],
        "overlap": [(0, 0x1000, 0x200, 0), (1, 0x1100, 16, 0)],
        "dup_id": [(0, 0x1000, 16, 0), (0, 0x2000, 16, 0)],
        "bad_kind": [(0, 0x1000, 16, 9)],
        "wraps": [(0, (1 << 64) - 16, 32, 0)],
    }
    for name, regs in bad.items():
        assert orc.plan(regs, 64, 64).rc == orc.EINVAL, name
    for C, A in [(8, 64), (64, 8), (48, 64), (64, 100), (0, 64)]:
        assert orc.plan(ok, C, A).rc == orc.EINVAL
    # touching (adjacent) regions and zero-size regions at the same address are fine
    assert orc.plan([(0, 0x1000, 16, 0), (1, 0x1010, 16, 0), (2, 0x1010, 0, 0)], 16, 16).rc == 0
    # world/rank
    mem = np.zeros(0x3000, np.uint8)
    assert orc.checkpoint(ok, mem, 0, orc.CRC32C, 64, 64, rank=1, world=1)[0] == orc.EINVAL
    assert orc.checkpoint(ok, mem, 0, 3, 64, 64)[0] == orc.EINVAL


def test_degenerate_tables(orc):
    p = orc.plan([(0, 0, 0, 0), (1, 16, 0, 0)], 64, 4096)
    assert (p.rc, p.payload_bytes, p.n_chunks) == (0, 0, 0)
    assert p.image_bytes == orc.manifest_bytes(2, 0) == 64 + 96 + 8


# ------------------------------------------------------------------ round trip and detection
def make_case(specs, seed):
    arena, offs = W.host_arena(specs, seed)
    base = 0x7F00_0000_0000
    regs = [(100 + i, base + o, r.nbytes, r.kind) for i, (r, o) in enumerate(zip(specs, offs))]
    return arena, base, regs


@pytest.mark.parametrize("seed", [0, 1])
@pytest.mark.parametrize("C", [4096, 1 << 20])
@pytest.mark.parametrize("kind", [1, 2])
def test_roundtrip_config_a(orc, seed, C, kind):
    specs = W.config_a(seed)
    arena, base, regs = make_case(specs, seed)
    orig = arena.copy()
    rc, image, moff = orc.checkpoint(regs, arena, base, kind, C, 4096, threads=4)
    assert rc == 0
    man = image[moff:]
    assert orc.manifest_ok(man)
    h = parse_manifest(man.tobytes())
    assert (h["magic"], h["ver"], h["kind"], h["C"], h["A"], h["n"]) == (b"SWAPMAN1", 1, kind, C, 4096, len(regs))
    first = 0
    for (rid, addr, nb, k), rr in zip(regs, h["regs"]):
        assert rr[:4] == (rid, k, addr, nb)
        n_i = len(range(0, nb, C))  # chunk starts 0, C, 2C, ... below nb
        assert (rr[5], rr[6]) == (first, n_i)
        assert [c[0] for c in h["chunks"][first:first + n_i]] == [regs.index((rid, addr, nb, k))] * n_i
        first += n_i
        o = rr[4]
        assert np.array_equal(image[o:o + nb], arena[addr - base:addr - base + nb])
    assert first == h["m"]
    # poison every region, restore, compare all bytes (guards included)
    for (_, addr, nb, _) in regs:
        arena[addr - base:addr - base + nb] = W.POISON_BYTE
    rc, nbad, fb = orc.restore(image, moff, arena, base, threads=4)
    assert (rc, nbad, fb) == (0, 0, (1 << 64) - 1)
    assert np.array_equal(arena, orig)
    # the "fast" timing variant (SSE4.2 CRC) restores the same bytes with the same verdict
    for (_, addr, nb, _) in regs:
        arena[addr - base:addr - base + nb] = W.POISON_BYTE
    assert orc.restore(image, moff, arena, base, threads=4, fast=True) == (0, 0, (1 << 64) - 1)
    assert np.array_equal(arena, orig)
    assert orc.verify(man, arena, base)[:2] == (0, 0)


def test_single_bit_flips(orc):
    C = 4096
    specs = W.edge_tables(C)["chunk_pm1"] + [W.RegionSpec("x", 0, 10000)]
    arena, base, regs = make_case(specs, 7)
    rc, image, moff = orc.checkpoint(regs, arena, base, orc.CRC32C, C, 4096)
    h = parse_manifest(image[moff:].tobytes())
    rng = np.random.default_rng(5)
    # (a) a flip inside chunk g is reported as exactly chunk g
    for g in rng.choice(h["m"], 6, replace=False):
        ri, _, lo, ln, _ = h["chunks"][g]
        pos = h["regs"][ri][4] + lo + int(rng.integers(0, ln))
        img = image.copy()
        img[pos] ^= np.uint8(1 << int(rng.integers(0, 8)))
        mem = arena.copy()
        rc, nbad, fb = orc.restore(img, moff, mem, base)
        assert (rc, nbad, fb) == (0, 1, g)
        assert orc.verify(img[moff:], mem, base)[1:] == (1, g)
    # (b) a flip in inter-region padding is not covered by any checksum
    pad = h["regs"][0][4] + h["regs"][0][3]
    assert pad < h["regs"][1][4]
    img = image.copy()
    img[pad] ^= 0xFF
    assert orc.restore(img, moff, arena.copy(), base)[:2] == (0, 0)
    # (c) a flip anywhere in the manifest is caught by the manifest CRC; nothing is written
    for pos in [moff, moff + 20, moff + 64 + 3, image.size - 20, image.size - 1]:
        img = image.copy()
        img[pos] ^= 0x10
        mem = arena.copy()
        for (_, addr, nb, _) in regs:
            mem[addr - base:addr - base + nb] = W.POISON_BYTE
        before = mem.copy()
        assert orc.restore(img, moff, mem, base)[0] == orc.ECORRUPT
        assert np.array_equal(mem, before)
    # (d) device-side corruption after restore is caught by verify
    mem = arena.copy()
    g = 3
    ri, _, lo, ln, _ = h["chunks"][g]
    mem[regs[ri][1] - base + lo + ln - 1] ^= 0x80
    assert orc.verify(image[moff:], mem, base)[1:] == (1, g)


def test_summary_and_global_digest(orc):
    specs = W.config_a(3)
    arena, base, regs = make_case(specs, 3)
    rc, image, moff = orc.checkpoint(regs, arena, base, orc.XXH64, 1 << 16, 4096, rank=2, world=4)
    man = image[moff:]
    s = orc.summary(man, image.size)
    rank, world, kind, n, m, payload, ib, mcrc, digest, res = SUM.unpack(s)
    h = parse_manifest(man.tobytes())
    assert (rank, world, kind, n, m, payload, ib, res) == (2, 4, 2, 16, h["m"], h["payload"], image.size, 0)
    assert mcrc == h["crc"] == orc.crc32c_sse42(man[:-8])
    cs = b"".join(struct.pack("<Q", c[4]) for c in h["chunks"])
    assert digest == orc.crc32c_sse42(cs)
    # payload == sum of region sizes plus alignment padding (closed form)
    exp, pos = 0, 0
    for i, r in enumerate(specs):
        pos = pos if i == 0 else -(-pos // 4096) * 4096
        pos += r.nbytes
    assert payload == pos
    # global digest of fabricated rank-ordered summaries
    fab = b"".join(SUM.pack(r, 4, 1, 3, 10 + r, 1000 * r, 5000, r * 7, r * 11, 0) for r in range(4))
    assert orc.global_digest(fab) == orc.crc32c_sse42(fab)


# ------------------------------------------------------------------ touched-chunk masks (reading 25)
def test_policy_view_chunk_masks(orc):
    """Pins for the mask rule of oracle.policy_view against independent statements of it: an all-zero
    mask is the DISCARD policy, an all-one mask (or none) is SAVE, and byte k of a region is zeroed
    iff keep[k // C] == 0 (brute force over tiny regions, byte by byte)."""
    import xxhash

    C = 16
    specs = [W.RegionSpec(f"r{i}", W.KIND_KV, n) for i, n in enumerate([0, 1, 15, 16, 17, 31, 32, 33, 48, 50])]
    arena, base, regs = make_case(specs, 11)
    n_ch = [-(-r[2] // C) for r in regs]
    save = [orc.SAVE] * len(regs)
    # all-zero mask == DISCARD, all-one / absent mask == SAVE
    zero = {i: np.zeros(n, np.uint8) for i, n in enumerate(n_ch)}
    ones = {i: np.ones(n, np.uint8) for i, n in enumerate(n_ch)}
    assert np.array_equal(orc.policy_view(regs, save, arena, arena, base, C, zero),
                          orc.policy_view(regs, [orc.DISCARD] * len(regs), arena, arena, base))
    assert np.array_equal(orc.policy_view(regs, save, arena, arena, base, C, ones), arena)
    assert np.array_equal(orc.policy_view(regs, save, arena, arena, base), arena)
    # random masks, checked byte by byte
    rng = np.random.default_rng(5)
    for _ in range(20):
        masks = {i: rng.integers(0, 2, n).astype(np.uint8) for i, n in enumerate(n_ch)}
        view = orc.policy_view(regs, save, arena, arena, base, C, masks)
        want = arena.copy()
        for i, (_, addr, nb, _) in enumerate(regs):
            for k in range(nb):
                if masks[i][k // C] == 0:
                    want[addr - base + k] = 0
        assert np.array_equal(view, want)
        # the captured image: masked chunks are zero bytes with the checksum of a zero chunk
        for kind in (orc.CRC32C, orc.XXH64):
            rc, image, moff = orc.checkpoint(regs, view, base, kind, C, 16)
            assert rc == 0
            h = parse_manifest(image[moff:].tobytes())
            for i, rr in enumerate(h["regs"]):
                first = rr[5]
                for j, keep in enumerate(masks[i]):
                    if keep:
                        continue
                    ln = h["chunks"][first + j][3]
                    assert np.all(image[rr[4] + j * C:rr[4] + j * C + ln] == 0)
                    z = bytes(ln)
                    want_cs = orc.crc32c_bitwise(z) if kind == orc.CRC32C else xxhash.xxh64_intdigest(z, 0)
                    assert h["chunks"][first + j][4] == want_cs
