"""CPU-side checks of the C-ABI library: it loads, exports exactly what include/swap.h
declares, and its host-only logic behaves (no compute calls: there is no GPU here)."""
import ctypes
import os
import re
import struct

import pytest

from conftest import ROOT

HEADER = os.path.join(ROOT, "include", "swap.h")


def declared_symbols():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^SWAP_API\s+[\w\s\*]+?\b(swap_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def swp():
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for core in ("swap_register_regions", "swap_checkpoint", "swap_restore", "swap_verify"):
        assert core in syms  # BASELINE.json north_star's call set
    assert len(syms) >= 19


def test_library_exports_every_declared_symbol(swp):
    L = swp.load()
    for name in declared_symbols():
        assert hasattr(L, name), name
    assert sorted(swp.EXPORTS) == declared_symbols()


def test_no_torch_or_cuda_types_in_header():
    src = open(HEADER).read()
    assert "torch" not in src.split("*/", 1)[1]
    assert "#include <cuda" not in src


def test_struct_sizes_match_header(swp):
    assert ctypes.sizeof(swp.swap_shard_summary_t) == 64
    assert ctypes.sizeof(swp.swap_region_t) == 24
    assert ctypes.sizeof(swp.swap_verify_result_t) == 40
    assert ctypes.sizeof(swp.swap_config_t) == 56


def test_config_default(swp):
    c = swp.swap_config_default()
    assert (c.chunk_bytes, c.align, c.checksum, c.mechanism, c.world, c.seg_bytes) == (1 << 20, 4096, 1, 0, 1, 0)
    assert (c.host_numa, c.reserved0) == (0, 0)  # auto NUMA placement


def test_status_strings(swp):
    L = swp.load()
    assert L.swap_status_str(0) == b"SWAP_OK"
    assert L.swap_status_str(-5) == b"SWAP_ECORRUPT"
    assert L.swap_last_error(None) == b"null ctx"
    L.swap_destroy(None)  # no-op


def test_create_validates_before_touching_cuda(swp):
    c = swp.swap_config_default()
    c.chunk_bytes = 100
    st, h = swp.swap_create(c)
    assert st == swp.SWAP_EINVAL and not h.value
    c = swp.swap_config_default()
    c.chunk_bytes = 1 << 32
    assert swp.swap_create(c)[0] == swp.SWAP_EUNSUPPORTED


@pytest.mark.skipif(os.path.exists("/dev/nvidia0"), reason="CPU-only check")
def test_create_fails_loudly_without_gpu(swp):
    st, h = swp.swap_create(swp.swap_config_default())
    assert st == swp.SWAP_ECUDA and not h.value


def test_null_args(swp):
    L = swp.load()
    assert L.swap_register_regions(None, None, 0) == swp.SWAP_EINVAL
    assert L.swap_checkpoint(None, None) == swp.SWAP_EINVAL
    assert L.swap_restore(None, None) == swp.SWAP_EINVAL
    assert L.swap_verify(None, None, 1, None) == swp.SWAP_EINVAL
    assert L.swap_sync(None, None) == swp.SWAP_EINVAL
    # round-2 entry points: argument checks come first and need no device
    assert L.swap_get_mechanism_dir(None, 0, None) == swp.SWAP_EINVAL
    assert L.swap_get_numa(None, None, None) == swp.SWAP_EINVAL
    assert L.swap_restore_stripe(None, 0, 2, None) == swp.SWAP_EINVAL
    assert L.swap_pull_stripes(None, 0, 2, None, None) == swp.SWAP_EINVAL
    assert L.swap_get_restore_spans(None, None, 0, None) == swp.SWAP_EINVAL
    assert L.swap_ipc_export(0, None, None, None) == swp.SWAP_EINVAL
    assert L.swap_ipc_import(0, None, 0, None, None) == swp.SWAP_EINVAL
    assert L.swap_ipc_close(0, None) == swp.SWAP_EINVAL


SUM = struct.Struct("<IIIIQQQQQQ")


def test_merge_global_vs_oracle(swp, orc):
    world = 4
    allb = b"".join(SUM.pack(r, world, 1, 16, 64 + r, 10 ** 9 + r, 10 ** 9 + 8192, 0xABC + r, 0xDEF * r, 0)
                    for r in range(world))
    st, d = swp.swap_merge_global(allb, world)
    assert st == 0 and d == orc.global_digest(allb)
    swapped = allb[64:128] + allb[:64] + allb[128:]
    assert swp.swap_merge_global(swapped, world)[0] == swp.SWAP_ENCCL
    wrong_world = SUM.pack(0, 2, 1, 1, 1, 1, 1, 1, 1, 0) + SUM.pack(1, 3, 1, 1, 1, 1, 1, 1, 1, 0)
    assert swp.swap_merge_global(wrong_world, 2)[0] == swp.SWAP_ENCCL


def test_host_crc_paths_vs_oracle(swp, orc):
    """libswap's host CRC-32C (hardware crc32 in three interleaved streams for long inputs, merged with
    GF(2) shifts) against the oracle's table CRC, through swap_merge_global's digest."""
    for world in (1, 3, 64, 193, 1000, 4099):
        allb = b"".join(SUM.pack(r, world, 1 + r % 2, r % 7, r * 3, r * 5 + 1, r * 7 + 2, r * 11, r * 13, 0)
                        for r in range(world))
        st, d = swp.swap_merge_global(allb, world)
        assert st == 0 and d == orc.global_digest(allb), world
