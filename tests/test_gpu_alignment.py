"""GPU parity with device addresses that are only 16-B aligned (the ABI's minimum, DESIGN.md
reading 8) and image alignments below the 4 KiB default.

The other parity tests place every region at a 256-B aligned base (cudaMalloc-like). Here region i
starts at a 256-B base + 16 * k_i bytes (k_i = 1..15), so the 256-bit-load kernels take their 16-B
fallback paths (ld32_v4x2 in the CRC-32C hash kernel and the XXH64 lane kernel), the SM movers see
512-B warp steps straddling cache lines, and the copy engine gets unaligned spans; with A = 16 the
image offsets are misaligned the same way. Bit-exact against the oracle: image (payload, padding,
manifest) and the restored arena with its guard bands.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import workloads as W
from conftest import ROOT
from gpu_util import device_case, poison

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
U64_MAX = (1 << 64) - 1


def skewed_case(seed: int, n: int = 24):
    rng = np.random.default_rng(seed)
    sizes = [int(x) for x in rng.integers(1, 3 << 20, n)]
    sizes[3], sizes[7], sizes[11] = 5, 100, 4096 + 48  # tiny and just-past-a-page regions
    specs = [W.RegionSpec(f"r{i}", i % 4, s, "bf16" if i % 3 == 0 and s % 2 == 0 else "bytes") for i, s in enumerate(sizes)]
    skew = [16 * (1 + (7 * i) % 15) for i in range(n)]
    return specs, skew


@pytest.fixture(scope="module")
def swp():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


@pytest.mark.parametrize("align", [16, 4096])
@pytest.mark.parametrize("C", [4096, 1 << 16, 1 << 20], ids=["4K", "64K", "1M"])
@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
@pytest.mark.parametrize("mech", ["sm", "ce_region", "ce_batch", "ce_pipe"])
def test_skewed_addresses_bit_exact(swp, orc, mech, kind, C, align):
    specs, skew = skewed_case(31)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 31, skew)
    assert all((base + o) % 32 == 16 or (base + o) % 32 == 0 for o in offs)
    assert any((base + o) % 32 == 16 for o in offs)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, C, align, threads=8)
    assert rc == 0
    stream = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=mech, align=align, pipe_mib=2) as sw, \
            torch.cuda.stream(stream):
        sw.checkpoint(stream)
        img = sw.image()
        diff = np.flatnonzero(img != ref)
        assert diff.size == 0, f"image differs at {diff[:8]} (manifest at {moff})"
        poison(arena, specs, offs)
        sw.restore(stream)
        res = sw.verify(stream, hbm_pass=True)
        assert (res["status"], res["n_bad"], res["hbm_n_bad"], res["first_bad_chunk"]) == (0, 0, 0, U64_MAX)
    torch.cuda.synchronize()
    back = arena.cpu().numpy()
    diff = np.flatnonzero(back != host)
    assert diff.size == 0, f"restored arena differs at {diff[:8]}"


SCRIPT = r'''
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1]); sys.path.insert(0, sys.argv[1] + "/tests")
import oracle as orc
from gpu_util import device_case, poison
from test_gpu_alignment import skewed_case
from paper_conf_sc_stoyanovsracb25_b200 import swap
specs, skew = skewed_case(32, 40)
arena, host, base, offs, sw_regions, or_regions = device_case(specs, 32, skew)
s = torch.cuda.Stream()
for kind, C in ((2, 1024), (2, 1 << 20), (1, 1024)):
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, C, 4096, threads=8)
    with swap.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism="ce_region") as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        assert np.array_equal(sw.image(), ref), (kind, C)
        poison(arena, specs, offs)
        sw.restore(s)
        r = sw.verify(s)
        assert r["status"] == 0 and r["hbm_n_bad"] == 0, (kind, C, r)
        assert np.array_equal(arena.cpu().numpy(), host), (kind, C)
print("skew ok")
'''


@pytest.mark.parametrize("variant", ["lane8", "bal", "dyn", "coop", "coop16", "coop8", "ring"])
def test_skewed_xxh64_hash_kernels(variant):
    """The XXH64 HBM hash kernels forced in turn (SWAP_XXH_KERNEL) on 16-B-aligned chunk starts."""
    env = dict(os.environ, SWAP_XXH_KERNEL=variant)
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], capture_output=True, text=True, env=env, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    assert "skew ok" in out.stdout
