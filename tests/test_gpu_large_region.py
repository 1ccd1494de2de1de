"""Maximum-size parity: one region larger than 4 GiB (offsets, segment and chunk indices past 32 bits
of bytes), plus ragged neighbours, with the largest chunk the product accepts (2 GiB, SURVEY §8(c)
reading 5 / DESIGN.md reading 5) and the default 1 MiB. Whole image (payload, padding, manifest) and
the whole restored arena compared byte for byte with the oracle, through the C ABI."""
import numpy as np
import pytest

import workloads as W
from gpu_util import device_case, poison

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

BIG = (5 << 30) + 13  # > 4 GiB, ragged tail
SPECS = [W.RegionSpec("big", W.KIND_KV, BIG), W.RegionSpec("r1", W.KIND_OTHER, (1 << 20) + 1),
         W.RegionSpec("r2", W.KIND_OTHER, 17)]


@pytest.fixture(scope="module")
def case():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    free, _ = torch.cuda.mem_get_info()
    if free < 2 * BIG:
        pytest.skip("needs ~11 GB of free HBM")
    return device_case(SPECS, 7)


@pytest.mark.parametrize("C,kind,mech", [(1 << 20, 1, "auto"), (1 << 20, 2, "auto"), (1 << 31, 1, "sm"),
                                         (1 << 31, 1, "ce_pipe"), (1 << 31, 2, "sm")],
                         ids=["1MiB-crc-auto", "1MiB-xxh-auto", "2GiB-crc-sm", "2GiB-crc-cepipe", "2GiB-xxh-sm"])
def test_region_over_4gib(case, C, kind, mech):
    import oracle as orc
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    arena, host, base, offs, sw_regions, or_regions = case
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, C, 4096, threads=16)
    assert rc == 0
    s = torch.cuda.Stream()
    with swap.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=mech) as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        img = sw.image()
        assert img.size == ref.size
        diff = np.flatnonzero(img != ref)
        assert diff.size == 0, f"image differs at {diff[:8]} (manifest at {moff})"
        poison(arena, SPECS, offs)
        sw.restore(s)
        res = sw.verify(s, hbm_pass=True)
        assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0
    torch.cuda.synchronize()
    back = arena.cpu().numpy()
    assert np.array_equal(back, host), "restored arena differs"
