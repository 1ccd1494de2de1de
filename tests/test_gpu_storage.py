"""NEXT-4 storage tier: swap_save / swap_load persist a sealed image and bring it back bit-exactly
(the file is the image the oracle defines); corrupt or foreign files are refused."""
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


@pytest.mark.parametrize("kind", [1, 2], ids=["crc32c", "xxh64"])
def test_save_load_roundtrip(swp, orc, tmp_path, kind):
    specs = W.config_a(9) + W.edge_tables(4096)["edge_sizes"]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 9)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, 1 << 16, 4096, threads=8)
    path = str(tmp_path / "engine.swapimg")
    s = torch.cuda.Stream()
    with swp.Swapper(sw_regions, chunk_bytes=1 << 16, checksum=kind) as sw:
        with pytest.raises(swp.SwapError) as e:
            sw.save(path)  # nothing sealed yet
        assert e.value.status == swp.SWAP_ESTATE
        sw.checkpoint(s)
        sw.save(path)
    data = np.fromfile(path, dtype=np.uint8)
    assert np.array_equal(data, ref)  # the file is exactly the oracle's image
    poison(arena, specs, offs)
    with swp.Swapper(sw_regions, chunk_bytes=1 << 16, checksum=kind) as sw2, torch.cuda.stream(s):
        sw2.load_image(path)  # a fresh process would do exactly this
        sw2.restore(s)
        assert sw2.verify(s)["status"] == 0
        assert np.array_equal(arena.cpu().numpy(), host)
        # a flipped manifest byte is refused by the import checks
        bad = data.copy()
        bad[moff + 70] ^= 1
        bad.tofile(path)
        with pytest.raises(swp.SwapError) as e:
            sw2.load_image(path)
        assert e.value.status == swp.SWAP_ECORRUPT
        data[:-1].tofile(path)  # wrong size: not an image of this layout
        with pytest.raises(swp.SwapError) as e:
            sw2.load_image(path)
        assert e.value.status == swp.SWAP_ECORRUPT
