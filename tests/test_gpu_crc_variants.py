"""Each CRC-32C HBM hash kernel (quad-line: base / b0f / zb; strand-staged with the per-chunk tensor-map
path and per-lane bulk copies for other segments: ts (19 warps), ts16) forced in turn through SWAP_CRC_KERNEL, in
a subprocess: the checkpoint's hash pass (HASH_STORE, copy-engine movers) must give the oracle's image byte
for byte, the restore's per-group checks and the HBM verify (HASH_CHECK) must pass, and a single flipped
byte in HBM must be reported as exactly its chunk. Chunk / segment sizes cover L1 = 1 KiB (strands shorter
than a stage), 4 KiB segments of 64 KiB chunks, the 256-KiB auto segments, 16 MiB chunks; regions are
placed 16-B skewed (tensor rows not aligned to the arena), with ragged and empty regions, and a DISCARD
region (its chunks hashed from the zero buffer: never the tensor path)."""
import os
import subprocess
import sys

import pytest

from conftest import ROOT

pytestmark = pytest.mark.gpu

SCRIPT = r'''
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1]); sys.path.insert(0, sys.argv[1] + "/tests")
import oracle as orc, workloads as W
from gpu_util import device_case, poison
from paper_conf_sc_stoyanovsracb25_b200 import swap
s = torch.cuda.Stream()
for C, seg in ((1024, 0), (1 << 16, 4096), (1 << 20, 0), (1 << 20, 1 << 18), (16 << 20, 0)):
    E = W.edge_tables(C)
    specs = W.config_a(12) + E["chunk_pm1"] + E["with_empty"]
    skew = [16 * ((i * 7) % 9) for i in range(len(specs))]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 12, skew)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, 1, C, 4096, threads=8)
    assert rc == 0
    firsts, g = [], 0
    for r in specs:
        firsts.append(g)
        g += -(-r.nbytes // C)
    big = max(range(len(specs)), key=lambda i: specs[i].nbytes)
    for mech in ("ce_region", "ce_pipe"):
        with swap.Swapper(sw_regions, chunk_bytes=C, checksum=1, mechanism=mech, pipe_mib=8, seg_bytes=seg) as sw, \
                torch.cuda.stream(s):
            sw.checkpoint(s)
            assert np.array_equal(sw.image(), ref), (C, seg, mech)
            poison(arena, specs, offs)
            sw.restore(s)
            r = sw.verify(s)
            assert r["status"] == 0 and r["n_bad"] == 0 and r["hbm_n_bad"] == 0, (C, seg, mech, r)
            assert np.array_equal(arena.cpu().numpy(), host), (C, seg, mech)
            for o in (0, specs[big].nbytes // 2 + 5, specs[big].nbytes - 1):
                pos = offs[big] + o
                arena[pos] ^= 0x20
                torch.cuda.synchronize()
                r = sw.verify(s, raise_on_corrupt=False)
                want = firsts[big] + o // C
                assert (r["hbm_n_bad"], r["hbm_first_bad"]) == (1, want), (C, seg, mech, o, r)
                arena[pos] ^= 0x20
                torch.cuda.synchronize()
    # DISCARD: the region's chunks are hashed from the zero buffer at checkpoint
    pol = [orc.DISCARD if i == big else orc.SAVE for i in range(len(specs))]
    with swap.Swapper(sw_regions, chunk_bytes=C, checksum=1, mechanism="ce_region", seg_bytes=seg) as sw, \
            torch.cuda.stream(s):
        sw.set_region_policy(big, "discard")
        sw.checkpoint(s)
        rc, ref2, _ = orc.checkpoint(or_regions, orc.policy_view(or_regions, pol, host, host, base), base, 1, C, 4096,
                                     threads=8)
        assert np.array_equal(sw.image(), ref2), (C, seg, "discard")
        sw.restore(s)
        r = sw.verify(s)
        assert r["status"] == 0 and r["hbm_n_bad"] == 0, (C, seg, "discard", r)
print("variant ok")
'''


@pytest.mark.parametrize("variant", ["base", "b0f", "zb", "ts", "ts16", "mx", "mx16"])
def test_crc32c_kernel_variant(variant):
    env = dict(os.environ, SWAP_CRC_KERNEL=variant)
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], capture_output=True, text=True, env=env, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    assert "variant ok" in out.stdout
