"""Each XXH64 HBM hash kernel (lane per chunk 8 deep; balanced 4 / 8 deep; dynamic; warp-cooperative with
32 / 16 / 8 chunks per warp; TMA ring) forced in turn through
SWAP_XXH_KERNEL, in a subprocess, on many small chunks and on few large ones: images and verify
results bit-exact against the oracle."""
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
for C in (1024, 1 << 16, 16 << 20):
    specs = W.config_a(12) + W.edge_tables(C)["chunk_pm1"]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 12)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, 2, C, 4096, threads=8)
    for mech in ("ce_region", "ce_pipe"):
        with swap.Swapper(sw_regions, chunk_bytes=C, checksum=2, mechanism=mech, pipe_mib=8) as sw, torch.cuda.stream(s):
            sw.checkpoint(s)
            assert np.array_equal(sw.image(), ref), (C, mech)
            poison(arena, specs, offs)
            sw.restore(s)
            r = sw.verify(s)
            assert r["status"] == 0 and r["hbm_n_bad"] == 0, (C, mech, r)
            assert np.array_equal(arena.cpu().numpy(), host), (C, mech)
print("variant ok")
'''


@pytest.mark.parametrize("variant", ["lane8", "bal", "bal8", "dyn", "coop", "coop16", "coop8", "ring", "quad", "quad1k", "quad4k", "quad_x", "dyn_x", "quad2", "pair", "pair2"])
def test_xxh64_kernel_variant(variant):
    env = dict(os.environ, SWAP_XXH_KERNEL=variant)
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], capture_output=True, text=True, env=env, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    assert "variant ok" in out.stdout
