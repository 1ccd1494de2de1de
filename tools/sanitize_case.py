"""compute-sanitizer workload: every kernel family and mover on small images (tools/sanitize.sh)."""
import os
import sys

ROOT = os.environ.get("GRAFT_REPO_ROOT", os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from gpu_util import device_case, poison  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200 import swap  # noqa: E402

s = torch.cuda.Stream()
specs = W.config_a(3)[:6] + W.edge_tables(4096)["edge_sizes"]
arena, host, base, offs, regions, _ = device_case(specs, 3)
for kind in (1, 2):
    for mech, extra in (("sm", {}), ("ce_pipe", {"pipe_mib": 4}), ("ce_region", {}), ("ce_batch", {})):
        for C in (4096, 1 << 20):
            with swap.Swapper(regions, chunk_bytes=C, checksum=kind, mechanism=mech, **extra) as sw, \
                    torch.cuda.stream(s):
                if mech == "ce_pipe":
                    sw.set_helpers([0])
                sw.set_region_policy(1, "discard")
                sw.checkpoint(s)
                poison(arena, specs, offs)
                sw.restore(s)
                assert sw.verify(s)["status"] == 0, (kind, mech, C)
# touched-chunk masks (zero-filled chunks, fragmented group copies under CE_PIPE, image zeroing)
for mech in ("ce_pipe", "sm"):
    with swap.Swapper(regions, chunk_bytes=4096, mechanism=mech, pipe_mib=1) as sw, torch.cuda.stream(s):
        big = max(range(len(specs)), key=lambda i: specs[i].nbytes)
        n = -(-specs[big].nbytes // 4096)
        for keep in (np.arange(n) % 3 == 0, np.arange(n) % 2 == 0):
            sw.set_chunk_mask(big, keep.astype(np.uint8))
            sw.checkpoint(s)
            poison(arena, specs, offs)
            sw.restore(s)
            assert sw.verify(s)["status"] == 0, mech
# XXH64 kernel variants are chosen by chunk count; a 1 KiB-chunk case exercises the lane kernel
with swap.Swapper(regions, chunk_bytes=1024, checksum=2, mechanism="ce_region") as sw, torch.cuda.stream(s):
    sw.checkpoint(s)
    sw.restore(s)
    assert sw.verify(s)["status"] == 0
# every XXH64 hash kernel, forced per launch through SWAP_XXH_KERNEL (the CE movers hash from HBM)
for v in ("lane8", "bal", "bal8", "dyn", "coop", "coop16", "coop8", "ring", "quad", "quad1k", "quad4k", "quad_x",
          "dyn_x", "quad2", "pair", "pair2", "quad3k"):
    os.environ["SWAP_XXH_KERNEL"] = v
    with swap.Swapper(regions, chunk_bytes=1024, checksum=2, mechanism="ce_region") as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        poison(arena, specs, offs)
        sw.restore(s)
        assert sw.verify(s)["status"] == 0, v
os.environ.pop("SWAP_XXH_KERNEL")
# the quad kernels' multi-stage rings: chunks of several stages (64 KiB) and a ragged tail
for v in ("quad", "quad2", "quad3k"):
    os.environ["SWAP_XXH_KERNEL"] = v
    with swap.Swapper(regions, chunk_bytes=1 << 16, checksum=2, mechanism="ce_region") as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        poison(arena, specs, offs)
        sw.restore(s)
        assert sw.verify(s)["status"] == 0, v
os.environ.pop("SWAP_XXH_KERNEL")
# CRC-32C hash kernel variants (fixed shared layout at the 0x400 dynamic base; the strand-staged ts kernels
# with their tensor-map path on standard segments and per-lane bulk copies on ragged ones, also with
# 128 KiB segments of 1 MiB chunks)
for v in ("base", "b0f", "zb", "zbb0f", "ts", "ts16", "mx", "mx16"):
    os.environ["SWAP_CRC_KERNEL"] = v
    for C, seg in ((1 << 16, 0), (1 << 20, 1 << 17)):
        with swap.Swapper(regions, chunk_bytes=C, checksum=1, mechanism="ce_region", seg_bytes=seg) as sw, \
                torch.cuda.stream(s):
            sw.checkpoint(s)
            poison(arena, specs, offs)
            sw.restore(s)
            assert sw.verify(s)["status"] == 0, v
os.environ.pop("SWAP_CRC_KERNEL")
# DP replicas in one process: stripe restore of replica A, then the fused pull of the other stripe from
# replica B (a second arena with the same bytes at a constant shift)
arena_b = arena.clone()
delta = arena_b.data_ptr() - arena.data_ptr()
for kind in (1, 2):
    with swap.Swapper(regions, chunk_bytes=4096, checksum=kind, pipe_mib=1) as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        poison(arena, specs, offs)
        sw.restore_stripe(0, 2, s)
        sw.pull_stripes(0, 2, [0, delta], s)
        assert sw.verify(s)["status"] == 0, kind
del arena_b
# VMM arenas + full-duplex exchange
def engine(seed):
    sp = W.scaled(W.config_b(), 48 << 20)
    of, total = W.place(sp)
    a = swap.Arena(total)
    b, view = a.alloc(total)
    W.fill_device_arena(view, sp, of, seed=seed)
    sw = swap.Swapper([(b + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(sp, of))], mechanism="ce_pipe",
                      pipe_mib=4)
    sw.bind_arena(a)
    return a, sw
a1, v1 = engine(1)
a2, inc = engine(2)
inc.swap_out(a2, s)
swap.exchange([v1], inc, s, s, headroom=0)
assert inc.verify(s)["status"] == 0
print("sanitize case ok")
