"""Touched-block mask probe: scaled config-B image, a fresh random KV mask per checkpoint, phase times
from the library's CUDA events (checkpoint / restore / verify) — for ncu launch lists of the mask path."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
import time  # noqa: E402

from paper_conf_sc_stoyanovsracb25_b200.swap import Arena, Swapper  # noqa: E402

GIB = float(os.environ.get("GIB", "8"))
FRAC = float(os.environ.get("TOUCHED", "0.25"))
specs = W.scaled(W.config_b(), int(GIB * (1 << 30)))
offs, total = W.place(specs)
ARENA = os.environ.get("ARENA") == "1"  # VMM arena released between checkpoint and restore
if ARENA:
    vmm = Arena(total)
    base, arena = vmm.alloc(total)
else:
    arena = torch.empty(total, dtype=torch.uint8, device="cuda")
    base = arena.data_ptr()
W.fill_device_arena(arena, specs, offs, seed=0)
C = 1 << 20
rng = np.random.default_rng(0)
s = torch.cuda.Stream()
with Swapper([(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]) as sw, \
        torch.cuda.stream(s):
    if ARENA:
        sw.bind_arena(vmm)
    for rep in range(int(os.environ.get("REPS", "3"))):
        for i, r in enumerate(specs):
            if r.kind == W.KIND_KV:
                sw.set_chunk_mask(i, (rng.random(-(-r.nbytes // C)) < FRAC).astype(np.uint8))
        t0 = time.perf_counter()
        sw.checkpoint(s)
        t1 = time.perf_counter()
        if ARENA:
            vmm.release()
        t2 = time.perf_counter()
        sw.restore(s)
        assert sw.verify(s)["status"] == 0
        t3 = time.perf_counter()
        print(rep, sw.mechanism(), {k: round(v, 2) for k, v in sw.timings().items()},
              f"wall ckpt {1e3 * (t1 - t0):.1f} ms swap-in {1e3 * (t3 - t2):.1f} ms", flush=True)
    if ARENA:
        sw.bind_arena(None)
