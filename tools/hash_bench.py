#!/usr/bin/env python
"""HBM verify-pass timing (a8) on the config-B region mix: checkpoint once, restore once, then
--reps verify passes timed with the library's CUDA events (swap_get_timings). Prints one JSON line.
Kernel variants are picked with SWAP_XXH_KERNEL / SWAP_CRC_KERNEL in the environment."""
import argparse
import json
import os
import statistics
import time
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Swapper  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gib", type=float, default=0, help="0 = full config B")
ap.add_argument("--checksum", default="crc32c")
ap.add_argument("--chunk", type=int, default=1 << 20)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--gap-ms", type=float, default=0, help="idle time before each verify (bench-like boost clocks)")
ap.add_argument("--variants", default="", help="comma list of kernel variants (SWAP_XXH_KERNEL for xxh64, "
                "SWAP_CRC_KERNEL for crc32c), interleaved in-process")
ap.add_argument("--all", action="store_true", help="print every rep's time")
a = ap.parse_args()
specs = W.config_b() if not a.gib else W.scaled(W.config_b(), int(a.gib * (1 << 30)))
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=1)
regions = [(arena.data_ptr() + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
payload = sum(r.nbytes for r in specs)
s = torch.cuda.Stream()
with Swapper(regions, mechanism="sm", checksum=1 if a.checksum == "crc32c" else 2, chunk_bytes=a.chunk) as sw, \
        torch.cuda.stream(s):
    sw.checkpoint(s)
    sw.restore(s)
    variants = a.variants.split(",") if a.variants else [None]
    env_key = "SWAP_XXH_KERNEL" if a.checksum == "xxh64" else "SWAP_CRC_KERNEL"
    ms = {v: [] for v in variants}
    for r in range(a.reps + 2):
        for v in variants:
            if v is not None:
                os.environ[env_key] = v
            if a.gap_ms:
                torch.cuda.synchronize()
                time.sleep(a.gap_ms * 1e-3)
            assert sw.verify(s)["status"] == 0
            if r >= 2:
                ms[v].append(sw.timings()["verify_ms"])
for v in variants:
    med = statistics.median(ms[v])
    print(json.dumps({"checksum": a.checksum, "chunk": a.chunk, "payload": payload,
                      "variant": v if v is not None else os.environ.get("SWAP_XXH_KERNEL", "") + os.environ.get("SWAP_CRC_KERNEL", ""),
                      "verify_ms": round(med, 3), "min_ms": round(min(ms[v]), 3), "max_ms": round(max(ms[v]), 3),
                      "TBps": round(payload / (med * 1e-3) / 1e12, 3),
                      "all_ms": [round(x, 2) for x in ms[v]] if a.all else None}), flush=True)
