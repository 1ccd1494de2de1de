#!/usr/bin/env python
"""A short, profiler-friendly round trip (checkpoint + restore + HBM verify) of the config-B region mix
scaled to --gib GiB, for ncu captures of one kernel at a realistic size (no timing printed)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Swapper  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gib", type=float, default=8)
ap.add_argument("--config", default="scaled", choices=["scaled", "A", "B", "D"],
                help="A: the 64-MiB parity/bench case (seed 0); B/D: the full bench workloads")
ap.add_argument("--mechanism", default="auto")
ap.add_argument("--checksum", default="crc32c")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--chunk", type=int, default=1 << 20)
a = ap.parse_args()
specs = {"A": lambda: W.config_a(0), "B": W.config_b, "D": lambda: W.config_d(0)}.get(a.config, lambda: W.scaled(W.config_b(), int(a.gib * (1 << 30))))()
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=1)
regions = [(arena.data_ptr() + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
s = torch.cuda.Stream()
with Swapper(regions, mechanism=a.mechanism, checksum=1 if a.checksum == "crc32c" else 2, chunk_bytes=a.chunk) as sw, \
        torch.cuda.stream(s):
    for _ in range(a.reps):
        sw.checkpoint(s)
        sw.restore(s)
        assert sw.verify(s)["status"] == 0
print("prof_case ok", a.mechanism)
