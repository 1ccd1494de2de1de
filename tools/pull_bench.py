#!/usr/bin/env python
"""Throughput of the fused pull kernel (swap_pull_stripes: SM mover SCATTER reading a replica's copy, chunk
check from the same registers) on one GPU, the "peer" being a second arena in this process: the kernel's
own capacity, to set against the ~770 GB/s per direction a real NVLink peer read would offer.

    python tools/pull_bench.py [--gib 8] [--checksum crc32c] [--chunk 1048576] [--stripes 2]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200 import swap  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gib", type=float, default=8)
ap.add_argument("--checksum", default="crc32c")
ap.add_argument("--chunk", type=int, default=1 << 20)
ap.add_argument("--stripes", type=int, default=2)
ap.add_argument("--reps", type=int, default=5)
a = ap.parse_args()
specs = W.scaled(W.config_b(), int(a.gib * (1 << 30)))
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=2)
peer = arena.clone()
base = arena.data_ptr()
regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
kind = 1 if a.checksum == "crc32c" else 2
s = torch.cuda.Stream()
k = a.stripes
with swap.Swapper(regions, chunk_bytes=a.chunk, checksum=kind, pipe_mib=64) as sw, torch.cuda.stream(s):
    sw.checkpoint(s)
    spans = sw.restore_spans()
    pulled = sum(nb for (g, _, _, nb) in spans if g % k != 0)
    deltas = [0] + [peer.data_ptr() - base] * (k - 1)
    ms = []
    for r in range(a.reps + 1):
        sw.restore_stripe(0, k, s)
        s.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        sw.pull_stripes(0, k, deltas, s)
        e1.record(s)
        res = sw.verify(s)
        assert res["status"] == 0 and res["n_bad"] == 0, res
        if r:
            ms.append(e0.elapsed_time(e1))
t = statistics.median(ms)
print(json.dumps({"checksum": a.checksum, "chunk": a.chunk, "stripes": k, "pulled_bytes": pulled, "pull_ms": round(t, 3),
                  "GBps": round(pulled / (t * 1e-3) / 1e9, 1),
                  "note": "HBM -> HBM on one device (read + write per pulled byte); an NVLink peer read offers ~770 GB/s"}))
