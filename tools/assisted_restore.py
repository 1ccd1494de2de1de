#!/usr/bin/env python
"""NEXT-2 experiment for a multi-GPU node (not runnable on the one-GPU pool of round 1): restore the
config B image (52.57 GB) onto GPU 0 with k idle peers helping (k = 0, 1, 3, 7 by default): each helper
pulls its share of the pipeline groups over its own PCIe link into HBM staging and forwards it over
NVLink. Prints one JSON line with swap-in seconds and GB/s per k.

    python tools/assisted_restore.py --helpers 0,1,3,7
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Swapper  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--helpers", default="0,1,3,7")
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
ndev = torch.cuda.device_count()
specs = W.config_b()
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda:0")
W.fill_device_arena(arena, specs, offs, seed=0)
regions = [(arena.data_ptr() + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
payload = sum(r.nbytes for r in specs)
out = {"workload": "B: Llama-3.1-8B engine image restored onto GPU 0", "devices": ndev, "results": {}}
s = torch.cuda.Stream(device=0)
with Swapper(regions, mechanism="ce_pipe", device=0) as sw, torch.cuda.stream(s):
    sw.checkpoint(s)
    for k in [int(x) for x in a.helpers.split(",")]:
        if k >= ndev:
            out["results"][k] = "skipped: not enough GPUs"
            continue
        sw.set_helpers(list(range(1, k + 1)))
        ts = []
        for rep in range(a.reps + 1):
            arena.fill_(0x5A)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            sw.restore(s)
            res = sw.verify(s)
            t1 = time.perf_counter()
            assert res["status"] == 0, res
            if rep:
                ts.append(t1 - t0)
        out["results"][k] = {"swap_in_s": round(statistics.mean(ts), 4),
                             "GBps": round(payload / statistics.mean(ts) / 1e9, 2)}
    sw.set_helpers([])
print(json.dumps(out), flush=True)
