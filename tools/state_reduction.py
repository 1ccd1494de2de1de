#!/usr/bin/env python
"""NEXT-3 measurement on config B (Llama-3.1-8B engine, 52.57 GB): swap-out / swap-in through a VMM
arena (real HBM release + re-acquire) with every region SAVE (full image, the bench's workload) vs the
engine-aware policy (weights SAVE_ONCE, KV pool DISCARD, workspace SAVE — the analogue of vLLM sleep
level 2), and weights SAVE_ONCE + KV SAVE with a touched-block mask (a fresh random
25 % of the KV pool's 1-MiB chunks per swap-out: only those move, the rest come back as zeros —
swap_set_chunk_mask, reading 25). Times are host wall clock around the C-ABI calls; prints one JSON line."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Arena, Swapper  # noqa: E402

REPS = int(os.environ.get("REPS", "3"))
specs = W.config_b()
offs, total = W.place(specs)
stream = torch.cuda.Stream()
out = {"workload": "B: Llama-3.1-8B engine image, 291 regions, 52.57 GB", "reps": REPS}
arena = Arena(total)
base, view = arena.alloc(total)
W.fill_device_arena(view, specs, offs, seed=0)
regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
TOUCHED = float(os.environ.get("TOUCHED", "0.25"))
C = 1 << 20
rng = np.random.default_rng(0)
for name, pol in [("full", None), ("engine_aware", {W.KIND_WEIGHTS: "save_once", W.KIND_KV: "discard"}),
                  ("touched_kv", {W.KIND_WEIGHTS: "save_once"})]:
    with Swapper(regions) as sw, torch.cuda.stream(stream):
        if pol:
            for i, r in enumerate(specs):
                if r.kind in pol:
                    sw.set_region_policy(i, pol[r.kind])
        sw.bind_arena(arena)  # restore re-acquires the HBM itself, overlapped with the copies
        t_out, t_in, t_ck, t_rel, moved = [], [], [], [], []
        for rep in range(REPS + 1):
            kept_kv = 0
            if name == "touched_kv":  # the engine touched a new random subset of KV blocks
                for i, r in enumerate(specs):
                    if r.kind == W.KIND_KV:
                        keep = (rng.random(-(-r.nbytes // C)) < TOUCHED).astype(np.uint8)
                        sw.set_chunk_mask(i, keep)
                        kept_kv += int(keep.sum()) * C
            t0 = time.perf_counter()
            sw.checkpoint(stream, sync=True)  # gather + seal
            tc = time.perf_counter()
            arena.release()  # HBM back to the device
            t1 = time.perf_counter()
            t2 = time.perf_counter()
            sw.restore(stream)
            res = sw.verify(stream, hbm_pass=True)
            t3 = time.perf_counter()
            assert res["status"] == 0, res
            if rep:  # rep 0 is the snapshot after init (gathers SAVE_ONCE regions too)
                t_out.append(t1 - t0)
                t_ck.append(tc - t0)
                t_rel.append(t1 - tc)
                t_in.append(t3 - t1)
                moved.append(kept_kv)
        restored = sum(r.nbytes for r in specs if not pol or pol.get(r.kind) is None and r.kind != W.KIND_KV)
        restored += sum(r.nbytes for r in specs if pol and pol.get(r.kind) == "save_once")
        saved = sum(r.nbytes for r in specs if not pol or pol.get(r.kind) is None and r.kind != W.KIND_KV)
        if not pol:
            restored = saved = sum(r.nbytes for r in specs)
        if name == "touched_kv":  # + the touched KV blocks (mean over the timed reps)
            restored += int(statistics.mean(moved))
            saved += int(statistics.mean(moved))
        out[name] = {"bytes_saved_per_swap_out": saved, "bytes_restored_per_swap_in": restored, "swap_out_s": round(statistics.mean(t_out), 4),
                     "checkpoint_s": round(statistics.mean(t_ck), 4), "release_s": round(statistics.mean(t_rel), 4),
                     "swap_in_s": round(statistics.mean(t_in), 4), 
                     "swap_in_GBps_of_full_image": round(sum(r.nbytes for r in specs) / statistics.mean(t_in) / 1e9, 2),
                     "mechanism": sw.mechanism()}
        if name == "touched_kv":
            out[name]["kv_touched_fraction"] = TOUCHED
print(json.dumps(out), flush=True)
arena.close()
