#!/usr/bin/env python
"""Mechanism x chunk-size x checksum sweep (SURVEY.md §8(d) "Baseline mechanisms in the same run";
BASELINE.json north_star: "evidence which mechanism wins at each chunk size").

For one seeded engine image (config B's region mix scaled to --gib GiB) and every chunk size,
checksum and mover: checkpoint / restore / HBM-verify throughput from libswap's own CUDA-event
timings (swap_get_timings), after one warm-up round trip. Writes JSON lines and a markdown table.

    python tools/sweep.py --gib 8 --out profiles/r01_sweep
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
ap.add_argument("--chunks", default="4096,65536,1048576,16777216")
ap.add_argument("--mechs", default="sm,ce_region,ce_chunk,ce_batch,ce_pipe")
ap.add_argument("--checksums", default="crc32c,xxh64")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--out", default="gpurun_out/sweep")
args = ap.parse_args()

specs = W.scaled(W.config_b(), int(args.gib * (1 << 30)))
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=5)
base = arena.data_ptr()
regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
payload = sum(r.nbytes for r in specs)
stream = torch.cuda.Stream()
rows = []
with open(args.out + ".jsonl", "w") as jf:
    for ck in args.checksums.split(","):
        kind = swap.SWAP_CHECKSUM_CRC32C if ck == "crc32c" else swap.SWAP_CHECKSUM_XXH64
        for C in [int(x) for x in args.chunks.split(",")]:
            sw = swap.Swapper(regions, chunk_bytes=C, checksum=kind, mechanism="sm")
            for m in args.mechs.split(","):
                sw.set_mechanism(m)
                t = {"checkpoint_ms": [], "restore_ms": [], "verify_ms": []}
                with torch.cuda.stream(stream):
                    for rep in range(args.reps + 1):
                        sw.checkpoint(stream)
                        for r, o in zip(specs, offs):
                            arena[o:o + r.nbytes].fill_(W.POISON_BYTE)
                        sw.restore(stream)
                        res = sw.verify(stream, hbm_pass=True)
                        assert res["status"] == 0, res
                        if rep:
                            for k, v in sw.timings().items():
                                t[k].append(v)
                rec = {"checksum": ck, "chunk": C, "mechanism": m, "payload": payload,
                       **{k.replace("_ms", "_GBps"): round(payload / (statistics.mean(v) * 1e-3) / 1e9, 2)
                          for k, v in t.items()}}
                rows.append(rec)
                jf.write(json.dumps(rec) + "\n")
                jf.flush()
                print(json.dumps(rec), flush=True)
            sw.close()

with open(args.out + ".md", "w") as f:
    f.write(f"# Mechanism sweep: config-B mix scaled to {payload / 1e9:.2f} GB, one B200\n\n")
    f.write("GB/s from libswap CUDA-event timings (mean of %d after 1 warm-up). verify = HBM pass.\n\n" % args.reps)
    f.write("| checksum | chunk | mechanism | checkpoint | restore | verify |\n|---|---|---|---|---|---|\n")
    for r in rows:
        f.write(f"| {r['checksum']} | {r['chunk']} | {r['mechanism']} | {r['checkpoint_GBps']} | "
                f"{r['restore_GBps']} | {r['verify_GBps']} |\n")
print("wrote", args.out + ".md")
