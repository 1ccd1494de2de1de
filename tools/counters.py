#!/usr/bin/env python
"""Counter evidence for the mechanism crossover (BASELINE.json north_star: "ncu counters (achieved host-link
and HBM GB/s, DRAM and PCIe throughput) evidence which mechanism wins at each chunk size").

Each case -- mechanism x chunk size x direction -- is one cudaProfilerStart/Stop range around a single
checkpoint or restore of a config-B-shaped image (--gib GiB), so that under

    ncu --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,\
        dram__bytes_write.sum,gpu__time_duration.sum --csv --log-file gpurun_out/counters.csv \
        python tools/counters.py --cases-out gpurun_out/counter_cases.json

the counters cover the copy-engine transfers too (kernel replay sees only kernels). The ranges come in the
order written to --cases-out; tools/counters_table.py joins the two into the per-payload-byte table.
Run without ncu it just times the same ranges with CUDA events (a sanity check of the case list)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Swapper  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gib", type=float, default=1.0)
ap.add_argument("--chunks", default="4096,65536,1048576,16777216")
ap.add_argument("--mechs", default="sm,ce_region,ce_batch,ce_pipe")
ap.add_argument("--checksum", default="crc32c")
ap.add_argument("--cases-out", default=None)
a = ap.parse_args()

specs = W.scaled(W.config_b(), int(a.gib * (1 << 30)))
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=1)
regions = [(arena.data_ptr() + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
payload = sum(r.nbytes for r in specs)
s = torch.cuda.Stream()
cases = []


def poison():
    with torch.cuda.stream(s):
        for r, o in zip(specs, offs):
            if r.nbytes:
                arena[o:o + r.nbytes].fill_(W.POISON_BYTE)
    torch.cuda.synchronize()


def profiled(fn):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.profiler.start()
    e0.record(s)
    fn()
    e1.record(s)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    return e0.elapsed_time(e1)


for C in [int(x) for x in a.chunks.split(",")]:
    with Swapper(regions, chunk_bytes=C, checksum=1 if a.checksum == "crc32c" else 2) as sw, torch.cuda.stream(s):
        for m in a.mechs.split(","):
            sw.set_mechanism(m)
            sw.checkpoint(s)  # warm (unprofiled)
            ms = profiled(lambda: sw.checkpoint(s, sync=True))
            cases.append({"mechanism": m, "chunk": C, "phase": "checkpoint", "payload": payload, "event_ms": round(ms, 3)})
            poison()

            def rst():
                sw.restore(s)
                assert sw.verify(s, hbm_pass=False)["status"] == 0

            ms = profiled(rst)
            cases.append({"mechanism": m, "chunk": C, "phase": "restore", "payload": payload, "event_ms": round(ms, 3)})
for c in cases:
    print(json.dumps(c))
if a.cases_out:
    with open(a.cases_out, "w") as f:
        json.dump(cases, f)
