#!/usr/bin/env python
"""Config A (64 MiB) verify-pass time per CRC segment size (seg_bytes), interleaved in one process."""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from gpu_util import device_case, poison  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200 import swap  # noqa: E402

specs = W.config_a(0)
arena, host, base, offs, regions, _ = device_case(specs, 0)
s = torch.cuda.Stream()
segs = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "4096,8192,16384,32768,65536").split(",")]
sws = {g: swap.Swapper(regions, seg_bytes=g) for g in segs}
with torch.cuda.stream(s):
    for g, sw in sws.items():
        sw.checkpoint(s)
        sw.restore(s)
    ms = {g: [] for g in segs}
    for r in range(12):
        for g, sw in sws.items():
            assert sw.verify(s)["status"] == 0
            if r >= 2:
                ms[g].append(sw.timings()["verify_ms"])
for g in segs:
    print(f"seg {g >> 10:3d} KiB: verify {statistics.median(ms[g]) * 1e3:.1f} us")
