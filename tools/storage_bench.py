#!/usr/bin/env python
"""NEXT-4 measurement: swap_save / swap_load throughput of the config B image (52.57 GB) on the GPU
box's local filesystem (O_DIRECT, multi-threaded), then a restore from the loaded image. One JSON line."""
import json
import os
import shutil
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_sc_stoyanovsracb25_b200.swap import Swapper  # noqa: E402

path = sys.argv[1] if len(sys.argv) > 1 else "/tmp/swap_bench.img"
specs = W.config_b()
offs, total = W.place(specs)
arena = torch.empty(total, dtype=torch.uint8, device="cuda")
W.fill_device_arena(arena, specs, offs, seed=0)
base = arena.data_ptr()
regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
s = torch.cuda.Stream()
rec = {"workload": "B: Llama-3.1-8B engine image, 52.57 GB", "path": path}
st = os.statvfs(os.path.dirname(path) or ".")
rec["fs_free_GB"] = round(st.f_bavail * st.f_frsize / 1e9, 1)
with Swapper(regions) as sw, torch.cuda.stream(s):
    sw.checkpoint(s)
    n = sw.image().size
    if st.f_bavail * st.f_frsize < n * 1.05:
        rec["skipped"] = "not enough free space"
        print(json.dumps(rec))
        sys.exit(0)
    t0 = time.perf_counter()
    sw.save(path)
    t1 = time.perf_counter()
    rec["save_GBps"] = round(n / (t1 - t0) / 1e9, 2)
os.system("sync; echo 3 > /proc/sys/vm/drop_caches 2>/dev/null")
with Swapper(regions) as sw2, torch.cuda.stream(s):
    t0 = time.perf_counter()
    sw2.load_image(path)
    t1 = time.perf_counter()
    sw2.restore(s)
    res = sw2.verify(s)
    t2 = time.perf_counter()
    assert res["status"] == 0
    rec.update(load_GBps=round(n / (t1 - t0) / 1e9, 2), restore_after_load_s=round(t2 - t1, 3),
               image_bytes=n)
os.unlink(path)
print(json.dumps(rec), flush=True)
