"""bench.py's reference arm (the CPU oracle) — runs without a GPU, single process and under torchrun."""
import json
import os
import subprocess
import sys

import pytest

from conftest import ROOT


def _lines(out):
    return [l for l in out.stdout.splitlines() if l.startswith("{")]


@pytest.mark.timeout(300)
def test_reference_arm_single():
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "A", "--steps", "2",
           "--warmup", "1", "--sample-bytes", str(1 << 24)]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=280, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    (line,) = _lines(out)
    rec = json.loads(line)
    assert rec["impl"] == "reference" and rec["unit"] == "GB/s" and rec["value"] > 0
    assert rec["e2e"]["h2d_bytes_per_step"] == 0 and rec["cpu_baseline"]["cores"] >= 1


@pytest.mark.timeout(300)
def test_reference_arm_two_ranks():
    # only rank 0 runs and prints; the other rank exits 0 without work
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29534", os.path.join(ROOT, "bench.py"), "--impl", "reference",
           "--gpus", "2", "--config", "A", "--steps", "2", "--warmup", "1", "--sample-bytes", str(1 << 24)]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=280, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    rec = json.loads(lines[0])
    assert rec["impl"] == "reference" and rec["cpu_baseline"]["kind"] == "oracle"


def test_host_helpers():
    sys.path.insert(0, ROOT)
    import bench
    import workloads as W

    assert bench.parse_cpulist("0-3,8,10-11") == [0, 1, 2, 3, 8, 10, 11]
    assert bench.parse_cpulist("") == []
    assert bench.numa_nodes()  # at least node 0
    topo = bench.topology()
    assert topo["numa_nodes"] and topo["cpu_model"]
    specs = W.config_d(0)
    # an image set that cannot fit is refused unless the shrink is asked for (and then it is named)
    with pytest.raises(SystemExit):
        bench.check_host(specs, 10 ** 4, allow_shrink=False)
    shrunk, scale = bench.check_host(specs, 10 ** 4, allow_shrink=True)
    assert scale < 1.0 and sum(r.nbytes for r in shrunk) < sum(r.nbytes for r in specs)
    assert bench.check_host(W.config_a(0), 1, allow_shrink=False) == (W.config_a(0), 1.0)
