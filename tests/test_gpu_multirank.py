"""N>1 path of bench.py (torchrun, one process per rank) on a single GPU: ranks share cuda:0
and the collectives (K5 summary all-gather, K6 mismatch all-reduce, max-over-ranks timing)
run over gloo. The NCCL variant differs only in where the 64-B / 8-B tensors live."""
import json
import os
import subprocess
import sys

import pytest

from conftest import ROOT

pytestmark = pytest.mark.gpu


@pytest.mark.timeout(600)
def test_bench_two_ranks_gloo():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29533", os.path.join(ROOT, "bench.py"), "--gpus", "2",
           "--config", "A", "--steps", "2", "--warmup", "1", "--no-compare", "--no-cpu-baseline",
           "--dist-backend", "gloo", "--force-legs"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=540, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout  # rank 0 alone prints
    rec = json.loads(lines[0])
    assert rec["n_gpus"] == 2 and rec["scaling"] == "weak" and rec["value"] > 0
    assert rec["config"]["payload_bytes_per_rank"] == 1 << 26
    assert rec["gpu_launches"] > 0
    # the N>1 legs, forced on one device: helper = the target GPU (degenerate), two DP replicas over gloo
    for mode in ("fused", "copy"):
        assert "error" not in rec["assisted_swap_in"]["1"][mode], rec["assisted_swap_in"]
        assert rec["assisted_swap_in"]["1"][mode]["GBps"] > 0
    dp = rec["dp_replicas"]
    assert "error" not in dp and dp["replicas"] == 2 and dp["striped_swap_in_s"] > 0, dp
    assert isinstance(dp["striped_fused_pull_swap_in_s"], float), dp


@pytest.mark.timeout(900)
def test_bench_two_ranks_gloo_config_d():
    """The N>1 code path at full per-rank size: two config-D shards (Llama-3.1-70B TP=8, 30.5 GB each) share
    cuda:0; the line carries per-rank placement, the copy-engine peak measured on all ranks at once, the
    topology record and clock samples; per-step max over ranks drives the value."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29535", os.path.join(ROOT, "bench.py"), "--gpus", "2",
           "--config", "D", "--steps", "2", "--warmup", "1", "--no-compare", "--no-cpu-baseline",
           "--dist-backend", "gloo"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=840, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    rec = json.loads(lines[0])
    assert rec["n_gpus"] == 2 and rec["value"] > 0 and "shrunk" not in rec["metric"]
    assert rec["config"]["payload_bytes_per_rank"] > 30e9
    assert [p["rank"] for p in rec["placement"]] == [0, 1]
    assert len(rec["measured_ce_GBps_all_ranks"]) == 2
    assert rec["topology"]["numa_nodes"] and rec["clocks"]["samples"] > 0
    lo, hi = rec["swap_in_latency_s_range"]
    assert lo <= rec["swap_in_latency_s"] <= hi


@pytest.mark.timeout(600)
def test_bench_two_ranks_legs_watchdog():
    """A hang in the N>1 legs must not cost the measured line: with a legs timeout shorter than the legs, every
    rank abandons them, rank 0 prints the line (with a legs_note and what the legs had recorded) and the job
    exits 0."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29537", os.path.join(ROOT, "bench.py"), "--gpus", "2",
           "--config", "A", "--steps", "2", "--warmup", "1", "--no-compare", "--no-cpu-baseline",
           "--dist-backend", "gloo", "--force-legs", "--legs-timeout", "0.01"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=540, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    rec = json.loads(lines[0])
    assert rec["n_gpus"] == 2 and rec["value"] > 0
    assert "timeout" in rec["legs_note"]
