"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests, smoke() and bench.py.

This module holds NONE of the method's arithmetic (no layout, chunking, checksum or
manifest code). It only says which regions an engine registers (sizes, kinds and the
model shapes behind them), where the harness places them in one device arena, and
what bytes they hold. Recipes follow SURVEY.md §8(d) "Synthetic inputs per config",
restated in DESIGN.md §"Input recipe"; the model shapes are the public HF configs of
SURVEY.md Appendix A (BASELINE.json configs[0..3]).
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np

KIND_WEIGHTS, KIND_KV, KIND_WORKSPACE, KIND_OTHER = 0, 1, 2, 3
GUARD_BYTE = 0xA5  # fills the gaps between regions in the arena (must never change)
POISON_BYTE = 0x5A  # written over every region between checkpoint and restore
BASE_ALIGN = 256  # cudaMalloc-like base alignment of each region in the arena
GUARD_BYTES = 4096  # gap before/after every region

GiB = 1 << 30
MiB = 1 << 20
KiB = 1 << 10


@dataclass(frozen=True)
class RegionSpec:
    name: str
    kind: int
    nbytes: int
    dtype: str = "bytes"  # "bf16" (weights, N(0, 0.02)) or "bytes" (uniform random bytes)


# ---------------------------------------------------------------- config A
def config_a(seed: int) -> list[RegionSpec]:
    """BASELINE.json configs[0]: 64 MiB, 16 random-size regions.

    15 cut points uniform in [1, 2^26 - 1] (numpy PCG64 seeded), sorted; sizes are the
    differences, so they sum to exactly 2^26 and are generally not multiples of 16.
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    cuts = np.sort(rng.integers(1, (1 << 26) - 1, size=15, endpoint=True))
    edges = np.concatenate([[0], cuts, [1 << 26]])
    sizes = np.diff(edges).astype(np.int64)
    kinds = [KIND_WEIGHTS] * 8 + [KIND_KV] * 4 + [KIND_WORKSPACE] * 3 + [KIND_OTHER]
    return [RegionSpec(f"a{seed}.r{i}", kinds[i], int(s)) for i, s in enumerate(sizes)]


# ---------------------------------------------------------------- engine images
def _workspace(seed: int, total: int, count: int = 64) -> list[RegionSpec]:
    """count workspace regions, log-uniform 4 KiB .. 256 MiB, scaled to sum exactly `total`."""
    rng = np.random.Generator(np.random.PCG64(seed))
    raw = np.exp(rng.uniform(math.log(4 * KiB), math.log(256 * MiB), size=count))
    sizes = np.floor(raw / raw.sum() * total).astype(np.int64)
    sizes[-1] += total - int(sizes.sum())
    return [RegionSpec(f"ws{i}", KIND_WORKSPACE, int(s)) for i, s in enumerate(sizes)]


def _bf16(name: str, *shape: int) -> RegionSpec:
    return RegionSpec(name, KIND_WEIGHTS, 2 * math.prod(shape), "bf16")


def _decoder_weights(vocab_shard: int, hidden: int, layers: int, qkv_rows: int, o_cols: int,
                     inter_shard: int, qkv_bias: bool) -> list[RegionSpec]:
    """vLLM-style fused layout: embed, lm_head, final norm, then per layer
    qkv [qkv_rows, hidden] (+bias), o [hidden, o_cols], gate_up [2*inter_shard, hidden],
    down [hidden, inter_shard], input/post-attention norms [hidden]."""
    out = [_bf16("embed", vocab_shard, hidden), _bf16("lm_head", vocab_shard, hidden), _bf16("norm", hidden)]
    for l in range(layers):
        out.append(_bf16(f"l{l}.qkv", qkv_rows, hidden))
        if qkv_bias:
            out.append(_bf16(f"l{l}.qkv_bias", qkv_rows))
        out += [
            _bf16(f"l{l}.o", hidden, o_cols),
            _bf16(f"l{l}.gate_up", 2 * inter_shard, hidden),
            _bf16(f"l{l}.down", hidden, inter_shard),
            _bf16(f"l{l}.in_norm", hidden),
            _bf16(f"l{l}.post_norm", hidden),
        ]
    return out


def config_b() -> list[RegionSpec]:
    """BASELINE.json configs[1]: Llama-3.1-8B bf16 engine on 1 GPU.

    195 weight regions (16.06 GB) + 32 KV regions x 1 GiB (2^18 tokens x 4 KiB/token/layer)
    + 64 workspace regions (2 GiB) = 291 regions, 52.57 GB.
    """
    w = _decoder_weights(128256, 4096, 32, 6144, 4096, 14336, qkv_bias=False)
    kv = [RegionSpec(f"kv{l}", KIND_KV, GiB) for l in range(32)]
    return w + kv + _workspace(1, 2 * GiB)


def config_c(rank: int) -> list[RegionSpec]:
    """BASELINE.json configs[2]: Qwen2.5-32B bf16 TP=2, one rank's shard (579 regions, 69.27 GB)."""
    w = _decoder_weights(76032, 5120, 64, 3584, 2560, 13824, qkv_bias=True)
    kv = [RegionSpec(f"kv{l}", KIND_KV, 512 * MiB) for l in range(64)]
    return w + kv + _workspace(100 + rank, 2 * GiB)


def config_d(rank: int) -> list[RegionSpec]:
    """BASELINE.json configs[3]: Llama-3.1-70B bf16 TP=8, one rank's shard (627 regions, 30.53 GB)."""
    w = _decoder_weights(16032, 8192, 80, 1280, 1024, 3584, qkv_bias=False)
    kv = [RegionSpec(f"kv{l}", KIND_KV, 128 * MiB) for l in range(80)]
    return w + kv + _workspace(200 + rank, 2 * GiB)


# ---------------------------------------------------------------- config E engines (hot-swap trace)
# BASELINE.json configs[4]: three engines (8B / 14B / 32B TP=2) swapped on GPU pairs. Per-GPU KV pool
# bytes/token/layer = 2 (K,V) x kv_heads/TP x head_dim 128 x 2 B. SURVEY.md §8(d) E uses 2^17 tokens;
# the one-GPU replay in tools/trace_e.py uses kv_tokens = 2^16 so that every engine's pinned image
# (about 158 GB in total) fits the GPU box's 196 GB of host RAM (DESIGN.md §"Config E").
def engine_e(model: str, rank: int = 0, kv_tokens: int = 1 << 16) -> list[RegionSpec]:
    if model == "8b":  # Llama-3.1-8B, TP=1
        w = _decoder_weights(128256, 4096, 32, 6144, 4096, 14336, qkv_bias=False)
        layers, kv_per_tok = 32, 2 * 8 * 128 * 2
    elif model == "14b":  # DeepSeek-R1-Distill-Qwen-14B / Qwen2.5-14B, TP=1
        w = _decoder_weights(152064, 5120, 48, 7168, 5120, 13824, qkv_bias=True)
        layers, kv_per_tok = 48, 2 * 8 * 128 * 2
    elif model == "32b":  # Qwen2.5-32B, TP=2 shard `rank`
        w = _decoder_weights(76032, 5120, 64, 3584, 2560, 13824, qkv_bias=True)
        layers, kv_per_tok = 64, 2 * 4 * 128 * 2
    else:
        raise ValueError(model)
    kv = [RegionSpec(f"kv{l}", KIND_KV, kv_tokens * kv_per_tok) for l in range(layers)]
    return w + kv + _workspace(300 + 10 * {"8b": 0, "14b": 1, "32b": 2}[model] + rank, 2 * GiB)


def trace_e(seed: int, duration_s: float, rate_per_s: float = 0.25, day_s: float = 600.0,
            shares=(("8b", 0.5), ("14b", 0.3), ("32b", 0.2)), burst_on_s: float = 30.0,
            burst_off_s: float = 120.0, burst_factor: float = 10.0, service_mean_s: float = 2.0):
    """Azure-shaped arrivals for config E (Fig. 1 shape):
    non-homogeneous Poisson with a diurnal sinusoid (one "day" = day_s seconds) times an on/off
    burst process (exponential ON/OFF periods, rate x burst_factor while ON), model shares, and
    lognormal service times with the given mean (sigma 0.5). Returns [(t, model, service_s)]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    # burst switching times
    edges, t, on = [], 0.0, False
    while t < duration_s:
        t += rng.exponential(burst_on_s if on else burst_off_s)
        edges.append((t, not on))
        on = not on
    lam_max = rate_per_s * 1.8 * burst_factor
    out, t, k, on = [], 0.0, 0, False
    names = [m for m, _ in shares]
    probs = np.array([p for _, p in shares]) / sum(p for _, p in shares)
    sigma = 0.5
    mu = math.log(service_mean_s) - sigma * sigma / 2
    while True:
        t += rng.exponential(1.0 / lam_max)  # thinning
        if t >= duration_s:
            break
        while k < len(edges) and edges[k][0] <= t:
            on = edges[k][1]
            k += 1
        lam = rate_per_s * (1.0 + 0.8 * math.sin(2 * math.pi * t / day_s)) * (burst_factor if on else 1.0)
        if rng.random() * lam_max <= lam:
            out.append((t, names[int(rng.choice(len(names), p=probs))], float(rng.lognormal(mu, sigma))))
    return out


def scaled(specs: list[RegionSpec], total: int) -> list[RegionSpec]:
    """Same region mix with every size scaled so the sum is about `total` (cheap GPU cases)."""
    s = sum(r.nbytes for r in specs)
    out = []
    for r in specs:
        nb = r.nbytes * total // s
        if r.dtype == "bf16":
            nb -= nb % 2
        out.append(RegionSpec(r.name, r.kind, nb, r.dtype))
    return out


# ---------------------------------------------------------------- edge tables
EDGE_SIZES = [1, 15, 16, 17, 511, 512, 513]


def edge_tables(chunk: int) -> dict[str, list[RegionSpec]]:
    """Degenerate and ragged tables (SURVEY §4 parity row)."""
    mk = lambda sizes, k=KIND_OTHER: [RegionSpec(f"e{i}", k, s) for i, s in enumerate(sizes)]
    return {
        "edge_sizes": mk(EDGE_SIZES),
        "one_chunk": mk([chunk]),
        "chunk_pm1": mk([chunk - 1, chunk + 1, 2 * chunk, 3 * chunk - 16]),
        "with_empty": mk([0, 100, 0, 4096 + 3, 0]),
        "many_tiny": mk([(i * 37) % 61 + 1 for i in range(300)]),
        "single_byte": mk([1]),
        "all_empty": mk([0, 0]),
    }


# ---------------------------------------------------------------- arena placement + contents
def place(specs: list[RegionSpec], skew: list[int] | None = None) -> tuple[list[int], int]:
    """Offsets of each region inside one device arena: BASE_ALIGN-aligned (plus skew[i] bytes, a
    multiple of 16, to exercise less-aligned device addresses), with GUARD_BYTES of guard before
    the first region, between regions and after the last."""
    offs, pos = [], GUARD_BYTES
    for i, r in enumerate(specs):
        pos = (pos + BASE_ALIGN - 1) // BASE_ALIGN * BASE_ALIGN + (skew[i] if skew else 0)
        offs.append(pos)
        pos += r.nbytes + GUARD_BYTES
    return offs, pos


def random_bytes(seed: int, nbytes: int) -> np.ndarray:
    """Uniform random bytes from numpy PCG64."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.integers(0, 256, size=nbytes, dtype=np.uint8)


def host_arena(specs: list[RegionSpec], seed: int, skew: list[int] | None = None) -> tuple[np.ndarray, list[int]]:
    """Arena bytes on the host: guard bytes everywhere, region contents seeded per region
    (uniform bytes; bf16 regions get N(0, 0.02) rounded to bf16)."""
    offs, total = place(specs, skew)
    arena = np.full(total, GUARD_BYTE, dtype=np.uint8)
    for i, (r, o) in enumerate(zip(specs, offs)):
        arena[o:o + r.nbytes] = region_bytes(r, seed * 1000003 + i)
    return arena, offs


def region_bytes(r: RegionSpec, seed: int) -> np.ndarray:
    if r.dtype == "bf16" and r.nbytes >= 2:
        rng = np.random.Generator(np.random.PCG64(seed))
        f = (rng.standard_normal(r.nbytes // 2).astype(np.float32) * np.float32(0.02))
        bits = f.view(np.uint32)
        bf = ((bits + 0x7FFF + ((bits >> 16) & 1)) >> 16).astype(np.uint16)  # round to nearest even
        out = bf.view(np.uint8)
        if r.nbytes % 2:
            out = np.concatenate([out, random_bytes(seed, 1)])
        return out
    return random_bytes(seed, r.nbytes)


def fill_device_arena(arena, specs: list[RegionSpec], offs: list[int], seed: int) -> None:
    """Fill a torch uint8 CUDA arena on the device (large configs): guards = GUARD_BYTE,
    weights N(0, 0.02) bf16, everything else uniform random bytes, from a seeded
    torch generator. Used where host generation of tens of GB would be too slow."""
    import torch

    arena.fill_(GUARD_BYTE)
    g = torch.Generator(device=arena.device)
    for i, (r, o) in enumerate(zip(specs, offs)):
        if r.nbytes == 0:
            continue
        g.manual_seed(seed * 1000003 + i)
        view = arena[o:o + r.nbytes]
        if r.dtype == "bf16" and r.nbytes % 2 == 0:
            w = torch.empty(r.nbytes // 2, dtype=torch.bfloat16, device=arena.device)
            w.normal_(0.0, 0.02, generator=g)
            view.copy_(w.view(torch.uint8))
            del w
        else:
            view.copy_(torch.randint(0, 256, (r.nbytes,), dtype=torch.uint8, device=arena.device, generator=g))
