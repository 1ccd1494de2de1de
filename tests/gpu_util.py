"""Helpers shared by the GPU parity tests (harness only: placement, poisoning, comparisons)."""
from __future__ import annotations

import struct

import numpy as np

import workloads as W

CHK = struct.Struct("<IIQQQ")


def device_case(specs, seed, skew=None):
    """Seeded arena on the GPU plus the region tables for the Swapper and for the oracle."""
    import torch

    host, offs = W.host_arena(specs, seed, skew)
    arena = torch.from_numpy(host).cuda()
    base = arena.data_ptr()
    sw_regions = [(base + o, r.nbytes, r.kind, 100 + i) for i, (r, o) in enumerate(zip(specs, offs))]
    or_regions = [(100 + i, base + o, r.nbytes, r.kind) for i, (r, o) in enumerate(zip(specs, offs))]
    return arena, host, base, offs, sw_regions, or_regions


def poison(arena, specs, offs):
    for r, o in zip(specs, offs):
        if r.nbytes:
            arena[o:o + r.nbytes].fill_(W.POISON_BYTE)


def chunk_records(manifest: np.ndarray, n_regions: int, n_chunks: int):
    base = 64 + 48 * n_regions
    return [CHK.unpack_from(manifest, base + 32 * g) for g in range(n_chunks)]
