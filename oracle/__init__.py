"""CPU oracle of the swap-image hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package. The product package
(``paper_conf_sc_stoyanovsracb25_b200``) never imports it and shares no code with it.

The arithmetic lives in ``oracle.c`` (plain C, one function per step of SURVEY.md
§8(c), the DESIGN.md reading of PAPER.md L130 §3.2 / L171 §4.2 "in-memory snapshot
of the GPU state"). This module is ctypes marshalling only.

Parity status: every function here is pinned by an external fact (tests/test_oracle.py):
RFC 3720 §B.4 CRC-32C vectors, the xxHash spec vectors and the ``xxhash`` library,
SSE4.2 hardware CRC, the zlib CRC combine algebra, a byte-at-a-time layout builder
(brute force), round-trip identity and single-bit fault detection. Against the paper
itself parity is unpinned: the paper prints no image or checksum values.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liboracle.so")

OK, EINVAL, ECORRUPT = 0, -1, -5
CRC32C, XXH64 = 1, 2


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so with gcc (plain C11 + OpenMP)."""
    src = os.path.join(HERE, "oracle.c")
    if not force and os.path.exists(LIB_PATH) and os.path.getmtime(LIB_PATH) >= max(
        os.path.getmtime(src), os.path.getmtime(os.path.join(HERE, "oracle.h"))
    ):
        return LIB_PATH
    tmp = LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(
        ["gcc", "-std=c11", "-O2", "-fopenmp", "-fPIC", "-shared", "-Wall", "-o", tmp, src]
    )
    os.replace(tmp, LIB_PATH)
    return LIB_PATH


class _Region(ctypes.Structure):
    _fields_ = [
        ("addr", ctypes.c_uint64),
        ("bytes", ctypes.c_uint64),
        ("id", ctypes.c_uint32),
        ("kind", ctypes.c_uint32),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        u8p, u64, u32, u64p = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint64)
        L = _lib
        for name in ("oracle_crc32c_bitwise", "oracle_crc32c_table", "oracle_crc32c_sse42"):
            getattr(L, name).argtypes = [u8p, u64]
            getattr(L, name).restype = u32
        L.oracle_have_sse42.restype = ctypes.c_int
        L.oracle_crc32c_combine.argtypes = [u32, u32, u64]
        L.oracle_crc32c_combine.restype = u32
        L.oracle_xxh64.argtypes = [u8p, u64, u64]
        L.oracle_xxh64.restype = u64
        L.oracle_chunk_hash.argtypes = [u32, u8p, u64]
        L.oracle_chunk_hash.restype = u64
        L.oracle_plan.argtypes = [ctypes.c_void_p, u64, u64, u64, u64p, u64p, u64p, u64p, u64p]
        L.oracle_plan.restype = ctypes.c_int
        L.oracle_manifest_bytes.argtypes = [u64, u64]
        L.oracle_manifest_bytes.restype = u64
        L.oracle_image_layout.argtypes = [ctypes.c_void_p, u64, u64, u64, u64p, u64p]
        L.oracle_image_layout.restype = ctypes.c_int
        L.oracle_checkpoint.argtypes = [ctypes.c_void_p, u64, u8p, u64, u64, u32, u64, u64, u32, u32, u8p, u64, ctypes.c_int]
        L.oracle_checkpoint.restype = ctypes.c_int
        L.oracle_summary.argtypes = [u8p, u64, u64, u8p]
        L.oracle_summary.restype = ctypes.c_int
        L.oracle_global_digest.argtypes = [u8p, u64]
        L.oracle_global_digest.restype = u32
        for name in ("oracle_restore", "oracle_restore_fast"):
            getattr(L, name).argtypes = [u8p, u64, u8p, u64, u64, u64p, u64p, ctypes.c_int]
            getattr(L, name).restype = ctypes.c_int
        L.oracle_verify.argtypes = [u8p, u8p, u64, u64, u64p, u64p, ctypes.c_int]
        L.oracle_verify.restype = ctypes.c_int
        L.oracle_manifest_ok.argtypes = [u8p]
        L.oracle_manifest_ok.restype = ctypes.c_int
    return _lib


def _ptr(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def _buf(data) -> np.ndarray:
    if isinstance(data, np.ndarray):
        return np.ascontiguousarray(data).view(np.uint8).reshape(-1)
    return np.frombuffer(bytes(data), dtype=np.uint8) if len(data) else np.zeros(1, np.uint8)[:0]


def crc32c_bitwise(data) -> int:
    b = _buf(data)
    return lib().oracle_crc32c_bitwise(_ptr(b) if b.size else None, b.size)


def crc32c(data) -> int:
    b = _buf(data)
    return lib().oracle_crc32c_table(_ptr(b) if b.size else None, b.size)


def crc32c_sse42(data) -> int:
    b = _buf(data)
    return lib().oracle_crc32c_sse42(_ptr(b) if b.size else None, b.size)


def have_sse42() -> bool:
    return bool(lib().oracle_have_sse42())


def crc32c_combine(crc_a: int, crc_b: int, len_b: int) -> int:
    return lib().oracle_crc32c_combine(crc_a, crc_b, len_b)


def xxh64(data, seed: int = 0) -> int:
    b = _buf(data)
    return lib().oracle_xxh64(_ptr(b) if b.size else None, b.size, seed)


def chunk_hash(kind: int, data) -> int:
    b = _buf(data)
    return lib().oracle_chunk_hash(kind, _ptr(b) if b.size else None, b.size)


def _regions(regions) -> ctypes.Array:
    """regions: iterable of (id, addr, bytes, kind)."""
    regions = list(regions)
    arr = (_Region * max(1, len(regions)))()
    for k, (rid, addr, nbytes, kind) in enumerate(regions):
        arr[k].id, arr[k].addr, arr[k].bytes, arr[k].kind = rid, addr, nbytes, kind
    return arr, len(regions)


@dataclass
class Plan:
    rc: int
    off: list
    first: list
    nchunks: list
    payload_bytes: int
    n_chunks: int
    image_bytes: int = 0
    manifest_off: int = 0


def plan(regions, chunk_bytes: int, align: int) -> Plan:
    arr, n = _regions(regions)
    off = (ctypes.c_uint64 * max(1, n))()
    first = (ctypes.c_uint64 * max(1, n))()
    nch = (ctypes.c_uint64 * max(1, n))()
    payload, m = ctypes.c_uint64(), ctypes.c_uint64()
    rc = lib().oracle_plan(arr, n, chunk_bytes, align, off, first, nch, ctypes.byref(payload), ctypes.byref(m))
    if rc:
        return Plan(rc, [], [], [], 0, 0)
    ib, mo = ctypes.c_uint64(), ctypes.c_uint64()
    lib().oracle_image_layout(arr, n, chunk_bytes, align, ctypes.byref(ib), ctypes.byref(mo))
    return Plan(rc, list(off[:n]), list(first[:n]), list(nch[:n]), payload.value, m.value, ib.value, mo.value)


def manifest_bytes(n_regions: int, n_chunks: int) -> int:
    return lib().oracle_manifest_bytes(n_regions, n_chunks)


def checkpoint(regions, mem: np.ndarray, mem_base: int, kind: int, chunk_bytes: int, align: int,
               rank: int = 0, world: int = 1, threads: int = 1):
    """Returns (rc, image uint8 array, manifest_off)."""
    arr, n = _regions(regions)
    ib, mo = ctypes.c_uint64(), ctypes.c_uint64()
    rc = lib().oracle_image_layout(arr, n, chunk_bytes, align, ctypes.byref(ib), ctypes.byref(mo))
    if rc:
        return rc, None, 0
    image = np.empty(ib.value, dtype=np.uint8)
    rc = lib().oracle_checkpoint(arr, n, _ptr(mem), mem_base, mem.size, kind, chunk_bytes, align,
                                 rank, world, _ptr(image), image.size, threads)
    return rc, (image if rc == 0 else None), mo.value


SAVE, SAVE_ONCE, DISCARD = 0, 1, 2


def policy_view(regions, policies, mem_now: np.ndarray, mem_first: np.ndarray, mem_base: int,
                chunk_bytes: int | None = None, masks: dict | None = None) -> np.ndarray:
    """The bytes a checkpoint captures under per-region swap policies (reading 24):
    SAVE -> the region now; SAVE_ONCE -> the region as it was at the first checkpoint;
    DISCARD -> zeros. Touched-chunk masks (reading 25): masks = {region index: keep[0..n_i)} for SAVE
    regions; chunk j with keep[j] == 0 covers region bytes [j*C, min((j+1)*C, bytes)) (SURVEY §8(c)
    step 3) and is captured as zeros, like DISCARD. Feed the result to checkpoint()."""
    view = mem_now.copy()
    for i, ((rid, addr, nbytes, kind), pol) in enumerate(zip(regions, policies)):
        lo = addr - mem_base
        if pol == DISCARD:
            view[lo:lo + nbytes] = 0
        elif pol == SAVE_ONCE:
            view[lo:lo + nbytes] = mem_first[lo:lo + nbytes]
        elif masks and i in masks and masks[i] is not None:
            keep = masks[i]
            assert len(keep) == -(-nbytes // chunk_bytes), "one mask entry per chunk"
            for j, k in enumerate(keep):
                if not k:
                    view[lo + j * chunk_bytes:lo + min((j + 1) * chunk_bytes, nbytes)] = 0
    return view


def summary(manifest: np.ndarray, image_bytes: int) -> bytes:
    out = np.zeros(64, np.uint8)
    rc = lib().oracle_summary(_ptr(manifest), manifest.size, image_bytes, _ptr(out))
    if rc:
        raise ValueError(f"oracle_summary rc={rc}")
    return out.tobytes()


def global_digest(summaries: bytes) -> int:
    b = _buf(summaries)
    return lib().oracle_global_digest(_ptr(b), b.size // 64)


def restore(image: np.ndarray, manifest_off: int, mem: np.ndarray, mem_base: int, threads: int = 1,
            fast: bool = False):
    """Returns (rc, n_bad, first_bad); writes mem in place. fast: CRC-32C by the SSE4.2 instruction
    instead of the Sarwate table (same results; the bench's "fast" CPU timing)."""
    nb, fb = ctypes.c_uint64(), ctypes.c_uint64()
    fn = lib().oracle_restore_fast if fast else lib().oracle_restore
    rc = fn(_ptr(image), manifest_off, _ptr(mem), mem_base, mem.size, ctypes.byref(nb), ctypes.byref(fb), threads)
    return rc, nb.value, fb.value


def verify(manifest: np.ndarray, mem: np.ndarray, mem_base: int, threads: int = 1):
    nb, fb = ctypes.c_uint64(), ctypes.c_uint64()
    rc = lib().oracle_verify(_ptr(manifest), _ptr(mem), mem_base, mem.size, ctypes.byref(nb), ctypes.byref(fb), threads)
    return rc, nb.value, fb.value


def manifest_ok(manifest: np.ndarray) -> bool:
    return bool(lib().oracle_manifest_ok(_ptr(manifest)))
