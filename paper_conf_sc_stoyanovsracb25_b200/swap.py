"""ctypes binding of libswap (include/swap.h) — argument marshalling only.

Every step of the checkpoint/restore path runs in libswap's CUDA kernels or copy-engine
calls; this module only converts Python values to the C ABI and back. There is no CPU
fallback: if libswap.so is missing or no sm_100 GPU is present, calls fail loudly.

The low-level functions keep the C names (``swap_create``, ``swap_register_regions``,
``swap_checkpoint``, ``swap_restore``, ``swap_verify``, ...) and return the raw status;
``Swapper`` is the convenience wrapper tests and bench.py use (it raises ``SwapError``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import build as _build

SWAP_OK, SWAP_EINVAL, SWAP_ENOMEM, SWAP_ECUDA, SWAP_ESTATE = 0, -1, -2, -3, -4
SWAP_ECORRUPT, SWAP_ENCCL, SWAP_EUNSUPPORTED, SWAP_EINTERNAL = -5, -6, -7, -8
SWAP_CHECKSUM_CRC32C, SWAP_CHECKSUM_XXH64 = 1, 2
SWAP_MECH_AUTO, SWAP_MECH_SM, SWAP_MECH_CE_REGION, SWAP_MECH_CE_CHUNK = 0, 1, 2, 3
SWAP_MECH_CE_BATCH, SWAP_MECH_CE_PIPE, SWAP_MECH_SM_NOCHECK = 4, 5, 6
MECHANISMS = {"auto": 0, "sm": 1, "ce_region": 2, "ce_chunk": 3, "ce_batch": 4, "ce_pipe": 5, "sm_nocheck": 6}
SWAP_KIND_WEIGHTS, SWAP_KIND_KV, SWAP_KIND_WORKSPACE, SWAP_KIND_OTHER = 0, 1, 2, 3
SWAP_POLICY_SAVE, SWAP_POLICY_SAVE_ONCE, SWAP_POLICY_DISCARD = 0, 1, 2
POLICIES = {"save": 0, "save_once": 1, "discard": 2}
U64_MAX = (1 << 64) - 1

EXPORTS = [
    "swap_config_default", "swap_create", "swap_register_regions", "swap_checkpoint", "swap_sync",
    "swap_restore", "swap_verify", "swap_set_mechanism", "swap_get_mechanism", "swap_get_mechanism_dir", "swap_get_numa", "swap_restore_stripe", "swap_get_restore_spans", "swap_pull_stripes", "swap_ipc_export", "swap_ipc_import", "swap_ipc_close", "swap_set_region_policy", "swap_set_chunk_mask", "swap_get_manifest", "swap_get_image",
    "swap_get_summary", "swap_import", "swap_save", "swap_load", "swap_set_global", "swap_merge_global", "swap_plan_layout", "swap_plan_manifest", "swap_get_timings",
    "swap_get_launch_count", "swap_status_str", "swap_last_error", "swap_destroy",
    "swap_arena_create", "swap_arena_info", "swap_arena_release", "swap_arena_reacquire", "swap_arena_last_error",
    "swap_arena_reacquire_range", "swap_bind_arena", "swap_exchange", "swap_set_helpers",
    "swap_arena_destroy", "swap_arena_export", "swap_arena_import", "swap_arena_unimport", "swap_sched_create", "swap_sched_add_backend", "swap_sched_touch", "swap_sched_lock",
    "swap_sched_plan", "swap_sched_reserve", "swap_sched_cancel", "swap_sched_grant", "swap_sched_release",
    "swap_sched_query", "swap_sched_free", "swap_sched_destroy",
]


class swap_region_t(ctypes.Structure):
    _fields_ = [("dev_addr", ctypes.c_uint64), ("bytes", ctypes.c_uint64), ("id", ctypes.c_uint32),
                ("kind", ctypes.c_uint32)]


class swap_config_t(ctypes.Structure):
    _fields_ = [("chunk_bytes", ctypes.c_uint64), ("align", ctypes.c_uint64), ("checksum", ctypes.c_uint32),
                ("mechanism", ctypes.c_uint32), ("device", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("world", ctypes.c_int32), ("grid_ctas", ctypes.c_uint32), ("seg_bytes", ctypes.c_uint32),
                ("pipe_mib", ctypes.c_uint32), ("host_numa", ctypes.c_int32), ("reserved0", ctypes.c_uint32)]


class swap_verify_result_t(ctypes.Structure):
    _fields_ = [("n_bad", ctypes.c_uint64), ("first_bad_chunk", ctypes.c_uint64), ("hbm_n_bad", ctypes.c_uint64),
                ("hbm_first_bad", ctypes.c_uint64), ("manifest_ok", ctypes.c_uint32),
                ("hbm_checked", ctypes.c_uint32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class swap_span_t(ctypes.Structure):
    _fields_ = [("group", ctypes.c_uint32), ("reserved", ctypes.c_uint32), ("dev_addr", ctypes.c_uint64),
                ("image_offset", ctypes.c_uint64), ("bytes", ctypes.c_uint64)]


class swap_shard_summary_t(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_uint32), ("world", ctypes.c_uint32), ("checksum", ctypes.c_uint32),
                ("n_regions", ctypes.c_uint32), ("n_chunks", ctypes.c_uint64), ("payload_bytes", ctypes.c_uint64),
                ("image_bytes", ctypes.c_uint64), ("manifest_crc", ctypes.c_uint64),
                ("chunk_digest", ctypes.c_uint64), ("reserved", ctypes.c_uint64)]


class swap_timings_t(ctypes.Structure):
    _fields_ = [("checkpoint_ms", ctypes.c_float), ("restore_ms", ctypes.c_float), ("verify_ms", ctypes.c_float),
                ("check_ms", ctypes.c_float)]


assert ctypes.sizeof(swap_shard_summary_t) == 64 and ctypes.sizeof(swap_config_t) == 56

_lib = None


def lib_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = True) -> ctypes.CDLL:
    """Loads the in-tree libswap.so (building it with nvcc if absent). Raises if unavailable."""
    global _lib
    if _lib is not None:
        return _lib
    if not _build.up_to_date():
        if not build_if_missing:
            raise RuntimeError(f"libswap.so missing or stale at {_build.LIB}; run paper_conf_sc_stoyanovsracb25_b200.build")
        _build.build()
    L = ctypes.CDLL(_build.LIB)
    vp, st, u32, sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_uint32, ctypes.c_size_t
    P = ctypes.POINTER
    sig = {
        "swap_config_default": (None, [P(swap_config_t)]),
        "swap_create": (st, [P(swap_config_t), P(vp)]),
        "swap_register_regions": (st, [vp, P(swap_region_t), sz]),
        "swap_checkpoint": (st, [vp, vp]),
        "swap_sync": (st, [vp, vp]),
        "swap_restore": (st, [vp, vp]),
        "swap_verify": (st, [vp, vp, ctypes.c_int, P(swap_verify_result_t)]),
        "swap_set_mechanism": (st, [vp, u32]),
        "swap_get_mechanism": (st, [vp, P(u32)]),
        "swap_get_mechanism_dir": (st, [vp, ctypes.c_int, P(u32)]),
        "swap_get_numa": (st, [vp, P(ctypes.c_int32), P(ctypes.c_double)]),
        "swap_restore_stripe": (st, [vp, u32, u32, vp]),
        "swap_get_restore_spans": (st, [vp, vp, ctypes.c_size_t, P(ctypes.c_size_t)]),
        "swap_pull_stripes": (st, [vp, u32, u32, P(ctypes.c_int64), vp]),
        "swap_ipc_export": (st, [ctypes.c_int, vp, vp, P(ctypes.c_uint64)]),
        "swap_ipc_import": (st, [ctypes.c_int, vp, ctypes.c_uint64, P(vp), P(vp)]),
        "swap_ipc_close": (st, [ctypes.c_int, vp]),
        "swap_set_region_policy": (st, [vp, u32, u32]),
        "swap_set_chunk_mask": (st, [vp, u32, vp, ctypes.c_uint64]),
        "swap_get_manifest": (st, [vp, P(vp), P(sz)]),
        "swap_get_image": (st, [vp, P(vp), P(sz)]),
        "swap_get_summary": (st, [vp, P(swap_shard_summary_t)]),
        "swap_import": (st, [vp]),
        "swap_save": (st, [vp, ctypes.c_char_p]),
        "swap_load": (st, [vp, ctypes.c_char_p]),
        "swap_set_global": (st, [vp, P(swap_shard_summary_t), ctypes.c_int, P(ctypes.c_uint64)]),
        "swap_merge_global": (st, [P(swap_shard_summary_t), ctypes.c_int, P(ctypes.c_uint64)]),
        "swap_plan_layout": (st, [P(swap_region_t), sz, P(swap_config_t), P(ctypes.c_uint64), P(ctypes.c_uint64),
                                  P(ctypes.c_uint64), P(ctypes.c_uint64)]),
        "swap_plan_manifest": (st, [P(swap_region_t), sz, P(swap_config_t), P(ctypes.c_uint64), vp, sz, P(sz)]),
        "swap_get_timings": (st, [vp, P(swap_timings_t)]),
        "swap_get_launch_count": (st, [vp, P(ctypes.c_uint64)]),
        "swap_status_str": (ctypes.c_char_p, [st]),
        "swap_last_error": (ctypes.c_char_p, [vp]),
        "swap_destroy": (None, [vp]),
        "swap_arena_create": (st, [ctypes.c_int, ctypes.c_uint64, P(vp)]),
        "swap_arena_info": (st, [vp, P(ctypes.c_uint64), P(ctypes.c_uint64), P(ctypes.c_int)]),
        "swap_arena_release": (st, [vp]),
        "swap_arena_reacquire": (st, [vp]),
        "swap_arena_reacquire_range": (st, [vp, ctypes.c_uint64, ctypes.c_uint64]),
        "swap_bind_arena": (st, [vp, vp]),
        "swap_set_helpers": (st, [vp, P(ctypes.c_int), ctypes.c_int]),
        "swap_exchange": (st, [P(vp), sz, vp, vp, vp, ctypes.c_uint64, P(ctypes.c_uint64)]),
        "swap_arena_last_error": (ctypes.c_char_p, [vp]),
        "swap_arena_destroy": (None, [vp]),
        "swap_arena_export": (st, [vp, P(ctypes.c_int), ctypes.c_size_t, P(ctypes.c_size_t), P(ctypes.c_uint64)]),
        "swap_arena_import": (st, [ctypes.c_int, P(ctypes.c_int), ctypes.c_size_t, ctypes.c_uint64, ctypes.c_uint64,
                                   P(vp), P(ctypes.c_uint64)]),
        "swap_arena_unimport": (None, [vp]),
        "swap_sched_create": (st, [u32, P(ctypes.c_uint64), P(vp)]),
        "swap_sched_add_backend": (st, [vp, u32, P(ctypes.c_uint64), ctypes.c_int]),
        "swap_sched_touch": (st, [vp, u32, u32, ctypes.c_double]),
        "swap_sched_lock": (st, [vp, u32, ctypes.c_int]),
        "swap_sched_plan": (st, [vp, u32, P(u32), u32, P(u32)]),
        "swap_sched_reserve": (st, [vp, u32, ctypes.c_double]),
        "swap_sched_cancel": (st, [vp, u32]),
        "swap_sched_grant": (st, [vp, P(u32), P(u32), u32, P(u32)]),
        "swap_sched_release": (st, [vp, u32]),
        "swap_sched_query": (st, [vp, u32, P(ctypes.c_int), P(ctypes.c_int)]),
        "swap_sched_free": (st, [vp, u32, P(ctypes.c_uint64)]),
        "swap_sched_destroy": (None, [vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype, f.argtypes = res, args
    _lib = L
    return L


class SwapError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__(f"{load().swap_status_str(status).decode()} ({status}): {msg}")


# ------------------------------------------------------------------ thin C-named wrappers
def swap_config_default() -> swap_config_t:
    cfg = swap_config_t()
    load().swap_config_default(ctypes.byref(cfg))
    return cfg


def swap_create(cfg: swap_config_t):
    h = ctypes.c_void_p()
    st = load().swap_create(ctypes.byref(cfg), ctypes.byref(h))
    return st, h


def swap_register_regions(ctx, regions) -> int:
    """regions: sequence of (dev_addr, nbytes, id, kind)."""
    arr = (swap_region_t * max(1, len(regions)))()
    for i, (addr, nb, rid, kind) in enumerate(regions):
        arr[i].dev_addr, arr[i].bytes, arr[i].id, arr[i].kind = addr, nb, rid, kind
    return load().swap_register_regions(ctx, arr, len(regions))


def swap_checkpoint(ctx, stream: int = 0) -> int:
    return load().swap_checkpoint(ctx, ctypes.c_void_p(stream))


def swap_sync(ctx, stream: int = 0) -> int:
    return load().swap_sync(ctx, ctypes.c_void_p(stream))


def swap_restore(ctx, stream: int = 0) -> int:
    return load().swap_restore(ctx, ctypes.c_void_p(stream))


def swap_verify(ctx, stream: int = 0, hbm_pass: bool = True):
    res = swap_verify_result_t()
    st = load().swap_verify(ctx, ctypes.c_void_p(stream), 1 if hbm_pass else 0, ctypes.byref(res))
    return st, res


def arena_import(device: int, fds: list[int], slab_bytes: int, total_bytes: int) -> tuple[int, int]:
    """Maps a peer's exported arena slabs on `device` (swap_arena_import): (view handle, device address)."""
    arr = (ctypes.c_int * max(1, len(fds)))(*fds)
    view, addr = ctypes.c_void_p(), ctypes.c_uint64()
    st = load().swap_arena_import(device, arr, len(fds), slab_bytes, total_bytes, ctypes.byref(view), ctypes.byref(addr))
    if st:
        raise SwapError(st, "swap_arena_import failed")
    return view.value, addr.value


def arena_unimport(view: int):
    load().swap_arena_unimport(ctypes.c_void_p(view))


def ipc_export(device: int, ptr: int) -> tuple[bytes, int]:
    """(64-B CUDA IPC handle of the allocation holding ptr, ptr's offset in it) -- swap_ipc_export."""
    h = (ctypes.c_uint8 * 64)()
    off = ctypes.c_uint64()
    st = load().swap_ipc_export(device, ctypes.c_void_p(ptr), h, ctypes.byref(off))
    if st:
        raise SwapError(st, "swap_ipc_export failed (not a cudaMalloc allocation?)")
    return bytes(h), off.value


def ipc_import(device: int, handle: bytes, offset: int) -> tuple[int, int]:
    """Maps another process's allocation: (base to close, mapped address of the exported pointer)."""
    h = (ctypes.c_uint8 * 64).from_buffer_copy(handle)
    base, mapped = ctypes.c_void_p(), ctypes.c_void_p()
    st = load().swap_ipc_import(device, h, offset, ctypes.byref(base), ctypes.byref(mapped))
    if st:
        raise SwapError(st, "swap_ipc_import failed")
    return base.value, mapped.value


def ipc_close(device: int, base: int):
    load().swap_ipc_close(device, ctypes.c_void_p(base))


def swap_merge_global(summaries: bytes, world: int):
    arr = (swap_shard_summary_t * world).from_buffer_copy(summaries)
    d = ctypes.c_uint64()
    st = load().swap_merge_global(arr, world, ctypes.byref(d))
    return st, d.value


def _region_array(regions):
    arr = (swap_region_t * max(1, len(regions)))()
    for i, (addr, nb, rid, kind) in enumerate(regions):
        arr[i].dev_addr, arr[i].bytes, arr[i].id, arr[i].kind = addr, nb, rid, kind
    return arr


def swap_plan_layout(regions, cfg: swap_config_t):
    """(status, payload_bytes, n_chunks, manifest_off, image_bytes) for (dev_addr, nbytes, id, kind) rows."""
    vals = [ctypes.c_uint64() for _ in range(4)]
    st = load().swap_plan_layout(_region_array(regions), len(regions), ctypes.byref(cfg), *[ctypes.byref(v) for v in vals])
    return (st, *[v.value for v in vals])


def swap_plan_manifest(regions, cfg: swap_config_t, checksums=None):
    """(status, manifest bytes) with the given chunk checksums (list of ints) or zeros."""
    st, payload, m, moff, ib = swap_plan_layout(regions, cfg)
    if st:
        return st, b""
    cs = (ctypes.c_uint64 * max(1, m))(*(checksums or []))
    n = ctypes.c_size_t()
    buf = ctypes.create_string_buffer(ib - moff)
    st = load().swap_plan_manifest(_region_array(regions), len(regions), ctypes.byref(cfg),
                                   cs if checksums is not None else None, buf, len(buf), ctypes.byref(n))
    return st, buf.raw[:n.value]


def _torch_stream(stream) -> int:
    if stream is None:
        import torch

        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------------ Swapper
class Swapper:
    """One registered engine shard on one device.

    regions: sequence of torch CUDA tensors (whole storages are registered), or of
    (dev_addr, nbytes, kind) / (dev_addr, nbytes, kind, id) tuples.
    """

    def __init__(self, regions, chunk_bytes: int = 1 << 20, checksum: int = SWAP_CHECKSUM_CRC32C,
                 mechanism: int | str = SWAP_MECH_AUTO, device: int | None = None, rank: int = 0, world: int = 1,
                 align: int = 4096, grid_ctas: int = 0, seg_bytes: int = 0, pipe_mib: int = 0,
                 host_numa: int = 0):
        """host_numa: 0 = place the pinned image on the device's NUMA node (auto), -1 = no placement,
        n >= 1 = NUMA node n-1 (swap_config_t.host_numa)."""
        L = load()
        table = []
        for i, r in enumerate(regions):
            if hasattr(r, "data_ptr"):
                if device is None:
                    device = r.device.index
                table.append((r.untyped_storage().data_ptr(), r.untyped_storage().nbytes(), i, SWAP_KIND_OTHER))
            else:
                addr, nb, kind = r[0], r[1], r[2]
                table.append((addr, nb, r[3] if len(r) > 3 else i, kind))
        if isinstance(mechanism, str):
            mechanism = MECHANISMS[mechanism]
        if device is None:  # raw addresses: the caller's current device (torch's, when torch is in use)
            try:
                import torch

                device = torch.cuda.current_device() if torch.cuda.is_available() else 0
            except ImportError:
                device = 0
        cfg = swap_config_default()
        cfg.chunk_bytes, cfg.checksum, cfg.mechanism, cfg.align = chunk_bytes, checksum, mechanism, align
        cfg.device, cfg.rank, cfg.world = device, rank, world
        cfg.grid_ctas, cfg.seg_bytes, cfg.pipe_mib = grid_ctas, seg_bytes, pipe_mib
        cfg.host_numa = host_numa
        st, h = swap_create(cfg)
        if st:
            raise SwapError(st, "swap_create failed (no sm_100 GPU / bad config)")
        self._ctx = h
        self.device = cfg.device
        self.rank, self.world = rank, world
        st = swap_register_regions(h, table)
        if st:
            msg = L.swap_last_error(h).decode()
            self.close()
            raise SwapError(st, msg)
        self.regions = table
        C = chunk_bytes or (1 << 20)
        self._n_chunks = [(nb + C - 1) // C for (_, nb, _, _) in table]

    # -- helpers
    def _check(self, st: int):
        if st:
            raise SwapError(st, load().swap_last_error(self._ctx).decode())

    @property
    def ctx(self):
        return self._ctx

    def checkpoint(self, stream=None, sync: bool = True):
        s = _torch_stream(stream)
        self._check(swap_checkpoint(self._ctx, s))
        if sync:
            self._check(swap_sync(self._ctx, s))

    def sync(self, stream=None):
        self._check(swap_sync(self._ctx, _torch_stream(stream)))

    def restore(self, stream=None):
        self._check(swap_restore(self._ctx, _torch_stream(stream)))

    def verify(self, stream=None, hbm_pass: bool = True, raise_on_corrupt: bool = True) -> dict:
        st, res = swap_verify(self._ctx, _torch_stream(stream), hbm_pass)
        if st and (raise_on_corrupt or st != SWAP_ECORRUPT):
            self._check(st)
        d = res.as_dict()
        d["status"] = st
        return d

    def swap_out(self, arena: "Arena | None" = None, stream=None):
        """Preempt: checkpoint + seal the manifest, then free the arena's HBM."""
        self.checkpoint(stream, sync=True)
        if arena is not None:
            arena.release()

    def set_helpers(self, devices):
        """NVLink-assisted restore: stripe CE_PIPE restore groups over these (idle) peer GPUs."""
        arr = (ctypes.c_int * max(1, len(devices)))(*devices)
        self._check(load().swap_set_helpers(self._ctx, arr, len(devices)))

    def bind_arena(self, arena: "Arena | None"):
        """Let restore re-acquire this arena's HBM itself (group by group under CE_PIPE)."""
        self._check(load().swap_bind_arena(self._ctx, arena._h if arena is not None else None))
        self._arena = arena

    def swap_in(self, arena: "Arena | None" = None, stream=None, hbm_pass: bool = True) -> dict:
        """Swap-in: re-acquire HBM at the recorded addresses, restore, verify. With an
        arena bound (bind_arena) the re-acquire happens inside the restore, overlapped."""
        if arena is not None and getattr(self, "_arena", None) is not arena and not arena.resident:
            arena.reacquire()
        self.restore(stream)
        return self.verify(stream, hbm_pass=hbm_pass)

    def set_mechanism(self, mechanism: int | str):
        if isinstance(mechanism, str):
            mechanism = MECHANISMS[mechanism]
        self._check(load().swap_set_mechanism(self._ctx, mechanism))

    def set_region_policy(self, region_index: int, policy: int | str):
        """SAVE / SAVE_ONCE / DISCARD for one region (before the first checkpoint)."""
        if isinstance(policy, str):
            policy = POLICIES[policy]
        self._check(load().swap_set_region_policy(self._ctx, region_index, policy))

    def set_chunk_mask(self, region_index: int, keep=None):
        """Touched-chunk mask of a SAVE region for the next checkpoint (None = keep every chunk):
        chunks with keep[j] == 0 are captured as zeros and not moved (include/swap.h)."""
        if keep is None:
            self._check(load().swap_set_chunk_mask(self._ctx, region_index, None, self._n_chunks[region_index]))
            return
        k = np.ascontiguousarray(np.asarray(keep, dtype=np.uint8))
        self._check(load().swap_set_chunk_mask(self._ctx, region_index, k.ctypes.data, k.size))

    def mechanism(self, direction: str = "restore") -> str:
        """Name of the mover the next call of `direction` ("restore" or "checkpoint") uses, AUTO
        resolved per direction (swap_get_mechanism_dir)."""
        m = ctypes.c_uint32()
        d = {"checkpoint": 0, "restore": 1}[direction]
        self._check(load().swap_get_mechanism_dir(self._ctx, d, ctypes.byref(m)))
        return {v: k for k, v in MECHANISMS.items()}[m.value]

    def save(self, path: str):
        """Persist the sealed image to `path` (swap_save)."""
        self._check(load().swap_save(self._ctx, os.fsencode(path)))

    def load_image(self, path: str):
        """Load an image file written by save() and validate it (swap_load)."""
        self._check(load().swap_load(self._ctx, os.fsencode(path)))

    def import_image(self):
        self._check(load().swap_import(self._ctx))

    def image(self) -> np.ndarray:
        """Borrowed, writable uint8 view of the library's pinned image (valid until close)."""
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        self._check(load().swap_get_image(self._ctx, ctypes.byref(p), ctypes.byref(n)))
        return np.ctypeslib.as_array(ctypes.cast(p, ctypes.POINTER(ctypes.c_uint8)), shape=(n.value,))

    def manifest(self) -> np.ndarray:
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        self._check(load().swap_get_manifest(self._ctx, ctypes.byref(p), ctypes.byref(n)))
        return np.ctypeslib.as_array(ctypes.cast(p, ctypes.POINTER(ctypes.c_uint8)), shape=(n.value,))

    def restore_stripe(self, stripe: int, n_stripes: int, stream=None):
        """Restore only CE_PIPE groups g with g % n_stripes == stripe (swap_restore_stripe; DP replicas)."""
        self._check(load().swap_restore_stripe(self._ctx, stripe, n_stripes, _torch_stream(stream)))

    def pull_stripes(self, stripe: int, n_stripes: int, peer_delta: list[int], stream=None):
        """Fused NVLink pull of the other replicas' stripes with the chunk check (swap_pull_stripes);
        peer_delta[o] = replica o's mapped address of a byte minus this replica's (ignored for o == stripe)."""
        arr = (ctypes.c_int64 * n_stripes)(*peer_delta)
        self._check(load().swap_pull_stripes(self._ctx, stripe, n_stripes, arr, _torch_stream(stream)))

    def restore_spans(self) -> list[tuple[int, int, int, int]]:
        """(group, dev_addr, image_offset, bytes) of every coalesced restore copy (swap_get_restore_spans)."""
        n = ctypes.c_size_t()
        self._check(load().swap_get_restore_spans(self._ctx, None, 0, ctypes.byref(n)))
        arr = (swap_span_t * max(1, n.value))()
        self._check(load().swap_get_restore_spans(self._ctx, arr, n.value, ctypes.byref(n)))
        return [(x.group, x.dev_addr, x.image_offset, x.bytes) for x in arr[:n.value]]

    def numa(self) -> dict:
        """Host NUMA placement of the image (swap_get_numa): the node targeted (-1 none) and the
        sampled share of its pages on that node."""
        node, frac = ctypes.c_int32(), ctypes.c_double()
        self._check(load().swap_get_numa(self._ctx, ctypes.byref(node), ctypes.byref(frac)))
        return {"node": node.value, "local_fraction": round(frac.value, 4)}

    def summary(self) -> bytes:
        s = swap_shard_summary_t()
        self._check(load().swap_get_summary(self._ctx, ctypes.byref(s)))
        return bytes(s)

    def set_global(self, summaries: bytes) -> int:
        world = len(summaries) // 64
        arr = (swap_shard_summary_t * world).from_buffer_copy(summaries)
        d = ctypes.c_uint64()
        self._check(load().swap_set_global(self._ctx, arr, world, ctypes.byref(d)))
        return d.value

    def timings(self) -> dict:
        """Device ms of the last checkpoint / restore / HBM verify movers (CUDA events), and the summed
        device ms of the last CE_PIPE restore's per-group check launches (check_ms)."""
        t = swap_timings_t()
        self._check(load().swap_get_timings(self._ctx, ctypes.byref(t)))
        return {"checkpoint_ms": t.checkpoint_ms, "restore_ms": t.restore_ms, "verify_ms": t.verify_ms,
                "check_ms": t.check_ms}

    def launch_count(self) -> int:
        n = ctypes.c_uint64()
        self._check(load().swap_get_launch_count(self._ctx, ctypes.byref(n)))
        return n.value

    def close(self):
        if getattr(self, "_ctx", None):
            load().swap_destroy(self._ctx)
            self._ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def exchange(victims, incoming, stream_out=None, stream_in=None, headroom: int = 0) -> int:
    """swap_exchange: victims (Swappers with bound, mapped arenas) out, `incoming` (bound, released) in,
    overlapped on the duplex link within the victims' HBM + headroom. Returns the peak extra HBM."""
    arr = (ctypes.c_void_p * max(1, len(victims)))(*[v.ctx.value if hasattr(v.ctx, "value") else v.ctx for v in victims])
    peak = ctypes.c_uint64()
    so = _torch_stream(stream_out)
    si = _torch_stream(stream_in)
    st = load().swap_exchange(arr, len(victims), incoming.ctx if incoming is not None else None,
                              ctypes.c_void_p(so), ctypes.c_void_p(si), headroom, ctypes.byref(peak))
    if st:
        who = incoming if incoming is not None else victims[0]
        raise SwapError(st, load().swap_last_error(who.ctx).decode())
    return peak.value


# ------------------------------------------------------------------ Arena (releasable HBM)
class _CudaArray:
    """Minimal __cuda_array_interface__ exporter so torch can view arena memory (no ownership)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False), "version": 3,
                                         "strides": None, "stream": None}


class Arena:
    """Device memory whose physical HBM can be released and re-acquired at the same addresses
    (swap_arena_* in include/swap.h). Carve engine tensors out of it with `tensor()`."""

    def __init__(self, nbytes: int, device: int = 0):
        h = ctypes.c_void_p()
        st = load().swap_arena_create(device, nbytes, ctypes.byref(h))
        if st:
            raise SwapError(st, f"swap_arena_create({nbytes} B on device {device}) failed")
        self._h = h
        self.device = device
        self._used = 0
        addr, size, res = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_int()
        load().swap_arena_info(h, ctypes.byref(addr), ctypes.byref(size), ctypes.byref(res))
        self.base, self.nbytes = addr.value, size.value

    def _check(self, st):
        if st:
            raise SwapError(st, load().swap_arena_last_error(self._h).decode())

    @property
    def resident(self) -> bool:
        res = ctypes.c_int()
        load().swap_arena_info(self._h, None, None, ctypes.byref(res))
        return bool(res.value)

    def tensor(self, offset: int, nbytes: int):
        """A torch uint8 CUDA tensor viewing arena bytes [offset, offset + nbytes)."""
        import torch

        assert 0 <= offset and offset + nbytes <= self.nbytes
        return torch.as_tensor(_CudaArray(self.base + offset, nbytes), device=f"cuda:{self.device}")

    def export(self) -> tuple[list[int], int]:
        """POSIX file descriptors of the arena's slabs (the caller owns and must close them) and the slab
        size -- swap_arena_export; pass them to a peer process (dist.map_replicas_arena does, over a Unix
        socket) for arena_import."""
        n, slab = ctypes.c_size_t(), ctypes.c_uint64()
        self._check(load().swap_arena_export(self._h, None, 0, ctypes.byref(n), ctypes.byref(slab)))
        fds = (ctypes.c_int * max(1, n.value))()
        self._check(load().swap_arena_export(self._h, fds, n.value, ctypes.byref(n), ctypes.byref(slab)))
        return list(fds[:n.value]), slab.value

    def alloc(self, nbytes: int, align: int = 256):
        """Bump-allocates `nbytes` (aligned) and returns (dev_addr, torch view)."""
        off = (self._used + align - 1) // align * align
        if off + nbytes > self.nbytes:
            raise SwapError(SWAP_ENOMEM, "arena full")
        self._used = off + nbytes
        return self.base + off, self.tensor(off, nbytes)

    def release(self):
        self._check(load().swap_arena_release(self._h))

    def reacquire_range(self, offset: int, nbytes: int):
        self._check(load().swap_arena_reacquire_range(self._h, offset, nbytes))

    def reacquire(self):
        self._check(load().swap_arena_reacquire(self._h))

    def close(self):
        if getattr(self, "_h", None):
            load().swap_arena_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------------------------ Scheduler (task manager)
class Scheduler:
    """Reservations + demand-aware preemption (swap_sched_* in include/swap.h; §3.3-3.5, §6)."""

    MAX_VICTIMS = 4096

    def __init__(self, capacity_per_gpu):
        caps = (ctypes.c_uint64 * len(capacity_per_gpu))(*capacity_per_gpu)
        h = ctypes.c_void_p()
        st = load().swap_sched_create(len(capacity_per_gpu), caps, ctypes.byref(h))
        if st:
            raise SwapError(st, "swap_sched_create")
        self._h, self.n_gpus = h, len(capacity_per_gpu)
        self._buf = (ctypes.c_uint32 * self.MAX_VICTIMS)()

    def _check(self, st, what):
        if st:
            raise SwapError(st, what)

    def add_backend(self, bid: int, need_per_gpu, resident: bool = False):
        need = (ctypes.c_uint64 * self.n_gpus)(*need_per_gpu)
        self._check(load().swap_sched_add_backend(self._h, bid, need, int(resident)), f"add_backend({bid})")

    def touch(self, bid: int, queue_len: int, last_access: float):
        self._check(load().swap_sched_touch(self._h, bid, queue_len, last_access), "touch")

    def lock(self, bid: int, locked: bool = True):
        self._check(load().swap_sched_lock(self._h, bid, int(locked)), "lock")

    def plan(self, bid: int):
        """Victims in eviction order, or None if infeasible."""
        n = ctypes.c_uint32()
        st = load().swap_sched_plan(self._h, bid, self._buf, self.MAX_VICTIMS, ctypes.byref(n))
        if st == SWAP_ENOMEM:
            return None
        self._check(st, "plan")
        return list(self._buf[:n.value])

    def reserve(self, bid: int, priority: float):
        self._check(load().swap_sched_reserve(self._h, bid, priority), f"reserve({bid})")

    def cancel(self, bid: int):
        self._check(load().swap_sched_cancel(self._h, bid), "cancel")

    def grant(self):
        """(backend, victims) for the head reservation; None if the queue is empty;
        ('blocked', backend) if the head cannot be satisfied now."""
        bid, n = ctypes.c_uint32(), ctypes.c_uint32()
        st = load().swap_sched_grant(self._h, ctypes.byref(bid), self._buf, self.MAX_VICTIMS, ctypes.byref(n))
        if st == SWAP_ENOMEM:
            return ("blocked", bid.value)
        self._check(st, "grant")
        if bid.value == 0xFFFFFFFF:
            return None
        return bid.value, list(self._buf[:n.value])

    def release(self, bid: int):
        self._check(load().swap_sched_release(self._h, bid), "release")

    def state(self, bid: int):
        r, q = ctypes.c_int(), ctypes.c_int()
        self._check(load().swap_sched_query(self._h, bid, ctypes.byref(r), ctypes.byref(q)), "query")
        return {"resident": bool(r.value), "queued": bool(q.value)}

    def free(self, gpu: int) -> int:
        f = ctypes.c_uint64()
        self._check(load().swap_sched_free(self._h, gpu, ctypes.byref(f)), "free")
        return f.value

    def close(self):
        if getattr(self, "_h", None):
            load().swap_sched_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
