"""Multi-GPU shard coordinator (§6 "Multi-GPU Orchestration").

A tensor-parallel engine's device memory is already per rank: rank r checkpoints and
restores its own shard on its own device and stream with no data-path collective. The
only exchanges are
  K5  all-gather of the 64-B shard summaries -> one rank-ordered global manifest + digest,
  K6  all-reduce(SUM) of the mismatch counts after restore/verify, so every rank agrees
      the engine is whole before serving resumes ("verifies that the inference
      engine API is active").
Both go through torch.distributed (NCCL over NVLink on the GPU box; gloo in CPU tests).
Validation and the digest run in libswap (swap_set_global / swap_merge_global).

Data-parallel replicas (NEXT-2) are the one place payload crosses NVLink: restore_replicas pulls
1/k of the image per replica over its own PCIe link (swap_restore_stripe) and broadcasts each
replica's stripe to the others in place, then every replica runs the HBM verify pass.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

import os
import socket
import tempfile
import threading

from .swap import Arena, SWAP_OK, SwapError, Swapper, arena_import, ipc_export, ipc_import, swap_merge_global


def _comm_device(group=None) -> torch.device:
    backend = dist.get_backend(group)
    if backend == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def all_gather_summaries(summary: bytes, group=None) -> bytes:
    """K5: every rank contributes its 64-B summary; returns the world*64 bytes in rank order."""
    assert len(summary) == 64
    world = dist.get_world_size(group)
    dev = _comm_device(group)
    mine = torch.frombuffer(bytearray(summary), dtype=torch.uint8).to(dev)
    out = torch.empty(world * 64, dtype=torch.uint8, device=dev)
    dist.all_gather_into_tensor(out, mine, group=group)
    return out.cpu().numpy().tobytes()


def merge_global(summaries: bytes) -> int:
    """Validates rank order and returns the global digest (libswap swap_merge_global)."""
    st, digest = swap_merge_global(summaries, len(summaries) // 64)
    if st != SWAP_OK:
        raise SwapError(st, "global manifest is not a rank-ordered set of summaries")
    return digest


def gather_manifest(sw: Swapper, group=None) -> tuple[bytes, int]:
    """After a checkpoint on every rank: all-gather summaries, install them in the ctx."""
    allb = all_gather_summaries(sw.summary(), group)
    return allb, sw.set_global(allb)


class _DeviceBytes:
    """A raw device range as a uint8 tensor (zero-copy, __cuda_array_interface__)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def device_view(ptr: int, nbytes: int, device: int) -> torch.Tensor:
    return torch.as_tensor(_DeviceBytes(ptr, nbytes), device=torch.device("cuda", device))


def restore_replicas(sw: Swapper, group=None, stream=None) -> dict:
    """Swap-in of k data-parallel replicas of one engine image (NEXT-2; PAPER.md L203 latency grows with
    the bytes moved, L230 one backend per GPU set). Replica r = rank r of `group`: swap_restore_stripe
    moves groups g = r (mod k) from its pinned image over its own PCIe link (with the fused per-group
    check); then, in group order, the owner of every restore span broadcasts it in place to the other
    replicas (NCCL over NVLink on the GPU box); finally every replica verifies all chunks from HBM.
    Returns the verify result (swap_verify with the HBM pass) of this replica."""
    k, r = dist.get_world_size(group), dist.get_rank(group)
    s = stream if stream is not None else torch.cuda.current_stream(sw.device)
    with torch.cuda.stream(s):
        sw.restore_stripe(r, k, s)
        spans = sw.restore_spans()
        # collectives are issued on `s`, after the stripe's copies; each span comes from its owner
        works = [dist.broadcast(device_view(dev, nb, sw.device), src=dist.get_global_rank(group, g % k) if group else g % k,
                                group=group, async_op=True)
                 for (g, dev, _, nb) in spans]
        for w in works:
            w.wait()
        return sw.verify(s, hbm_pass=True, raise_on_corrupt=False)


def map_replicas(local_ptr: int, device: int, group=None) -> tuple[list[int], list[int]]:
    """CUDA IPC mapping of every other replica's arena into this process (for pull_replicas): all-gathers
    each replica's (handle, offset, address) of its arena base; returns (peer_delta, bases to close) with
    peer_delta[o] = mapped address of replica o's arena base - local_ptr (0 for this replica)."""
    k, r = dist.get_world_size(group), dist.get_rank(group)
    h, off = ipc_export(device, local_ptr)
    allh = [None] * k
    dist.all_gather_object(allh, (h, off), group=group)
    deltas, bases = [], []
    for o, (ho, offo) in enumerate(allh):
        if o == r:
            deltas.append(0)
            continue
        base, mapped = ipc_import(device, ho, offo)
        bases.append(base)
        deltas.append(mapped - local_ptr)
    return deltas, bases


def _exchange_fds(my_fds: list[int], group=None) -> dict[int, list[int]]:
    """Every rank sends its file descriptors to every other rank over Unix-domain sockets (SCM_RIGHTS;
    the rendezvous paths travel through torch.distributed); returns {peer rank: its fds, now valid here}."""
    k, r = dist.get_world_size(group), dist.get_rank(group)
    path = os.path.join(tempfile.gettempdir(), f"swapserve-{os.getpid()}-{r}-{id(my_fds)}.sock")
    srv = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
    srv.bind(path)
    srv.listen(max(1, k - 1))
    got: dict[int, list[int]] = {}

    def accept_all():
        for _ in range(k - 1):
            conn, _ = srv.accept()
            with conn:
                fds, peer, expect = [], None, None
                while expect is None or len(fds) < expect:
                    msg, part, _, _ = socket.recv_fds(conn, 64, 253)
                    if not msg:
                        break
                    peer, expect = (int(x) for x in msg.decode().split(":")[:2])
                    fds.extend(part)
                got[peer] = fds

    t = threading.Thread(target=accept_all, daemon=True)
    t.start()
    paths = [None] * k
    dist.all_gather_object(paths, path, group=group)
    for o in range(k):
        if o == r:
            continue
        with socket.socket(socket.AF_UNIX, socket.SOCK_STREAM) as c:
            c.connect(paths[o])
            for i in range(0, max(1, len(my_fds)), 200):  # SCM_RIGHTS carries at most 253 fds per message
                socket.send_fds(c, [f"{r}:{len(my_fds)}:".encode()], my_fds[i:i + 200])
    t.join()
    srv.close()
    os.unlink(path)
    dist.barrier(group=group)
    return got


def map_replicas_arena(arena: Arena, group=None) -> tuple[list[int], list[int]]:
    """map_replicas for VMM arenas (releasable HBM, swap.Arena): every replica exports its arena's slabs as
    file descriptors (swap_arena_export), the descriptors are exchanged over Unix sockets, and each peer's
    slabs are mapped here (swap_arena_import). The arena must be resident; after a release / re-acquire the
    physical slabs are new, so map again. Returns (peer_delta, views to swap.arena_unimport)."""
    k, r = dist.get_world_size(group), dist.get_rank(group)
    fds, slab = arena.export()
    try:
        peers = _exchange_fds(fds, group)
    finally:
        for f in fds:
            os.close(f)
    sizes = [None] * k
    dist.all_gather_object(sizes, arena.nbytes, group=group)
    deltas, views = [], []
    for o in range(k):
        if o == r:
            deltas.append(0)
            continue
        try:
            view, addr = arena_import(arena.device, peers[o], slab, sizes[o])
        finally:
            for f in peers[o]:
                os.close(f)
        views.append(view)
        deltas.append(addr - arena.base)
    return deltas, views


def pull_replicas(sw: Swapper, peer_delta: list[int] | None = None, group=None, stream=None,
                  arena: Arena | None = None) -> dict:
    """Swap-in of k data-parallel replicas with the fused NVLink pull (NEXT-2): replica r restores its
    stripe over its own PCIe link (swap_restore_stripe); once every stripe has landed (barrier), one SM
    kernel per replica pulls the other stripes straight from the owners' HBM and checks every chunk from the
    registers that carried it (swap_pull_stripes); then the HBM verify pass. A closing barrier keeps any
    replica from overwriting its stripe while a peer may still be reading it. With `arena` (the replicas'
    regions live in VMM arenas, possibly released before the swap-in: the stripe restore re-acquires every
    slab) the peers' arenas are mapped after the stripe restores (map_replicas_arena) and unmapped at the end;
    otherwise `peer_delta` comes from map_replicas. Returns the verify result."""
    from .swap import arena_unimport

    k, r = dist.get_world_size(group), dist.get_rank(group)
    s = stream if stream is not None else torch.cuda.current_stream(sw.device)
    sw.restore_stripe(r, k, s)
    s.synchronize()
    dist.barrier(group=group)
    views = []
    if arena is not None:
        peer_delta, views = map_replicas_arena(arena, group)
    sw.pull_stripes(r, k, peer_delta, s)
    res = sw.verify(s, hbm_pass=True, raise_on_corrupt=False)
    dist.barrier(group=group)
    for v in views:
        arena_unimport(v)
    return res


def agree_restore(verify_result: dict, group=None) -> int:
    """K6: global number of bad chunks (fused restore check + HBM pass) over all ranks."""
    dev = _comm_device(group)
    t = torch.tensor([verify_result["n_bad"] + verify_result["hbm_n_bad"] + (0 if verify_result["manifest_ok"] else 1)],
                     dtype=torch.int64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return int(t.item())
