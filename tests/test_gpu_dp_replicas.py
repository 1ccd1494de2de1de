"""Data-parallel replica swap-in (NEXT-2 second half): two replicas of the same engine
image share cuda:0 over gloo; each restores only its stripe of the restore groups (swap_restore_stripe)
and the stripes are exchanged by in-place broadcasts (dist.restore_replicas), then every replica verifies
all chunks from HBM. Checked against the oracle: the restored arenas equal the original bytes, a bit
flipped in replica 1's image inside a group replica 1 owns is reported (same chunk) by both replicas' HBM
passes and by replica 1's fused check, and a flip inside a group replica 0 owns is never read. The fused
NVLink pull variant (CUDA IPC mapping of the other replica's arena, swap_pull_stripes) restores the same
bytes, and there replica 0's pull kernel itself reports the chunk it read corrupted from replica 1."""
import os
import tempfile

import pytest
import torch.multiprocessing as mp

from conftest import ROOT

pytestmark = pytest.mark.gpu
C = 1 << 16


def _worker(rank, world, init_file, q):
    import sys

    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import numpy as np
    import torch
    import torch.distributed as dist

    import oracle as orc
    import workloads as W
    from gpu_util import device_case, poison
    from paper_conf_sc_stoyanovsracb25_b200 import dist as sdist
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    dist.init_process_group("gloo", init_method=f"file://{init_file}", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        specs = W.config_a(3)  # the same engine on both replicas
        arena, host, base, offs, sw_regions, or_regions = device_case(specs, 3)
        rc, ref, moff = orc.checkpoint(or_regions, host, base, orc.CRC32C, C, 4096, threads=4)
        s = torch.cuda.Stream()
        out = {}
        with swap.Swapper(sw_regions, chunk_bytes=C, checksum=swap.SWAP_CHECKSUM_CRC32C, pipe_mib=4) as sw, \
                torch.cuda.stream(s):
            sw.checkpoint(s)
            out["image_equal"] = bool(np.array_equal(sw.image(), ref))
            spans = sw.restore_spans()
            out["n_groups"] = len({g for (g, _, _, _) in spans})
            out["spans_cover"] = sum(nb for (_, _, _, nb) in spans) == sum(r.nbytes for r in specs)
            poison(arena, specs, offs)
            res = sdist.restore_replicas(sw, None, s)
            out["clean"] = (res["n_bad"], res["hbm_n_bad"], res["manifest_ok"])
            out["mem_equal"] = bool(np.array_equal(arena.cpu().numpy(), host))
            # flips in replica 1's image: one in a group replica 1 owns, one in a group replica 0 owns
            img = sw.image()
            own1 = next(sp for sp in spans if sp[0] % world == 1)
            own0 = next(sp for sp in spans if sp[0] % world == 0)  # replica 0's stripe
            p1, p0 = own1[2] + own1[3] // 2, own0[2] + own0[3] // 2
            chunk_of = {}
            for pos in (p1, p0):  # the chunk holding image offset pos, from the oracle manifest
                man = ref[moff:]
                n, m = int.from_bytes(man[32:40].tobytes(), "little"), int.from_bytes(man[40:48].tobytes(), "little")
                for gi in range(m):
                    rec = man[64 + 48 * n + 32 * gi:64 + 48 * n + 32 * gi + 32].tobytes()
                    ri, lo, ln = int.from_bytes(rec[0:4], "little"), int.from_bytes(rec[8:16], "little"), int.from_bytes(rec[16:24], "little")
                    off = int.from_bytes(man[64 + 48 * ri + 24:64 + 48 * ri + 32].tobytes(), "little")
                    if off + lo <= pos < off + lo + ln:
                        chunk_of[pos] = gi
            if rank == 1:
                img[p1] ^= 0x01
                img[p0] ^= 0x01
            poison(arena, specs, offs)
            res = sdist.restore_replicas(sw, None, s)
            out["flip"] = (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"], res["hbm_first_bad"])
            out["flip_chunk"] = chunk_of[p1]
            # the same with the fused NVLink pull (CUDA IPC of the other replica's arena; same device here):
            # replica 0's pull kernel reads replica 1's corrupted stripe and its fused check reports it
            deltas, bases = sdist.map_replicas(base, 0, None)
            poison(arena, specs, offs)
            res = sdist.pull_replicas(sw, deltas, None, s)
            out["pull_flip"] = (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"], res["hbm_first_bad"])
            if rank == 1:  # undo the flips: a clean pulled swap-in restores every byte
                img[p1] ^= 0x01
                img[p0] ^= 0x01
            dist.barrier()
            poison(arena, specs, offs)
            res = sdist.pull_replicas(sw, deltas, None, s)
            out["pull_clean"] = (res["n_bad"], res["hbm_n_bad"], res["manifest_ok"])
            out["pull_mem_equal"] = bool(np.array_equal(arena.cpu().numpy(), host))
            for b in bases:
                swap.ipc_close(0, b)
        q.put((rank, out))
    except Exception:  # report instead of leaving the parent waiting on the queue
        import traceback

        q.put((rank, {"error": traceback.format_exc()}))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(400)
@pytest.mark.parametrize("world", [2, 3])
def test_replicas_striped_restore(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with tempfile.TemporaryDirectory() as d:
        init_file = os.path.join(d, "pg")
        procs = [ctx.Process(target=_worker, args=(r, world, init_file, q)) for r in range(world)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=240) for _ in range(world))
        for p in procs:
            p.join(60)
            assert p.exitcode == 0
    for r in range(world):
        assert "error" not in res[r], res[r].get("error")
        assert res[r]["image_equal"] and res[r]["spans_cover"] and res[r]["n_groups"] >= 2 * world
        assert res[r]["clean"] == (0, 0, 1) and res[r]["mem_equal"]
    g = res[1]["flip_chunk"]
    # replica 1 moved the flipped chunk itself (fused check) and broadcast it: every HBM pass sees it;
    # the flip in replica 0's stripe was never read
    assert res[1]["flip"] == (1, g, 1, g)
    for r in range(world):
        if r != 1:
            assert res[r]["flip"] == (0, (1 << 64) - 1, 1, g), r
            # fused pull: replica r's pull kernel checks the chunk it read from replica 1's HBM
            assert res[r]["pull_flip"] == (1, g, 1, g), r
    assert res[1]["pull_flip"] == (1, g, 1, g)
    for r in range(world):
        assert res[r]["pull_clean"] == (0, 0, 1) and res[r]["pull_mem_equal"], r


@pytest.mark.parametrize("kind", [1, 2])
def test_fused_pull_in_process(kind):
    """swap_pull_stripes with the peer replica as a second arena of this process (the same bytes at a
    constant shift): every byte restored, and a corruption of the peer's HBM copy inside the pulled stripe
    is reported by the pull kernel's fused check as exactly its chunk (the oracle's chunk of that byte)."""
    import sys

    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import numpy as np
    import torch

    import oracle as orc
    import workloads as W
    from gpu_util import device_case, poison
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    specs = W.config_a(5) + W.edge_tables(4096)["chunk_pm1"]
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, 5)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, kind, 4096, 4096, threads=4)
    peer = arena.clone()
    delta = peer.data_ptr() - base
    s = torch.cuda.Stream()
    with swap.Swapper(sw_regions, chunk_bytes=4096, checksum=kind, pipe_mib=2) as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        assert np.array_equal(sw.image(), ref)
        poison(arena, specs, offs)
        sw.restore_stripe(0, 2, s)
        sw.pull_stripes(0, 2, [0, delta], s)
        res = sw.verify(s)
        assert (res["n_bad"], res["hbm_n_bad"]) == (0, 0)
        assert np.array_equal(arena.cpu().numpy(), host)
        # corrupt one byte of the peer copy inside a group of stripe 1
        g1 = next(sp for sp in sw.restore_spans() if sp[0] % 2 == 1)
        dev = g1[1] + g1[3] // 3
        peer[dev - base] ^= 0x40
        # the oracle's chunk of that byte: region i holding it, chunk (dev - addr_i) // C
        i = next(k for k, (_, a, nb, _) in enumerate(or_regions) if a <= dev < a + nb)
        chunk = sum(-(-r.nbytes // 4096) for r in specs[:i]) + (dev - or_regions[i][1]) // 4096
        poison(arena, specs, offs)
        sw.restore_stripe(0, 2, s)
        sw.pull_stripes(0, 2, [0, delta], s)
        res = sw.verify(s, raise_on_corrupt=False)
        assert (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"], res["hbm_first_bad"]) == (1, chunk, 1, chunk)


def test_stripe_pull_with_policies_masks_and_released_arena():
    """Replica A in a released, bound VMM arena with a DISCARD region and a touched-chunk mask: the stripe
    restore re-acquires HBM for *every* group (the pulled ones included), zero-fills the zero chunks in full,
    and the fused pull from replica B (a cudaMalloc copy) fills the rest -- equal to the oracle's
    policy_view, the image equal to the oracle's checkpoint of that view."""
    import sys

    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import numpy as np
    import torch

    import oracle as orc
    import workloads as W
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    C = 1 << 16
    specs = W.scaled(W.config_b(), 96 << 20)
    offs, total = W.place(specs)
    arena = swap.Arena(total)
    base, view = arena.alloc(total)
    W.fill_device_arena(view, specs, offs, seed=9)
    peer = view.clone()  # replica B: the same bytes, cudaMalloc'd
    host = view.cpu().numpy()
    regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
    or_regions = [(i, a, n, k) for (a, n, k, i) in regions]
    big = max(range(len(specs)), key=lambda i: specs[i].nbytes)
    disc = next(i for i in range(len(specs)) if i != big and specs[i].nbytes > C)
    keep = (np.arange(-(-specs[big].nbytes // C)) % 3 != 1).astype(np.uint8)
    s = torch.cuda.Stream()
    with swap.Swapper(regions, chunk_bytes=C, pipe_mib=4) as sw, torch.cuda.stream(s):
        sw.set_region_policy(disc, "discard")
        sw.set_chunk_mask(big, keep)
        sw.bind_arena(arena)
        sw.checkpoint(s)
        pol = [orc.SAVE] * len(specs)
        pol[disc] = orc.DISCARD
        want = orc.policy_view(or_regions, pol, host, host, base, C, {big: keep})
        rc, ref, _ = orc.checkpoint(or_regions, want, base, orc.CRC32C, C, 4096, threads=8)
        assert rc == 0 and np.array_equal(sw.image(), ref)
        arena.release()
        sw.restore_stripe(1, 2, s)
        sw.pull_stripes(1, 2, [peer.data_ptr() - base, 0], s)
        res = sw.verify(s)
        assert (res["n_bad"], res["hbm_n_bad"]) == (0, 0) and arena.resident
        back = arena.tensor(0, total).cpu().numpy()
        for r, o in zip(specs, offs):
            assert np.array_equal(back[o:o + r.nbytes], want[o:o + r.nbytes]), r.name
        sw.bind_arena(None)
    arena.close()


def _arena_worker(rank, world, init_file, q):
    import sys

    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import numpy as np
    import torch
    import torch.distributed as dist

    import workloads as W
    from paper_conf_sc_stoyanovsracb25_b200 import dist as sdist
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    dist.init_process_group("gloo", init_method=f"file://{init_file}", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        specs = W.scaled(W.config_b(), 2300 << 20)  # > 2 slabs
        offs, total = W.place(specs)
        arena = swap.Arena(total)
        base, view = arena.alloc(total)
        W.fill_device_arena(view, specs, offs, seed=4)  # the same engine on every replica
        host = view.cpu().numpy()
        regions = [(base + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
        s = torch.cuda.Stream()
        out = {}
        with swap.Swapper(regions, pipe_mib=64) as sw, torch.cuda.stream(s):
            sw.bind_arena(arena)
            for it in range(2):  # swap out (HBM released), then the cooperative swap-in; twice
                sw.swap_out(arena, s)
                assert not arena.resident
                res = sdist.pull_replicas(sw, None, None, s, arena=arena)
                out[f"res{it}"] = (res["status"], res["n_bad"], res["hbm_n_bad"])
                back = arena.tensor(0, total).cpu().numpy()  # guards are fresh HBM after the release: regions only
                out[f"eq{it}"] = all(np.array_equal(back[o:o + r.nbytes], host[o:o + r.nbytes]) for r, o in zip(specs, offs))
            sw.bind_arena(None)
        arena.close()
        q.put((rank, out))
    except Exception:
        import traceback

        q.put((rank, {"error": traceback.format_exc()}))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(400)
def test_replicas_fused_pull_released_vmm_arenas():
    """DP replicas whose regions live in released VMM arenas (NEXT-1 + NEXT-2): the stripe restore
    re-acquires every slab, the replicas exchange their arenas' slab file descriptors over Unix sockets and
    map each other (swap_arena_export / swap_arena_import), the fused pull fills the other stripes, and the
    regions equal the original bytes on every replica, twice."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with tempfile.TemporaryDirectory() as d:
        init_file = os.path.join(d, "pg")
        procs = [ctx.Process(target=_arena_worker, args=(r, world, init_file, q)) for r in range(world)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=360) for _ in range(world))
        for p in procs:
            p.join(60)
            assert p.exitcode == 0
    for r in range(world):
        assert "error" not in res[r], res[r].get("error")
        for it in range(2):
            assert res[r][f"res{it}"] == (0, 0, 0) and res[r][f"eq{it}"], (r, it, res[r])
