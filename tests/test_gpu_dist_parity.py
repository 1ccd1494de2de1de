"""Global-manifest parity across real ranks (SURVEY.md §4 distributed row, §8(e); §6).

Two processes share cuda:0 over gloo; each checkpoints its own real config-A shard (seed = rank) through
the C ABI, then the K5 all-gather, swap_set_global and the K6 agreement run exactly as in bench.py.
Every value is compared with the oracle: each rank's summary with oracle.summary over the oracle image
of the same shard; the gathered bytes with the concatenation of those oracle summaries; the installed
global digest with oracle.global_digest; and after a single-bit flip injected into rank 1's image, the
K6 count on both ranks is exactly rank 1's two detections of that chunk (fused restore check + HBM pass),
the chunk the oracle restore of the same flipped image reports."""
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
        specs = W.config_a(rank)
        arena, host, base, offs, sw_regions, or_regions = device_case(specs, rank)
        rc, ref, moff = orc.checkpoint(or_regions, host, base, orc.CRC32C, C, 4096, rank=rank, world=world, threads=4)
        assert rc == 0
        ref_summary = orc.summary(ref[moff:], ref.size)
        s = torch.cuda.Stream()
        out = {}
        with swap.Swapper(sw_regions, chunk_bytes=C, checksum=swap.SWAP_CHECKSUM_CRC32C, rank=rank, world=world) as sw, \
                torch.cuda.stream(s):
            sw.checkpoint(s)
            out["image_equal"] = bool(np.array_equal(sw.image(), ref))
            out["summary"] = sw.summary()
            out["ref_summary"] = ref_summary
            allb, digest = sdist.gather_manifest(sw, None)  # K5 + swap_set_global
            out["gathered"], out["digest"] = allb, digest
            # clean restore: every rank agrees on zero bad chunks
            poison(arena, specs, offs)
            sw.restore(s)
            out["bad_clean"] = sdist.agree_restore(sw.verify(s, raise_on_corrupt=False), None)
            out["mem_equal"] = bool(np.array_equal(arena.cpu().numpy(), host))
            # rank 1 flips one payload bit of its image: K6 must count exactly that chunk on both ranks
            if rank == 1:
                img = sw.image()
                pos = specs[0].nbytes // 2  # inside region 0, whose image offset is 0
                img[pos] ^= 0x10
                flipped = ref.copy()
                flipped[pos] ^= 0x10
                mem = host.copy()
                out["oracle_bad"] = orc.restore(flipped, moff, mem, base)[1:]
                out["flip_chunk"] = pos // C
            poison(arena, specs, offs)
            sw.restore(s)
            res = sw.verify(s, raise_on_corrupt=False)
            out["verify_flip"] = (res["n_bad"], res["first_bad_chunk"], res["hbm_n_bad"])
            out["bad_flip"] = sdist.agree_restore(res, None)
        q.put((rank, out))
    except Exception:  # report instead of leaving the parent waiting on the queue
        import traceback

        q.put((rank, {"error": traceback.format_exc()}))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_ranks_global_manifest_vs_oracle(orc):
    world = 2
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
    for rank in range(world):
        assert "error" not in res[rank], res[rank].get("error")
    want = res[0]["ref_summary"] + res[1]["ref_summary"]
    for rank in range(world):
        r = res[rank]
        assert r["image_equal"], rank
        assert r["summary"] == r["ref_summary"], rank
        assert r["gathered"] == want, rank
        assert r["digest"] == orc.global_digest(want), rank
        assert r["bad_clean"] == 0 and r["mem_equal"], rank
        # rank 1's flipped chunk is seen by the fused restore check and by the HBM pass: K6 sums both
        assert r["bad_flip"] == 2, rank
    g = res[1]["flip_chunk"]
    assert res[0]["verify_flip"] == (0, (1 << 64) - 1, 0)
    assert res[1]["verify_flip"] == (1, g, 1)
    assert res[1]["oracle_bad"] == (1, g)
