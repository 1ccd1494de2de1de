"""world_size-2 gloo run of the shard coordinator's host logic:
K5 all-gather of the 64-B summaries -> libswap's merge/digest, checked against the oracle;
K6 all-reduce of mismatch counts."""
import os
import struct
import tempfile

import pytest
import torch.multiprocessing as mp

from conftest import ROOT

SUM = struct.Struct("<IIIIQQQQQQ")


def _worker(rank, world, init_file, q):
    import sys

    sys.path.insert(0, ROOT)
    import torch.distributed as dist

    dist.init_process_group("gloo", init_method=f"file://{init_file}", rank=rank, world_size=world)
    try:
        from paper_conf_sc_stoyanovsracb25_b200 import dist as sdist

        mine = SUM.pack(rank, world, 2, 10 + rank, 100 * (rank + 1), 10 ** 9 * (rank + 1), 10 ** 9 * (rank + 1) + 4096,
                        0x1234 + rank, 0x9876 * (rank + 1), 0)
        allb = sdist.all_gather_summaries(mine, None)
        digest = sdist.merge_global(allb)
        bad = sdist.agree_restore({"n_bad": rank, "hbm_n_bad": 0, "manifest_ok": 1}, None)
        q.put((rank, allb, digest, bad))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(120)
def test_gloo_world2_gather_and_agree(orc):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with tempfile.TemporaryDirectory() as d:
        init_file = os.path.join(d, "pg")
        procs = [ctx.Process(target=_worker, args=(r, world, init_file, q)) for r in range(world)]
        for p in procs:
            p.start()
        out = [q.get(timeout=100) for _ in range(world)]
        for p in procs:
            p.join(30)
            assert p.exitcode == 0
    out.sort()
    expect = b"".join(
        SUM.pack(r, world, 2, 10 + r, 100 * (r + 1), 10 ** 9 * (r + 1), 10 ** 9 * (r + 1) + 4096, 0x1234 + r,
                 0x9876 * (r + 1), 0) for r in range(world))
    for rank, allb, digest, bad in out:
        assert allb == expect
        assert digest == orc.global_digest(expect)
        assert bad == 0 + 1  # ranks contributed 0 and 1 bad chunks
