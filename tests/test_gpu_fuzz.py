"""Seeded random parity sweep over the whole configuration space (SURVEY §4 parity row, widened):
each case draws a region table (1-40 regions; sizes 0 B - 6 MiB with ragged tails, log-uniform so
tiny, one-chunk and many-chunk regions mix), device-address skews (multiples of 16 B), a chunk size C
(16 B - 16 MiB), an image alignment A (16 B - 64 KiB), a CRC segment size, a mover grid, a CE_PIPE group
size, a checksum and a mechanism. Through the C ABI, compared with the oracle byte for byte: the whole
image (payload, zero padding, manifest), the restored arena (regions and guard bands) and the verify
counters; then a single-bit flip in the image must be reported as exactly its chunk."""
import numpy as np
import pytest

import workloads as W
from gpu_util import device_case, poison

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MECHS = ["auto", "sm", "ce_region", "ce_chunk", "ce_batch", "ce_pipe"]
U64_MAX = (1 << 64) - 1


def draw(seed: int):
    rng = np.random.Generator(np.random.PCG64(1000 + seed))
    n = int(rng.integers(1, 41))
    sizes = []
    for _ in range(n):
        r = rng.random()
        if r < 0.08:
            sizes.append(0)
        elif r < 0.3:
            sizes.append(int(rng.integers(1, 600)))
        else:
            sizes.append(int(np.exp(rng.uniform(np.log(600), np.log(6 << 20)))))
    kind = int(rng.integers(1, 3))
    C = 1 << int(rng.integers(4, 25))  # 16 B .. 16 MiB
    if C < 4096 and sum(sizes) // C > 400_000:  # keep the manifest (32 B per chunk) small
        C = 4096
    A = 1 << int(rng.integers(4, 17))
    mech = MECHS[int(rng.integers(0, len(MECHS)))]
    seg = 0 if rng.random() < 0.5 else 1 << int(rng.integers(12, 19))
    grid = 0 if rng.random() < 0.6 else int(rng.choice([1, 3, 37, 148, 296]))
    pipe = 0 if rng.random() < 0.5 else int(rng.choice([1, 2, 5]))
    skew = [16 * int(rng.integers(0, 16)) for _ in range(n)]
    specs = [W.RegionSpec(f"f{i}", int(rng.integers(0, 4)), s) for i, s in enumerate(sizes)]
    return specs, skew, dict(kind=kind, C=C, A=A, mech=mech, seg=seg, grid=grid, pipe=pipe), int(rng.integers(0, 1 << 30))


@pytest.mark.parametrize("seed", range(160))
def test_random_configuration(seed):
    import oracle as orc
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    specs, skew, k, flip = draw(seed)
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, seed, skew)
    rc, ref, moff = orc.checkpoint(or_regions, host, base, k["kind"], k["C"], k["A"], threads=8)
    assert rc == 0
    s = torch.cuda.Stream()
    with swap.Swapper(sw_regions, chunk_bytes=k["C"], checksum=k["kind"], mechanism=k["mech"], align=k["A"],
                      seg_bytes=k["seg"], grid_ctas=k["grid"], pipe_mib=k["pipe"]) as sw, torch.cuda.stream(s):
        sw.checkpoint(s)
        img = sw.image()
        diff = np.flatnonzero(img != ref)
        assert diff.size == 0, f"{k}: image differs at {diff[:8]} (manifest at {moff})"
        poison(arena, specs, offs)
        sw.restore(s)
        res = sw.verify(s, hbm_pass=True)
        assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0, (k, res)
        torch.cuda.synchronize()
        back = arena.cpu().numpy()
        assert np.array_equal(back, host), f"{k}: restored arena differs at {np.flatnonzero(back != host)[:8]}"
        # one flipped payload bit -> exactly the chunk holding it
        nonempty = [i for i, r in enumerate(specs) if r.nbytes]
        if nonempty:
            plan = orc.plan(or_regions, k["C"], k["A"])
            i = nonempty[flip % len(nonempty)]
            byte = (flip >> 3) % specs[i].nbytes
            img[plan.off[i] + byte] ^= 1 << (flip & 7)
            want = plan.first[i] + byte // k["C"]
            poison(arena, specs, offs)
            sw.restore(s)
            res = sw.verify(s, hbm_pass=True, raise_on_corrupt=False)
            img[plan.off[i] + byte] ^= 1 << (flip & 7)
            assert (res["n_bad"], res["first_bad_chunk"]) == (1, want), (k, res, want)


@pytest.mark.parametrize("seed", range(60))
def test_random_policies_and_sequences(seed):
    """Random per-region SAVE / SAVE_ONCE / DISCARD policies (reading 24) over a random
    configuration, through a sequence: checkpoint, the engine mutates memory, checkpoint again, restore
    twice (restore-many), mutate, checkpoint a third time, restore. Every image and every
    restored arena equals the oracle applied to oracle.policy_view."""
    import oracle as orc
    from paper_conf_sc_stoyanovsracb25_b200 import swap

    specs, skew, k, flip = draw(10_000 + seed)
    rng = np.random.Generator(np.random.PCG64(flip))
    arena, host, base, offs, sw_regions, or_regions = device_case(specs, seed, skew)
    pol = [int(rng.choice([orc.SAVE, orc.SAVE_ONCE, orc.DISCARD], p=[0.5, 0.3, 0.2])) for _ in specs]
    C, A, kind = k["C"], k["A"], k["kind"]

    def mutate(mem):
        out = mem.copy()
        for r, o in zip(specs, offs):
            if r.nbytes and rng.random() < 0.6:
                lo = int(rng.integers(0, r.nbytes))
                out[o + lo:o + min(r.nbytes, lo + 1 + int(rng.integers(0, 5000)))] ^= np.uint8(rng.integers(1, 256))
        return out

    s = torch.cuda.Stream()
    with swap.Swapper(sw_regions, chunk_bytes=C, checksum=kind, mechanism=k["mech"], align=A, seg_bytes=k["seg"],
                      grid_ctas=k["grid"], pipe_mib=k["pipe"]) as sw, torch.cuda.stream(s):
        for i, p in enumerate(pol):
            sw.set_region_policy(i, p)
        first = host.copy()
        now = host
        for step in range(3):
            if step:
                now = mutate(now)
                arena.copy_(torch.from_numpy(now).cuda())
                torch.cuda.synchronize()
            sw.checkpoint(s)
            view = orc.policy_view(or_regions, pol, now, first, base)
            rc, ref, _ = orc.checkpoint(or_regions, view, base, kind, C, A, threads=8)
            assert rc == 0
            diff = np.flatnonzero(sw.image() != ref)
            assert diff.size == 0, f"step {step} {k} pol={pol}: image differs at {diff[:8]}"
            for _ in range(2 if step == 1 else 1):
                poison(arena, specs, offs)
                sw.restore(s)
                res = sw.verify(s, hbm_pass=True)
                assert res["status"] == 0 and res["n_bad"] == 0 and res["hbm_n_bad"] == 0, (step, k, res)
                torch.cuda.synchronize()
                back = arena.cpu().numpy()
                assert np.array_equal(back, view), f"step {step} {k}: restored arena differs at {np.flatnonzero(back != view)[:8]}"
