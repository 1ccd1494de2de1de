"""Product planner + manifest writer (libswap, host-only entry points) vs the oracle, on CPU:
layout closed forms and byte-identical sealed manifests for random region tables (hypothesis)."""
import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

SIZES = st.one_of(st.integers(0, 64), st.integers(0, 5000), st.sampled_from([16, 4095, 4096, 4097, 1 << 16]))


@pytest.fixture(scope="module")
def swp():
    import paper_conf_sc_stoyanovsracb25_b200.swap as swap

    swap.load()
    return swap


def mk_regions(sizes, kinds, gaps):
    regs, pos = [], 0x10000
    for i, (s, k, gp) in enumerate(zip(sizes, kinds, gaps)):
        regs.append((pos, s, 1000 + i, k))
        pos += (s + 16 * gp + 15) // 16 * 16 + 16
    return regs


@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(sizes=st.lists(SIZES, min_size=1, max_size=12), C=st.sampled_from([16, 32, 64, 4096, 1 << 16]),
       A=st.sampled_from([16, 64, 4096]), kind=st.sampled_from([1, 2]), data=st.data())
def test_manifest_bytes_match_oracle(swp, orc, sizes, C, A, kind, data):
    kinds = data.draw(st.lists(st.integers(0, 3), min_size=len(sizes), max_size=len(sizes)))
    gaps = data.draw(st.lists(st.integers(0, 40), min_size=len(sizes), max_size=len(sizes)))
    regs = mk_regions(sizes, kinds, gaps)
    cfg = swp.swap_config_default()
    cfg.chunk_bytes, cfg.align, cfg.checksum = C, A, kind
    st_, payload, m, moff, ib = swp.swap_plan_layout(regs, cfg)
    assert st_ == 0
    # oracle: build the image from random memory, take its chunk checksums and manifest
    base = regs[0][0]
    span = regs[-1][0] + regs[-1][1] - base + 16
    mem = np.random.default_rng(len(sizes) * 7 + C).integers(0, 256, span, dtype=np.uint8)
    orc_regs = [(rid, a, nb, k) for (a, nb, rid, k) in regs]
    rc, img, omoff = orc.checkpoint(orc_regs, mem, base, kind, C, A)
    assert rc == 0 and (omoff, img.size) == (moff, ib)
    p = orc.plan(orc_regs, C, A)
    assert (p.payload_bytes, p.n_chunks) == (payload, m)
    man = img[moff:]
    cs = [int(man[64 + 48 * len(regs) + 32 * g + 24:64 + 48 * len(regs) + 32 * g + 32].view("<u8")[0]) for g in range(m)]
    st2, ours = swp.swap_plan_manifest(regs, cfg, cs)
    assert st2 == 0 and ours == man.tobytes()


def test_plan_rejects_like_oracle(swp, orc):
    cfg = swp.swap_config_default()
    for regs in ([(0x1008, 10, 1, 0)], [(0x1000, 0x200, 1, 0), (0x1100, 16, 2, 0)],
                 [(0x1000, 16, 1, 0), (0x2000, 16, 1, 0)], [(0x1000, 16, 1, 7)], []):
        st_ = swp.swap_plan_layout(regs, cfg)[0]
        assert st_ == swp.SWAP_EINVAL
        assert orc.plan([(rid, a, nb, k) for (a, nb, rid, k) in regs], 1 << 20, 4096).rc == orc.EINVAL
