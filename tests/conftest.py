import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running (full-size configs)")


def read_golden(name):
    """Rows of a tests/golden/*.txt fixture: '|'-separated fields, '#' comments skipped."""
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.rstrip("\n")
            if not line.strip() or line.lstrip().startswith("#"):
                continue
            rows.append([x.strip() for x in line.split("|")])
    return rows


def decode_input(spec: str) -> bytes:
    if spec.startswith("@ascii:"):
        return spec[len("@ascii:"):].encode()
    if spec.startswith("@fill:"):
        b, n = spec[len("@fill:"):].split("x")
        return bytes([int(b, 16)]) * int(n)
    if spec.startswith("@sanity:"):
        n = int(spec[len("@sanity:"):])
        g, out = 2654435761, bytearray()
        for _ in range(n):
            out.append(g >> 56)
            g = (g * 11400714785074694797) % (1 << 64)
        return bytes(out)
    return bytes.fromhex(spec)


@pytest.fixture(scope="session")
def orc():
    import oracle

    oracle.lib()
    return oracle
