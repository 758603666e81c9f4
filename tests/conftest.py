import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def load_golden(name):
    """Parse a tests/golden/*.txt fixture: key/value lines and named int matrices."""
    path = os.path.join(ROOT, "tests", "golden", name)
    out, cur = {}, None
    with open(path) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            toks = line.split()
            if len(toks) == 1 and not toks[0].lstrip("-").isdigit():
                cur = toks[0]
                out[cur] = []
            elif len(toks) == 2 and not toks[0].lstrip("-").isdigit():
                out[toks[0]] = toks[1]
                cur = None
            else:
                out[cur].append([int(t) for t in toks])
    return out


@pytest.fixture
def golden():
    return load_golden
