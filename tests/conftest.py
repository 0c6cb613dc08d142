import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: multi-second CPU test")


def read_golden(name):
    """Parse a tests/golden/*.txt fixture: 'key value...' lines, '#' comments."""
    d = {"mem": [], "hit": []}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *v = line.split()
            if k == "mem":
                d["mem"].append(tuple(int(x) for x in v))
            elif k == "hit":
                d["hit"].append(v)
            elif k in ("R", "Q"):
                d[k] = v[0]
            elif k in ("ptrs", "locs"):
                d[k] = [int(x) for x in v]
            elif k[0] == "k" and k[1:].isdigit():  # expected triples at a parameter k (rare MEMs)
                d.setdefault(k, []).append(tuple(int(x) for x in v))
            else:
                d[k] = int(v[0])
    return d
