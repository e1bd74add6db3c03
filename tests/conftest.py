import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: full-size configs (minutes)")


def load_golden(name):
    """Parse a tests/golden/*.txt fixture -> dict(n, source, arcs, dist, V, E)."""
    d = {"arcs": []}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *vals = line.split()
            if k == "arc":
                d["arcs"].append(tuple(int(x) for x in vals))
            elif k == "dist":
                d["dist"] = [int(x) for x in vals]
            else:
                d[k if k != "source" else "source"] = int(vals[0])
    return d


def golden_names():
    return sorted(f for f in os.listdir(GOLDEN) if f.endswith(".txt") and not f.startswith("bucket"))
