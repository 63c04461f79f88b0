import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU test")


GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_grid(name):
    """Parse a tests/golden figure: returns (params dict, rows list, comment lines)."""
    params, rows, comments = {}, [], []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line:
                continue
            if line.startswith("#"):
                comments.append(line[1:].strip())
                continue
            if "=" in line:
                for tok in line.split():
                    k, v = tok.split("=")
                    params[k] = int(v)
                continue
            rows.append([int(x) for x in line.split()])
    return params, rows, comments


def grid_to_cells(rows):
    """rows[bank][column] -> flat list indexed by address column*w + bank."""
    w = len(rows)
    ncol = len(rows[0])
    return [rows[addr % w][addr // w] for addr in range(w * ncol)]


def splits_from_comments(comments):
    for c in comments:
        if c.startswith("splits:"):
            return [tuple(int(x) for x in t.split(",")) for t in c[len("splits:"):].split()]
    return None


@pytest.fixture
def golden():
    return load_grid
