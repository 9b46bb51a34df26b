import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
HERE = os.path.dirname(os.path.abspath(__file__))
if HERE not in sys.path:
    sys.path.insert(0, HERE)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run with -m gpu)")
    config.addinivalue_line("markers", "slow: long-running (full-size oracle runs)")


@pytest.fixture(scope="session")
def fig2():
    """Fig. 2 database and printed vertical lists (tests/golden/fig2.txt)."""
    txs, vert = {}, []
    with open(os.path.join(HERE, "golden", "fig2.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            if line.startswith("T "):
                tid, items = line[2:].split(":")
                txs[int(tid)] = [int(x) for x in items.split()]
            elif line.startswith("V "):
                cand, tids, bits = [p.strip() for p in line[2:].split("|")]
                vert.append((tuple(int(x) for x in cand.split()), [int(x) for x in tids.split()], bits))
    ordered = [txs[i] for i in sorted(txs)]
    return ordered, vert
