import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the built CUDA library")
    config.addinivalue_line("markers", "slow: large-size parity cases")
    config.addinivalue_line("markers", "c5: the Kronecker scale-26 config (2.1e9 entries; minutes of host work)")


def tiny_graphs():
    """Hand-built graphs: path, star, cycle, complete, grid, disconnected,
    isolated vertices, plus a multigraph with parallel edges."""
    import gen
    g = {}
    g["path5"] = gen.from_edges(5, [(i, i + 1) for i in range(4)])
    g["star5"] = gen.from_edges(5, [(0, i) for i in range(1, 5)])
    g["cycle6"] = gen.from_edges(6, [(i, (i + 1) % 6) for i in range(6)])
    g["k5"] = gen.from_edges(5, [(i, j) for i in range(5) for j in range(i + 1, 5)])
    g["grid3x4"] = gen.grid(3, 4)
    g["two_comp"] = gen.from_edges(7, [(0, 1), (1, 2), (3, 4), (4, 5), (5, 3)])
    g["isolated"] = gen.from_edges(6, [(1, 3), (3, 5)])
    g["single"] = gen.from_edges(1, [])
    g["fig4"] = gen.from_edges(6, [(0, 1), (1, 2), (1, 3), (2, 4), (3, 4), (4, 5)])
    return g


@pytest.fixture(scope="session")
def tiny():
    return tiny_graphs()
