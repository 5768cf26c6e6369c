"""BC parity: CUDA Brandes (forward sigma push/pull, backward dependency pull) vs the oracle,
max |x - r| / max(|r|, 1) <= 1e-4 (north_star; reading R11)."""
import itertools

import numpy as np
import pytest

import gen
import oracle
from tests import brute
from tests.conftest import tiny_graphs

pytestmark = pytest.mark.gpu
TOL = 1e-4
VARIANTS = list(itertools.product(["push", "pull"], ["thread", "twc", "wm", "cm", "strict"]))


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _close(x, r):
    err = np.abs(x - r) / np.maximum(np.abs(r), 1.0)
    assert err.max() <= TOL, err.max()


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny_all_sources(gsw, name):
    g = tiny_graphs()[name]
    x, _ = gsw.Graph(g.off, g.col).bc(list(range(g.n)))
    _close(x.cpu().numpy(), oracle.bc(g, list(range(g.n))))


def test_multigraph_and_random(gsw):
    g = gen.from_edges(4, [(0, 1), (0, 1), (1, 3), (0, 2), (2, 3)], dedupe=False)
    x, _ = gsw.Graph(g.off, g.col).bc([0, 3])
    _close(x.cpu().numpy(), oracle.bc(g, [0, 3]))
    for seed in range(4):
        g = brute.random_graph(np.random.default_rng(seed), 12, 0.3)
        x, _ = gsw.Graph(g.off, g.col).bc(list(range(g.n)))
        _close(x.cpu().numpy(), oracle.bc(g, list(range(g.n))))


@pytest.mark.parametrize("variant", VARIANTS, ids=["-".join(v) for v in VARIANTS])
def test_forced_variants(gsw, variant):
    for g in (gen.rmat(12, seed=8), gen.grid(30, 20)):
        G = gsw.Graph(g.off, g.col)
        G.force_config(direction=variant[0], load_balance=variant[1])
        srcs = gen.sources(g, 4)
        x, _ = G.bc(srcs)
        _close(x.cpu().numpy(), oracle.bc(g, srcs))


def test_c1_16_sources(gsw):
    g = gen.config_graph("C1")
    srcs = gen.sources(g, 16)
    x, st = gsw.Graph(g.off, g.col).bc(srcs, records=4096)
    _close(x.cpu().numpy(), oracle.bc(g, srcs))
    assert st["iterations"] > 16


def test_errors_and_empty(gsw):
    g = gen.rmat(8)
    G = gsw.Graph(g.off, g.col)
    with pytest.raises(gsw.GswError):
        G.bc([g.n])
    x, _ = G.bc([])
    assert np.all(x.cpu().numpy() == 0)


@pytest.mark.slow
def test_c4_16_sources(gsw):
    g = gen.config_graph("C4")
    srcs = gen.sources(g, 16)
    x, _ = gsw.Graph(g.off, g.col).bc(srcs)
    _close(x.cpu().numpy(), oracle.bc(g, srcs))
