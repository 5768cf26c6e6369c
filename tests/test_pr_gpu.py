"""PageRank parity: CUDA power iteration vs the fp64 oracle, max relative per-vertex error <= 1e-5
(north_star; reading R10), every direction x load-balance candidate."""
import itertools

import numpy as np
import pytest

import gen
import oracle
from tests.conftest import tiny_graphs

pytestmark = pytest.mark.gpu
RTOL = 1e-5
VARIANTS = list(itertools.product(["push", "pull"], ["thread", "twc", "wm", "cm", "strict"]))


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _close(x, r):
    rel = np.abs(x - r) / r
    assert rel.max() <= RTOL, rel.max()


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny(gsw, name):
    g = tiny_graphs()[name]
    x, _ = gsw.Graph(g.off, g.col).pr(0.85, 20)
    _close(x.cpu().numpy(), oracle.pr(g, 0.85, 20))


@pytest.mark.parametrize("variant", VARIANTS, ids=["-".join(v) for v in VARIANTS])
def test_forced_variants(gsw, variant):
    for g in (gen.rmat(12, seed=4), gen.grid(40, 17)):
        G = gsw.Graph(g.off, g.col)
        G.force_config(direction=variant[0], load_balance=variant[1])
        for iters in (0, 1, 20):
            x, st = G.pr(0.85, iters, records=64)
            _close(x.cpu().numpy(), oracle.pr(g, 0.85, iters))
            assert st["iterations"] == iters


def test_survey_pins_and_mass(gsw):
    x, _ = gsw.Graph(*(lambda g: (g.off, g.col))(gen.from_edges(4, [(0, 1), (1, 2)]))).pr(0.85, 20)
    # exact-rational survey values; the GPU stores contributions in fp32 (accumulation fp64), so
    # the bar is the north_star's 1e-5 (R10), not the oracle's own 1e-9 pin
    np.testing.assert_allclose(x.cpu().numpy(), [0.246311087850, 0.459758776680, 0.246311087850, 0.047619047619],
                               rtol=RTOL)
    g = gen.rmat(14, seed=2)
    x, _ = gsw.Graph(g.off, g.col).pr(0.85, 20)
    assert abs(x.sum().item() - 1.0) < 1e-6


def test_directed_csc(gsw):
    rng = np.random.default_rng(3)
    n = 500
    edges = [(int(u), int(v)) for u, v in rng.integers(0, n, size=(3000, 2)) if u != v]
    g = gen.from_edges(n, edges, symmetric=False)
    csc = gen.from_edges(n, [(v, u) for u, v in edges], symmetric=False)
    G = gsw.Graph(g.off, g.col, csc=(csc.off, csc.col))
    x, _ = G.pr(0.85, 20)
    _close(x.cpu().numpy(), oracle.pr(g, 0.85, 20, csc=csc))


def test_c1_full(gsw):
    g = gen.config_graph("C1")
    x, _ = gsw.Graph(g.off, g.col).pr(0.85, 20)
    _close(x.cpu().numpy(), oracle.pr(g, 0.85, 20))


@pytest.mark.slow
def test_c3_full(gsw):
    g = gen.config_graph("C3")
    x, _ = gsw.Graph(g.off, g.col).pr(0.85, 20)
    _close(x.cpu().numpy(), oracle.pr(g, 0.85, 20))


def _stream_graph():
    """Rows that span several 8192-edge tiles (two hubs), a run of degree-1 rows with isolated
    vertices interleaved (more than 8192 rows inside one tile's edge range without relabeling),
    and random short rows."""
    rng = np.random.default_rng(5)
    n = 60000
    edges = [(0, v) for v in range(2, 26000)] + [(1, v) for v in range(3, 12000, 2)]
    edges += [(v, v + 1) for v in range(30000, 58000, 3)]          # v+2 stays isolated
    edges += [(int(u), int(v)) for u, v in rng.integers(2, 30000, size=(20000, 2)) if u != v]
    return gen.from_edges(n, edges)


@pytest.mark.parametrize("relabel", [True, False])
@pytest.mark.parametrize("cache", [None, "0", "1000"])
def test_stream_tiles(gsw, monkeypatch, relabel, cache):
    """The edge-tiled stream kernel (AUTO = pull + STRICT): tile-crossing rows, the shared-memory
    slice and the global-memory fallback, the contribution cache on and off."""
    if not relabel:
        monkeypatch.setenv("GSW_NO_RELABEL", "1")
    if cache is not None:
        monkeypatch.setenv("GSW_PR_CACHE", cache)
    g = _stream_graph()
    G = gsw.Graph(g.off, g.col)
    for iters in (1, 2, 20):
        x, st = G.pr(0.85, iters, records=64)
        _close(x.cpu().numpy(), oracle.pr(g, 0.85, iters))
        assert st["records"][0]["load_balance"] == gsw.LB_STRICT


@pytest.mark.parametrize("blocks", ["1", "2", "3", "8"])
def test_source_blocked(gsw, monkeypatch, blocks):
    """The source-blocked gather (pr_blocked.cu; AUTO when pr/deg overflows L2, i.e. C5): forced
    on small graphs with 1-8 source blocks, heavy rows (> 4096 in-edges) as chunk tasks, with
    and without relabeling, 0 / 1 / 20 iterations."""
    monkeypatch.setenv("GSW_PR_BLOCKED", "1")
    monkeypatch.setenv("GSW_PR_BLOCKS", blocks)
    for g in (_stream_graph(), gen.rmat(13, seed=2), gen.from_edges(10, [(0, 1), (2, 3)])):
        G = gsw.Graph(g.off, g.col)
        for iters in (0, 1, 20):
            x, st = G.pr(0.85, iters)
            _close(x.cpu().numpy(), oracle.pr(g, 0.85, iters))
            assert st["iterations"] == iters
