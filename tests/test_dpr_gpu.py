"""Delta-PageRank parity (reading R16): gsw_dpr vs oracle.dpr.

Tolerance, derived from the invariant x = r + (I - dM)^{-1} delta (oracle.c orc_dpr): a run with
threshold eps = tol (1-d)/N ends with every residual <= eps, so its result r satisfies
0 <= x - r and ||x - r||_1 <= N eps / (1-d) = tol, whatever order the residuals were pushed in.
The GPU and the oracle therefore each lie in that band (pinned against dense solves in
test_oracle.py), and ||r_gpu - r_orc||_1 <= 2 tol.  fp64 atomics reorder sums, so a residual
within an ulp of eps may activate one iteration apart on the two sides: the comparison is the
band, not bit equality.  Inputs whose residuals stay far from eps (regular graphs) must follow
the oracle's trajectory: same iteration count, 1e-12 relative agreement.
"""
import numpy as np
import pytest

import gen
import oracle
from tests.conftest import tiny_graphs

pytestmark = pytest.mark.gpu
D = 0.85


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _fixed_point(g, csc=None, d=D):
    x, _ = oracle.dpr(g, d, -1.0, max_iters=300, csc=csc)   # Neumann sum, d^300 < 1e-21
    return x


def _band(r, x, tol):
    gap = x - r
    assert gap.min() >= -1e-12 * x.max(), gap.min()
    assert gap.sum() <= tol * (1 + 1e-9), (gap.sum(), tol)


def _check(gsw, g, tol, direction=None, csc=None):
    G = gsw.Graph(g.off, g.col) if csc is None else gsw.Graph(g.off, g.col, csc=(csc.off, csc.col))
    if direction:
        G.force_config(direction=direction)
    r, st = G.dpr(D, tol, records=4096)
    r = r.cpu().numpy()
    eps = tol * (1 - D) / g.n
    ro, it_o = oracle.dpr(g, D, eps, csc=csc)
    x = _fixed_point(g, csc)
    _band(r, x, tol)
    _band(ro, x, tol)
    assert np.abs(r - ro).sum() <= 2 * tol
    assert abs(st["iterations"] - it_o) <= 2
    return r, st


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny(gsw, name):
    g = tiny_graphs()[name]
    for tol in (1e-3, 1e-8):
        _check(gsw, g, tol)


@pytest.mark.parametrize("direction", [None, "push", "pull"])
def test_rmat_grid_directions(gsw, direction):
    for g in (gen.rmat(12, seed=4), gen.grid(40, 17), gen.rmat(10, 4, seed=9)):
        for tol in (1e-2, 1e-6):
            r, st = _check(gsw, g, tol, direction)
            dirs = {rec["direction"] for rec in st["records"]}
            if direction:
                assert dirs == {1 if direction == "push" else 2}
            assert st["iterations"] == len(st["records"])


def test_auto_switches_pull_then_push(gsw):
    g = gen.rmat(14, seed=2)
    _, st = _check(gsw, g, 1e-6)
    recs = st["records"]
    assert recs[0]["direction"] == 2                       # every vertex active: pull
    assert recs[-1]["direction"] == 1                      # shrinking tail: push
    for rec in recs:                                       # the rule itself
        assert rec["direction"] == (2 if rec["Ea"] > g.nnz - rec["Ea"] else 1)
    va = [rec["Va"] for rec in recs]
    assert va[0] == g.n and va[-1] < va[0]


def test_regular_graph_trajectory(gsw):
    ring = 5000   # a long cycle: 2-regular, several filter chunks and a ragged tail
    for g in (gen.from_edges(ring, [(i, (i + 1) % ring) for i in range(ring)]),
              gen.from_edges(6, [(i, j) for i in range(6) for j in range(i + 1, 6)])):
        for tol in (1e-2, 1e-5):
            eps = tol * (1 - D) / g.n
            T = next(t for t in range(10 ** 4) if not (1 - D) * D ** t / g.n > eps)
            r, st = gsw.Graph(g.off, g.col).dpr(D, tol)
            assert st["iterations"] == T
            np.testing.assert_allclose(r.cpu().numpy(), (1 - D ** T) / g.n, rtol=1e-12)


def test_directed_csc(gsw):
    rng = np.random.default_rng(5)
    n = 700
    edges = [(int(u), int(v)) for u, v in rng.integers(0, n, size=(5000, 2)) if u != v]
    g = gen.from_edges(n, edges, symmetric=False)
    csc = gen.from_edges(n, [(v, u) for u, v in edges], symmetric=False)
    for direction in (None, "push", "pull"):
        _check(gsw, g, 1e-6, direction, csc=csc)


def test_max_iters_and_errors(gsw):
    g = gen.rmat(10, seed=1)
    G = gsw.Graph(g.off, g.col)
    r, st = G.dpr(D, 1e-9, max_iters=3)
    assert st["iterations"] == 3
    ro, _ = oracle.dpr(g, D, 1e-9 * (1 - D) / g.n, max_iters=3)
    np.testing.assert_allclose(r.cpu().numpy(), ro, rtol=1e-12)     # 3 full pull steps
    for bad in (dict(damping=1.0), dict(tol=-1.0), dict(max_iters=0), dict(max_iters=65537)):
        kw = dict(damping=D, tol=1e-6, max_iters=10)
        kw.update(bad)
        with pytest.raises(Exception):
            G.dpr(**kw)


def test_host_output_buffer(gsw):
    import torch
    g = gen.rmat(11, seed=3)
    out = torch.empty(g.n, dtype=torch.float64)       # host tensor: library copies out
    r, _ = gsw.Graph(g.off, g.col).dpr(D, 1e-6, out=out)
    _band(out.numpy(), _fixed_point(g), 1e-6)


def test_c1_full(gsw):
    g = gen.config_graph("C1")
    _check(gsw, g, 1e-6)


@pytest.mark.slow
@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_full_mass_band(gsw, cfg):
    """Full C3 / C4: x's total mass is known in closed form ((N - iso) + iso (1-d)) / N for an
    undirected graph (M column-stochastic off the isolated vertices), so 0 <= sum(x - r) <= tol
    is checked at full size without the fixed point."""
    g = gen.config_graph(cfg)
    tol = 1e-6
    r, st = gsw.Graph(g.off, g.col).dpr(D, tol)
    r = r.cpu().numpy()
    iso = int((np.diff(np.asarray(g.off)) == 0).sum())
    mass = ((g.n - iso) + iso * (1 - D)) / g.n
    gap = mass - r.sum()
    assert -1e-9 <= gap <= tol * (1 + 1e-6), gap
    assert r.min() >= (1 - D) / g.n * (1 - 1e-12)      # every vertex is active at t = 0


@pytest.mark.parametrize("direction", [None, "push", "pull"])
def test_heavy_row_chunks(gsw, direction):
    """Rows above the 1024-edge chunk (two hubs of 2,500 and 5,000 edges, ragged last chunks)
    next to short and mid rows: every tier of both expand kernels."""
    n = 6000
    edges = [(0, i) for i in range(1, 5001)] + [(1, i) for i in range(2000, 4500)]
    edges += [(i, i + 1) for i in range(5000, n - 1)] + [(i, i + 100) for i in range(100, 1100)]
    g = gen.from_edges(n, edges)
    for tol in (1e-4, 1e-8):
        _check(gsw, g, tol, direction)


def test_max_iters_limit_fits_small_graphs(gsw):
    """The documented maximum (65,536 iterations) is a valid call even on a tiny graph: the
    per-iteration records are budgeted in the workspace (ENOMEM before)."""
    g = gen.from_edges(6, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5)])
    r, st = gsw.Graph(g.off, g.col).dpr(D, 0.0, max_iters=65536)
    assert 1 <= st["iterations"] <= 65536
    ro, _ = oracle.dpr(g, D, 0.0, max_iters=st["iterations"])
    np.testing.assert_allclose(r.cpu().numpy(), ro, rtol=1e-9, atol=1e-300)
