"""Pins for the CPU oracle: brute force, closed forms, invariants,
independent library routines (scipy.sparse.csgraph, networkx) and the paper's record R.

None of these tests calls the CUDA path.  A plausible mistake in the oracle (dropped term, wrong
sign or index, transposed operand, wrong dangling convention) fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

import gen
import oracle
from tests import brute
from tests.conftest import tiny_graphs

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _scipy_csr(g, weighted=False):
    import scipy.sparse as sp
    data = g.w.astype(np.float64) if weighted else np.ones(g.nnz)
    return sp.csr_matrix((data, g.col, g.off), shape=(g.n, g.n))


RNG_CASES = [(s, n, p) for s, (n, p) in enumerate([(6, .3), (8, .25), (10, .2), (12, .15), (12, .35),
                                                    (9, .5), (11, .1), (7, .6)])]


# ------------------------------------------------------------------ BFS (c1)
@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_bfs_tiny_vs_floyd(tiny, name):
    g = tiny[name]
    for s in range(g.n):
        assert np.array_equal(oracle.bfs(g, s), brute.bfs_depth(g, s))


@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_bfs_random_vs_floyd(seed, n, p):
    g = brute.random_graph(np.random.default_rng(seed), n, p)
    for s in range(n):
        assert np.array_equal(oracle.bfs(g, s), brute.bfs_depth(g, s))


def test_bfs_grid_closed_form():
    W, H = 37, 23
    g = gen.grid(W, H)
    d = oracle.bfs(g, 0).reshape(H, W)
    i, j = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    assert np.array_equal(d, i + j)


def _graph500_validate(g, s, depth):
    assert depth[s] == 0
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    du, dv = depth[src], depth[g.col]
    both = (du >= 0) & (dv >= 0)
    assert np.all(np.abs(du[both] - dv[both]) <= 1)
    assert not np.any((du >= 0) & (dv < 0))                      # no reached -> unreached edge
    has_parent = np.zeros(g.n, bool)
    has_parent[g.col[(du >= 0) & (dv == du + 1)]] = True
    reached = depth >= 0
    reached[s] = False
    assert np.all(has_parent[reached])


def test_bfs_rmat16_graph500_and_scipy():
    import scipy.sparse.csgraph as cg
    g = gen.rmat(16)
    for s in gen.sources(g, 3):
        d = oracle.bfs(g, s)
        _graph500_validate(g, s, d)
        ref = cg.shortest_path(_scipy_csr(g), unweighted=True, indices=s)
        ref = np.where(np.isinf(ref), -1, ref).astype(np.int32)
        assert np.array_equal(d, ref)


def test_bfs_features_vs_depths():
    """Per-level Va/Ea/Via/Eia recomputed by brute force from Floyd depths, and the identities
    N = Va + Via + Fixed, 2M = Ea + Eia + E_fixed (record R: 62 fixed vertices, 826 edges)."""
    for seed, n, p in RNG_CASES:
        g = brute.random_graph(np.random.default_rng(seed), n, p)
        deg = g.deg
        for s in range(n):
            Va, Ea, Via, Eia = oracle.bfs_features(g, s)
            depth = brute.bfs_depth(g, s)
            L = depth.max() + 1
            assert len(Va) == L
            for t in range(L):
                act = depth == t
                ina = (depth < 0) | (depth > t)
                assert Va[t] == act.sum() and Ea[t] == deg[act].sum()
                assert Via[t] == ina.sum() and Eia[t] == deg[ina].sum()
                fixed = (depth >= 0) & (depth < t)
                assert Va[t] + Via[t] + fixed.sum() == n
                assert Ea[t] + Eia[t] + deg[fixed].sum() == g.nnz


def test_fig4_active_set():
    """Fig. 4: the second-level active set of the example BFS is {2,3}."""
    g = tiny_graphs()["fig4"]
    d = oracle.bfs(g, 0)
    assert set(np.flatnonzero(d == 2).tolist()) == {2, 3}


# ------------------------------------------------------------------ SSSP (c2)
@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_sssp_random_vs_floyd(seed, n, p):
    g = brute.random_graph(np.random.default_rng(100 + seed), n, p, weighted=True)
    for s in range(n):
        assert np.array_equal(oracle.sssp(g, s), brute.sssp_dist(g, s))


def test_sssp_unit_weights_equal_bfs():
    g = gen.rmat(12)
    g1 = gen.Graph(g.n, g.off, g.col, np.ones(g.nnz, np.uint32))
    for s in gen.sources(g, 3):
        d = oracle.sssp(g1, s).astype(np.int64)
        b = oracle.bfs(g, s).astype(np.int64)
        assert np.array_equal(np.where(d == 2**32 - 1, -1, d), b)


def test_sssp_grid_survey_pins_and_invariants():
    pins = _gold("survey_pins.json")["grid512_sssp"]
    g = gen.with_hash_weights(gen.grid(pins["width"]), seed=12345, maxw=64)
    d = oracle.sssp(g, 0).astype(np.int64)
    assert d.max() == pins["max_dist"] and d[-1] == pins["dist_last"]
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    assert np.all(d[g.col] <= d[src] + g.w)                       # triangle inequality
    tight = np.zeros(g.n, bool)
    tight[g.col[d[g.col] == d[src] + g.w]] = True                 # every v != s has a tight edge
    tight[0] = True
    assert tight.all()
    w = g.w.astype(np.int64)
    assert w.min() >= 1 and w.max() <= 64


def test_sssp_rmat_vs_scipy():
    import scipy.sparse.csgraph as cg
    g = gen.with_hash_weights(gen.rmat(14), seed=5, maxw=64)
    for s in gen.sources(g, 2):
        d = oracle.sssp(g, s)
        ref = cg.dijkstra(_scipy_csr(g, weighted=True), indices=s)
        ref = np.where(np.isinf(ref), 2**32 - 1, ref).astype(np.uint32)
        assert np.array_equal(d, ref)


# ------------------------------------------------------------------ CC (c3)
@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_cc_tiny_vs_closure(tiny, name):
    g = tiny[name]
    assert np.array_equal(oracle.cc(g), brute.cc_labels(g))


@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_cc_random_vs_closure(seed, n, p):
    g = brute.random_graph(np.random.default_rng(200 + seed), n, p / 2)
    assert np.array_equal(oracle.cc(g), brute.cc_labels(g))


def test_cc_rmat_invariants_and_scipy():
    import scipy.sparse.csgraph as cg
    g = gen.rmat(16)
    lab = oracle.cc(g)
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    assert np.all(lab[src] == lab[g.col])
    assert np.all(lab <= np.arange(g.n))
    assert np.array_equal(lab[lab], lab)
    ncomp, ref = cg.connected_components(_scipy_csr(g), directed=False)
    assert len(np.unique(lab)) == ncomp
    # same partition: min id per scipy component
    mn = np.full(ncomp, g.n)
    np.minimum.at(mn, ref, np.arange(g.n))
    assert np.array_equal(lab, mn[ref])
    assert np.all(oracle.cc(gen.grid(40)) == 0)


# ------------------------------------------------------------------ PR (c4)
@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_pr_tiny_vs_dense_google(tiny, name):
    g = tiny[name]
    np.testing.assert_allclose(oracle.pr(g), brute.pagerank_dense(g), rtol=1e-12, atol=0)


@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_pr_random_vs_dense_google(seed, n, p):
    g = brute.random_graph(np.random.default_rng(300 + seed), n, p)
    for iters in (0, 1, 7, 20):
        np.testing.assert_allclose(oracle.pr(g, iters=iters), brute.pagerank_dense(g, iters=iters),
                                   rtol=1e-12, atol=0)


def test_pr_directed_vs_dense_google():
    rng = np.random.default_rng(7)
    n = 9
    edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < 0.25]
    g = gen.from_edges(n, edges, symmetric=False)
    csc = gen.from_edges(n, [(v, u) for u, v in edges], symmetric=False)
    np.testing.assert_allclose(oracle.pr(g, csc=csc), brute.pagerank_dense(g), rtol=1e-12)


def test_pr_survey_exact_rationals():
    pins = _gold("survey_pins.json")
    s = oracle.pr(gen.from_edges(5, [(0, i) for i in range(1, 5)]))
    assert abs(s[0] - pins["pr_star_k14"]["centre"]) < 1e-11
    assert np.all(np.abs(s[1:] - pins["pr_star_k14"]["leaf"]) < 1e-11)
    p = oracle.pr(gen.from_edges(4, [(0, 1), (1, 2)]))
    np.testing.assert_allclose(p, pins["pr_path3_plus_isolated"]["values"], atol=1e-11, rtol=0)
    assert abs(p[3] - 1 / 21) < 1e-11       # fixed point of p = 0.0375 + 0.2125 p


def test_pr_regular_graphs_uniform_and_mass():
    for g in (gen.from_edges(10, [(i, (i + 1) % 10) for i in range(10)]),
              gen.from_edges(6, [(i, j) for i in range(6) for j in range(i + 1, 6)])):
        np.testing.assert_allclose(oracle.pr(g), 1.0 / g.n, rtol=1e-14)
    g = gen.rmat(14)
    d = 0.85
    x = oracle.pr(g, d, 20)
    assert abs(x.sum() - 1.0) < 1e-12
    assert x.min() >= (1 - d) / g.n * (1 - 1e-12)
    # L1 contraction ||x_{t+1}-x_t|| <= d^t ||x_1-x_0||
    xs = [oracle.pr(g, d, t) for t in range(6)]
    base = np.abs(xs[1] - xs[0]).sum()
    for t in range(1, 5):
        assert np.abs(xs[t + 1] - xs[t]).sum() <= d ** t * base * (1 + 1e-9)


# ------------------------------------------------------------------ Delta-PR
@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_dpr_tiny_vs_dense_solve(tiny, name):
    g = tiny[name]
    x = brute.dpr_fixed_point(g)
    # eps < 0: every vertex active every iteration -> Neumann partial sums converge to x
    r, it = oracle.dpr(g, eps=-1.0, max_iters=400)
    assert it == 400
    np.testing.assert_allclose(r, x, rtol=1e-12, atol=0)
    # thresholded: 0 <= x - r and ||x - r||_1 <= ||delta_final||_1/(1-d) <= N eps/(1-d)
    for eps in (1e-3 / g.n, 1e-6 / g.n):
        r, _ = oracle.dpr(g, eps=eps)
        assert np.all(x - r >= -1e-15)
        assert (x - r).sum() <= g.n * eps / 0.15 * (1 + 1e-9)


@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_dpr_random_vs_dense_solve(seed, n, p):
    g = brute.random_graph(np.random.default_rng(700 + seed), n, p)
    x = brute.dpr_fixed_point(g)
    eps = 1e-7 / g.n
    r, it = oracle.dpr(g, eps=eps)
    assert it > 0
    assert np.all(x - r >= -1e-15) and (x - r).sum() <= g.n * eps / 0.15 * (1 + 1e-9)
    # one iteration from delta_0: active vertices gain (1-d)/N, the rest keep 0
    r1, it1 = oracle.dpr(g, eps=eps, max_iters=1)
    assert it1 == 1 and np.allclose(r1, 0.15 / g.n, rtol=1e-15)


def test_dpr_directed_vs_dense_solve():
    rng = np.random.default_rng(11)
    n = 9
    edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < 0.25]
    g = gen.from_edges(n, edges, symmetric=False)
    csc = gen.from_edges(n, [(v, u) for u, v in edges], symmetric=False)
    r, _ = oracle.dpr(g, eps=-1.0, max_iters=400, csc=csc)
    np.testing.assert_allclose(r, brute.dpr_fixed_point(g), rtol=1e-12)


def test_dpr_regular_closed_form():
    # k-regular graph: every delta_t = (1-d) d^t / N, all active together, so after the T
    # iterations with delta_t > eps, r = (1-d^T)/N exactly (geometric series), x = 1/N
    d = 0.85
    for g in (gen.from_edges(10, [(i, (i + 1) % 10) for i in range(10)]),
              gen.from_edges(6, [(i, j) for i in range(6) for j in range(i + 1, 6)])):
        for tol in (1e-2, 1e-5):
            eps = tol * (1 - d) / g.n
            T = next(t for t in range(10 ** 4) if not (1 - d) * d ** t / g.n > eps)
            r, it = oracle.dpr(g, d, eps)
            assert it == T
            np.testing.assert_allclose(r, (1 - d ** T) / g.n, rtol=1e-12)
    # isolated vertex: active once with (1-d)/N, never receives mass
    r, it = oracle.dpr(gen.from_edges(3, [(0, 1)]), d, 1e-9)
    assert abs(r[2] - (1 - d) / 3) < 1e-17


def test_dpr_rmat_mass_and_bound():
    g = gen.rmat(12)
    d, eps = 0.85, 1e-6 / g.n
    r, it = oracle.dpr(g, d, eps)
    x, _ = oracle.dpr(g, d, -1.0, max_iters=260)       # d^260 < 1e-18
    assert np.all(x - r >= -1e-15) and (x - r).sum() <= g.n * eps / (1 - d)
    # mass: M is column-stochastic on non-isolated vertices (they total (N-iso)/N); an isolated
    # vertex keeps its (1-d)/N (no dangling teleport, R16)
    iso = int((np.diff(np.asarray(g.off)) == 0).sum())
    assert iso > 0
    assert abs(x.sum() - ((g.n - iso) + iso * (1 - d)) / g.n) < 1e-12


# ------------------------------------------------------------------ BC (c5)
@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_bc_tiny_vs_pair_enumeration(tiny, name):
    g = tiny[name]
    srcs = list(range(g.n))
    np.testing.assert_allclose(oracle.bc(g, srcs), brute.bc_pairs(g, srcs), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("seed,n,p", RNG_CASES)
def test_bc_random_vs_pair_enumeration(seed, n, p):
    rng = np.random.default_rng(400 + seed)
    g = brute.random_graph(rng, n, p)
    srcs = sorted(set(rng.integers(0, n, size=3).tolist()))
    np.testing.assert_allclose(oracle.bc(g, srcs), brute.bc_pairs(g, srcs), rtol=1e-12, atol=1e-12)


def test_bc_multigraph_counts_parallel_edges():
    g = gen.from_edges(4, [(0, 1), (0, 1), (1, 3), (0, 2), (2, 3)], dedupe=False)
    np.testing.assert_allclose(oracle.bc(g, [0]), brute.bc_pairs(g, [0]), rtol=1e-12)


def test_bc_closed_forms():
    n = 7
    path = gen.from_edges(n, [(i, i + 1) for i in range(n - 1)])
    for s in range(n):
        b = oracle.bc(path, [s])
        exp = [(n - 1 - v) if v > s else (v if v < s else 0) for v in range(n)]
        np.testing.assert_allclose(b, exp)
    star = gen.from_edges(6, [(0, i) for i in range(1, 6)])
    np.testing.assert_allclose(oracle.bc(star, [3]), [4, 0, 0, 0, 0, 0])
    np.testing.assert_allclose(oracle.bc(star, [0]), 0)
    k = gen.from_edges(5, [(i, j) for i in range(5) for j in range(i + 1, 5)])
    np.testing.assert_allclose(oracle.bc(k, range(5)), 0)


def test_bc_sum_identity_and_networkx():
    """sum_v delta_s(v) = sum_{t reachable, t != s} (dist(s,t) - 1)  (SURVEY c5 ii)."""
    g = gen.rmat(10)
    for s in gen.sources(g, 4):
        b = oracle.bc(g, [s])
        d = oracle.bfs(g, s)
        reach = (d > 0)
        assert abs(b.sum() - (d[reach] - 1).sum()) < 1e-6 * max(1.0, b.sum())
    import networkx as nx
    h = gen.rmat(8)
    G = nx.Graph()
    G.add_nodes_from(range(h.n))
    src = np.repeat(np.arange(h.n), np.diff(h.off))
    G.add_edges_from(zip(src.tolist(), h.col.tolist()))
    ref = nx.betweenness_centrality(G, normalized=False)   # undirected: halves the pair sum
    b = oracle.bc(h, range(h.n))
    np.testing.assert_allclose(b, 2 * np.array([ref[v] for v in range(h.n)]), rtol=1e-9, atol=1e-9)


# ------------------------------------------------------------------ features (c6)
def test_record_R_ratio_arithmetic():
    R = _gold("record_R.json")
    r = oracle.ratios(R["N"], R["M"], R["Va"], R["Ea"], R["Via"], R["Eia"])
    for k in ("Vap", "Eap", "Eiap", "cd"):
        assert round(r[k], R["printed_decimals"][k]) == pytest.approx(R[k], abs=1e-12), k
    assert abs(r["Viap"] - R["Viap"]) < 1e-3            # printing slip, SURVEY Q15
    assert round(2 * R["M"] / R["N"], 1) == R["dbar"]
    assert R["N"] - R["Va"] - R["Via"] == 62            # Fixed vertices (consistent record)


def test_attrs_closed_forms():
    star = gen.from_edges(5, [(0, i) for i in range(1, 5)])     # degrees [4,1,1,1,1]
    a = oracle.attrs(star)
    assert a["N"] == 5 and a["M"] == 4 and a["dbar"] == 1.6
    assert abs(a["gini"] - 0.3) < 1e-15
    assert abs(a["h_er"] - 2 * math.log(2) / math.log(5)) < 1e-15
    assert abs(a["r_d"] - 3 / 1.6) < 1e-15
    assert abs(a["sigma_d"] - np.std([4, 1, 1, 1, 1])) < 1e-15
    cyc = gen.from_edges(8, [(i, (i + 1) % 8) for i in range(8)])
    a = oracle.attrs(cyc)
    assert a["gini"] == 0 and abs(a["h_er"] - 1) < 1e-15 and a["sigma_d"] == 0


def test_attrs_gini_mean_abs_difference():
    """Gini via the mean-absolute-difference definition (a different formula)."""
    g = gen.rmat(11)
    d = g.deg.astype(np.float64)
    mad = np.abs(d[:, None] - d[None, :]).sum() / (2 * len(d) ** 2 * d.mean())
    assert abs(oracle.attrs(g)["gini"] - mad) < 1e-12


def test_pr_dpr_thread_count_invariant():
    """oracle.c runs the per-vertex loops of PR / Delta-PR with OpenMP; each vertex's sum keeps
    its ascending order, so 1 thread and all threads give bit-identical results."""
    g = gen.rmat(13, seed=9)
    res = []
    for k in (1, 0):
        oracle.set_threads(k)
        res.append((oracle.pr(g, 0.85, 20), oracle.dpr(g, 0.85, 1e-7 * 0.15 / g.n)))
    oracle.set_threads(0)
    assert np.array_equal(res[0][0], res[1][0])
    assert np.array_equal(res[0][1][0], res[1][1][0]) and res[0][1][1] == res[1][1][1]
