"""Cluster launches of the persistent engine: the BFS
team tier (cluster 0's k CTAs run the small levels with a hardware cluster barrier and the
frontier parts in distributed shared memory), the single-cluster grid (its grid barrier is
barrier.cluster) and the reduced grid are all opt-in A/B shapes; each must reproduce the oracle
and the per-level Inspector features exactly."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

SHAPES = {
    "team16": {"GSW_TEAM": "16"},
    "team8": {"GSW_TEAM": "8"},
    "team4": {"GSW_TEAM": "4"},
    "team16_e512": {"GSW_TEAM": "16", "GSW_TEAM_E": "512"},
    "cluster16": {"GSW_CLUSTER": "16"},
    "cluster8_team": {"GSW_CLUSTER": "8", "GSW_TEAM_IN_CLUSTER": "1"},
    "grid16": {"GSW_GRID_CTAS": "16"},
}


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _graphs():
    rng = np.random.default_rng(11)
    sparse = [(int(a), int(b)) for a, b in rng.integers(0, 3000, size=(5000, 2)) if a != b]
    return (gen.grid(61, 47), gen.grid(300, 7), gen.rmat(13, seed=5),
            gen.from_edges(300, [(i, i + 1) for i in range(299)]), gen.from_edges(3000, sparse))


@pytest.mark.parametrize("shape", sorted(SHAPES))
def test_bfs_cluster_shapes(gsw, monkeypatch, shape):
    for k, v in SHAPES[shape].items():
        monkeypatch.setenv(k, v)
    team = "GSW_TEAM" in SHAPES[shape] or "GSW_TEAM_IN_CLUSTER" in SHAPES[shape]
    for g in _graphs():
        G = gsw.Graph(g.off, g.col)
        for s in gen.sources(g, 3, seed=4):
            d, st = G.bfs(s, records=4096)
            d = d.cpu().numpy()
            assert np.array_equal(d, oracle.bfs(g, s)), (shape, g.name, s)
            Va, Ea, Via, Eia = oracle.bfs_features(g, s)
            assert [r["Va"] for r in st["records"]] == Va.tolist(), (shape, g.name)
            assert [r["Ea"] for r in st["records"]] == Ea.tolist(), (shape, g.name)
            assert [r["Via"] for r in st["records"]] == Via.tolist(), (shape, g.name)
            assert [r["Eia"] for r in st["records"]] == Eia.tolist(), (shape, g.name)
            ctas = [r["ctas"] for r in st["records"]]
            if team and g.name.startswith("grid") and g.n > 2000:
                # road-like graph (mean degree < 8): the levels run by the team record k CTAs
                assert any(1 < c <= 16 for c in ctas), (shape, g.name, ctas[:20])


@pytest.mark.parametrize("shape", ["cluster16", "grid16"])
def test_other_algorithms_on_cluster_shapes(gsw, monkeypatch, shape):
    """The single-cluster grid and the reduced grid apply to every persistent kernel."""
    for k, v in SHAPES[shape].items():
        monkeypatch.setenv(k, v)
    g = gen.with_hash_weights(gen.grid(40, 30), 12345, 64)
    G = gsw.Graph(g.off, g.col, g.w)
    d, _ = G.sssp(0)
    assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, 0))
    r = gen.rmat(12, seed=3)
    H = gsw.Graph(r.off, r.col)
    lab, _ = H.cc()
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(r))
    pr, _ = H.pr(0.85, 20)
    ref = oracle.pr(r, 0.85, 20)
    assert np.max(np.abs(pr.cpu().numpy() - ref) / ref) <= 1e-5


def test_team_on_c2_grid(gsw, monkeypatch):
    """C2-shaped grid with the 16-CTA team: bit-exact, and most levels run on the team."""
    monkeypatch.setenv("GSW_TEAM", "16")
    g = gen.grid(2048)
    G = gsw.Graph(g.off, g.col)
    d, st = G.bfs(0, records=8192)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, 0))
    ctas = [r["ctas"] for r in st["records"]]
    assert sum(1 < c <= 16 for c in ctas) > 3000
