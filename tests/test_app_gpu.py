"""User-programmable front-end (Fig. 11): BFS and SSSP written with
filter / emit / comp / compAtomic (include/gsw_app.cuh, csrc/app.cu) must return exactly what the
oracle returns, under every forced pattern variant, like the hand-specialised gsw_bfs / gsw_sssp."""
import itertools

import numpy as np
import pytest

import gen
import oracle
from tests.conftest import tiny_graphs

pytestmark = pytest.mark.gpu
VARIANTS = list(itertools.product(["push", "pull"], ["bitmap", "queue", "sorted_queue"],
                                  ["thread", "twc", "wm", "cm", "strict"], ["standalone", "fused"]))


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny_all_sources(gsw, name):
    g = tiny_graphs()[name]
    gw = gen.with_hash_weights(g, 3, 64)
    G = gsw.Graph(gw.off, gw.col, gw.w)
    for s in range(g.n):
        d, _ = G.app_bfs(s)
        assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), (name, s)
        d, _ = G.app_sssp(s)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(gw, s)), (name, s)


@pytest.mark.parametrize("variant", VARIANTS, ids=["-".join(v) for v in VARIANTS])
def test_forced_variants(gsw, variant):
    d_, f_, l_, u_ = variant
    for g in (gen.with_hash_weights(gen.rmat(12, seed=3), 5, 64), gen.with_hash_weights(gen.grid(40, 23), 12345, 64)):
        G = gsw.Graph(g.off, g.col, g.w)
        G.force_config(direction=d_, format=f_, load_balance=l_, fusion=u_)
        for s in gen.sources(g, 2, seed=11):
            d, st = G.app_bfs(s, records=256)
            assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), (variant, g.name, s)
            assert all(r["direction"] == gsw.DIRECTIONS[d_] for r in st["records"])
            d, _ = G.app_sssp(s)
            assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, s)), (variant, g.name, s)


@pytest.mark.parametrize("step", ["auto", "static", "unordered"])
@pytest.mark.parametrize("delta0", [0, 1, 1000])
def test_sssp_stepping(gsw, step, delta0):
    for g in (gen.with_hash_weights(gen.rmat(12, seed=7), 9, 64), gen.with_hash_weights(gen.grid(50), 12345, 64)):
        G = gsw.Graph(g.off, g.col, g.w)
        G.force_config(stepping=step, delta0=delta0)
        s = gen.sources(g, 1, seed=5)[0]
        d, _ = G.app_sssp(s)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, s)), (step, delta0, g.name)


def test_features_per_level_match_oracle(gsw):
    """The engine's Inspector counts (Va, Ea, Via, Eia per level) for the BFS app equal the
    oracle's (Table 1), as for gsw_bfs."""
    g = gen.rmat(13, seed=2)
    G = gsw.Graph(g.off, g.col)
    s = gen.sources(g, 1)[0]
    _, st = G.app_bfs(s, records=64)
    Va, Ea, _, _ = oracle.bfs_features(g, s)
    assert [r["Va"] for r in st["records"]] == Va.tolist()
    assert [r["Ea"] for r in st["records"]] == Ea.tolist()


def test_c1_and_host_output(gsw):
    import torch
    g = gen.config_graph("C1")
    gw = gen.with_hash_weights(g, 12345, 64)
    G = gsw.Graph(gw.off, gw.col, gw.w)
    for s in gen.sources(g, 2):
        d, _ = G.app_bfs(s)
        assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))
        out = torch.empty(g.n, dtype=torch.int32)
        G.app_sssp(s, out=out)
        assert np.array_equal(out.numpy().view(np.uint32), oracle.sssp(gw, s))


@pytest.mark.slow
def test_c2_sssp_full(gsw):
    g = gen.config_graph("C2")
    d, _ = gsw.Graph(g.off, g.col, g.w).app_sssp(0)
    assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, 0))


def test_errors(gsw):
    g = gen.rmat(10)
    G = gsw.Graph(g.off, g.col)
    with pytest.raises(gsw.GswError):
        G.app_sssp(0)                    # no weights
    with pytest.raises(gsw.GswError):
        G.app_bfs(g.n)
