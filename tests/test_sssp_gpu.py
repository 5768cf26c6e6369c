"""SSSP parity: CUDA near/far stepping vs the Dijkstra oracle, bit-exact uint32 distances
(SURVEY 8(c) c2), every forced variant and every stepping candidate (P4)."""
import itertools
import json
import os

import numpy as np
import pytest

import gen
import oracle
from tests import brute

pytestmark = pytest.mark.gpu
VARIANTS = list(itertools.product(["push", "pull"], ["bitmap", "queue", "sorted_queue"],
                                  ["thread", "twc", "wm", "cm", "strict"], ["standalone", "fused"]))
STEPPING = ["auto", "static", "unordered", "increase", "decrease", "remain"]
GOLD = os.path.join(os.path.dirname(__file__), "golden", "survey_pins.json")


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _sssp(G, s, **kw):
    d, st = G.sssp(s, **kw)
    return d.cpu().numpy().view(np.uint32), st


def test_random_small(gsw):
    for seed in range(6):
        g = brute.random_graph(np.random.default_rng(seed), 12, 0.3, weighted=True)
        G = gsw.Graph(g.off, g.col, g.w)
        for s in range(g.n):
            d, _ = _sssp(G, s)
            assert np.array_equal(d, oracle.sssp(g, s)), (seed, s)


@pytest.mark.parametrize("variant", VARIANTS, ids=["-".join(v) for v in VARIANTS])
def test_forced_variant_sweep(gsw, variant):
    d_, f_, l_, u_ = variant
    for g in (gen.with_hash_weights(gen.rmat(12, seed=6), 5, 64), gen.with_hash_weights(gen.grid(40, 30), 12345, 64)):
        G = gsw.Graph(g.off, g.col, g.w)
        G.force_config(direction=d_, format=f_, load_balance=l_, fusion=u_)
        s = gen.sources(g, 1, seed=3)[0]
        d, _ = _sssp(G, s)
        assert np.array_equal(d, oracle.sssp(g, s)), (variant, g.name)


@pytest.mark.parametrize("step", STEPPING)
@pytest.mark.parametrize("delta0", [0, 1, 7, 100000])
def test_stepping_modes(gsw, step, delta0):
    for g in (gen.with_hash_weights(gen.rmat(12, seed=7), 9, 64), gen.with_hash_weights(gen.grid(64), 12345, 64)):
        G = gsw.Graph(g.off, g.col, g.w)
        G.force_config(stepping=step, delta0=delta0)
        s = gen.sources(g, 1, seed=5)[0]
        d, st = _sssp(G, s, records=8192)
        assert np.array_equal(d, oracle.sssp(g, s)), (step, delta0, g.name)
        if step == "unordered":
            assert all(r["theta"] == 0xFFFFFFFF for r in st["records"])


def test_grid512_survey_pin(gsw):
    pins = json.load(open(GOLD))["grid512_sssp"]
    g = gen.with_hash_weights(gen.grid(pins["width"]), 12345, 64)
    d, st = _sssp(gsw.Graph(g.off, g.col, g.w), 0)
    assert int(d.max()) == pins["max_dist"] and int(d[-1]) == pins["dist_last"]
    assert np.array_equal(d, oracle.sssp(g, 0))


def test_unit_weights_equal_bfs(gsw):
    g = gen.rmat(12, seed=2)
    G = gsw.Graph(g.off, g.col, np.ones(g.nnz, np.uint32))
    s = gen.sources(g, 1)[0]
    d, _ = _sssp(G, s)
    b = oracle.bfs(g, s).astype(np.int64)
    assert np.array_equal(np.where(d == 0xFFFFFFFF, -1, d.astype(np.int64)), b)


def test_errors(gsw):
    g = gen.rmat(8)
    G = gsw.Graph(g.off, g.col)
    with pytest.raises(gsw.GswError):
        G.sssp(0)                                  # no weights
    gw = gen.with_hash_weights(g, 1, 64)
    with pytest.raises(gsw.GswError):
        gsw.Graph(gw.off, gw.col, gw.w).sssp(g.n)  # source out of range


@pytest.mark.slow
def test_c2_full_size(gsw):
    g = gen.config_graph("C2")
    d, st = _sssp(gsw.Graph(g.off, g.col, g.w), 0)
    assert np.array_equal(d, oracle.sssp(g, 0))
    assert int(d.max()) == 62467 and int(d[-1]) == 62436
