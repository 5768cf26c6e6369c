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


def _hub_graph(n_leaves=3000, path=24):
    """A path 0..path-1 ending at a hub with n_leaves leaves, each leaf with its own pendant vertex:
    a solo round relaxing the hub's row claims n_leaves > 512 near vertices at once (VERDICT r1
    weak #1: the CTA-resident queue holds 512)."""
    edges = [(i, i + 1) for i in range(path - 1)]
    hub = path - 1
    leaves = range(path, path + n_leaves)
    edges += [(hub, v) for v in leaves]
    edges += [(v, v + n_leaves) for v in leaves]
    return gen.from_edges(path + 2 * n_leaves, edges)


@pytest.mark.parametrize("n_leaves", [511, 512, 513, 3000])
def test_solo_tier_overflow_claims(gsw, monkeypatch, n_leaves):
    """The SSSP solo tier with thresholds raised so a round claims more vertices than its shared
    queue holds: distances stay bit-exact and the byte model stays physical, on 5 reruns."""
    monkeypatch.setenv("GSW_SOLO_E", str(10 ** 7))
    monkeypatch.setenv("GSW_SOLO_V", "512")
    g = gen.with_hash_weights(_hub_graph(n_leaves), 77, 64)
    ref = oracle.sssp(g, 0)
    G = gsw.Graph(g.off, g.col, g.w)
    for delta0 in (0, 10 ** 6):
        G.force_config(delta0=delta0)
        for _ in range(5):
            d, st = _sssp(G, 0, records=4096)
            assert np.array_equal(d, ref), (n_leaves, delta0)
            # every counted byte is a touched CSR/state element: far below nnz*64 + n*64
            assert 0 < st["bytes_alg"] < 64 * (g.nnz + g.n) * max(1, st["iterations"]), st["bytes_alg"]
            assert st["edges_touched"] <= 64 * g.nnz


def test_solo_tier_overflow_rmat(gsw, monkeypatch):
    """Same on weighted R-MAT with a huge delta0 (every improved vertex near) and an unbounded
    solo edge budget: hub rows inside the tier claim thousands of vertices."""
    monkeypatch.setenv("GSW_SOLO_E", str(10 ** 7))
    monkeypatch.setenv("GSW_SOLO_V", "512")
    g = gen.with_hash_weights(gen.rmat(14, seed=11), 3, 64)
    G = gsw.Graph(g.off, g.col, g.w)
    for s in gen.sources(g, 3, seed=2):
        ref = oracle.sssp(g, s)
        for delta0 in (0, 10 ** 6):
            G.force_config(delta0=delta0)
            d, st = _sssp(G, s)
            assert np.array_equal(d, ref), (s, delta0)
            assert st["bytes_alg"] < 64 * (g.nnz + g.n) * max(1, st["iterations"])
