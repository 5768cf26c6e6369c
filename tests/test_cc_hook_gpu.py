"""Hooking + pointer-jumping CC (gsw_cc_hook; Soman et al. [53]) vs the
union-find oracle: bit-exact labels (minimum caller id of the component) under every forced
load-balance mapping of the hook sweep, on tiny, random, scale-free, grid and relabeled inputs."""
import numpy as np
import pytest

import gen
import oracle
from tests.conftest import tiny_graphs

pytestmark = pytest.mark.gpu
LBS = ["auto", "thread", "twc", "wm", "cm", "strict"]


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


def _hook(G, **kw):
    lab, st = G.cc_hook(**kw)
    return lab.cpu().numpy(), st


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny(gsw, name):
    g = tiny_graphs()[name]
    lab, _ = _hook(gsw.Graph(g.off, g.col))
    assert np.array_equal(lab, oracle.cc(g))


@pytest.mark.parametrize("lb", LBS)
def test_forced_lb(gsw, lb):
    rng = np.random.default_rng(1)
    graphs = [gen.rmat(12, seed=5), gen.grid(50, 21), gen.from_edges(3000, rng.integers(0, 3000, size=(2500, 2))),
              gen.from_edges(4000, [(i, i + 1) for i in range(0, 3999, 2)])]
    for g in graphs:
        G = gsw.Graph(g.off, g.col)
        if lb != "auto":
            G.force_config(load_balance=lb)
        lab, st = _hook(G, records=256)
        assert np.array_equal(lab, oracle.cc(g)), (lb, g.name)
        recs = st["records"]
        assert len(recs) == st["iterations"] >= 1
        assert recs[-1]["Va"] == 0                       # the last sweep hooks nothing
        assert all(r["Va"] > 0 for r in recs[:-1])


def test_same_as_label_propagation(gsw):
    """Both CC algorithms of the library agree (and with the oracle) on a relabeled R-MAT."""
    g = gen.rmat(14, seed=9)
    G = gsw.Graph(g.off, g.col)
    a, _ = G.cc()
    b, _ = _hook(G)
    assert np.array_equal(b, a.cpu().numpy())
    assert np.array_equal(b, oracle.cc(g))


def test_host_output_and_edge_cases(gsw):
    g = gen.from_edges(6, [(0, 5), (2, 3)])
    G = gsw.Graph(g.off, g.col)
    import torch
    out = torch.empty(6, dtype=torch.int32)             # host buffer through the C ABI
    lab, st = G.cc_hook(out=out)
    assert lab.tolist() == [0, 1, 2, 2, 4, 0]
    one = gen.from_edges(1, [])
    lab, st = _hook(gsw.Graph(one.off, one.col))
    assert lab.tolist() == [0] and st["iterations"] == 1


def test_c1_full_size(gsw):
    g = gen.config_graph("C1")
    lab, _ = _hook(gsw.Graph(g.off, g.col))
    assert np.array_equal(lab, oracle.cc(g))


@pytest.mark.slow
def test_c3_full_size(gsw):
    g = gen.config_graph("C3")
    lab, st = _hook(gsw.Graph(g.off, g.col), records=64)
    assert np.array_equal(lab, oracle.cc(g))


def test_directed_input_weak_components(gsw):
    """A directed CSR (with its CSC): every adjacency entry hooks both trees, so the labels are the
    weakly connected components, as the union-find oracle computes them over the same entries."""
    rng = np.random.default_rng(8)
    n = 700
    edges = [(int(u), int(v)) for u, v in rng.integers(0, n, size=(500, 2)) if u != v]
    g = gen.from_edges(n, edges, symmetric=False)
    csc = gen.from_edges(n, [(v, u) for u, v in edges], symmetric=False)
    G = gsw.Graph(g.off, g.col, csc=(csc.off, csc.col))
    for lb in ("auto", "thread", "strict"):
        if lb == "auto":
            G.force_config()
        else:
            G.force_config(load_balance=lb)
        lab, _ = _hook(G)
        assert np.array_equal(lab, oracle.cc(g)), lb
