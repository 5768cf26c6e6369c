"""CC parity: CUDA min-label propagation (through the C ABI) vs the union-find oracle, bit-exact
labels normalised to the minimum vertex id, every forced variant."""
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


def _cc(G, **kw):
    lab, st = G.cc(**kw)
    return lab.cpu().numpy(), st


@pytest.mark.parametrize("name", sorted(tiny_graphs()))
def test_tiny(gsw, name):
    g = tiny_graphs()[name]
    lab, _ = _cc(gsw.Graph(g.off, g.col))
    assert np.array_equal(lab, oracle.cc(g))


@pytest.mark.parametrize("variant", VARIANTS, ids=["-".join(v) for v in VARIANTS])
def test_forced_variant_sweep(gsw, variant):
    d_, f_, l_, u_ = variant
    graphs = [gen.rmat(12, seed=5), gen.grid(50, 21),
              gen.from_edges(3000, np.random.default_rng(1).integers(0, 3000, size=(2500, 2)))]
    for g in graphs:
        G = gsw.Graph(g.off, g.col)
        G.force_config(direction=d_, format=f_, load_balance=l_, fusion=u_)
        lab, _ = _cc(G)
        assert np.array_equal(lab, oracle.cc(g)), (variant, g.name)


def test_c1_full_and_invariants(gsw):
    g = gen.config_graph("C1")
    lab, st = _cc(gsw.Graph(g.off, g.col), records=1024)
    ref = oracle.cc(g)
    assert np.array_equal(lab, ref)
    assert st["iterations"] >= 1 and len(st["records"]) == st["iterations"]


def test_host_output(gsw):
    import torch
    g = gen.rmat(11, seed=9)
    out = torch.empty(g.n, dtype=torch.int32).pin_memory()
    gsw.Graph(g.off, g.col).cc(out=out)
    assert np.array_equal(out.numpy(), oracle.cc(g))


@pytest.mark.slow
def test_c3_full_size(gsw):
    g = gen.config_graph("C3")
    lab, _ = _cc(gsw.Graph(g.off, g.col))
    assert np.array_equal(lab, oracle.cc(g))


@pytest.mark.parametrize("switch", ["0", "1", "3", "32"])
def test_switch_to_hooking(gsw, monkeypatch, switch):
    """Autotuned CC hands over to hooking + pointer jumping after GSW_CC_SWITCH label-propagation
    iterations (0: never): bit-exact labels, records of both phases, host and device outputs."""
    import torch
    monkeypatch.setenv("GSW_CC_SWITCH", switch)
    rng = np.random.default_rng(4)
    graphs = [gen.grid(120, 40), gen.grid(500, 3), gen.rmat(12, seed=2),
              gen.from_edges(4000, [(i, i + 1) for i in range(3999) if i % 700 != 0]),
              gen.from_edges(3000, rng.integers(0, 3000, size=(2000, 2)))]
    for g in graphs:
        G = gsw.Graph(g.off, g.col)
        lab, st = _cc(G, records=8192)
        ref = oracle.cc(g)
        assert np.array_equal(lab, ref), (switch, g.name)
        assert len(st["records"]) == st["iterations"]
        assert [r["iteration"] for r in st["records"]] == list(range(st["iterations"]))
        out = torch.empty(g.n, dtype=torch.int32).pin_memory()
        G.cc(out=out)
        assert np.array_equal(out.numpy(), ref), (switch, g.name, "host output")


def test_switch_on_c2_grid(gsw):
    """C2-shaped road grid: the default switch turns ~4,000 label-propagation iterations into a
    few dozen plus two hooking sweeps."""
    g = gen.grid(2048)
    lab, st = _cc(gsw.Graph(g.off, g.col), records=8192)
    assert np.array_equal(lab, np.zeros(g.n, dtype=lab.dtype))
    assert st["iterations"] < 64
