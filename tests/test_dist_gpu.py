"""Multi-GPU path on one GPU: loopback partitions (the same partitioned kernels as
NCCL mode, exchange in device memory) and NCCL mode with one rank.  BFS bit-exact, PR <= 1e-5."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gsw():
    import paper_conf_ppopp_menglts19_b200 as m
    return m


@pytest.mark.parametrize("nparts", [1, 2, 3, 4, 8])
def test_loopback_bfs(gsw, nparts):
    for g in (gen.rmat(13, seed=4), gen.grid(37, 23), gen.from_edges(130, [(i, i + 1) for i in range(129)])):
        P = gsw.PartitionedGraph(g.off, g.col, nparts)
        for s in gen.sources(g, 3, seed=2):
            d, st = P.bfs(s, records=128)
            assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), (nparts, g.name, s)
            Va, Ea, Via, Eia = oracle.bfs_features(g, s)
            assert [r["Va"] for r in st["records"]] == Va.tolist()
            assert [r["Ea"] for r in st["records"]] == Ea.tolist()


@pytest.mark.parametrize("direction", ["push", "pull"])
def test_loopback_bfs_forced(gsw, direction):
    g = gen.rmat(12, seed=9)
    P = gsw.PartitionedGraph(g.off, g.col, 3)
    P.force_config(direction=direction)
    s = gen.sources(g, 1)[0]
    d, _ = P.bfs(s)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))


@pytest.mark.parametrize("nparts", [1, 2, 5])
def test_loopback_pr(gsw, nparts):
    g = gen.rmat(12, seed=6)
    x, _ = gsw.PartitionedGraph(g.off, g.col, nparts).pr(0.85, 20)
    r = oracle.pr(g, 0.85, 20)
    assert (np.abs(x.cpu().numpy() - r) / r).max() <= 1e-5


def test_nccl_single_rank(gsw):
    g = gen.rmat(12, seed=1)
    uid = gsw.dist_unique_id()
    off, col = gsw.owned_rows(g.off, g.col, 0, 1)
    D = gsw.DistGraph(off, col, g.n, uid, 1, 0)
    s = gen.sources(g, 1)[0]
    d, _ = D.bfs(s)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))
    x, _ = D.pr(0.85, 20)
    r = oracle.pr(g, 0.85, 20)
    assert (np.abs(x.cpu().numpy() - r) / r).max() <= 1e-5
    with pytest.raises(gsw.GswError):
        D.cc()


def test_c3_loopback_8(gsw):
    g = gen.config_graph("C3")
    P = gsw.PartitionedGraph(g.off, g.col, 8)
    s = gen.sources(g, 1)[0]
    d, _ = P.bfs(s)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))
