"""Multi-GPU path on one GPU: loopback partitions (the same partitioned kernels as
NCCL mode, exchange in device memory), NCCL mode with one rank (the collectives really run), and
the host-staged backend with 2-3 processes sharing the GPU over gloo.  BFS and CC bit-exact,
PR <= 1e-5."""
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
    lab, st = D.cc()
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))
    with pytest.raises(gsw.GswError):
        D.sssp(s)                                             # no weights on this handle
    D2 = gsw.DistGraph(off, col, g.n, None, 1, 0)            # private communicator, no id needed
    d, _ = D2.bfs(s)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))


@pytest.mark.parametrize("nparts", [1, 2, 3, 8])
def test_loopback_cc(gsw, nparts):
    for g in (gen.rmat(13, seed=4), gen.grid(37, 23), gen.from_edges(300, [(i, i + 1) for i in range(0, 299, 2)]),
              gen.from_edges(400, [(0, i) for i in range(1, 300)] + [(i, i + 1) for i in range(300, 399)])):
        lab, st = gsw.PartitionedGraph(g.off, g.col, nparts).cc()
        assert np.array_equal(lab.cpu().numpy(), oracle.cc(g)), (nparts, g.name)


def test_loopback_heavy_rows(gsw):
    """Rows above the 1024-edge task size (push tasks, PR / CC chunk partials) across parts."""
    n = 9000
    edges = [(0, i) for i in range(1, 6000)] + [(1, i) for i in range(3000, 8999, 2)] + [(i, i + 1) for i in range(6000, 8999)]
    g = gen.from_edges(n, edges)
    for p in (1, 2, 4):
        P = gsw.PartitionedGraph(g.off, g.col, p)
        for force in (None, "push", "pull"):
            P.force_config(direction=force)
            for s in (0, 7000, 8998):
                d, _ = P.bfs(s)
                assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), (p, force, s)
        P.force_config()
        x, _ = P.pr(0.85, 20)
        r = oracle.pr(g, 0.85, 20)
        assert (np.abs(x.cpu().numpy() - r) / r).max() <= 1e-5
        lab, _ = P.cc()
        assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))


def _host_worker(rank, ws, port, q):
    import os
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    try:
        dist.init_process_group("gloo", rank=rank, world_size=ws)
        import paper_conf_ppopp_menglts19_b200 as m
        g = gen.rmat(13, seed=8)
        off, col = m.owned_rows(g.off, g.col, rank, ws)
        S = m.dist_slice(g.n, ws)
        vb, ve = rank * S, min(g.n, (rank + 1) * S)
        ex = m.TorchHostExchange()
        D = m.HostDistGraph(off, col, g.n, ex, rank, device="cuda:0")
        bad = []
        for s in gen.sources(g, 3, seed=5):
            d, st = D.bfs(s, records=64)
            if not np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)[vb:ve]):
                bad.append(("bfs", s))
            Va, _, _, _ = oracle.bfs_features(g, s)
            if [r["Va"] for r in st["records"]] != Va.tolist():
                bad.append(("bfs-Va", s))
        x, _ = D.pr(0.85, 20)
        r = oracle.pr(g, 0.85, 20)[vb:ve]
        if (np.abs(x.cpu().numpy() - r) / r).max() > 1e-5:
            bad.append("pr")
        lab, _ = D.cc()
        if not np.array_equal(lab.cpu().numpy(), oracle.cc(g)[vb:ve]):
            bad.append("cc")
        gw = gen.with_hash_weights(g, 11, 64)
        wo, wc, ww = m.owned_rows(gw.off, gw.col, rank, ws, weights=gw.w)
        Dw = m.HostDistGraph(wo, wc, g.n, ex, rank, device="cuda:0", weights=ww)
        s0 = gen.sources(g, 1, seed=6)[0]
        dd, _ = Dw.sssp(s0)
        if not np.array_equal(dd.cpu().numpy().view(np.uint32), oracle.sssp(gw, s0)[vb:ve]):
            bad.append("sssp")
        srcs = gen.sources(g, 2, seed=8)
        bcx, _ = D.bc(srcs)
        bcr = oracle.bc(g, srcs)[vb:ve]
        if (np.abs(bcx.cpu().numpy() - bcr) / np.maximum(np.abs(bcr), 1.0)).max() > 1e-4:
            bad.append("bc")
        q.put((rank, bad))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:          # noqa: BLE001
        q.put((rank, [repr(e)]))


@pytest.mark.parametrize("ws", [2, 3])
def test_host_staged_processes(gsw, ws):
    """world_size 2 / 3 gloo processes, each driving the library's partitioned kernels on the same
    GPU through gsw_graph_create_dist_host: owned slices match the oracle."""
    import random
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 20000 + random.randint(0, 20000)
    procs = [ctx.Process(target=_host_worker, args=(r, ws, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(ws))
    for p in procs:
        p.join(timeout=120)
    assert all(not v for v in res.values()), res


def test_c3_loopback_8(gsw):
    g = gen.config_graph("C3")
    P = gsw.PartitionedGraph(g.off, g.col, 8)
    s = gen.sources(g, 1)[0]
    d, _ = P.bfs(s)
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s))


@pytest.mark.parametrize("nparts", [1, 2, 3, 8])
def test_loopback_sssp(gsw, nparts):
    """Partitioned SSSP (near/far with a static step, forced UNORDERED = Bellman-Ford): bit-exact
    distances against the Dijkstra oracle on scale-free, grid and path inputs."""
    for g in (gen.with_hash_weights(gen.rmat(12, seed=4), 3, 64), gen.with_hash_weights(gen.grid(41, 23), 12345, 64),
              gen.with_hash_weights(gen.from_edges(200, [(i, i + 1) for i in range(199)]), 5, 64)):
        P = gsw.PartitionedGraph(g.off, g.col, nparts, weights=g.w)
        for step in (None, "unordered"):
            P.force_config(stepping=step)
            for s in gen.sources(g, 2, seed=3):
                d, st = P.sssp(s, records=64)
                assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, s)), (nparts, g.name, step, s)
        P.force_config(delta0=1)
        s = gen.sources(g, 1, seed=9)[0]
        d, _ = P.sssp(s)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, s))


def test_nccl_single_rank_sssp(gsw):
    g = gen.with_hash_weights(gen.rmat(12, seed=5), 7, 64)
    off, col, w = gsw.owned_rows(g.off, g.col, 0, 1, weights=g.w)
    D = gsw.DistGraph(off, col, g.n, None, 1, 0, weights=w)
    s = gen.sources(g, 1)[0]
    d, _ = D.sssp(s)
    assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g, s))
    with pytest.raises(gsw.GswError):
        gsw.DistGraph(*gsw.owned_rows(g.off, g.col, 0, 1), g.n, None, 1, 0).sssp(s)   # no weights


def _bc_close(x, r):
    err = np.abs(x - r) / np.maximum(np.abs(r), 1.0)
    assert err.max() <= 1e-4, err.max()


@pytest.mark.parametrize("nparts", [1, 2, 3])
def test_loopback_bc(gsw, nparts):
    """Partitioned Brandes BC (forward sigma pull, backward omega pull, replicated level arrays)
    against the oracle, with heavy rows (> 1,024 entries) among the inputs."""
    n = 3000
    hub = gen.from_edges(n, [(0, i) for i in range(1, 1500)] + [(i, i + 1) for i in range(1500, n - 1)] +
                         [(i, (i * 7) % n) for i in range(1, n, 3)])
    for g in (gen.rmat(11, seed=3), gen.grid(19, 13), hub):
        P = gsw.PartitionedGraph(g.off, g.col, nparts)
        srcs = gen.sources(g, 3, seed=4)
        x, _ = P.bc(srcs)
        _bc_close(x.cpu().numpy(), oracle.bc(g, srcs))


def test_nccl_single_rank_bc(gsw):
    g = gen.rmat(12, seed=8)
    D = gsw.DistGraph(*gsw.owned_rows(g.off, g.col, 0, 1), g.n, None, 1, 0)
    srcs = gen.sources(g, 2)
    x, _ = D.bc(srcs)
    _bc_close(x.cpu().numpy(), oracle.bc(g, srcs))


KNOBS = {
    "graph_loop": {"GSW_DIST_GRAPH": "1"},
    "host_loop": {"GSW_DIST_GRAPH": "0"},
    "no_hub_first": {"GSW_DIST_HUBFIRST": "0"},
    "no_pr_hub_order": {"GSW_DIST_PR_HUBORDER": "0"},
    "plain": {"GSW_DIST_GRAPH": "0", "GSW_DIST_HUBFIRST": "0", "GSW_DIST_PR_HUBORDER": "0"},
}


@pytest.mark.parametrize("knob", sorted(KNOBS))
@pytest.mark.parametrize("nparts", [1, 3])
def test_loopback_execution_choices(gsw, monkeypatch, knob, nparts):
    """The partitioned path's execution choices (CUDA-graph level loop, hub-first
    rows, PR hub order) change nothing in the results: BFS depths and per-level features, CC labels,
    SSSP distances (weights follow the reordered columns), PR within 1e-5, BC within 1e-4."""
    for k, v in KNOBS[knob].items():
        monkeypatch.setenv(k, v)
    g = gen.rmat(13, seed=12)
    P = gsw.PartitionedGraph(g.off, g.col, nparts)
    for s in gen.sources(g, 2, seed=7):
        d, st = P.bfs(s, records=128)
        assert np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), (knob, nparts, s)
        Va, Ea, _, _ = oracle.bfs_features(g, s)
        assert [r["Va"] for r in st["records"]] == Va.tolist()
        d2, _ = P.bfs(s)                   # second call: the cached graph (graph mode) is re-launched
        assert np.array_equal(d2.cpu().numpy(), d.cpu().numpy())
    lab, _ = P.cc()
    assert np.array_equal(lab.cpu().numpy(), oracle.cc(g))
    x, _ = P.pr(0.85, 20)
    r = oracle.pr(g, 0.85, 20)
    assert (np.abs(x.cpu().numpy() - r) / r).max() <= 1e-5
    srcs = gen.sources(g, 3, seed=3)
    b, _ = P.bc(srcs)
    ref = oracle.bc(g, srcs)
    assert (np.abs(b.cpu().numpy() - ref) / np.maximum(np.abs(ref), 1.0)).max() <= 1e-4
    gw = gen.with_hash_weights(gen.grid(33, 21), 12345, 64)
    W = gsw.PartitionedGraph(gw.off, gw.col, nparts, weights=gw.w)
    dd, _ = W.sssp(0)
    assert np.array_equal(dd.cpu().numpy().view(np.uint32), oracle.sssp(gw, 0)), (knob, nparts)
