"""Host-side logic of the 1D partition (no GPU): slice sizes and owned-row extraction, checked
by reassembling the graph across world_size-2 gloo processes."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import gen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_slice_sizes():
    import paper_conf_ppopp_menglts19_b200 as gsw
    for n in (1, 10, 63, 64, 65, 1000, 4194304, 67108864):
        for p in (1, 2, 3, 4, 8):
            S = gsw.dist_slice(n, p)
            assert S % 64 == 0 and S * p >= n and (S - 64) * p < n + 64 * p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    import paper_conf_ppopp_menglts19_b200 as gsw
    g = gen.rmat(11, seed=3)
    off, col = gsw.owned_rows(g.off, g.col, rank, world)
    S = gsw.dist_slice(g.n, world)
    assert off.shape[0] - 1 == max(0, min(g.n, (rank + 1) * S) - rank * S)
    # all-gather the owned degree vectors and columns; the concatenation must be the input CSR
    degs = [None] * world
    cols = [None] * world
    dist.all_gather_object(degs, np.diff(off).tolist())
    dist.all_gather_object(cols, col.tolist())
    if rank == 0:
        deg = np.concatenate([np.asarray(d, dtype=np.int64) for d in degs])
        allc = np.concatenate([np.asarray(c, dtype=np.int64) for c in cols])
        q.put(bool(np.array_equal(deg, g.deg) and np.array_equal(allc, g.col.astype(np.int64))))
    dist.barrier()
    dist.destroy_process_group()


def test_owned_rows_reassemble_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    ok = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
    assert ok


def _protocol_worker(rank, world, port, q):
    """One rank of the SURVEY 8(e) BFS exchange protocol, executed on host arrays: destination
    ownership (pull over owned rows, push over the column slice "every u -> owned targets"),
    the replicated frontier bitmap all-gathered per level, the (Va, Ea) totals all-reduced, and
    the direction decided by the same rule on the global features on every rank."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    import paper_conf_ppopp_menglts19_b200 as gsw
    g = gen.rmat(10, seed=7)
    n = g.n
    S = gsw.dist_slice(n, world)
    off, col = gsw.owned_rows(g.off, g.col, rank, world)
    vb = rank * S
    nloc = off.shape[0] - 1
    # column slice for push: (u -> v) for every global u and owned v (symmetric graph: the
    # transpose of the owned rows)
    src_of = np.repeat(np.arange(vb, vb + nloc), np.diff(off))
    slice_u, slice_v = col.astype(np.int64), src_of
    results = {}
    for s in gen.sources(g, 3, seed=5):
        depth = np.full(nloc, -1, np.int64)
        if vb <= s < vb + nloc:
            depth[s - vb] = 0
        fb = np.zeros(S * world, bool)
        fb[s] = True
        Va, Ea = 1, int(g.deg[s])
        Via, Eia = n - 1, int(g.nnz) - Ea
        lvl = 0
        while Va > 0:
            if lvl > 0:
                Via -= Va
                Eia -= Ea
            pull = Ea * 16.0 > Eia and Va * 2048.0 > n          # select.cuh rule R6
            nfb_loc = np.zeros(S, bool)
            if pull:
                for v in range(nloc):
                    if depth[v] < 0:
                        nb = col[off[v]:off[v + 1]]
                        if nb.size and fb[nb].any():
                            nfb_loc[v] = True
            else:
                hit = fb[slice_u]
                for v in np.unique(slice_v[hit]):
                    if depth[v - vb] < 0:
                        nfb_loc[v - vb] = True
            depth[nfb_loc[:nloc]] = lvl + 1
            parts = [torch.zeros(S, dtype=torch.bool) for _ in range(world)]
            dist.all_gather(parts, torch.from_numpy(nfb_loc))
            fb = torch.cat(parts).numpy()
            tot = torch.tensor([int(nfb_loc.sum()), int(g.deg[vb:vb + nloc][nfb_loc[:nloc]].sum())], dtype=torch.int64)
            dist.all_reduce(tot)
            Va, Ea = int(tot[0]), int(tot[1])
            lvl += 1
        alld = [None] * world
        dist.all_gather_object(alld, depth.tolist())
        results[int(s)] = np.concatenate([np.asarray(d, np.int64) for d in alld])[:n]
    if rank == 0:
        import oracle
        q.put(all(np.array_equal(results[s], oracle.bfs(g, s)) for s in results))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_bfs_protocol_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_protocol_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    ok = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
    assert ok
