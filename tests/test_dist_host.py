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
