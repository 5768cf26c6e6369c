#!/usr/bin/env python
"""Graph-creation time (device CSR in, degree relabeling included) with the symmetric pair-sort
relabel vs the 64-bit key sort (GSW_RELABEL_KEYS64=1), and BFS parity between the two."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
off = torch.from_numpy(g.off).cuda()
col = torch.from_numpy(g.col).cuda()
s = int(gen.sources(g, 1)[0])
ref = None
for mode in ("pairs", "keys64", "pairs"):
    if mode == "keys64":
        os.environ["GSW_RELABEL_KEYS64"] = "1"
    else:
        os.environ.pop("GSW_RELABEL_KEYS64", None)
    best = 1e9
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        G = gsw.Graph(off, col)
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
        d = G.bfs(s)[0].cpu().numpy()
        del G
    if ref is None:
        ref = d
    print(f"{mode:7s} create {best * 1e3:7.2f} ms (host wall, device CSR)  bfs identical={bool(np.array_equal(d, ref))}", flush=True)
