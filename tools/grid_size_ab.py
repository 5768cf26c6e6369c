#!/usr/bin/env python
"""Persistent-grid size A/B on small graphs (GSW_GRID_CTAS): C1 BFS (64 roots, harmonic GTEPS) and
SSSP / CC on C1-sized inputs."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph("C1")
G = gsw.Graph(g.off, g.col)
roots = gen.sources(g, 64)
for grid in ("0", "148", "96", "64", "32", "16"):
    if grid == "0":
        os.environ.pop("GSW_GRID_CTAS", None)
    else:
        os.environ["GSW_GRID_CTAS"] = grid
    rates, tot = [], 0.0
    for s in roots:
        b = min(G.bfs(s)[1]["gpu_ms"] for _ in range(3))
        d = G.bfs(s)[0].cpu().numpy()
        m = int(g.deg[d >= 0].sum()) // 2
        rates.append(m / (b * 1e-3) / 1e9)
        tot += b
    hm = len(rates) / sum(1.0 / r for r in rates)
    cc = min(G.cc()[1]["gpu_ms"] for _ in range(3))
    print(f"grid={grid:4s} C1 BFS {tot / len(roots) * 1e3:7.1f} us/root  hmean {hm:6.2f} GTEPS   C1 CC {cc * 1e3:7.1f} us", flush=True)
