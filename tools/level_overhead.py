#!/usr/bin/env python
"""Per-iteration fixed cost of the persistent engine: BFS on a long path and on the C2-shaped grid
(tiny frontier every level), reported as microseconds per level."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

for name, g, src in [("path20000", gen.from_edges(20000, [(i, i + 1) for i in range(19999)]), 0),
                     ("grid512", gen.grid(512), 0), ("grid2048", gen.grid(2048), 0)]:
    G = gsw.Graph(g.off, g.col)
    for cfg in [dict(), dict(direction="push", format="queue", load_balance="wm", fusion="fused"),
                dict(direction="push", format="queue", load_balance="thread", fusion="fused"),
                dict(direction="push", format="queue", load_balance="thread", fusion="standalone")]:
        G.force_config(**cfg)
        best = None
        for _ in range(3):
            _, st = G.bfs(src)
            best = st if best is None or st["gpu_ms"] < best["gpu_ms"] else best
        print(f"{name:10s} {str(cfg):90s} levels={best['iterations']:6d} ms={best['gpu_ms']:8.3f} "
              f"us/level={best['gpu_ms'] * 1e3 / best['iterations']:.2f}", flush=True)
