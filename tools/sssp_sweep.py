#!/usr/bin/env python
"""C2 SSSP: rounds and device time over stepping modes and delta0 values (stepping calibration)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw
g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C2")
G = gsw.Graph(g.off, g.col, g.w)
for step in ["static", "auto", "increase", "remain"]:
    for d0 in [0, 128, 512, 1024, 2048, 4096, 8192]:
        G.force_config(stepping=step, delta0=d0)
        best = None
        for _ in range(2):
            _, st = G.sssp(0)
            best = st if best is None or st["gpu_ms"] < best["gpu_ms"] else best
        print(f"{step:9s} d0={d0:5d} rounds={best['iterations']:6d} ms={best['gpu_ms']:8.2f} "
              f"edges/nnz={best['edges_touched'] / g.nnz:6.2f}", flush=True)
