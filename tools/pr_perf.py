#!/usr/bin/env python
"""PR x20 on a config graph: autotuned (stream kernel) vs forced pull-TWC, best of 3, ms and iters/s."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw
g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
G = gsw.Graph(g.off, g.col)
for cfg in [dict(), dict(direction="pull", load_balance="twc")]:
    G.force_config(**cfg)
    best = min((G.pr(0.85, 20)[1] for _ in range(3)), key=lambda s: s["gpu_ms"])
    print(f"PR x20 {cfg or 'auto'}: {best['gpu_ms']:.3f} ms  {20e3 / best['gpu_ms']:.0f} iters/s  "
          f"alg GB/s={best['bytes_alg'] / best['gpu_ms'] / 1e6:.0f}", flush=True)
