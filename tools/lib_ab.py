#!/usr/bin/env python
"""Same-process-free A/B of two library builds on the headline workloads: run once per build
(GSW_LIB_PATH selects the .so) and print device time per C3 BFS root (16 roots, L2 flushed before
every call, best of 3), C2 BFS and C2 SSSP.  Usage: python tools/lib_ab.py [label]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

label = sys.argv[1] if len(sys.argv) > 1 else os.environ.get("GSW_LIB_PATH", "main")
flush = torch.empty(64 << 22, dtype=torch.float32, device="cuda")
g = gen.config_graph("C3")
G = gsw.Graph(g.off, g.col)
tot = 0.0
roots = [int(x) for x in gen.sources(g, 16)]
for s in roots:
    b = 1e9
    for k in range(3):
        flush.fill_(k)
        torch.cuda.synchronize()
        b = min(b, G.bfs(s)[1]["gpu_ms"])
    tot += b
print(f"{label}: C3 BFS {tot / len(roots):.4f} ms per root (16 roots)", flush=True)
del G
g2 = gen.config_graph("C2")
G2 = gsw.Graph(g2.off, g2.col, g2.w)
print(f"{label}: C2 BFS {min(G2.bfs(0)[1]['gpu_ms'] for _ in range(3)):.3f} ms  "
      f"C2 SSSP {min(G2.sssp(0)[1]['gpu_ms'] for _ in range(3)):.3f} ms", flush=True)
