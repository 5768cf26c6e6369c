#!/usr/bin/env python
"""Tiered-reduction A/B (GSW_LIB_PATH selects the build): C4 BC x16, C3/C4 CC, C3 SSSP-pull-free
sanity (device time, best of 3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

tag = os.environ.get("GSW_LIB_PATH", "main")
g = gen.config_graph("C4")
G = gsw.Graph(g.off, g.col)
srcs = gen.sources(g, 16)
print(f"{tag}: C4 BC x16 {min(G.bc(srcs)[1]['gpu_ms'] for _ in range(3)):.2f} ms", flush=True)
print(f"{tag}: C4 CC {min(G.cc()[1]['gpu_ms'] for _ in range(3)):.3f} ms", flush=True)
del G
g = gen.config_graph("C3")
G = gsw.Graph(g.off, g.col)
print(f"{tag}: C3 CC {min(G.cc()[1]['gpu_ms'] for _ in range(5)):.3f} ms", flush=True)
print(f"{tag}: C3 BC x4 {min(G.bc(gen.sources(g, 4))[1]['gpu_ms'] for _ in range(3)):.2f} ms", flush=True)
