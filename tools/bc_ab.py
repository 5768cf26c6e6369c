#!/usr/bin/env python
"""C4 BC (16 sources) device time, best of 3 (A/B of library builds via GSW_LIB_PATH)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C4")
G = gsw.Graph(g.off, g.col)
srcs = gen.sources(g, 16)
b = min(G.bc(srcs)[1]["gpu_ms"] for _ in range(3))
print(f"{os.environ.get('GSW_LIB_PATH', 'main')}: BC x16 {b:.2f} ms", flush=True)
