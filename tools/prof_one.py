#!/usr/bin/env python
"""Run one algorithm once on a config graph after a warm-up (for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw
algo, cfg = sys.argv[1], sys.argv[2]
kw = dict(a.split("=") for a in sys.argv[3:])
g = gen.config_graph(cfg)
G = gsw.Graph(g.off, g.col, g.w) if g.w is not None else gsw.Graph(g.off, g.col)
if kw:
    G.force_config(**kw)
for _ in range(2):
    if algo == "pr": G.pr(0.85, 4)
    elif algo == "bfs": G.bfs(gen.sources(g, 1)[0])
    elif algo == "cc": G.cc()
    elif algo == "sssp": G.sssp(0)
    elif algo == "bc": G.bc(gen.sources(g, 2))
    elif algo == "dpr": G.dpr(0.85, 1e-6)
    elif algo == "cc_hook": G.cc_hook()
print("done")
