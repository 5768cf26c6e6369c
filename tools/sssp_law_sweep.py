#!/usr/bin/env python
"""Dynamic-stepping control laws x c (delta0 = c*wbar/dbar) on a graph (P4 calibration)."""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
code = r'''
import os, sys
sys.path.insert(0, %r)
import gen, paper_conf_ppopp_menglts19_b200 as gsw
g = gen.config_graph(%r) if %r != "RMAT" else gen.with_hash_weights(gen.rmat(20), 5, 64)
G = gsw.Graph(g.off, g.col, g.w)
s = 0 if %r == "C2" else gen.sources(g, 1)[0]
for c in [0, 2, 4, 8]:
    d0 = 0 if c == 0 else int(c * 32 * %s)
    G.force_config(stepping="auto", delta0=d0)
    b = min((G.sssp(s)[1] for _ in range(2)), key=lambda st: st["gpu_ms"])
    print(f"law=%s d0={d0:6d} rounds={b['iterations']:6d} ms={b['gpu_ms']:8.2f} edges/nnz={b['edges_touched']/g.nnz:6.2f}", flush=True)
'''
graph = sys.argv[1] if len(sys.argv) > 1 else "C2"
wbar_dbar = "8.125" if graph == "C2" else "1.0"
for law in range(4):
    env = dict(os.environ, GSW_SSSP_LAW=str(law))
    subprocess.run([sys.executable, "-c", code % (ROOT, graph, graph, graph, wbar_dbar, law)], env=env)
