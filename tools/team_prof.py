#!/usr/bin/env python
"""Per-phase timing of the BFS team tier on C2 (diagnostic build: make flagvariant VNAME=tp
VFLAGS=-DGSW_TEAM_PROF=1; run with GSW_LIB_PATH=build/var_tp/libgsw.so).  The library prints the
per-level phase means on stderr."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C2")
G = gsw.Graph(g.off, g.col)
for team, extra in (("16", {}), ("16", {"GSW_CLUSTER": "16", "GSW_TEAM_IN_CLUSTER": "1"}),
                    ("8", {"GSW_CLUSTER": "8", "GSW_TEAM_IN_CLUSTER": "1"})):
    os.environ["GSW_TEAM"] = team
    for k in ("GSW_CLUSTER", "GSW_TEAM_IN_CLUSTER"):
        os.environ.pop(k, None)
    os.environ.update(extra)
    for _ in range(2):
        _, st = G.bfs(0)
    print(f"team {team} {extra}: {st['gpu_ms']:.3f} ms, {st['iterations']} levels", file=sys.stderr, flush=True)
