#!/usr/bin/env python
"""Per-level comparison of the partitioned path (loopback p=1) with the single-GPU engine on one
root: direction and edges scanned per level, total device time (where the partitioned path's time
goes)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
s = int(gen.sources(g, 1)[0])
for name, make in (("single", lambda: gsw.Graph(g.off, g.col)), ("loopback p=1", lambda: gsw.PartitionedGraph(g.off, g.col, 1))):
    G = make()
    best = None
    for _ in range(3):
        d, st = G.bfs(s, records=64)
        if best is None or st["gpu_ms"] < best["gpu_ms"]:
            best = st
    print(f"{name}: {best['gpu_ms']:.3f} ms, {best['iterations']} levels, edges {best['edges_touched']}", flush=True)
    for r in best["records"]:
        print(f"   it={r['iteration']} dir={'push' if r['direction'] == 1 else 'pull'} Va={r['Va']:9d} Ea={r['Ea']:11d} "
              f"edges={r['edges']:10d} filter_us={r['filter_us']:6.2f} expand_us={r['expand_us']:6.2f}", flush=True)
    del G
