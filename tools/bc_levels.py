#!/usr/bin/env python
"""Per-level records (direction, LB, Va, edges, Filter/Expand us) of BC from one source on C4."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C4")
G = gsw.Graph(g.off, g.col)
if len(sys.argv) > 2:
    G.force_config(**dict(a.split("=") for a in sys.argv[2:]))
src = gen.sources(g, 1)
for _ in range(2):
    _, st = G.bc(src, records=256)
print(f"gpu_ms={st['gpu_ms']:.3f} levels={st['iterations']}")
for r in st["records"]:
    print(f"it={r['iteration']:3d} dir={r['direction']} lb={r['load_balance']} Va={r['Va']:9d} Ea={r['Ea']:11d} "
          f"edges={r['edges']:11d} filter_us={r['filter_us']:7.2f} expand_us={r['expand_us']:8.2f}")
