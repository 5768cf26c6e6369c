#!/usr/bin/env python
"""PageRank: single-GPU engine with / without the degree relabeling (GSW_NO_RELABEL) vs the partitioned
path (loopback p=1, hub-order contribution layout): python tools/pr_relabel_ab.py [C3|C5]"""
import os, sys, time
sys.path.insert(0, os.getcwd())
import gen, paper_conf_ppopp_menglts19_b200 as gsw
cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
g = gen.config_graph(cfg)
for nr in ("0", "1"):
    os.environ["GSW_NO_RELABEL"] = nr
    G = gsw.Graph(g.off, g.col)
    b = min(G.pr(0.85, 20)[1]["gpu_ms"] for _ in range(2))
    print(f"{cfg} single-GPU relabel={'no' if nr == '1' else 'yes'}: PR {20 / b * 1e3:.1f} it/s", flush=True)
    del G
os.environ["GSW_NO_RELABEL"] = "0"
P = gsw.PartitionedGraph(g.off, g.col, 1)
b = min(P.pr(0.85, 20)[1]["gpu_ms"] for _ in range(2))
print(f"{cfg} partitioned p=1: PR {20 / b * 1e3:.1f} it/s", flush=True)
