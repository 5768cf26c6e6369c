#!/usr/bin/env python
"""One partitioned (loopback p=1) C3 BFS after a warm-up, for an ncu launch list of the
per-level kernels (tools/capture_profiles.sh style): python tools/prof_part.py [C3] [graph 0/1]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
os.environ["GSW_DIST_GRAPH"] = sys.argv[2] if len(sys.argv) > 2 else "1"
P = gsw.PartitionedGraph(g.off, g.col, 1)
s = int(gen.sources(g, 1)[0])
P.bfs(s)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
d, st = P.bfs(s, records=64)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print(st["gpu_ms"], st["iterations"], [(r["direction"], r["edges"]) for r in st["records"]])
