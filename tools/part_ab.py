"""Partitioned BFS per-level overhead: loopback p=1 (no collectives) vs NCCL with one rank vs the
single-GPU persistent engine, on C3 (device span per root, best of 3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402

g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
roots = gen.sources(g, 4)
RUNS = [("single-GPU engine", "1", lambda: gsw.Graph(g.off, g.col))]
for graph in ("1", "0"):       # GSW_DIST_GRAPH: level loop as one CUDA graph (1) or host-driven (0)
    tag = "graph" if graph == "1" else "host loop"
    RUNS += [(f"loopback p=1 {tag}", graph, lambda: gsw.PartitionedGraph(g.off, g.col, 1)),
             (f"loopback p=4 {tag}", graph, lambda: gsw.PartitionedGraph(g.off, g.col, 4)),
             (f"NCCL 1 rank {tag}", graph, lambda: gsw.DistGraph(*gsw.owned_rows(g.off, g.col, 0, 1), g.n, None, 1, 0))]
for name, graph, make in RUNS:
    os.environ["GSW_DIST_GRAPH"] = graph
    G = make()
    tot, lv = 0.0, 0
    for s in roots:
        best = min(G.bfs(s)[1]["gpu_ms"] for _ in range(3))
        tot += best
        lv += G.bfs(s)[1]["iterations"]
    print(f"{name:28s} {tot / len(roots):8.3f} ms per root, {lv / len(roots):.1f} levels", flush=True)
    pr = min(G.pr(0.85, 20)[1]["gpu_ms"] for _ in range(2))
    print(f"{name:28s} PR {20 / pr * 1e3:8.1f} it/s", flush=True)
    del G
