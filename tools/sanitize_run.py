"""Workload for compute-sanitizer (tools/sanitize.sh): every algorithm of libgsw on small seeded
graphs, including forced variants, the CTA-resident tiers (with a raised edge budget so a round
claims more than the shared queue holds) and the partitioned loopback path.  Checks parity with
the CPU oracle too (tests-only module, used here as a checker), so a sanitizer-clean run is also a
correct one.  Usage: python tools/sanitize_run.py [small|c1]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402


def main():
    size = sys.argv[1] if len(sys.argv) > 1 else "small"
    scale = 16 if size == "c1" else 11
    g = gen.rmat(scale, seed=1)
    gw = gen.with_hash_weights(g, 5, 64)
    grid = gen.with_hash_weights(gen.grid(64 if size == "c1" else 24), 12345, 64)
    ok = True

    def chk(name, a, b, tol=None):
        nonlocal ok
        if tol is None:
            good = np.array_equal(a, b)
        else:
            good = float(np.max(np.abs(a - b) / np.maximum(np.abs(b), tol[1]))) <= tol[0]
        print(f"{name}: {'ok' if good else 'MISMATCH'}", flush=True)
        ok &= good

    G = gsw.Graph(g.off, g.col)
    s = gen.sources(g, 1)[0]
    chk("bfs auto", G.bfs(s)[0].cpu().numpy(), oracle.bfs(g, s))
    for d, f, lb, fu in [("push", "queue", "twc", "fused"), ("pull", "bitmap", "thread", "fused"),
                         ("pull", "sorted_queue", "strict", "standalone"), ("push", "bitmap", "wm", "standalone"),
                         ("push", "sorted_queue", "cm", "fused")]:
        G.force_config(direction=d, format=f, load_balance=lb, fusion=fu)
        chk(f"bfs {d}/{f}/{lb}/{fu}", G.bfs(s)[0].cpu().numpy(), oracle.bfs(g, s))
    G.force_config()
    chk("cc", G.cc()[0].cpu().numpy(), oracle.cc(g))
    chk("pr", G.pr(0.85, 20)[0].cpu().numpy().astype(np.float64), oracle.pr(g, 0.85, 20), (1e-5, 0.0))
    srcs = gen.sources(g, 4)
    chk("bc", G.bc(srcs)[0].cpu().numpy(), oracle.bc(g, srcs), (1e-4, 1.0))
    r, st = G.dpr(0.85, 1e-6)
    ro, _ = oracle.dpr(g, 0.85, 1e-6 * 0.15 / g.n)
    chk("dpr (L1 <= 2 tol)", np.array([np.abs(r.cpu().numpy() - ro).sum() <= 2e-6]), np.array([True]))
    G.force_config(direction="push")
    r, st = G.dpr(0.85, 1e-6)
    chk("dpr push (L1 <= 2 tol)", np.array([np.abs(r.cpu().numpy() - ro).sum() <= 2e-6]), np.array([True]))
    del G

    Gw = gsw.Graph(gw.off, gw.col, gw.w)
    chk("sssp auto", Gw.sssp(s)[0].cpu().numpy().view(np.uint32), oracle.sssp(gw, s))
    Gw.force_config(direction="pull", format="bitmap", load_balance="twc", fusion="standalone", stepping="static")
    chk("sssp pull/static", Gw.sssp(s)[0].cpu().numpy().view(np.uint32), oracle.sssp(gw, s))
    del Gw
    Gg = gsw.Graph(grid.off, grid.col, grid.w)
    chk("sssp grid (solo tier)", Gg.sssp(0)[0].cpu().numpy().view(np.uint32), oracle.sssp(grid, 0))
    chk("bfs grid (solo tier)", Gg.bfs(0)[0].cpu().numpy(), oracle.bfs(grid, 0))
    os.environ["GSW_SOLO_E"] = str(10 ** 7)      # solo rounds that overflow the shared queues
    Gw = gsw.Graph(gw.off, gw.col, gw.w)
    Gw.force_config(delta0=10 ** 6)
    chk("sssp solo overflow", Gw.sssp(s)[0].cpu().numpy().view(np.uint32), oracle.sssp(gw, s))
    G = gsw.Graph(g.off, g.col)
    chk("bfs solo overflow", G.bfs(s)[0].cpu().numpy(), oracle.bfs(g, s))
    del os.environ["GSW_SOLO_E"]
    # hooking + pointer-jumping CC under every sweep mapping (round 2, session 3)
    G = gsw.Graph(g.off, g.col)
    for lb in ("auto", "thread", "twc", "wm", "cm", "strict"):
        if lb == "auto":
            G.force_config()
        else:
            G.force_config(load_balance=lb)
        chk(f"cc_hook {lb}", G.cc_hook()[0].cpu().numpy(), oracle.cc(g))
    G.force_config()
    Gg = gsw.Graph(grid.off, grid.col, grid.w)
    chk("cc_hook grid", Gg.cc_hook()[0].cpu().numpy(), oracle.cc(grid))
    # cluster launches: the BFS team tier (DSMEM frontier parts) and the single-cluster grid
    for env in ({"GSW_TEAM": "16"}, {"GSW_TEAM": "4"}, {"GSW_CLUSTER": "8"}):
        os.environ.update(env)
        tag = ",".join(f"{k}={v}" for k, v in env.items())
        chk(f"bfs grid [{tag}]", Gg.bfs(0)[0].cpu().numpy(), oracle.bfs(grid, 0))
        chk(f"bfs rmat [{tag}]", G.bfs(s)[0].cpu().numpy(), oracle.bfs(g, s))
        for k in env:
            del os.environ[k]
    os.environ.update({"GSW_CLUSTER": "8"})
    chk("sssp grid [GSW_CLUSTER=8]", Gg.sssp(0)[0].cpu().numpy().view(np.uint32), oracle.sssp(grid, 0))
    del os.environ["GSW_CLUSTER"]
    del G, Gg
    P = gsw.PartitionedGraph(g.off, g.col, 3)
    chk("partitioned bfs p=3", P.bfs(s)[0].cpu().numpy(), oracle.bfs(g, s))
    chk("partitioned pr p=3", P.pr(0.85, 20)[0].cpu().numpy().astype(np.float64), oracle.pr(g, 0.85, 20), (1e-5, 0.0))
    print("ALL OK" if ok else "FAILURES", flush=True)
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
