#!/usr/bin/env python
"""Training corpus for the learned selector (Sec. 4.4).

The paper brute-forces every pattern combination per iteration on 644 real graphs and trains one
CART tree per pattern on the 21 features of each iteration.  Here the corpus is
synthetic (R-MAT at several skews / edge factors / scales, 2D grids, Chung-Lu power-law graphs --
the evaluation graphs C1..C5 are NOT in it: other seeds and sizes), and the brute force uses the
fact that BFS levels are unique: iteration t processes the same active set under every forced
variant, so the per-iteration device times of the 60 forced runs (gsw_force_config) are directly
comparable (the methodology of Fig. 14).

Writes one JSON: for every (graph, root, level): the features and the time of every variant.

  python tools/selector_corpus.py --json gpurun_out/selector_corpus.json
"""
import argparse
import itertools
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

DIRS = ["push", "pull"]
FMTS = ["bitmap", "queue", "sorted_queue"]
LBS = ["thread", "twc", "wm", "cm", "strict"]
FUS = ["standalone", "fused"]


def corpus(gen, size="full"):
    """~110 synthetic graphs (none of them C1-C5: other seeds and sizes).  size="small" keeps the
    round-1 list of 24."""
    out = []
    if size == "large":
        # round-2 addition: graphs as large as the evaluation configs (the 106-graph corpus stops at
        # scale 20 / 3M vertices, and its trees lost on C3/C4); other seeds and skews than C1-C5
        for scale, ef, abc, seed in [(21, 16, (.57, .19, .19), 301), (22, 16, (.57, .19, .19), 302),
                                     (22, 8, (.60, .15, .15), 303), (21, 32, (.50, .20, .20), 304),
                                     (23, 16, (.57, .19, .19), 305), (22, 24, (.65, .15, .15), 306)]:
            out.append(gen.rmat(scale, ef, *abc, seed=seed))
        for k, (n, pairs, gamma) in enumerate([(4_000_000, 60_000_000, 2.3), (5_000_000, 70_000_000, 2.2),
                                               (3_500_000, 50_000_000, 2.5), (6_000_000, 90_000_000, 2.4)]):
            out.append(gen.chung_lu(n, pairs, gamma=gamma, i0=150.0, seed=310 + k))
        out.append(gen.grid(1800, 1800))
        return out
    if size == "small":
        for scale, ef, abc, seed in [(14, 8, (.57, .19, .19), 11), (14, 32, (.57, .19, .19), 12),
                                     (15, 16, (.45, .25, .15), 13), (15, 16, (.70, .10, .10), 14),
                                     (16, 8, (.57, .19, .19), 15), (16, 16, (.45, .15, .15), 16),
                                     (17, 16, (.57, .19, .19), 17), (17, 4, (.57, .19, .19), 18),
                                     (18, 16, (.57, .19, .19), 19), (18, 8, (.65, .15, .15), 20),
                                     (19, 16, (.57, .19, .19), 21), (19, 32, (.50, .20, .20), 22),
                                     (20, 16, (.57, .19, .19), 23), (20, 8, (.60, .15, .15), 24),
                                     (21, 16, (.57, .19, .19), 25), (21, 24, (.50, .20, .20), 26)]:
            out.append(gen.rmat(scale, ef, *abc, seed=seed))
        for w, h in [(192, 192), (400, 100), (700, 700), (1400, 1000)]:
            out.append(gen.grid(w, h))
        for n, pairs, gamma, seed in [(200_000, 2_000_000, 2.1, 31), (300_000, 3_000_000, 2.5, 32),
                                      (500_000, 4_000_000, 2.3, 33), (2_000_000, 24_000_000, 2.3, 34)]:
            out.append(gen.chung_lu(n, pairs, gamma=gamma, i0=50.0, seed=seed))
        return out
    skews = [(.45, .15, .15), (.50, .20, .20), (.57, .19, .19), (.60, .15, .15), (.65, .15, .15), (.70, .10, .10)]
    seed = 100
    # R-MAT / Kronecker: scales 12-20 x edge factors 4-48 x six skews (72 graphs)
    for scale in (12, 13, 14, 15, 16, 17, 18, 19, 20):
        for k, ef in enumerate((4, 8, 16, 24, 32, 48, 6, 12)):
            if scale >= 19 and ef > 16:
                continue
            seed += 1
            out.append(gen.rmat(scale, ef, *skews[(scale + k) % len(skews)], seed=seed))
    # road-like grids of several sizes and aspect ratios (16)
    for w, h in [(64, 64), (128, 32), (150, 150), (256, 256), (300, 80), (400, 400), (512, 128), (600, 600),
                 (800, 200), (1000, 1000), (1200, 300), (1400, 1400), (2000, 120), (90, 3000), (1700, 900),
                 (2400, 500)]:
        out.append(gen.grid(w, h))
    # Chung-Lu power laws (24)
    for k, (n, pairs, gamma) in enumerate([(50_000, 300_000, 2.1), (50_000, 800_000, 2.6), (80_000, 500_000, 2.3),
                                           (100_000, 1_000_000, 2.0), (100_000, 600_000, 2.8),
                                           (150_000, 2_000_000, 2.2), (200_000, 1_500_000, 2.5),
                                           (250_000, 3_000_000, 2.1), (300_000, 2_000_000, 2.9),
                                           (400_000, 5_000_000, 2.3), (500_000, 3_000_000, 2.7),
                                           (600_000, 8_000_000, 2.2), (700_000, 5_000_000, 2.5),
                                           (800_000, 10_000_000, 2.4), (1_000_000, 6_000_000, 2.8),
                                           (1_000_000, 15_000_000, 2.1), (1_200_000, 10_000_000, 2.3),
                                           (1_500_000, 12_000_000, 2.6), (1_500_000, 20_000_000, 2.2),
                                           (2_000_000, 16_000_000, 2.4), (2_000_000, 30_000_000, 2.1),
                                           (2_500_000, 20_000_000, 2.5), (3_000_000, 25_000_000, 2.3),
                                           (3_000_000, 40_000_000, 2.2)]):
        out.append(gen.chung_lu(n, pairs, gamma=gamma, i0=20.0 + 10 * (k % 5), seed=200 + k))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--json", required=True)
    ap.add_argument("--roots", type=int, default=2)
    ap.add_argument("--size", default="full", choices=["full", "small", "large"])
    a = ap.parse_args()
    import torch
    import gen
    import paper_conf_ppopp_menglts19_b200 as gsw
    variants = list(itertools.product(DIRS, FMTS, LBS, FUS))
    rows = []
    t0 = time.time()
    for g in corpus(gen, a.size):
        G = gsw.Graph(g.off, g.col)
        attrs = G.attributes()
        for s in gen.sources(g, a.roots, seed=99):
            per = {}
            levels = None
            for v in variants:
                G.force_config(direction=v[0], format=v[1], load_balance=v[2], fusion=v[3])
                G.bfs(s)
                _, st = G.bfs(s, records=1 << 15)
                recs = st["records"]
                # cost of iteration t's decision = its Expand + the NEXT iteration's Filter (the
                # active-set materialisation the decision's output format/fusion forces on t+1)
                per["-".join(v)] = [recs[i]["expand_us"] + (recs[i + 1]["filter_us"] if i + 1 < len(recs) else 0.0)
                                    + (recs[i]["filter_us"] if i == 0 else 0.0) for i in range(len(recs))]
                if levels is None:
                    levels = [(r["Va"], r["Ea"], r["Via"], r["Eia"]) for r in recs]
            G.force_config()
            # road-like graphs have thousands of near-identical levels: keep at most 200 per root
            keep = range(len(levels)) if len(levels) <= 200 else sorted({int(i * (len(levels) - 1) / 199) for i in range(200)})
            for t in keep:
                Va, Ea, Via, Eia = levels[t]
                rows.append({"graph": g.name, "root": int(s), "t": t, "Va": Va, "Ea": Ea, "Via": Via, "Eia": Eia,
                             "attrs": attrs, "times": {k: round(v[t], 2) for k, v in per.items() if t < len(v)}})
        print(f"{g.name}: n={g.n} nnz={g.nnz} levels={len(levels)} rows={len(rows)} {time.time() - t0:.0f}s", flush=True)
        del G
        torch.cuda.empty_cache()
    if a.json.endswith(".gz"):
        import gzip
        with gzip.open(a.json, "wt") as f:
            json.dump(rows, f)
    else:
        with open(a.json, "w") as f:
            json.dump(rows, f)


if __name__ == "__main__":
    main()
