#!/usr/bin/env python
"""Device time of the two CC algorithms (min-label propagation gsw_cc vs hooking + pointer
jumping gsw_cc_hook) on the BASELINE configs, per forced load balance of the hook sweep."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import gen
import paper_conf_ppopp_menglts19_b200 as gsw


def best(fn, reps=3):
    b = None
    for _ in range(reps):
        out, st = fn()
        if b is None or st["gpu_ms"] < b[1]["gpu_ms"]:
            b = (out, st)
    return b


for cfg in sys.argv[1:] or ["C1", "C3", "C4", "C2"]:
    g = gen.config_graph(cfg)
    G = gsw.Graph(g.off, g.col)
    a, sa = best(lambda: G.cc(records=64))
    print(f"{cfg} cc (label propagation) {sa['gpu_ms']:8.3f} ms  iters={sa['iterations']}", flush=True)
    for lb in ["auto", "thread", "twc", "wm", "cm", "strict"]:
        G.force_config(load_balance=None if lb == "auto" else lb) if lb != "auto" else G.force_config()
        b, sb = best(lambda: G.cc_hook(records=64))
        same = bool(np.array_equal(a.cpu().numpy(), b.cpu().numpy()))
        hooks = [r["Va"] for r in sb["records"]]
        print(f"{cfg} cc_hook lb={lb:6s} {sb['gpu_ms']:8.3f} ms  iters={sb['iterations']} hooks={hooks} "
              f"GB/s(alg)={sb['bytes_alg'] / sb['gpu_ms'] / 1e6:7.1f} same_as_cc={same}", flush=True)
    G.force_config()
    del G
