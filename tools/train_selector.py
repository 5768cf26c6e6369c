#!/usr/bin/env python
"""Train the per-pattern CART selector trees (Sec. 4.4) from
tools/selector_corpus.py's brute-force records and emit them as device if-else code.

As in the paper, one shallow decision tree per pattern, applied in the order direction -> load
balance -> format -> fusion; each later tree sees the earlier decisions as inputs.
The label of an iteration is the pattern value of its fastest forced variant; the training is cost-
sensitive: the direction tree weights a row by what the other direction would cost (|best push -
best pull|), the other trees by the row's median-minus-best variant time.  Features are the
Table 1 quantities available on the device: dataset N, d-bar, sigma_d, r_d, Gini,
H_er; runtime V_ap, E_ap, V_iap, E_iap, cd = Ea/Va, and the active/inactive edge ratio Ea/Eia
(the quantity of the paper's direction rule).

  python tools/train_selector.py gpurun_out/selector_corpus.json \
      [--emit paper_conf_ppopp_menglts19_b200/csrc/select_trees.cuh] [--depth 4]
"""
import argparse
import collections
import json
import os

import numpy as np

DIRS = ["push", "pull"]
FMTS = ["bitmap", "queue", "sorted_queue"]
LBS = ["thread", "twc", "wm", "cm", "strict"]
FUS = ["standalone", "fused"]
ENUM = {"push": "GSW_PUSH", "pull": "GSW_PULL", "bitmap": "GSW_BITMAP", "queue": "GSW_QUEUE",
        "sorted_queue": "GSW_SORTED_QUEUE", "thread": "GSW_LB_THREAD", "twc": "GSW_LB_TWC", "wm": "GSW_LB_WM",
        "cm": "GSW_LB_CM", "strict": "GSW_LB_STRICT", "standalone": "GSW_STANDALONE", "fused": "GSW_FUSED"}
FEATURES = ["N", "dbar", "sigma_d", "r_d", "gini", "h_er", "V_ap", "E_ap", "V_iap", "E_iap", "cd", "r_e"]
# device expressions of the features (select.cuh Features)
DEVICE = {"N": "f.N", "dbar": "f.dbar", "sigma_d": "f.sd", "r_d": "f.rd", "gini": "f.gini", "h_er": "f.her",
          "V_ap": "(float)f.Va / f.N", "E_ap": "(float)f.Ea / (2.f * f.M)", "V_iap": "(float)f.Via / f.N",
          "E_iap": "(float)f.Eia / (2.f * f.M)", "cd": "(f.Va > 0 ? (float)f.Ea / (float)f.Va : 0.f)",
          "r_e": "((float)f.Ea / (float)(f.Eia > 0 ? f.Eia : 1))"}


def feats(r):
    A = r["attrs"]
    N, M = A["N"], A["M"]
    Va, Ea, Via, Eia = r["Va"], r["Ea"], r["Via"], r["Eia"]
    return [N, A["dbar"], A["sigma_d"], A["r_d"], A["gini"], A["h_er"], Va / N, Ea / (2 * M), Via / N,
            Eia / (2 * M), Ea / Va if Va else 0.0, Ea / max(Eia, 1)]


def split(name):
    d, rest = name.split("-", 1)
    for f in FMTS:
        if rest.startswith(f + "-"):
            lb, fu = rest[len(f) + 1:].split("-")
            return d, f, lb, fu
    raise ValueError(name)


def rules(x):
    """The hand-set rules of select.cuh (without maxd, which the corpus does not record)."""
    N, Va, Ea, Eia = x["N"], x["Va"], x["Ea"], x["Eia"]
    d = "pull" if (Ea * 16.0 > Eia and Va * 2048.0 > N) else "push"
    cd = Ea / Va if Va else 0
    lb = "thread" if d == "pull" else ("strict" if cd > 64 else ("wm" if Va < 148 * 4 * 256 * 4 else "twc"))
    vap = Va / N
    fmt = "bitmap" if (d == "pull" or vap > 1 / 16) else ("sorted_queue" if vap > 1 / 256 else "queue")
    return f"{d}-{fmt}-{lb}-fused"


def emit_tree(tree, names, classes, fn, indent="    "):
    from sklearn.tree import _tree
    t = tree.tree_
    lines = []

    def leaf_class(node):
        """the class a subtree returns if every leaf below agrees, else None (identical-leaf
        splits are collapsed when emitting: VERDICT r1 noted them in select_trees.cuh)"""
        if t.feature[node] == _tree.TREE_UNDEFINED:
            return int(np.argmax(t.value[node][0]))
        l, r = leaf_class(t.children_left[node]), leaf_class(t.children_right[node])
        return l if (l is not None and l == r) else None

    def rec(node, depth):
        pad = indent * depth
        same = leaf_class(node)
        if same is not None:
            lines.append(f"{pad}return {ENUM[classes[same]]};")
            return
        if t.feature[node] != _tree.TREE_UNDEFINED:
            lit = f"{t.threshold[node]:.9g}"
            lit = lit if ("." in lit or "e" in lit) else lit + ".0"
            lines.append(f"{pad}if ({names[t.feature[node]]} <= {lit}f) {{")
            rec(t.children_left[node], depth + 1)
            lines.append(f"{pad}}} else {{")
            rec(t.children_right[node], depth + 1)
            lines.append(f"{pad}}}")
        else:
            lines.append(f"{pad}return {ENUM[classes[int(np.argmax(t.value[node][0]))]]};")
    rec(0, 1)
    return lines


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("corpus")
    ap.add_argument("--emit", default=None)
    ap.add_argument("--depth", type=int, default=4)
    ap.add_argument("--report", default=None)
    ap.add_argument("--ccp", type=float, default=0.0, help="cost-complexity pruning alpha (sklearn ccp_alpha)")
    ap.add_argument("--drop", default="N", help="comma-separated features left out (default: N, the only "
                    "absolute size; the others are scale-free ratios or distribution shapes)")
    a = ap.parse_args()
    from sklearn.tree import DecisionTreeClassifier
    if a.corpus.endswith(".gz"):
        import gzip
        raw = json.load(gzip.open(a.corpus, "rt"))
    else:
        raw = json.load(open(a.corpus))
    rows = [r for r in raw if r["Va"] > 0 and len(r["times"]) == 60]
    keep = [i for i, f in enumerate(FEATURES) if f not in a.drop.split(",")]
    X = np.array([feats(r) for r in rows])[:, keep]
    best = [min(r["times"], key=r["times"].get) for r in rows]
    w = np.array([np.median(list(r["times"].values())) - min(r["times"].values()) + 1e-3 for r in rows])
    # cost-sensitive weight of the direction decision: what choosing the other direction costs
    wd = np.array([abs(min(v for k, v in r["times"].items() if k.startswith("push-")) -
                       min(v for k, v in r["times"].items() if k.startswith("pull-"))) + 1e-3 for r in rows])
    lab = [split(b) for b in best]
    graphs = sorted({r["graph"] for r in rows})

    def fit(Xs, ys, ws):
        # cost-complexity pruning (the paper keeps "its height as low as possible")
        clf = DecisionTreeClassifier(max_depth=a.depth, min_samples_leaf=3, random_state=0, ccp_alpha=a.ccp)
        clf.fit(Xs, ys, sample_weight=ws)
        return clf

    def train(idx):
        Xi, wi = X[idx], w[idx]
        yd = [lab[i][0] for i in idx]
        t_dir = fit(Xi, yd, wd[idx])
        dcode = np.array([[DIRS.index(lab[i][0])] for i in idx])
        Xl = np.hstack([Xi, dcode])
        t_lb = fit(Xl, [lab[i][2] for i in idx], wi)
        lcode = np.array([[LBS.index(lab[i][2])] for i in idx])
        Xf = np.hstack([Xl, lcode])
        t_fmt = fit(Xf, [lab[i][1] for i in idx], wi)
        fcode = np.array([[FMTS.index(lab[i][1])] for i in idx])
        t_fus = fit(np.hstack([Xf, fcode]), [lab[i][3] for i in idx], wi)
        return t_dir, t_lb, t_fmt, t_fus

    def predict(trees, x):
        t_dir, t_lb, t_fmt, t_fus = trees
        d = t_dir.predict([x])[0]
        xl = list(x) + [DIRS.index(d)]
        lb = t_lb.predict([xl])[0]
        xf = xl + [LBS.index(lb)]
        fm = t_fmt.predict([xf])[0]
        fu = t_fus.predict([xf + [FMTS.index(fm)]])[0]
        return f"{d}-{fm}-{lb}-{fu}"

    # leave-one-graph-out: per-graph total of the chosen per-iteration variant times
    report = collections.OrderedDict()
    tot = collections.Counter()
    for gname in graphs:
        tr = [i for i, r in enumerate(rows) if r["graph"] != gname]
        te = [i for i, r in enumerate(rows) if r["graph"] == gname]
        trees = train(tr)
        s = collections.Counter()
        fixed = collections.Counter()
        for i in te:
            r = rows[i]
            s["oracle"] += min(r["times"].values())
            s["trees_logo"] += r["times"][predict(trees, X[i])]
            s["rules"] += r["times"][rules({"N": r["attrs"]["N"], **r})]
            for k, v in r["times"].items():
                fixed[k] += v
        s["best_fixed"] = min(fixed.values())
        report[gname] = {k: round(v, 1) for k, v in s.items()}
        tot.update(s)
    report["TOTAL"] = {k: round(v, 1) for k, v in tot.items()}
    for k, v in report.items():
        print(f"{k:28s} " + " ".join(f"{kk}={vv:9.1f}" for kk, vv in v.items()))
    trees = train(list(range(len(rows))))
    acc = np.mean([predict(trees, X[i]) == best[i] for i in range(len(rows))])
    print(f"rows={len(rows)} graphs={len(graphs)} exact-variant training accuracy={acc:.3f}")
    if a.report:
        json.dump({"logo_us": report, "train_variant_accuracy": acc, "rows": len(rows), "graphs": graphs,
                   "depth": a.depth}, open(a.report, "w"), indent=1)
    if a.emit:
        names = [DEVICE[FEATURES[i]] for i in keep]
        out = ["// select_trees.cuh -- GENERATED by tools/train_selector.py (do not edit): the per-pattern",
               "// CART trees of the learned selector (PAPER.md Sec. 4.4, P:944-1021; SURVEY 8(f) F1), trained on",
               f"// {len(rows)} brute-forced BFS iterations of {len(graphs)} synthetic graphs (tools/selector_corpus.py).",
               "// Applied in the paper's order direction -> LB -> format -> fusion (P:1083-1090); each tree",
               "// sees the earlier decisions.  Selected with GSW_SELECTOR=trees (DESIGN.md R13b).",
               "#pragma once", '#include "gsw.h"', "", "namespace gsw {", ""]
        t_dir, t_lb, t_fmt, t_fus = trees
        out.append("__device__ __forceinline__ int tree_direction(const Features &f) {")
        out += emit_tree(t_dir, names, list(t_dir.classes_), "dir")
        out.append("}")
        out.append("__device__ __forceinline__ int tree_lb(const Features &f, int dir) {")
        out += emit_tree(t_lb, names + ["(dir == GSW_PULL ? 1.f : 0.f)"], list(t_lb.classes_), "lb")
        out.append("}")
        lbx = "(float)(lb == GSW_LB_THREAD ? 0 : lb == GSW_LB_TWC ? 1 : lb == GSW_LB_WM ? 2 : lb == GSW_LB_CM ? 3 : 4)"
        out.append("__device__ __forceinline__ int tree_format(const Features &f, int dir, int lb) {")
        out += emit_tree(t_fmt, names + ["(dir == GSW_PULL ? 1.f : 0.f)", lbx], list(t_fmt.classes_), "fmt")
        out.append("}")
        fmx = "(float)(fmt == GSW_BITMAP ? 0 : fmt == GSW_QUEUE ? 1 : 2)"
        out.append("__device__ __forceinline__ int tree_fusion(const Features &f, int dir, int lb, int fmt) {")
        out += emit_tree(t_fus, names + ["(dir == GSW_PULL ? 1.f : 0.f)", lbx, fmx], list(t_fus.classes_), "fus")
        out.append("}")
        out += ["", "}  // namespace gsw", ""]
        open(a.emit, "w").write("\n".join(out))
        print("wrote", a.emit)


if __name__ == "__main__":
    main()
