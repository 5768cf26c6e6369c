// select.cuh -- Inspector features + Selector (Sec. 4.3-4.5, Table 1, Fig. 12-13).
//
// The paper trains one CART tree per pattern offline on 386,780 records from 644 real graphs
// and applies them in the order direction -> load balance -> format -> stepping ->
// fusion.  Those trees are not printed and the corpus is out of scope, so the trees
// below are shallow hand-set if-else rules that encode the paper's stated findings (each rule
// cites the sentence it follows) with thresholds calibrated on B200.
// select_trees.cuh holds CART trees learned the paper's way on a synthetic brute-force corpus
// (tools/selector_corpus.py + tools/train_selector.py); GSW_SELECTOR=trees uses them for BFS.
// Every CTA evaluates the selector redundantly on identical inputs, so all CTAs agree on the
// configuration without an extra barrier.
#pragma once
#include "common.cuh"
#include "gsw.h"

namespace gsw {

struct Features {
    // dataset attributes (Table 1)
    float N, M, dbar, sd, rd, gini, her;
    // runtime characteristics of the current iteration
    long long Va, Ea, Via, Eia;
    unsigned maxd, mind;
    // historical information, lagged by one iteration (reading R9)
    float tf, te, Tf, Te;
    int iter;
    int selector;   // 0: the hand-set rules below; 1: the learned trees (select_trees.cuh, GSW_SELECTOR=trees)
};

struct DevCfg {
    int dir, fmt, lb, step, fused;
};

__device__ __forceinline__ int pick(int forced, int chosen) { return forced != GSW_AUTO ? forced : chosen; }

}  // namespace gsw
#include "select_trees.cuh"
namespace gsw {

// BFS-like traversal (BFS, BC forward): active = frontier, inactive = unvisited.
// Direction split (P1).  The paper's stated finding is "the pull mode is preferable ... when the
// number of the active edges is greater than that of inactive edges", i.e. a split on
// Ea/Eia at 1.  Its CART tree learns the split point per GPU (P:1220-1221 retrains for P100); on
// B200 the early-exit pull of tools/strategy_table.py wins already at Ea/Eia ~ 1/2 and loses at
// ~1/3600, and pulling a tiny frontier costs a full scan of the visited map, so the calibrated
// split is  pull <=> Ea * kPullAlpha > Eia  and  Va * kPullBeta > N   (reading R6).
constexpr float kPullAlpha = 16.f;
constexpr float kPullBeta = 2048.f;
constexpr long long kTwcMinActive = 148LL * 4 * kBlock * 4;   // items that fill every TWC tile once

__device__ __forceinline__ int traversal_direction(const Features &f) {
    return ((float)f.Ea * kPullAlpha > (float)f.Eia && (float)f.Va * kPullBeta > f.N) ? GSW_PULL : GSW_PUSH;
}

__device__ __forceinline__ DevCfg select_traversal(const Features &f, const gsw_config &force) {
    DevCfg c;
    if (f.selector == 1) {
        // learned CART trees (R13b), in the paper's order
        c.dir = pick(force.direction, tree_direction(f));
        c.lb = pick(force.load_balance, tree_lb(f, c.dir));
        c.fmt = pick(force.format, tree_format(f, c.dir, c.lb));
        c.fused = pick(force.fusion, tree_fusion(f, c.dir, c.lb, c.fmt));
        c.step = GSW_STEP_REMAIN;
        return c;
    }
    c.dir = pick(force.direction, traversal_direction(f));
    float cd = f.Va > 0 ? (float)f.Ea / (float)f.Va : 0.f;
    // P3 load balance: "TWC has the lowest overhead", "CM and WM perform better with irregular
    // workloads", "when the workload contains a hub vertex ... STRICT is the best".
    // Pull with early exit scans ~1-2 edges per vertex, so the per-thread mapping wins on B200.
    // On B200 TWC's tiles (blockDim x 4 items per CTA) only pay once the active set fills the
    // grid; below that WM with adaptive items per warp spreads the edges over every SM.
    int lb;
    if (c.dir == GSW_PULL) lb = GSW_LB_THREAD;
    else if (f.maxd > 1024u || cd > 64.f) lb = GSW_LB_STRICT;                // hub in workload
    else if (f.Va < kTwcMinActive) lb = GSW_LB_WM;                           // latency-bound
    else lb = GSW_LB_TWC;                                                    // regular degrees
    c.lb = pick(force.load_balance, lb);
    // P2 format: "bitmap is more friendly to dense workloads, the unsorted queue is more friendly
    // to sparse workloads, and the sorted queue is in the middle"; Fig. 12(b): queue
    // when the number of active vertices is small.
    float vap = f.N > 0 ? (float)f.Va / f.N : 0.f;
    int fmt;
    if (c.dir == GSW_PULL) fmt = GSW_BITMAP;
    else if (vap > 1.f / 16.f) fmt = GSW_BITMAP;
    else if (vap > 1.f / 256.f) fmt = GSW_SORTED_QUEUE;
    else fmt = GSW_QUEUE;
    c.fmt = pick(force.format, fmt);
    c.step = GSW_STEP_REMAIN;
    // P5 fusion: fused kernels are preferred when degrees are similar (Fig. 12(f));
    // fall back to standalone when the last iteration took far longer than the fused average
    // (P:681-682).  With atomic bitmap claiming the fused variant generates no
    // duplicates on B200, so it is also the default on skewed graphs.
    int fused = GSW_FUSED;
    if (f.iter >= 3 && f.Te > 0.f && (f.te + f.tf) > 4.f * (f.Te + f.Tf)) fused = GSW_STANDALONE;
    c.fused = pick(force.fusion, fused);
    return c;
}

}  // namespace gsw
