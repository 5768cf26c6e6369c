// launch.h -- host side of the persistent-kernel engine: grid sizing, control-block carving,
// cooperative launch, and copy-back of the per-iteration records (the paper's feedback stage,
// P:840-844, done once per run instead of once per iteration).
#pragma once
#include "engine.cuh"
#include "internal.h"

namespace gsw {

struct LaunchInfo {
    int grid = 0;
};

// Blocks per SM of every persistent kernel (kernels declare __launch_bounds__(kBlock, kMinBlocks)).
#ifndef GSW_MINB
#define GSW_MINB 4            // A/B builds: make variant MINB=3 (Makefile)
#endif
constexpr int kMinBlocks = GSW_MINB;

gsw_status prepare_common(gsw_graph g, Workspace &ws, const void *kernel, RunCommon &rc, LaunchInfo &li);
gsw_status launch_persistent(gsw_graph g, const void *kernel, void **args, const LaunchInfo &li);
gsw_status finish_run(gsw_graph g, const RunCommon &rc, const LaunchInfo &li, gsw_run_stats *st);

// entry points implemented per algorithm
gsw_status run_bfs(gsw_graph g, int32_t source, int32_t *depth, gsw_run_stats *st);
gsw_status run_sssp(gsw_graph g, int32_t source, uint32_t *dist, gsw_run_stats *st);
gsw_status run_cc(gsw_graph g, int32_t *label, gsw_run_stats *st);
gsw_status run_pr(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st);
gsw_status run_dpr(gsw_graph g, double damping, double tol, int32_t max_iters, double *rank, gsw_run_stats *st);
gsw_status run_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc, gsw_run_stats *st);

}  // namespace gsw
