// launch.h -- host side of the persistent-kernel engine: grid sizing, control-block carving,
// cooperative launch, and copy-back of the per-iteration records (the paper's feedback stage,
// P:840-844, done once per run instead of once per iteration).
#pragma once
#include "engine.cuh"
#include "internal.h"

namespace gsw {

struct LaunchInfo {
    int grid = 0;
    int cluster = 0;   // > 0: the grid is one thread-block cluster of this many CTAs (no cooperative launch)
    int team = 0;      // > 0: cooperative launch in clusters of this many CTAs (team tier)
};

// Blocks per SM of every persistent kernel (kernels declare __launch_bounds__(kBlock, kMinBlocks)).
// Resident CTAs per SM of each persistent kernel (its __launch_bounds__ minimum, hence its
// register budget 65536 / (256 * k)).  Measured on B200 (profiles/r2/minblocks_ab.txt): the
// latency-bound level loops of BFS and SSSP run faster with fewer, fatter CTAs (the grid barrier
// has fewer arrivals and ptxas stops spilling), CC's bandwidth-heavy pulls with more.
// GSW_MINB=k (make variant MINB=k) forces one value for every kernel (A/B builds).
constexpr int kMaxBlocksPerSm = 4;
#ifdef GSW_MINB
constexpr int kMinBlocks = GSW_MINB, kMinBlocksBfs = GSW_MINB, kMinBlocksSssp = GSW_MINB, kMinBlocksCc = GSW_MINB,
              kMinBlocksBc = GSW_MINB, kMinBlocksPr = GSW_MINB, kMinBlocksApp = GSW_MINB;
#else
constexpr int kMinBlocks = 4;
constexpr int kMinBlocksBfs = 2, kMinBlocksSssp = 2, kMinBlocksCc = 4, kMinBlocksBc = 4, kMinBlocksPr = 4,
              kMinBlocksApp = 2;
#endif

gsw_status prepare_common(gsw_graph g, Workspace &ws, const void *kernel, RunCommon &rc, LaunchInfo &li,
                          int max_per_sm);
// Team tier: pick the cluster size (16, else 8) for a cooperative clustered launch of `kernel` at
// one CTA per SM and set li.grid / li.team / rc.team_k; no-op (returns false) when clusters do not
// fit or GSW_TEAM=0.
bool setup_team(gsw_graph g, const void *kernel, RunCommon &rc, LaunchInfo &li);
gsw_status launch_persistent(gsw_graph g, const void *kernel, void **args, const LaunchInfo &li);
gsw_status finish_run(gsw_graph g, const RunCommon &rc, const LaunchInfo &li, gsw_run_stats *st);

// entry points implemented per algorithm
gsw_status run_bfs(gsw_graph g, int32_t source, int32_t *depth, gsw_run_stats *st);
gsw_status run_sssp(gsw_graph g, int32_t source, uint32_t *dist, gsw_run_stats *st);
gsw_status run_cc(gsw_graph g, int32_t *label, gsw_run_stats *st);
gsw_status run_cc_hook(gsw_graph g, int32_t *label, gsw_run_stats *st);
gsw_status run_cc_hook_seeded(gsw_graph g, int32_t *label, gsw_run_stats *st, const int *seed, size_t ws_used);
gsw_status run_pr(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st);
gsw_status run_dpr(gsw_graph g, double damping, double tol, int32_t max_iters, double *rank, gsw_run_stats *st);
gsw_status run_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc, gsw_run_stats *st);

}  // namespace gsw
