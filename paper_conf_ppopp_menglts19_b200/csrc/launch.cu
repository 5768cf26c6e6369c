// launch.cu -- persistent cooperative launch + run bookkeeping shared by all algorithms.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <mutex>

#include "launch.h"

namespace gsw {

static long long env_ll(const char *name, long long dflt) {
    const char *v = std::getenv(name);
    return (v && *v) ? std::atoll(v) : dflt;
}

// Can one k-CTA cluster of `kernel` be resident at once?  (Non-portable sizes > 8 need the opt-in
// attribute; a GPC of B200 has 16-20 SMs.)  Cached per (kernel, k).
bool cluster_fits(const void *kernel, int k) {
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, bool> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_pair(kernel, k);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    if (k > 8 && cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess)
        cudaGetLastError();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(k);
    cfg.blockDim = dim3(kBlock);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = k;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int nc = 0;
    if (cudaOccupancyMaxActiveClusters(&nc, kernel, &cfg) != cudaSuccess) {
        cudaGetLastError();
        nc = 0;
    }
    cache[key] = nc > 0;
    return nc > 0;
}

static int blocks_per_sm(const void *kernel, int max_per_sm) {
    static std::mutex mu;
    static std::map<const void *, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(kernel);
    if (it != cache.end()) return it->second;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kernel, kBlock, 0) != cudaSuccess) {
        cudaGetLastError();
        nb = 1;
    }
    nb = std::max(1, std::min(nb, max_per_sm));   // the kernel's launch-bounds minimum (launch.h)
    // optional shared-memory carveout hint (percent), for L1-vs-smem A/B measurements
    if (const char *c = std::getenv("GSW_CARVEOUT")) {
        if (cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, std::atoi(c)) != cudaSuccess)
            cudaGetLastError();
    }
    cache[kernel] = nb;
    return nb;
}


gsw_status prepare_common(gsw_graph g, Workspace &ws, const void *kernel, RunCommon &rc, LaunchInfo &li,
                          int max_per_sm) {
    li.grid = g->sms * blocks_per_sm(kernel, max_per_sm);
    li.cluster = 0;
    li.team = 0;
    rc.cluster = 0;
    rc.team_k = 0;
    rc.team_e = env_ll("GSW_TEAM_E", 1ll << 40);
    // A/B knobs for the latency-bound level loops: GSW_GRID_CTAS=k runs the persistent kernel on k
    // CTAs (software grid barrier); GSW_CLUSTER=k (2..16) launches it as ONE k-CTA thread-block
    // cluster whose grid barrier is the hardware cluster barrier
    if (long long k = env_ll("GSW_GRID_CTAS", 0); k > 0 && k < li.grid) li.grid = (int)k;
    if (long long k = env_ll("GSW_CLUSTER", 0); k >= 2 && k <= 16 && cluster_fits(kernel, (int)k)) {
        li.grid = (int)k;
        li.cluster = (int)k;
        rc.cluster = 1;
    }
    static_assert(sizeof(Ctl) <= 1024, "control block fits the handle's slot");
    const bool own_ctl = g->ctl != nullptr;   // handle-owned block: zeroed at create, never reset
    rc.ctl = own_ctl ? (Ctl *)g->ctl : (Ctl *)ws.take(sizeof(Ctl));
    rc.cnt = (IterCnt *)ws.take(3 * sizeof(IterCnt));
    rc.hist = (Hist *)ws.take(sizeof(Hist) * kMaxHist);
    rc.rec = (gsw_iter_record *)ws.take(sizeof(gsw_iter_record) * kMaxHist);
    rc.partial = (uint32_t *)ws.take(sizeof(uint32_t) * (li.grid + 1));
    rc.pub = (TeamPub *)ws.take(sizeof(TeamPub));
    if (!rc.ctl || !rc.cnt || !rc.hist || !rc.rec || !rc.partial || !rc.pub) {
        set_error("workspace too small for the run's control blocks");
        return GSW_ENOMEM;
    }
    rc.force = g->forced;
    const Attrs &A = g->attrs;
    Features f{};
    f.N = (float)A.N; f.M = (float)A.M; f.dbar = (float)A.dbar; f.sd = (float)A.sd; f.rd = (float)A.rd;
    f.gini = (float)A.gini; f.her = (float)A.her;
    rc.base = f;
    // the run's device time starts here: the control-block reset below is part of the call
    GSW_CUDA(cudaEventRecord(g->ev0, g->stream));
    // solo tier (CTA 0 alone for tiny active sets); GSW_SOLO_E / GSW_SOLO_V override (calibration)
    rc.solo_e = env_ll("GSW_SOLO_E", kSoloE);
    rc.solo_v = env_ll("GSW_SOLO_V", kSoloV);
    if (!own_ctl) GSW_CUDA(cudaMemsetAsync(rc.ctl, 0, sizeof(Ctl), g->stream));
    return GSW_OK;
}

// Clusters of k CTAs of `kernel` that can be co-resident (cooperative launch needs them all).
static int max_clusters(const void *kernel, int k, int sms) {
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_pair(kernel, k);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    if (k > 8 && cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess)
        cudaGetLastError();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(k * (sms / k)));
    cfg.blockDim = dim3(kBlock);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = k;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int nc = 0;
    if (cudaOccupancyMaxActiveClusters(&nc, kernel, &cfg) != cudaSuccess) {
        cudaGetLastError();
        nc = 0;
    }
    nc = std::min(nc, sms / k);
    cache[key] = nc;
    return nc;
}

bool setup_team(gsw_graph g, const void *kernel, RunCommon &rc, LaunchInfo &li) {
    // off by default: measured slower than the grid path on C2 (profiles/r2/team_*.txt)
    const long long want = env_ll("GSW_TEAM", 0);
    if (li.cluster && env_ll("GSW_TEAM_IN_CLUSTER", 0)) {   // A/B: the whole (single-cluster) grid is the team
        rc.team_k = li.cluster;
        return true;
    }
    if (want < 2 || rc.cluster || li.cluster) return false;
    for (int k : {16, 8, 4}) {
        if (k > want) continue;
        const int nc = max_clusters(kernel, k, g->sms);
        // keep at least ~3/4 of the SMs for the grid-wide levels
        if (nc * k * 4 < g->sms * 3) continue;
        li.grid = nc * k;
        li.team = k;
        rc.team_k = k;
        return true;
    }
    return false;
}

gsw_status launch_persistent(gsw_graph g, const void *kernel, void **args, const LaunchInfo &li) {
    if (li.team > 0) {
        if (li.team > 8) GSW_CUDA(cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(li.grid);
        cfg.blockDim = dim3(kBlock);
        cfg.stream = g->stream;
        cudaLaunchAttribute at[2];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = li.team;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        at[1].id = cudaLaunchAttributeCooperative;
        at[1].val.cooperative = 1;
        cfg.attrs = at;
        cfg.numAttrs = 2;
        GSW_CUDA(cudaLaunchKernelExC(&cfg, kernel, args));
        GSW_CUDA(cudaEventRecord(g->ev1, g->stream));
        return GSW_OK;
    }
    if (li.cluster > 0) {
        // one cluster: its CTAs are co-scheduled by construction (no cooperative attribute needed)
        if (li.cluster > 8) GSW_CUDA(cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(li.grid);
        cfg.blockDim = dim3(kBlock);
        cfg.stream = g->stream;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = li.cluster;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        GSW_CUDA(cudaLaunchKernelExC(&cfg, kernel, args));
        GSW_CUDA(cudaEventRecord(g->ev1, g->stream));
        return GSW_OK;
    }
    GSW_CUDA(cudaLaunchCooperativeKernel(kernel, dim3(li.grid), dim3(kBlock), args, 0, g->stream));
    GSW_CUDA(cudaEventRecord(g->ev1, g->stream));
    return GSW_OK;
}

gsw_status finish_run(gsw_graph g, const RunCommon &rc, const LaunchInfo &li, gsw_run_stats *st) {
    (void)li;
    Ctl h{};
    GSW_CUDA(cudaMemcpyAsync(&h, rc.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g->stream));
    GSW_CUDA(cudaStreamSynchronize(g->stream));
    if (h.err) { set_error("device error code " + std::to_string(h.err)); return GSW_ECUDA; }
    if (h.t_end && std::getenv("GSW_PHASES"))
        std::fprintf(stderr, "gsw phases: init %.2f us, iterations %.2f us, output %.2f us\n",
                     (h.t_phase - h.t_start) * 1e-3, (h.t_expand - h.t_phase) * 1e-3, (h.t_end - h.t_expand) * 1e-3);
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = (int32_t)h.iters;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)h.edges_total;
        st->bytes_alg = (int64_t)h.bytes_alg;
        if (st->records && st->max_records > 0) {
            int nr = std::min<int>({(int)h.iters, st->max_records, kMaxHist});
            if (nr > 0)
                GSW_CUDA(cudaMemcpy(st->records, rc.rec, sizeof(gsw_iter_record) * nr, cudaMemcpyDeviceToHost));
        }
    }
    return GSW_OK;
}

}  // namespace gsw
