// capi.cu -- the extern "C" boundary declared in include/gsw.h: argument validation, error
// plumbing, handle lifetime.  Every compute step runs in the kernels of the other .cu files.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "launch.h"

namespace gsw {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }

gsw_status cuda_fail(cudaError_t e, const char *what) {
    g_err = std::string("CUDA error ") + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ") at " + what;
    cudaGetLastError();
    return GSW_ECUDA;
}

size_t graph_bytes(int64_t n, int64_t nnz, int has_w, int has_csc);
gsw_status load_csr(gsw_graph g, const gsw_csr *c, Workspace &ws, uint32_t **off, int32_t **col, uint32_t **w,
                    int64_t *staging);
gsw_status compute_attrs(gsw_graph g, unsigned *iso_bitmap, void *tmp);
gsw_status validate_graph(gsw_graph g);
gsw_status relabel_graph(gsw_graph g, uint32_t *perm, uint32_t *inv, char *tmp, size_t tmp_bytes);
gsw_status build_first_nbr(gsw_graph g, int32_t *first);
// dist.cu
int64_t dist_slice(int64_t n, int32_t p);
gsw_status dist_create(const gsw_csr *rows, int64_t n, const void *nccl_id, const gsw_exchange *hx, int32_t nranks,
                       int32_t rank, int mode, void *workspace, size_t ws_bytes, void *stream, gsw_graph *out);
void dist_destroy(DistState *d);
gsw_status dist_bfs(gsw_graph g, int32_t source, int32_t *depth_out, gsw_run_stats *st);
gsw_status dist_pr(gsw_graph g, double damping, int32_t iters, double *rank_out, gsw_run_stats *st);
gsw_status dist_cc(gsw_graph g, int32_t *label_out, gsw_run_stats *st);
gsw_status dist_sssp(gsw_graph g, int32_t source, uint32_t *dist_out, gsw_run_stats *st);
gsw_status dist_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc_out, gsw_run_stats *st);
size_t dist_workspace(int64_t n, int64_t nnz, int32_t nranks, int32_t nparts, int mode, bool weighted);
enum { kModeNccl = 0, kModeLoopback = 1, kModeHost = 2 };   // dist.cu DistMode
gsw_status dist_unique_id(void *id128);

static gsw_status no_dist(gsw_graph g, const char *what) {
    if (g->dist) { set_error(std::string(what) + ": not supported on a distributed handle"); return GSW_EUNSUPPORTED; }
    return GSW_OK;
}

static gsw_status check_csr(const gsw_csr *c, const char *what) {
    if (!c) { set_error(std::string(what) + " is NULL"); return GSW_EINVAL; }
    if (c->n <= 0) { set_error(std::string(what) + ": n must be > 0"); return GSW_EINVAL; }
    if (c->n >= (int64_t(1) << 31) - 64) { set_error(std::string(what) + ": n >= 2^31"); return GSW_EOVERFLOW; }
    if (c->nnz < 0) { set_error(std::string(what) + ": nnz < 0"); return GSW_EINVAL; }
    if (c->nnz >= (int64_t(1) << 32)) { set_error(std::string(what) + ": nnz >= 2^32"); return GSW_EOVERFLOW; }
    if (!c->row_offsets || (c->nnz > 0 && !c->col_indices)) {
        set_error(std::string(what) + ": null array");
        return GSW_EINVAL;
    }
    return GSW_OK;
}

}  // namespace gsw

using namespace gsw;

extern "C" {

const char *gsw_last_error(void) { return g_err.c_str(); }
const char *gsw_version(void) { return "gsw-b200 0.1 (sm_100a)"; }

gsw_status gsw_workspace_size(int64_t n, int64_t nnz, int32_t has_weights, int32_t has_csc, size_t *bytes) {
    if (!bytes || n <= 0 || nnz < 0) { set_error("gsw_workspace_size: bad arguments"); return GSW_EINVAL; }
    if (nnz >= (int64_t(1) << 32) || n >= (int64_t(1) << 31) - 64) { set_error("graph too large"); return GSW_EOVERFLOW; }
    *bytes = graph_bytes(n, nnz, has_weights, has_csc) + scratch_bytes_for(n, nnz, has_weights) + 4096;
    return GSW_OK;
}

gsw_status gsw_graph_create(const gsw_csr *csr, const gsw_csr *csc, void *workspace, size_t ws_bytes,
                            void *cuda_stream, gsw_graph *out) {
    gsw_status s;
    if (!out) { set_error("gsw_graph_create: out is NULL"); return GSW_EINVAL; }
    *out = nullptr;
    if ((s = check_csr(csr, "csr")) != GSW_OK) return s;
    if (csc) {
        if ((s = check_csr(csc, "csc")) != GSW_OK) return s;
        if (csc->n != csr->n || csc->nnz != csr->nnz) { set_error("csc shape differs from csr"); return GSW_EINVAL; }
        if ((csr->weights == nullptr) != (csc->weights == nullptr)) { set_error("csr/csc weights mismatch"); return GSW_EINVAL; }
    }
    if (!workspace || is_device_ptr(workspace) != 1) { set_error("workspace must be a device pointer"); return GSW_EINVAL; }
    if (((uintptr_t)workspace & 255) != 0) { set_error("workspace must be 256-byte aligned"); return GSW_EINVAL; }
    size_t need = 0;
    if ((s = gsw_workspace_size(csr->n, csr->nnz, csr->weights != nullptr, csc != nullptr, &need)) != GSW_OK) return s;
    if (ws_bytes < need) { set_error("workspace too small: need " + std::to_string(need) + " bytes"); return GSW_ENOMEM; }
    // offsets[0] == 0 and offsets[n] == nnz (host-side check of two entries)
    int64_t ends[2] = {0, 0};
    auto read_i64 = [](const int64_t *p, int64_t *dst) -> cudaError_t {
        if (is_device_ptr(p)) return cudaMemcpy(dst, p, 8, cudaMemcpyDeviceToHost);
        *dst = *p;
        return cudaSuccess;
    };
    for (const gsw_csr *c : {csr, csc}) {
        if (!c) continue;
        GSW_CUDA(read_i64(c->row_offsets, &ends[0]));
        GSW_CUDA(read_i64(c->row_offsets + c->n, &ends[1]));
        if (ends[0] != 0 || ends[1] != c->nnz) { set_error("row_offsets[0] must be 0 and row_offsets[n] == nnz"); return GSW_EINVAL; }
    }
    gsw_graph g = new gsw_graph_s();
    g->stream = (cudaStream_t)cuda_stream;
    g->ws = (char *)workspace;
    g->ws_bytes = ws_bytes;
    cudaError_t e = cudaGetDevice(&g->device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g->sms, cudaDevAttrMultiProcessorCount, g->device);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev0);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev1);
    if (e != cudaSuccess) { delete g; return cuda_fail(e, "gsw_graph_create setup"); }
    Workspace ws{g->ws, ws_bytes, 0};
    size_t gb = graph_bytes(csr->n, csr->nnz, csr->weights != nullptr, csc != nullptr);
    Workspace gws{g->ws, gb + 1024, 0};   // graph region (CSR/CSC, isolated bitmap, perm/inv)
    g->scratch = g->ws + ((gb + 1024 + 255) & ~size_t(255));
    g->scratch_bytes = ws_bytes - ((gb + 1024 + 255) & ~size_t(255));
    int64_t *staging = (int64_t *)g->scratch;
    uint32_t *off, *woff;
    int32_t *col;
    uint32_t *w;
    if ((s = load_csr(g, csr, gws, &off, &col, &w, staging)) != GSW_OK) { gsw_graph_destroy(g); return s; }
    g->g.n = (int)csr->n;
    g->g.nnz = (uint32_t)csr->nnz;
    g->g.off = off; g->g.col = col; g->g.w = w;
    if (csc) {
        int32_t *icol;
        uint32_t *iw;
        // staging is reused: the offsets conversion of the CSR has been enqueued before on the same stream
        if ((s = load_csr(g, csc, gws, &woff, &icol, &iw, staging + (csr->n + 1))) != GSW_OK) { gsw_graph_destroy(g); return s; }
        g->g.in_off = woff; g->g.in_col = icol; g->g.in_w = iw;
        g->symmetric = false;
    } else {
        g->g.in_off = off; g->g.in_col = col; g->g.in_w = w;
        g->symmetric = true;
    }
    g->iso = (unsigned *)gws.take((size_t)((csr->n + 31) / 32) * 4);
    uint32_t *perm = (uint32_t *)gws.take((size_t)csr->n * 4), *inv = (uint32_t *)gws.take((size_t)csr->n * 4);
    if (!g->iso || !perm || !inv) { gsw_graph_destroy(g); set_error("workspace too small"); return GSW_ENOMEM; }
    // degree-ordered relabeling (graph.cu); GSW_NO_RELABEL=1 keeps caller order (A/B measurements)
    const char *nr = getenv("GSW_NO_RELABEL");
    if (!(nr && nr[0] == '1') && csr->nnz < (int64_t(1) << 31)) {
        if ((s = relabel_graph(g, perm, inv, g->scratch, g->scratch_bytes)) != GSW_OK) { gsw_graph_destroy(g); return s; }
    }
    int32_t *first = (int32_t *)gws.take((size_t)csr->n * 4 + 4);
    if (!first) { gsw_graph_destroy(g); set_error("workspace too small"); return GSW_ENOMEM; }
    if ((s = build_first_nbr(g, first)) != GSW_OK) { gsw_graph_destroy(g); return s; }
    if (g->g.inv) {
        g->iso_caller = (unsigned *)gws.take((size_t)((csr->n + 31) / 32) * 4);
        if (!g->iso_caller) { gsw_graph_destroy(g); set_error("workspace too small"); return GSW_ENOMEM; }
    }
    g->ctl = gws.take(1024);
    if (!g->ctl || cudaMemsetAsync(g->ctl, 0, 1024, g->stream) != cudaSuccess) {
        gsw_graph_destroy(g);
        set_error("workspace too small / control block");
        return GSW_ENOMEM;
    }
    void *tmp = (char *)g->scratch + (((csr->n + 1) * 16 + 4096 + 255) & ~int64_t(255));
    if ((s = compute_attrs(g, g->iso, tmp)) != GSW_OK) { gsw_graph_destroy(g); return s; }
    *out = g;
    return GSW_OK;
}

gsw_status gsw_graph_destroy(gsw_graph g) {
    if (!g) return GSW_OK;
    if (g->ev0) cudaEventDestroy(g->ev0);
    if (g->ev1) cudaEventDestroy(g->ev1);
    if (g->poll) cudaFreeHost(g->poll);
    dist_destroy(g->dist);
    delete g;
    return GSW_OK;
}

gsw_status gsw_graph_validate(gsw_graph g) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (gsw_status s = no_dist(g, "gsw_graph_validate")) return s;
    return validate_graph(g);
}

gsw_status gsw_graph_attributes(gsw_graph g, double out[7]) {
    if (!g || !out) { set_error("null argument"); return GSW_EINVAL; }
    const Attrs &A = g->attrs;
    out[0] = A.N; out[1] = A.M; out[2] = A.dbar; out[3] = A.sd; out[4] = A.rd; out[5] = A.gini; out[6] = A.her;
    return GSW_OK;
}

gsw_status gsw_force_config(gsw_graph g, const gsw_config *cfg) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (!cfg) { g->forced = gsw_config{}; return GSW_OK; }
    auto in = [](int v, int lo, int hi) { return v == GSW_AUTO || (v >= lo && v <= hi); };
    if (!in(cfg->direction, GSW_PUSH, GSW_PULL) || !in(cfg->format, GSW_BITMAP, GSW_SORTED_QUEUE) ||
        !in(cfg->load_balance, GSW_LB_THREAD, GSW_LB_STRICT) ||
        !in(cfg->stepping, GSW_STEP_INCREASE, GSW_STEP_UNORDERED) || !in(cfg->fusion, GSW_STANDALONE, GSW_FUSED)) {
        set_error("gsw_force_config: field out of range");
        return GSW_EINVAL;
    }
    g->forced = *cfg;
    return GSW_OK;
}

gsw_status gsw_bfs(gsw_graph g, int32_t source, int32_t *depth, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (g->dist) return dist_bfs(g, source, depth, stats);
    return run_bfs(g, source, depth, stats);
}

gsw_status gsw_sssp(gsw_graph g, int32_t source, uint32_t *dist, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (g->dist) return dist_sssp(g, source, dist, stats);
    return run_sssp(g, source, dist, stats);
}

gsw_status gsw_cc(gsw_graph g, int32_t *label, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (g->dist) return dist_cc(g, label, stats);
    return run_cc(g, label, stats);
}

gsw_status gsw_cc_hook(gsw_graph g, int32_t *label, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (gsw_status s = no_dist(g, "gsw_cc_hook")) return s;
    return run_cc_hook(g, label, stats);
}

gsw_status gsw_pr(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (g->dist) return dist_pr(g, damping, iters, rank, stats);
    return run_pr(g, damping, iters, rank, stats);
}

gsw_status gsw_dpr(gsw_graph g, double damping, double tol, int32_t max_iters, double *rank, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (gsw_status s = no_dist(g, "gsw_dpr")) return s;
    return run_dpr(g, damping, tol, max_iters, rank, stats);
}

gsw_status gsw_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc, gsw_run_stats *stats) {
    if (!g) { set_error("null graph"); return GSW_EINVAL; }
    if (g->dist) return dist_bc(g, sources, nsrc, bc, stats);
    return run_bc(g, sources, nsrc, bc, stats);
}

int64_t gsw_dist_slice(int64_t n, int32_t nranks) { return (n > 0 && nranks > 0) ? dist_slice(n, nranks) : 0; }

gsw_status gsw_dist_unique_id(void *id128) { return dist_unique_id(id128); }

gsw_status gsw_dist_workspace_size(int64_t n_global, int64_t nnz_owned, int32_t nranks, size_t *bytes) {
    if (!bytes || n_global <= 0 || nnz_owned < 0 || nranks < 1) { set_error("gsw_dist_workspace_size: bad arguments"); return GSW_EINVAL; }
    *bytes = dist_workspace(n_global, nnz_owned, nranks, 1, kModeNccl, false);
    return GSW_OK;
}

gsw_status gsw_dist_workspace_size_weighted(int64_t n_global, int64_t nnz_owned, int32_t nranks, int32_t has_weights,
                                            int32_t loopback, size_t *bytes) {
    if (!bytes || n_global <= 0 || nnz_owned < 0 || nranks < 1) { set_error("gsw_dist_workspace_size_weighted: bad arguments"); return GSW_EINVAL; }
    *bytes = dist_workspace(n_global, nnz_owned, nranks, loopback ? nranks : 1, loopback ? kModeLoopback : kModeNccl,
                            has_weights != 0);
    return GSW_OK;
}

gsw_status gsw_dist_loopback_workspace_size(int64_t n, int64_t nnz, int32_t nparts, size_t *bytes) {
    if (!bytes || n <= 0 || nnz < 0 || nparts < 1) { set_error("gsw_dist_loopback_workspace_size: bad arguments"); return GSW_EINVAL; }
    *bytes = dist_workspace(n, nnz, nparts, nparts, kModeLoopback, false);
    return GSW_OK;
}

gsw_status gsw_graph_create_dist(const gsw_csr *owned, int64_t n_global, const void *nccl_id128, int32_t nranks,
                                 int32_t rank, void *workspace, size_t ws_bytes, void *cuda_stream, gsw_graph *out) {
    if (!out) { set_error("out is NULL"); return GSW_EINVAL; }
    if (nranks > 1 && !nccl_id128) { set_error("nccl_id128 is NULL"); return GSW_EINVAL; }
    unsigned char own_id[128];
    if (!nccl_id128) {                      // one rank: a private communicator, the collectives still run
        if (gsw_status s = dist_unique_id(own_id)) return s;
        nccl_id128 = own_id;
    }
    return dist_create(owned, n_global, nccl_id128, nullptr, nranks, rank, kModeNccl, workspace, ws_bytes, cuda_stream,
                       out);
}

gsw_status gsw_graph_create_dist_host(const gsw_csr *owned, int64_t n_global, const gsw_exchange *exchange,
                                      int32_t nranks, int32_t rank, void *workspace, size_t ws_bytes,
                                      void *cuda_stream, gsw_graph *out) {
    if (!out || !exchange) { set_error("null argument"); return GSW_EINVAL; }
    return dist_create(owned, n_global, nullptr, exchange, nranks, rank, kModeHost, workspace, ws_bytes, cuda_stream,
                       out);
}

gsw_status gsw_graph_create_partitioned(const gsw_csr *csr, int32_t nparts, void *workspace, size_t ws_bytes,
                                        void *cuda_stream, gsw_graph *out) {
    if (!out || !csr) { set_error("null argument"); return GSW_EINVAL; }
    return dist_create(csr, csr->n, nullptr, nullptr, nparts, 0, kModeLoopback, workspace, ws_bytes, cuda_stream, out);
}

}  // extern "C"
