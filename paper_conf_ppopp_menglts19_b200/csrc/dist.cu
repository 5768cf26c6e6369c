// dist.cu -- multi-GPU frontier step: 1D vertex partition with destination
// ownership, frontier-bitmap all-gather and feature all-reduce over NCCL (NVLink 5 / NVSwitch),
// plus a loopback mode that runs p virtual ranks on one GPU through the same partitioned kernels.
//
// BFS level t (every rank):  [host] same direction rule as the single-GPU selector on the GLOBAL
//   features -> [kernel] push: for every frontier vertex u (replicated bitmap FB_t), walk the
//   column slice u -> owned targets and claim them; pull: for every owned unvisited v, scan its row
//   (global in-neighbours) until a frontier bit is found -> each rank writes only its slice of
//   FB_{t+1} -> [NCCL] in-place AllGather of the slices (n/8 bytes) + AllReduce of (Va, Ea, edges)
//   -> [host] read the 24-byte totals (termination, next decision).
// PR iteration: owned rows pull the replicated fp64 contributions, each rank writes its slice of
//   the next contributions, AllGather + AllReduce(dangling mass) on the stream (no host sync).
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include <cub/device/device_scan.cuh>
#include <nccl.h>

#include "launch.h"

namespace gsw {

// ------------------------------------------------------------------ NCCL, loaded at run time
struct NcclApi {
    bool tried = false, ok = false;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclGetErrorString) errStr = nullptr;
};
static NcclApi g_nccl;

static bool nccl_load() {
    if (g_nccl.tried) return g_nccl.ok;
    g_nccl.tried = true;
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) {
        const char *p = getenv("GSW_NCCL_PATH");
        if (p) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) { set_error(std::string("NCCL not loadable: ") + dlerror()); return false; }
    g_nccl.getUniqueId = (decltype(g_nccl.getUniqueId))dlsym(h, "ncclGetUniqueId");
    g_nccl.commInitRank = (decltype(g_nccl.commInitRank))dlsym(h, "ncclCommInitRank");
    g_nccl.commDestroy = (decltype(g_nccl.commDestroy))dlsym(h, "ncclCommDestroy");
    g_nccl.allGather = (decltype(g_nccl.allGather))dlsym(h, "ncclAllGather");
    g_nccl.allReduce = (decltype(g_nccl.allReduce))dlsym(h, "ncclAllReduce");
    g_nccl.errStr = (decltype(g_nccl.errStr))dlsym(h, "ncclGetErrorString");
    g_nccl.ok = g_nccl.getUniqueId && g_nccl.commInitRank && g_nccl.commDestroy && g_nccl.allGather &&
                g_nccl.allReduce && g_nccl.errStr;
    if (!g_nccl.ok) set_error("NCCL symbols missing");
    return g_nccl.ok;
}

#define GSW_NCCL(call)                                                                      \
    do {                                                                                    \
        ncclResult_t _r = (call);                                                           \
        if (_r != ncclSuccess) {                                                            \
            set_error(std::string("NCCL error ") + g_nccl.errStr(_r) + " at " + #call);     \
            return GSW_ENCCL;                                                               \
        }                                                                                   \
    } while (0)

// ------------------------------------------------------------------ partition state
struct DPart {
    int64_t vb = 0;           // first owned vertex (multiple of 64)
    int nloc = 0;             // owned vertices
    uint32_t nnz = 0;         // owned adjacency entries
    uint32_t *roff = nullptr; // nloc+1, rebased to 0
    const int32_t *rcol = nullptr;   // global neighbour ids
    uint32_t *soff = nullptr; // n_global+1: global source u -> owned targets
    int32_t *scol = nullptr;  // local target ids
    unsigned *vis = nullptr;  // visited words of the owned slice (S/32)
};

struct DistState {
    int nranks = 1, rank = 0;
    bool loopback = false;
    int64_t n = 0, S = 0, npad = 0;
    std::vector<DPart> parts;
    unsigned *FB[2] = {nullptr, nullptr};   // replicated frontier bitmaps, npad/32 words
    double *contrib[2] = {nullptr, nullptr};// replicated PR contributions, npad entries
    unsigned long long *cnt = nullptr;      // per part {va, ea, edges}, then the totals
    double *dang = nullptr;                 // per part dangling mass, then the total
    ncclComm_t comm = nullptr;
};

int64_t dist_slice(int64_t n, int32_t p) {
    int64_t per = (n + p - 1) / p;
    return (per + 63) / 64 * 64;
}

// ------------------------------------------------------------------ kernels
namespace {

inline int grid_for(long long work, int sms) {
    long long b = (work + kBlock - 1) / kBlock;
    return (int)std::max(1LL, std::min(b, (long long)sms * 8));
}

__global__ void k_rebase_offsets(const int64_t *in, int64_t base, uint32_t *out, long long n1) {
    for (long long i = gtid(); i < n1; i += gthreads()) out[i] = (uint32_t)(in[i] - base);
}
__global__ void k_rebase_offsets_u32(const uint32_t *in, uint32_t base, uint32_t *out, long long n1) {
    for (long long i = gtid(); i < n1; i += gthreads()) out[i] = in[i] - base;
}
// slice CSR: count global sources
__global__ void k_slice_count(const uint32_t *roff, const int32_t *rcol, int nloc, uint32_t *cnt) {
    for (long long v = gtid(); v < nloc; v += gthreads())
        for (uint32_t e = roff[v]; e < roff[v + 1]; ++e) atomicAdd(cnt + rcol[e], 1u);
}
__global__ void k_slice_fill(const uint32_t *roff, const int32_t *rcol, int nloc, uint32_t *cursor, int32_t *scol) {
    for (long long v = gtid(); v < nloc; v += gthreads())
        for (uint32_t e = roff[v]; e < roff[v + 1]; ++e) scol[atomicAdd(cursor + rcol[e], 1u)] = (int32_t)v;
}

struct BfsPartArgs {
    const uint32_t *roff;
    const int32_t *rcol;
    const uint32_t *soff;
    const int32_t *scol;
    unsigned *vis;
    int *depth;               // owned slice
    int64_t vb;
    int nloc;
    int64_t npad;
    const unsigned *fb;       // FB_t (global)
    unsigned *nfb;            // FB_{t+1} (global; this part writes its slice)
    int lvl;
    unsigned long long *cnt;  // {va, ea, edges}
};

__device__ __forceinline__ void add_counts(unsigned long long va, unsigned long long ea, unsigned long long ed,
                                           unsigned long long *cnt) {
    va = warp_sum(va); ea = warp_sum(ea); ed = warp_sum(ed);
    if (lane_id() == 0 && (va | ed)) { atomicAdd(cnt, va); atomicAdd(cnt + 1, ea); atomicAdd(cnt + 2, ed); }
}

__global__ void k_bfs_init(BfsPartArgs a, int64_t src) {
    const int W = (a.nloc + 31) >> 5;
    for (long long v = gtid(); v < a.nloc; v += gthreads()) a.depth[v] = (a.vb + v == src) ? 0 : -1;
    for (long long w = gtid(); w < W; w += gthreads()) {
        unsigned m = 0;
        for (int b = 0; b < 32; ++b) {
            long long v = w * 32 + b;
            bool done = v >= a.nloc || a.roff[v + 1] == a.roff[v] || a.vb + v == src;
            m |= (done ? 1u : 0u) << b;
        }
        a.vis[w] = m;
    }
}

// push: warp per frontier word, lanes stride over the slice rows of its set bits
__global__ void k_bfs_push(BfsPartArgs a) {
    const long long FW = a.npad >> 5;
    unsigned long long va = 0, ea = 0, ed = 0;
    for (long long w = gwarp(); w < FW; w += gwarps()) {
        unsigned word = a.fb[w];
        while (word) {
            const int b = __ffs(word) - 1;
            word &= word - 1;
            const long long u = w * 32 + b;
            const uint32_t s0 = a.soff[u], s1 = a.soff[u + 1];
            for (uint32_t e = s0 + lane_id(); e < s1; e += 32) {
                const int v = a.scol[e];
                ed++;
                const unsigned bit = 1u << (v & 31);
                if (a.vis[v >> 5] & bit) continue;
                if (atomicOr(a.vis + (v >> 5), bit) & bit) continue;
                a.depth[v] = a.lvl + 1;
                atomicOr(a.nfb + ((a.vb + v) >> 5), bit);      // vb is a multiple of 64
                va++;
                ea += a.roff[v + 1] - a.roff[v];
            }
        }
    }
    add_counts(va, ea, ed, a.cnt);
}

// pull: warp per owned 32-vertex word, lane = vertex, early exit at the first frontier parent
__global__ void k_bfs_pull(BfsPartArgs a) {
    const int W = (a.nloc + 31) >> 5;
    unsigned long long va = 0, ea = 0, ed = 0;
    for (long long w = gwarp(); w < W; w += gwarps()) {
        const unsigned vis = a.vis[w];
        const long long v = w * 32 + lane_id();
        bool found = false;
        uint32_t deg = 0;
        if (!((vis >> lane_id()) & 1u)) {
            const uint32_t b = a.roff[v], e = a.roff[v + 1];
            deg = e - b;
            for (uint32_t k = b; k < e; ++k) {
                const int u = a.rcol[k];
                ed++;
                if ((a.fb[u >> 5] >> (u & 31)) & 1u) { found = true; break; }
            }
        }
        const unsigned hits = __ballot_sync(0xffffffffu, found);
        if (found) { a.depth[v] = a.lvl + 1; va++; ea += deg; }
        if (lane_id() == 0 && hits) {
            a.vis[w] = vis | hits;
            a.nfb[(a.vb >> 5) + w] = hits;
        }
    }
    add_counts(va, ea, ed, a.cnt);
}

__global__ void k_set_bit(unsigned *fb, int64_t v) { atomicOr(fb + (v >> 5), 1u << (v & 31)); }

__global__ void k_sum_parts(unsigned long long *cnt, int parts) {
    if (threadIdx.x < 3) {
        unsigned long long s = 0;
        for (int p = 0; p < parts; ++p) s += cnt[3 * p + threadIdx.x];
        cnt[3 * parts + threadIdx.x] = s;
    }
}

struct PrPartArgs {
    const uint32_t *roff;
    const int32_t *rcol;
    int64_t vb;
    int nloc;
    const double *cur;        // replicated contributions
    double *next;             // replicated next contributions (this part writes its slice)
    const double *dtot;       // D_t
    double *dpart;            // this part's dangling accumulator for D_{t+1}
    double *out;              // owned slice output (last iteration) or nullptr
    double base, d, invN;
};

__global__ void k_pr_init(PrPartArgs a) {
    double dang = 0.0;
    for (long long v = gtid(); v < a.nloc; v += gthreads()) {
        uint32_t dg = a.roff[v + 1] - a.roff[v];
        a.next[a.vb + v] = dg ? a.invN / dg : 0.0;
        if (!dg) dang += a.invN;
        if (a.out) a.out[v] = a.invN;
    }
    dang = warp_sum(dang);
    if (lane_id() == 0 && dang != 0.0) atomicAdd(a.dpart, dang);
}

// warp per 32 owned rows: short rows one lane each, long rows warp-cooperative
__global__ void k_pr_iter(PrPartArgs a) {
    const double D = *a.dtot;
    const double base = a.base + a.d * D * a.invN;
    double dang = 0.0;
    for (long long wb = gwarp() * 32; wb < a.nloc; wb += gwarps() * 32) {
        const long long v = wb + lane_id();
        uint32_t b = 0, e = 0;
        if (v < a.nloc) { b = a.roff[v]; e = a.roff[v + 1]; }
        double s = 0.0;
        if (e - b < 32) for (uint32_t k = b; k < e; ++k) s += a.cur[a.rcol[k]];
        unsigned longrows = __ballot_sync(0xffffffffu, v < a.nloc && e - b >= 32);
        while (longrows) {
            const int j = __ffs(longrows) - 1;
            longrows &= longrows - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), ej = __shfl_sync(0xffffffffu, e, j);
            double t = 0.0;
            for (uint32_t k = bj + lane_id(); k < ej; k += 32) t += a.cur[a.rcol[k]];
            t = warp_sum(t);
            if ((int)lane_id() == j) s = t;
        }
        if (v < a.nloc) {
            const double p = base + a.d * s;
            const uint32_t dg = e - b;
            a.next[a.vb + v] = dg ? p / dg : 0.0;
            if (!dg) dang += p;
            if (a.out) a.out[v] = p;
        }
    }
    dang = warp_sum(dang);
    if (lane_id() == 0 && dang != 0.0) atomicAdd(a.dpart, dang);
}

__global__ void k_sum_dang(double *dang, int parts) {
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int p = 0; p < parts; ++p) s += dang[p];
        dang[parts] = s;
    }
}

}  // namespace

// ------------------------------------------------------------------ workspace + creation
static size_t al(size_t x) { return (x + 255) & ~size_t(255); }

static size_t dist_bytes(int64_t n, int64_t nnz_owned_total, int32_t nranks, int32_t nparts, bool own_copy_rows) {
    const int64_t S = dist_slice(n, nranks), npad = S * nranks;
    size_t b = 0;
    b += al((size_t)npad / 8) * 2;                           // FB[2]
    b += al((size_t)npad * 8) * 2;                           // contrib[2]
    b += al(64 * 8 * (nparts + 1)) + al(8 * (nparts + 1));  // counters
    for (int p = 0; p < nparts; ++p) {
        b += al((size_t)(S + 1) * 4);                        // roff
        b += al((size_t)(n + 1) * 4);                        // soff
        b += al((size_t)S / 8);                              // vis
    }
    b += al((size_t)nnz_owned_total * 4);                    // scol (all parts)
    if (own_copy_rows) b += al((size_t)nnz_owned_total * 4); // rcol copy (NCCL mode)
    else b += al((size_t)nnz_owned_total * 4) + al((size_t)(n + 1) * 4);   // full CSR (loopback)
    size_t cub = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, cub, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)(n + 1));
    b += al(cub) + al((size_t)(n + 1) * 4);                  // scan temp + cursor
    b += al((size_t)(n + 1) * 8);                            // i64 staging
    b += al((size_t)npad * 8) * 2;                           // output staging (depth / rank)
    return b + (1 << 20);
}

static gsw_status build_slice(gsw_graph g, DPart &p, int64_t n, Workspace &tmp_ws, int32_t *scol, void *cub_tmp,
                              size_t cub_bytes, uint32_t *cursor) {
    cudaStream_t s = g->stream;
    GSW_CUDA(cudaMemsetAsync(p.soff, 0, (size_t)(n + 1) * 4, s));
    k_slice_count<<<grid_for(p.nloc, g->sms), kBlock, 0, s>>>(p.roff, p.rcol, p.nloc, p.soff);
    GSW_CUDA(cudaGetLastError());
    size_t cb = cub_bytes;
    GSW_CUDA(cub::DeviceScan::ExclusiveSum(cub_tmp, cb, p.soff, p.soff, (int)(n + 1), s));
    GSW_CUDA(cudaMemcpyAsync(cursor, p.soff, (size_t)(n + 1) * 4, cudaMemcpyDeviceToDevice, s));
    k_slice_fill<<<grid_for(p.nloc, g->sms), kBlock, 0, s>>>(p.roff, p.rcol, p.nloc, cursor, scol);
    GSW_CUDA(cudaGetLastError());
    p.scol = scol;
    (void)tmp_ws;
    return GSW_OK;
}

gsw_status dist_create(const gsw_csr *rows, int64_t n, const void *nccl_id, int32_t nranks, int32_t rank,
                       bool loopback, void *workspace, size_t ws_bytes, void *stream, gsw_graph *out) {
    *out = nullptr;
    if (!rows || !rows->row_offsets || (rows->nnz > 0 && !rows->col_indices) || n <= 0 || nranks < 1 ||
        rank < 0 || rank >= nranks) {
        set_error("dist create: bad arguments");
        return GSW_EINVAL;
    }
    if (n >= (int64_t(1) << 31) - 64 || rows->nnz >= (int64_t(1) << 32)) { set_error("graph too large"); return GSW_EOVERFLOW; }
    const int64_t S = dist_slice(n, nranks);
    const int nparts = loopback ? nranks : 1;
    if (!loopback) {
        const int64_t own = std::max<int64_t>(0, std::min<int64_t>(n, (int64_t)(rank + 1) * S) - (int64_t)rank * S);
        if (rows->n != own) { set_error("owned rows must be exactly the rank's slice (gsw_dist_slice)"); return GSW_EINVAL; }
    } else if (rows->n != n) {
        set_error("loopback mode takes the full graph");
        return GSW_EINVAL;
    }
    const size_t need = dist_bytes(n, rows->nnz, nranks, nparts, !loopback);
    if (!workspace || is_device_ptr(workspace) != 1 || ws_bytes < need) {
        set_error("dist workspace must be a device buffer of >= " + std::to_string(need) + " bytes");
        return GSW_ENOMEM;
    }
    gsw_graph g = new gsw_graph_s();
    g->stream = (cudaStream_t)stream;
    g->ws = (char *)workspace;
    g->ws_bytes = ws_bytes;
    cudaError_t e = cudaGetDevice(&g->device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g->sms, cudaDevAttrMultiProcessorCount, g->device);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev0);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev1);
    if (e != cudaSuccess) { delete g; return cuda_fail(e, "dist create setup"); }
    DistState *d = new DistState();
    g->dist = d;
    d->nranks = nranks; d->rank = rank; d->loopback = loopback;
    d->n = n; d->S = S; d->npad = S * nranks;
    g->g.n = (int)n;
    g->g.nnz = (uint32_t)rows->nnz;
    Workspace ws{g->ws, ws_bytes, 0};
    d->FB[0] = (unsigned *)ws.take(d->npad / 8);
    d->FB[1] = (unsigned *)ws.take(d->npad / 8);
    d->contrib[0] = (double *)ws.take(d->npad * 8);
    d->contrib[1] = (double *)ws.take(d->npad * 8);
    d->cnt = (unsigned long long *)ws.take(64 * 8 * (nparts + 1));
    d->dang = (double *)ws.take(8 * (nparts + 1));
    int64_t *staging = (int64_t *)ws.take((size_t)(n + 1) * 8);
    size_t cub_bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, cub_bytes, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)(n + 1));
    void *cub_tmp = ws.take(cub_bytes);
    uint32_t *cursor = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    int32_t *scol_all = (int32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4);
    cudaStream_t s = g->stream;
    auto fail = [&](gsw_status st) { gsw_graph_destroy(g); return st; };
    // adjacency on the device
    const int64_t *off64 = rows->row_offsets;
    if (!is_device_ptr(off64)) {
        if (cudaMemcpyAsync(staging, off64, (size_t)(rows->n + 1) * 8, cudaMemcpyHostToDevice, s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "copy offsets"));
        off64 = staging;
    }
    int32_t *col = (int32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4);
    uint32_t *full_off = loopback ? (uint32_t *)ws.take((size_t)(n + 1) * 4) : nullptr;
    if (!d->FB[1] || !d->contrib[1] || !d->cnt || !d->dang || !staging || !cub_tmp || !cursor || !scol_all || !col ||
        (loopback && !full_off)) {
        set_error("dist workspace too small");
        return fail(GSW_ENOMEM);
    }
    if (rows->nnz > 0 && cudaMemcpyAsync(col, rows->col_indices, (size_t)rows->nnz * 4,
                                         is_device_ptr(rows->col_indices) ? cudaMemcpyDeviceToDevice
                                                                          : cudaMemcpyHostToDevice, s) != cudaSuccess)
        return fail(cuda_fail(cudaGetLastError(), "copy columns"));
    if (loopback) {
        k_rebase_offsets<<<grid_for(n + 1, g->sms), kBlock, 0, s>>>(off64, 0, full_off, n + 1);
    }
    // partitions
    std::vector<int64_t> hoff;
    if (loopback) {
        hoff.resize(n + 1);
        if (cudaMemcpyAsync(hoff.data(), off64, (size_t)(n + 1) * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "read offsets"));
    }
    int32_t *scol_cur = scol_all;
    for (int p = 0; p < nparts; ++p) {
        DPart P;
        const int r = loopback ? p : rank;
        P.vb = (int64_t)r * S;
        P.nloc = (int)std::max<int64_t>(0, std::min<int64_t>(n, P.vb + S) - P.vb);
        P.roff = (uint32_t *)ws.take((size_t)(S + 1) * 4);
        P.soff = (uint32_t *)ws.take((size_t)(n + 1) * 4);
        P.vis = (unsigned *)ws.take((size_t)S / 8);
        if (!P.roff || !P.soff || !P.vis) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
        if (loopback) {
            const int64_t e0 = P.nloc ? hoff[P.vb] : 0, e1 = P.nloc ? hoff[P.vb + P.nloc] : 0;
            P.nnz = (uint32_t)(e1 - e0);
            P.rcol = col + e0;
            if (P.nloc) k_rebase_offsets_u32<<<grid_for(P.nloc + 1, g->sms), kBlock, 0, s>>>(full_off + P.vb, (uint32_t)e0,
                                                                                             P.roff, P.nloc + 1);
        } else {
            P.nnz = (uint32_t)rows->nnz;
            P.rcol = col;
            k_rebase_offsets<<<grid_for(P.nloc + 1, g->sms), kBlock, 0, s>>>(off64, 0, P.roff, P.nloc + 1);
        }
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "rebase"));
        Workspace none{nullptr, 0, 0};
        gsw_status st = build_slice(g, P, n, none, scol_cur, cub_tmp, cub_bytes, cursor);
        if (st != GSW_OK) return fail(st);
        scol_cur += P.nnz;
        d->parts.push_back(P);
    }
    // output staging lives after the partitions
    g->scratch = (char *)ws.take((size_t)d->npad * 8 * 2);
    g->scratch_bytes = (size_t)d->npad * 8 * 2;
    if (!g->scratch) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "dist create"));
    if (!loopback && nranks > 1) {
        if (!nccl_load()) return fail(GSW_ENCCL);
        ncclUniqueId id;
        std::memcpy(&id, nccl_id, sizeof(id));
        ncclResult_t r = g_nccl.commInitRank(&d->comm, nranks, id, rank);
        if (r != ncclSuccess) { set_error(std::string("ncclCommInitRank: ") + g_nccl.errStr(r)); return fail(GSW_ENCCL); }
    }
    *out = g;
    return GSW_OK;
}

void dist_destroy(DistState *d) {
    if (!d) return;
    if (d->comm && g_nccl.ok) g_nccl.commDestroy(d->comm);
    delete d;
}

// ------------------------------------------------------------------ exchange
static gsw_status allgather_u32(DistState *d, unsigned *buf, size_t words_per_rank, cudaStream_t s) {
    if (d->loopback || d->nranks == 1) return GSW_OK;                 // shared replica / single rank
    GSW_NCCL(g_nccl.allGather(buf + (size_t)d->rank * words_per_rank, buf, words_per_rank, ncclUint32, d->comm, s));
    return GSW_OK;
}
static gsw_status allgather_f64(DistState *d, double *buf, size_t per_rank, cudaStream_t s) {
    if (d->loopback || d->nranks == 1) return GSW_OK;
    GSW_NCCL(g_nccl.allGather(buf + (size_t)d->rank * per_rank, buf, per_rank, ncclFloat64, d->comm, s));
    return GSW_OK;
}
static gsw_status reduce_counts(DistState *d, cudaStream_t s) {
    const int parts = (int)d->parts.size();
    k_sum_parts<<<1, 32, 0, s>>>(d->cnt, parts);
    GSW_CUDA(cudaGetLastError());
    if (!d->loopback && d->nranks > 1)
        GSW_NCCL(g_nccl.allReduce(d->cnt + 3 * parts, d->cnt + 3 * parts, 3, ncclUint64, ncclSum, d->comm, s));
    return GSW_OK;
}
static gsw_status reduce_dang(DistState *d, cudaStream_t s) {
    const int parts = (int)d->parts.size();
    k_sum_dang<<<1, 32, 0, s>>>(d->dang, parts);
    GSW_CUDA(cudaGetLastError());
    if (!d->loopback && d->nranks > 1)
        GSW_NCCL(g_nccl.allReduce(d->dang + parts, d->dang + parts, 1, ncclFloat64, ncclSum, d->comm, s));
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed BFS
gsw_status dist_bfs(gsw_graph g, int32_t source, int32_t *depth_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (source < 0 || source >= d->n) { set_error("gsw_bfs: source out of range"); return GSW_EINVAL; }
    if (!depth_out) { set_error("gsw_bfs: depth is NULL"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->loopback ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(depth_out) == 1;
    int *depth = dev_out ? depth_out : (int *)g->scratch;
    const size_t FBW = (size_t)d->npad / 32;
    std::vector<gsw_iter_record> recs;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemsetAsync(d->FB[0], 0, FBW * 4, s));
    std::vector<BfsPartArgs> pa(parts);
    for (int p = 0; p < parts; ++p) {
        const DPart &P = d->parts[p];
        pa[p] = BfsPartArgs{P.roff, P.rcol, P.soff, P.scol, P.vis, depth + (d->loopback ? P.vb : 0), P.vb, P.nloc,
                            d->npad, nullptr, nullptr, 0, d->cnt + 3 * p};
        if (P.nloc) k_bfs_init<<<grid_for(P.nloc, g->sms), kBlock, 0, s>>>(pa[p], source);
    }
    k_set_bit<<<1, 1, 0, s>>>(d->FB[0], source);
    GSW_CUDA(cudaGetLastError());
    // global features of level 0: Va = 1, Ea = deg(source)
    unsigned long long tot[3] = {1, 0, 0};
    {
        // degree of the source: row length in the owning partition (host read of two offsets)
        const int owner = d->loopback ? (int)(source / d->S) : -1;
        unsigned long long dsrc = 0;
        if (d->loopback || source / d->S == d->rank) {
            const DPart &P = d->parts[d->loopback ? owner : 0];
            uint32_t o[2];
            GSW_CUDA(cudaMemcpyAsync(o, P.roff + (source - P.vb), 8, cudaMemcpyDeviceToHost, s));
            GSW_CUDA(cudaStreamSynchronize(s));
            dsrc = o[1] - o[0];
        }
        GSW_CUDA(cudaMemsetAsync(d->cnt, 0, 8 * 3 * (parts + 1), s));
        GSW_CUDA(cudaMemcpyAsync(d->cnt + 1, &dsrc, 8, cudaMemcpyHostToDevice, s));
        gsw_status r = reduce_counts(d, s);
        if (r != GSW_OK) return r;
        GSW_CUDA(cudaMemcpyAsync(tot, d->cnt + 3 * parts, 24, cudaMemcpyDeviceToHost, s));
        GSW_CUDA(cudaStreamSynchronize(s));
        tot[0] = 1;
    }
    long long Via = d->n - 1, Eia = (long long)g->g.nnz;   // per rank nnz is local: use the global sum below
    {
        // global nnz = sum of owned nnz over ranks
        unsigned long long loc = 0;
        for (auto &P : d->parts) loc += P.nnz;
        GSW_CUDA(cudaMemsetAsync(d->cnt, 0, 8 * 3 * (parts + 1), s));
        GSW_CUDA(cudaMemcpyAsync(d->cnt, &loc, 8, cudaMemcpyHostToDevice, s));
        gsw_status r = reduce_counts(d, s);
        if (r != GSW_OK) return r;
        unsigned long long gn[3];
        GSW_CUDA(cudaMemcpyAsync(gn, d->cnt + 3 * parts, 24, cudaMemcpyDeviceToHost, s));
        GSW_CUDA(cudaStreamSynchronize(s));
        Eia = (long long)gn[0] - (long long)tot[1];
    }
    unsigned long long edges_total = 0, bytes = 0;
    int t = 0;
    for (;; ++t) {
        const long long Va = (long long)tot[0], Ea = (long long)tot[1];
        if (Va == 0) break;
        if (t > 0) { Via -= Va; Eia -= Ea; }
        // same direction split as the single-GPU selector (select.cuh, R6)
        int dir = ((double)Ea * 16.0 > (double)Eia && (double)Va * 2048.0 > (double)d->n) ? GSW_PULL : GSW_PUSH;
        if (g->forced.direction != GSW_AUTO) dir = g->forced.direction;
        unsigned *fb = d->FB[t & 1], *nfb = d->FB[(t + 1) & 1];
        GSW_CUDA(cudaMemsetAsync(nfb, 0, FBW * 4, s));
        GSW_CUDA(cudaMemsetAsync(d->cnt, 0, 8 * 3 * (parts + 1), s));
        for (int p = 0; p < parts; ++p) {
            BfsPartArgs a = pa[p];
            a.fb = fb; a.nfb = nfb; a.lvl = t;
            if (!a.nloc) continue;
            if (dir == GSW_PUSH) k_bfs_push<<<g->sms * 8, kBlock, 0, s>>>(a);
            else k_bfs_pull<<<g->sms * 8, kBlock, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        gsw_status r = allgather_u32(d, nfb, (size_t)d->S / 32, s);
        if (r != GSW_OK) return r;
        r = reduce_counts(d, s);
        if (r != GSW_OK) return r;
        gsw_iter_record rec{};
        rec.iteration = t; rec.direction = dir; rec.format = GSW_BITMAP;
        rec.load_balance = dir == GSW_PULL ? GSW_LB_THREAD : GSW_LB_WM; rec.fusion = GSW_FUSED;
        rec.Va = Va; rec.Ea = Ea; rec.Via = Via; rec.Eia = Eia;
        GSW_CUDA(cudaMemcpyAsync(tot, d->cnt + 3 * parts, 24, cudaMemcpyDeviceToHost, s));
        GSW_CUDA(cudaStreamSynchronize(s));
        rec.edges = (long long)tot[2];
        edges_total += tot[2];
        bytes += dir == GSW_PUSH ? 12ull * Va + 4ull * tot[2] + 8ull * tot[0]
                                 : (unsigned long long)d->n / 4 + 4ull * tot[2] + 4ull * tot[0] + 8ull * Via;
        recs.push_back(rec);
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(depth_out, depth, (size_t)out_len * 4, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = t;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)edges_total;
        st->bytes_alg = (int64_t)bytes;
        if (st->records && st->max_records > 0)
            std::memcpy(st->records, recs.data(), sizeof(gsw_iter_record) * std::min<size_t>(recs.size(), st->max_records));
    }
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed PageRank
gsw_status dist_pr(gsw_graph g, double damping, int32_t iters, double *rank_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (!rank_out || iters < 0 || !(damping >= 0.0 && damping <= 1.0)) { set_error("gsw_pr: bad arguments"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->loopback ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(rank_out) == 1;
    double *out = dev_out ? rank_out : (double *)g->scratch;
    const double invN = 1.0 / (double)d->n;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemsetAsync(d->dang, 0, 8 * (parts + 1), s));
    GSW_CUDA(cudaMemsetAsync(d->contrib[0], 0, (size_t)d->npad * 8, s));
    for (int p = 0; p < parts; ++p) {
        const DPart &P = d->parts[p];
        PrPartArgs a{P.roff, P.rcol, P.vb, P.nloc, nullptr, d->contrib[0], nullptr, d->dang + p,
                     iters == 0 ? out + (d->loopback ? P.vb : 0) : nullptr, 0.0, damping, invN};
        if (P.nloc) k_pr_init<<<grid_for(P.nloc, g->sms), kBlock, 0, s>>>(a);
    }
    GSW_CUDA(cudaGetLastError());
    gsw_status r = allgather_f64(d, d->contrib[0], (size_t)d->S, s);
    if (r != GSW_OK) return r;
    r = reduce_dang(d, s);
    if (r != GSW_OK) return r;
    unsigned long long nnz_loc = 0;
    for (auto &P : d->parts) nnz_loc += P.nnz;
    for (int t = 0; t < iters; ++t) {
        const double *cur = d->contrib[t & 1];
        double *next = d->contrib[(t + 1) & 1];
        // D_t sits at dang[parts]; the per-part accumulators are reused for D_{t+1}
        GSW_CUDA(cudaMemsetAsync(d->dang, 0, 8 * parts, s));
        for (int p = 0; p < parts; ++p) {
            const DPart &P = d->parts[p];
            PrPartArgs a{P.roff, P.rcol, P.vb, P.nloc, cur, next, d->dang + parts, d->dang + p,
                         t == iters - 1 ? out + (d->loopback ? P.vb : 0) : nullptr, (1.0 - damping) * invN, damping, invN};
            // dtot is read before the per-part accumulators are summed into it by reduce_dang below
            if (P.nloc) k_pr_iter<<<g->sms * 8, kBlock, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        r = allgather_f64(d, next, (size_t)d->S, s);
        if (r != GSW_OK) return r;
        r = reduce_dang(d, s);
        if (r != GSW_OK) return r;
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank_out, out, (size_t)out_len * 8, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = iters;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)nnz_loc * iters;
        st->bytes_alg = (int64_t)((4ull * nnz_loc + 20ull * (unsigned long long)out_len) * iters);
    }
    return GSW_OK;
}

size_t dist_workspace(int64_t n, int64_t nnz, int32_t nranks, int32_t nparts, bool own_copy) {
    return dist_bytes(n, nnz, nranks, nparts, own_copy);
}

gsw_status dist_unique_id(void *id128) {
    if (!id128) { set_error("null id"); return GSW_EINVAL; }
    if (!nccl_load()) return GSW_ENCCL;
    ncclUniqueId id;
    GSW_NCCL(g_nccl.getUniqueId(&id));
    std::memcpy(id128, &id, sizeof(id));
    return GSW_OK;
}

}  // namespace gsw
