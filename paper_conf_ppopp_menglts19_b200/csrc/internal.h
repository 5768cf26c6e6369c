// internal.h -- host-side internals of libgsw (graph handle, workspace carving, error plumbing).
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>
#include <cuda_runtime.h>

#include "gsw.h"

namespace gsw {

// Device view of the graph: u32 offsets (nnz < 2^32), int32 columns, optional u32 weights.
// For symmetric inputs the CSC fields alias the CSR (all graphs undirected).
struct DevGraph {
    int n;
    uint32_t nnz;
    const uint32_t *off;      // n+1  (out-edges, push)
    const int32_t *col;       // nnz
    const uint32_t *w;        // nnz or nullptr
    const uint32_t *in_off;   // n+1  (in-edges, pull)
    const int32_t *in_col;
    const uint32_t *in_w;
    // in_first[v] = in_col[in_off[v]] (-1 for empty rows): the first in-neighbour, i.e. the
    // highest-degree one after relabeling, read coalesced by the pull's first probe (graph.cu)
    const int32_t *in_first;
    // degree-ordered relabeling (graph.cu): internal id i is caller id perm[i]; inv[caller] = i.
    // nullptr when the graph is kept in caller order.
    const uint32_t *perm;
    const uint32_t *inv;
};

// Dataset attributes (Table 1), computed once at load.
struct Attrs {
    double N, M, dbar, sd, rd, gini, her;
    uint32_t maxdeg, mindeg, maxw;
    int64_t isolated;
    double wbar;              // mean edge weight (SSSP static step c*wbar/dbar)
};

// Packed per-iteration configuration (Fig. 13: one choice per pattern).
struct Cfg {
    int8_t dir, fmt, lb, step, fused;
};

struct Workspace {
    char *base = nullptr;
    size_t size = 0, used = 0;
    void *take(size_t bytes) {
        size_t a = (used + 255) & ~size_t(255);
        if (a + bytes > size) return nullptr;
        used = a + bytes;
        return base + a;
    }
};

}  // namespace gsw

namespace gsw {
struct DistState;
}

struct gsw_graph_s {
    gsw::DistState *dist = nullptr;   // multi-GPU / partitioned handle (dist.cu), else nullptr
    gsw::DevGraph g{};
    gsw::Attrs attrs{};
    bool symmetric = true;
    cudaStream_t stream = nullptr;
    int device = 0, sms = 0;
    gsw_config forced{};
    unsigned *iso = nullptr;      // isolated-vertex bitmap (no in-edges, or padding), W words
    unsigned *iso_caller = nullptr;  // the same bits in caller order (relabeled graphs), W words
    void *ctl = nullptr;          // the persistent kernels' control block (grid barrier word,
                                  // run totals), zeroed once at create: runs need no reset
                                  // (the flip-bit barrier works from any counter value)
    // workspace regions
    char *ws = nullptr;
    size_t ws_bytes = 0;
    char *scratch = nullptr;      // per-run scratch (after the graph copy)
    size_t scratch_bytes = 0;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    unsigned long long *poll = nullptr;   // 2 pinned host slots for gsw_dpr's termination poll (lazy)
};

namespace gsw {

void set_error(const std::string &msg);
gsw_status cuda_fail(cudaError_t e, const char *what);

#define GSW_CUDA(call)                                                   \
    do {                                                                 \
        cudaError_t _e = (call);                                         \
        if (_e != cudaSuccess) return ::gsw::cuda_fail(_e, #call);       \
    } while (0)

constexpr int kDprMaxIters = 1 << 16;   // gsw_dpr: per-iteration records held in the scratch

// scratch bytes for a graph of n vertices (max over algorithms), see DESIGN.md "HBM layout"
size_t scratch_bytes_for(int64_t n, int64_t nnz, int has_w);

// 1 if p is device (or managed) memory, 0 if host, -1 on error
int is_device_ptr(const void *p);

// records copy-out helper
struct RunRecords;

}  // namespace gsw
