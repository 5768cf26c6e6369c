// graph.cu -- step a0 of the hot path: ingest + dataset attributes (Table 1; "computed
// only once while loading the data into the memory").  Not inside any timed run.
#include <cstdlib>
#include <cmath>
#include <cstring>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>

#include "common.cuh"
#include "internal.h"

namespace gsw {

namespace {

__global__ void k_offsets_to_u32(const int64_t *in, uint32_t *out, long long n1) {
    for (long long i = gtid(); i < n1; i += gthreads()) out[i] = (uint32_t)in[i];
}

// caller-order copy of the isolated bitmap: bit j = isolated(inv[j]) (padding bits set)
__global__ void k_iso_caller(const uint32_t *inv, const unsigned *iso, int n, unsigned *isoc, int W) {
    for (long long w = gwarp(); w < W; w += gwarps()) {
        const int j = (int)(w * 32 + lane_id());
        bool b = true;
        if (j < n) { const uint32_t v = inv[j]; b = (iso[v >> 5] >> (v & 31)) & 1u; }
        const unsigned m = __ballot_sync(0xffffffffu, b);
        if (lane_id() == 0) isoc[w] = m;
    }
}
// isolated bitmap: bit v = 1 if deg(v) == 0 or v >= n (padding bits)
__global__ void k_isolated_bitmap(const uint32_t *off, int n, unsigned *iso, int W) {
    for (long long w = gwarp(); w < W; w += gwarps()) {
        int v = (int)(w * 32 + lane_id());
        bool b = v >= n || off[v + 1] == off[v];
        unsigned m = __ballot_sync(0xffffffffu, b);
        if (lane_id() == 0) iso[w] = m;
    }
}

struct AttrAcc {
    unsigned long long sum, iso, wsum;
    double sumsq, dlnd;
    unsigned maxd, mind, maxw, bad;
};

__global__ void k_attrs(const uint32_t *off, int n, AttrAcc *acc) {
    __shared__ double sd[kWarps];
    __shared__ unsigned long long su[kWarps];
    unsigned long long s = 0, iso = 0;
    double sq = 0, dl = 0;
    unsigned mx = 0, mn = 0xffffffffu;
    for (long long v = gtid(); v < n; v += gthreads()) {
        unsigned d = off[v + 1] - off[v];
        s += d; sq += (double)d * d;
        if (d) dl += (double)d * log((double)d); else iso++;
        mx = max(mx, d); mn = min(mn, d);
    }
    s = block_sum(s, su);
    iso = block_sum(iso, su);
    sq = block_sum(sq, sd);
    dl = block_sum(dl, sd);
    __shared__ unsigned smx[kWarps], smn[kWarps];
    mx = warp_max(mx); mn = warp_min(mn);
    if (lane_id() == 0) { smx[threadIdx.x >> 5] = mx; smn[threadIdx.x >> 5] = mn; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < kWarps; ++i) { mx = max(mx, smx[i]); mn = min(mn, smn[i]); }
        atomicAdd(&acc->sum, s); atomicAdd(&acc->iso, iso);
        atomicAdd(&acc->sumsq, sq); atomicAdd(&acc->dlnd, dl);
        atomicMax(&acc->maxd, mx); atomicMin(&acc->mind, mn);
    }
}

// degree histogram: small degrees (the hot bins of power-law graphs) are counted in a per-CTA
// shared-memory histogram and merged once; large degrees go straight to global atomics
constexpr int kHistSmem = 2048;
__global__ void k_degree_hist(const uint32_t *off, int n, unsigned long long *hist, unsigned nbins) {
    __shared__ unsigned sh[kHistSmem];
    for (int i = threadIdx.x; i < kHistSmem; i += blockDim.x) sh[i] = 0u;
    __syncthreads();
    for (long long v = gtid(); v < n; v += gthreads()) {
        const unsigned d = off[v + 1] - off[v];
        if (d < (unsigned)kHistSmem) atomicAdd(&sh[d], 1u);
        else atomicAdd(&hist[d], 1ull);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kHistSmem && i < (int)nbins; i += blockDim.x)
        if (sh[i]) atomicAdd(&hist[i], (unsigned long long)sh[i]);
}

__global__ void k_maxw(const uint32_t *w, long long nnz, AttrAcc *acc) {
    unsigned mx = 0;
    unsigned long long s = 0;
    for (long long e = gtid(); e < nnz; e += gthreads()) { mx = max(mx, w[e]); s += w[e]; }
    mx = warp_max(mx);
    s = warp_sum(s);
    if (lane_id() == 0) { atomicMax(&acc->maxw, mx); atomicAdd(&acc->wsum, s); }
}

__global__ void k_validate(const uint32_t *off, const int32_t *col, int n, long long nnz, unsigned *bad) {
    for (long long v = gtid(); v < n; v += gthreads())
        if (off[v + 1] < off[v]) atomicOr(bad, 1u);
    for (long long e = gtid(); e < nnz; e += gthreads())
        if (col[e] < 0 || col[e] >= n) atomicOr(bad, 2u);
}

__global__ void k_first_nbr(const uint32_t *off, const int32_t *col, int n, int32_t *first) {
    for (long long v = gtid(); v < n; v += gthreads()) {
        const uint32_t b = off[v];
        first[v] = off[v + 1] > b ? col[b] : -1;
    }
}
// ---- degree-ordered relabeling
__global__ void k_deg_iota(const uint32_t *off, int n, uint32_t *deg, uint32_t *ids) {
    for (long long v = gtid(); v < n; v += gthreads()) { deg[v] = off[v + 1] - off[v]; ids[v] = (uint32_t)v; }
}
__global__ void k_invert(const uint32_t *perm, int n, uint32_t *inv) {
    for (long long i = gtid(); i < n; i += gthreads()) inv[perm[i]] = (uint32_t)i;
}
// new row i = old row perm[i], columns renamed through inv; one warp per row
// rows in the new order, columns renamed, as 64-bit keys (new row << 32 | new column): one
// device-wide radix sort of the keys then yields every row sorted (stable, ties keep weights)
__global__ void k_permute_rows_keys(const uint32_t *noff, const uint32_t *off, const int32_t *col, const uint32_t *w,
                                    const uint32_t *perm, const uint32_t *inv, int n, unsigned long long *keys,
                                    uint32_t *nw) {
    for (long long i = gwarp(); i < n; i += gwarps()) {
        const uint32_t o = perm[i];
        const uint32_t b = off[o], e = off[o + 1], nb = noff[i];
        const unsigned long long hi = (unsigned long long)i << 32;
        for (uint32_t k = b + lane_id(); k < e; k += 32) {
            keys[nb + (k - b)] = hi | inv[col[k]];
            if (w) nw[nb + (k - b)] = w[k];
        }
    }
}
// symmetric unweighted fast path (relabel_csr): (new column, new row) pairs in new-row order;
// rows of kRelabelHeavy+ edges are skipped here and written by k_permute_heavy (a warp walking a
// 163K-edge hub row serially was most of this pass)
constexpr uint32_t kRelabelHeavy = 8192;
__global__ void k_permute_rows_pairs(const uint32_t *noff, const uint32_t *off, const int32_t *col, const uint32_t *perm,
                                     const uint32_t *inv, int n, uint32_t *keys, uint32_t *vals, uint32_t *heavy,
                                     unsigned *nheavy) {
    for (long long i = gwarp(); i < n; i += gwarps()) {
        const uint32_t o = perm[i];
        const uint32_t b = off[o], e = off[o + 1], nb = noff[i];
        if (e - b >= kRelabelHeavy) {
            if (lane_id() == 0) heavy[atomicAdd(nheavy, 1u)] = (uint32_t)i;
            continue;
        }
        for (uint32_t k = b + lane_id(); k < e; k += 32) {
            keys[nb + (k - b)] = inv[col[k]];
            vals[nb + (k - b)] = (uint32_t)i;
        }
    }
}
__global__ void k_permute_heavy(const uint32_t *noff, const uint32_t *off, const int32_t *col, const uint32_t *perm,
                                const uint32_t *inv, uint32_t *keys, uint32_t *vals, const uint32_t *heavy,
                                const unsigned *nheavy) {
    const unsigned nh = *nheavy;
    for (unsigned h = blockIdx.x; h < nh; h += gridDim.x) {
        const uint32_t i = heavy[h], o = perm[i];
        const uint32_t b = off[o], e = off[o + 1], nb = noff[i];
        for (uint32_t k = b + threadIdx.x; k < e; k += blockDim.x) {
            keys[nb + (k - b)] = inv[col[k]];
            vals[nb + (k - b)] = i;
        }
    }
}
__global__ void k_key_cols(const unsigned long long *keys, long long m, int32_t *col) {
    for (long long k = gtid(); k < m; k += gthreads()) col[k] = (int32_t)(uint32_t)keys[k];
}
__global__ void k_set_u32(uint32_t *p, uint32_t v) { *p = v; }
__global__ void k_perm_deg(const uint32_t *off, const uint32_t *perm, int n, uint32_t *degp) {
    for (long long i = gtid(); i < n; i += gthreads()) { const uint32_t o = perm[i]; degp[i] = off[o + 1] - off[o]; }
}

inline int grid_for(long long work, int sms) {
    long long b = (work + kBlock - 1) / kBlock;
    long long cap = (long long)sms * 8;
    return (int)std::max(1LL, std::min(b, cap));
}

}  // namespace

size_t graph_bytes(int64_t n, int64_t nnz, int has_w, int has_csc) {
    size_t W = (size_t)((n + 31) / 32);
    size_t b = 0;
    auto add = [&](size_t x) { b += (x + 255) & ~size_t(255); };
    add((n + 1) * 4); add(nnz * 4); if (has_w) add(nnz * 4);
    if (has_csc) { add((n + 1) * 4); add(nnz * 4); if (has_w) add(nnz * 4); }
    add(W * 4);  // isolated bitmap
    add(n * 4); add(n * 4);  // relabeling: perm, inv
    add(n * 4);              // first in-neighbour
    add(W * 4);              // isolated bitmap in caller order
    add(1024);               // persistent-kernel control block
    return b;
}

// Per-run scratch: the maximum over algorithms.
size_t relabel_temp_bytes(int64_t n, int64_t nnz, int has_w);
size_t scratch_bytes_for(int64_t n, int64_t nnz, int has_w) {
    size_t W = (size_t)((n + 31) / 32);
    size_t per_v = 64;                         // BC: depth 4 + sigma 8 + delta 8 + stack 4 + bc 8 + queues
    size_t b = per_v * (size_t)(n + 64) + 16 * W * 4;
    b += (size_t)(n + 1) * 8;                  // i64 offset staging at ingest / scan arrays
    b += 16u << 20;                            // control blocks, per-CTA partials, history, records (x2: gsw_cc's
                                               // label-propagation run and the hooking run it hands over to)
    // gsw_dpr: two heavy-row chunk tables (<= nnz/128 + 1 entries of 12 B, dpr.cu k_dpr_chunks)
    // and kDprMaxIters per-iteration records (queue length 4 B + counters 32 B)
    b += 2 * ((size_t)nnz / 128 + 1) * 12 + 1024 + (size_t)kDprMaxIters * 36;
    if (nnz < (int64_t(1) << 31)) b = std::max(b, relabel_temp_bytes(n, nnz, has_w));   // ingest temp
    return b;
}

int is_device_ptr(const void *p) {
    if (!p) return 0;
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) { cudaGetLastError(); return 0; }
    return (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) ? 1 : 0;
}

static gsw_status copy_in(void *dst, const void *src, size_t bytes, cudaStream_t s) {
    if (bytes == 0) return GSW_OK;
    cudaMemcpyKind k = is_device_ptr(src) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    GSW_CUDA(cudaMemcpyAsync(dst, src, bytes, k, s));
    return GSW_OK;
}

gsw_status load_csr(gsw_graph g, const gsw_csr *c, Workspace &ws, uint32_t **off, int32_t **col,
                    uint32_t **w, int64_t *staging) {
    int64_t n = c->n, nnz = c->nnz;
    *off = (uint32_t *)ws.take((n + 1) * 4);
    *col = (int32_t *)ws.take(std::max<int64_t>(nnz, 1) * 4);
    *w = nullptr;
    if (c->weights) *w = (uint32_t *)ws.take(std::max<int64_t>(nnz, 1) * 4);
    if (!*off || !*col || (c->weights && !*w)) { set_error("workspace too small for the graph"); return GSW_ENOMEM; }
    gsw_status st;
    const int64_t *off64 = c->row_offsets;
    if (!is_device_ptr(off64)) {
        if ((st = copy_in(staging, off64, (n + 1) * 8, g->stream)) != GSW_OK) return st;
        off64 = staging;
    }
    k_offsets_to_u32<<<grid_for(n + 1, g->sms), kBlock, 0, g->stream>>>(off64, *off, n + 1);
    GSW_CUDA(cudaGetLastError());
    if ((st = copy_in(*col, c->col_indices, nnz * 4, g->stream)) != GSW_OK) return st;
    if (c->weights && (st = copy_in(*w, c->weights, nnz * 4, g->stream)) != GSW_OK) return st;
    return GSW_OK;
}

gsw_status compute_attrs(gsw_graph g, unsigned *iso_bitmap, void *tmp) {
    const DevGraph &G = g->g;
    int n = G.n;
    int W = (n + 31) / 32;
    // "isolated" for the traversals = no in-edges (never discovered; pre-marked visited); for the
    // symmetric inputs of every config that is degree 0 (Table 1's isolated count, k_attrs)
    k_isolated_bitmap<<<grid_for((long long)W * 32, g->sms), kBlock, 0, g->stream>>>(G.in_off, n, iso_bitmap, W);
    if (G.inv && g->iso_caller)
        k_iso_caller<<<grid_for((long long)W * 32, g->sms), kBlock, 0, g->stream>>>(G.inv, iso_bitmap, n, g->iso_caller, W);
    AttrAcc *acc = (AttrAcc *)tmp;
    AttrAcc init{};
    init.mind = 0xffffffffu;
    GSW_CUDA(cudaMemcpyAsync(acc, &init, sizeof(init), cudaMemcpyHostToDevice, g->stream));
    k_attrs<<<grid_for(n, g->sms), kBlock, 0, g->stream>>>(G.off, n, acc);
    if (G.w) k_maxw<<<grid_for(G.nnz, g->sms), kBlock, 0, g->stream>>>(G.w, G.nnz, acc);
    GSW_CUDA(cudaGetLastError());
    AttrAcc h;
    GSW_CUDA(cudaMemcpyAsync(&h, acc, sizeof(h), cudaMemcpyDeviceToHost, g->stream));
    GSW_CUDA(cudaStreamSynchronize(g->stream));
    // degree histogram -> Gini over ascending degrees (counting sort order)
    size_t nb = (size_t)h.maxd + 1;
    unsigned long long *hist = (unsigned long long *)((char *)tmp + 256);
    GSW_CUDA(cudaMemsetAsync(hist, 0, nb * 8, g->stream));
    k_degree_hist<<<grid_for(n, g->sms), kBlock, 0, g->stream>>>(G.off, n, hist, (unsigned)nb);
    GSW_CUDA(cudaGetLastError());
    std::vector<unsigned long long> hh(nb);
    GSW_CUDA(cudaMemcpyAsync(hh.data(), hist, nb * 8, cudaMemcpyDeviceToHost, g->stream));
    GSW_CUDA(cudaStreamSynchronize(g->stream));
    double N = n, S = (double)h.sum, dbar = S / N;
    double gnum = 0.0, r = 0.0;                 // sum_i (2i - N - 1) d_(i), ranks r+1..r+c
    for (size_t k = 0; k < nb; ++k) {
        double c = (double)hh[k];
        if (c == 0) continue;
        gnum += (double)k * (c * (2.0 * r + c + 1.0) - c * (N + 1.0));
        r += c;
    }
    Attrs &A = g->attrs;
    A.N = N;
    A.M = S / 2.0;
    A.dbar = dbar;
    double var = h.sumsq / N - dbar * dbar;
    A.sd = std::sqrt(std::max(0.0, var));
    A.rd = dbar > 0 ? (double)(h.maxd - h.mind) / dbar : 0.0;
    A.gini = S > 0 ? gnum / (N * S) : 0.0;
    // H_er = -sum (d/S) ln(d/S) / ln N = (ln S - (1/S) sum d ln d) / ln N
    A.her = (S > 0 && n > 1) ? (std::log(S) - h.dlnd / S) / std::log(N) : 0.0;
    A.maxdeg = h.maxd;
    A.mindeg = h.mind;
    A.maxw = h.maxw;
    A.wbar = G.nnz ? (double)h.wsum / (double)G.nnz : 0.0;
    A.isolated = (int64_t)h.iso;
    return GSW_OK;
}

// ---------------------------------------------------------------- degree-ordered relabeling
// Internal vertex ids are assigned by descending degree (stable: ties keep caller order) and every
// row is sorted ascending in the new ids.  Hubs then share a few cache lines in every per-vertex
// array (frontier bits, labels, PR contributions) and come first in each adjacency row, which
// helps the early-exit pull.  Outputs are gathered back to caller ids by each kernel.
static size_t al256(size_t x) { return (x + 255) & ~size_t(255); }

static int key_end_bit(int64_t n) {
    int b = 1;
    while ((int64_t(1) << b) < n) ++b;
    return 32 + b;
}

size_t relabel_temp_bytes(int64_t n, int64_t nnz, int has_w) {
    size_t t1 = 0, t2 = 0, t3 = 0;
    cub::DeviceRadixSort::SortPairsDescending(nullptr, t1, (uint32_t *)nullptr, (uint32_t *)nullptr,
                                              (uint32_t *)nullptr, (uint32_t *)nullptr, (int)n);
    cub::DeviceScan::InclusiveSum(nullptr, t2, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)n);
    cub::DoubleBuffer<unsigned long long> kb(nullptr, nullptr);
    cub::DoubleBuffer<uint32_t> vb(nullptr, nullptr);
    if (has_w) cub::DeviceRadixSort::SortPairs(nullptr, t3, kb, vb, (int)nnz, 0, key_end_bit(n));
    else cub::DeviceRadixSort::SortKeys(nullptr, t3, kb, (int)nnz, 0, key_end_bit(n));
    size_t t4 = 0;
    cub::DoubleBuffer<uint32_t> kb32(nullptr, nullptr), vb32(nullptr, nullptr);
    cub::DeviceRadixSort::SortPairs(nullptr, t4, kb32, vb32, (int)nnz, 0, key_end_bit(n) - 32);
    size_t t = std::max(std::max(t1, t4), std::max(t2, t3));
    const size_t m = (size_t)std::max<int64_t>(nnz, 1);
    return al256(t) + 3 * al256((size_t)n * 4) + al256((size_t)(n + 1) * 4) + 2 * al256(m * 8) +
           (has_w ? 2 * al256(m * 4) : 0) + 4096;
}

// Rows of the relabeled graph: permuted, columns renamed through inv, sorted ascending (so the
// highest-degree neighbour comes first).  One 64-bit radix sort of (row, column) keys over all
// edges -- a segmented sort spent most of its time in one CTA per hub row (C3: ~10 ms).
static gsw_status relabel_csr(gsw_graph g, uint32_t *off, int32_t *col, uint32_t *w, const uint32_t *perm,
                              const uint32_t *inv, uint32_t *degp, uint32_t *noff, unsigned long long *k0,
                              unsigned long long *k1, uint32_t *w0, uint32_t *w1, void *cub_tmp, size_t cub_bytes) {
    const int n = g->g.n;
    const int64_t nnz = g->g.nnz;
    cudaStream_t s = g->stream;
    k_perm_deg<<<grid_for(n, g->sms), kBlock, 0, s>>>(off, perm, n, degp);
    size_t cb = cub_bytes;
    GSW_CUDA(cub::DeviceScan::InclusiveSum(cub_tmp, cb, degp, noff + 1, n, s));
    k_set_u32<<<1, 1, 0, s>>>(noff, 0u);
    if (g->symmetric && !w && nnz > 0 && !std::getenv("GSW_RELABEL_KEYS64")) {
        // Symmetric graph: new row x holds {y : x in N(y)}.  Emitting (x, y) pairs in ascending y
        // (new rows in order) and sorting them STABLY by x alone yields every row's columns in
        // ascending order -- a radix sort over log2(n) key bits with 32-bit keys and values
        // instead of the (row << 32 | column) 64-bit keys below (C3: half the passes).
        uint32_t *ka = reinterpret_cast<uint32_t *>(k0), *kb2 = ka + nnz;
        uint32_t *va = reinterpret_cast<uint32_t *>(k1), *vb2 = va + nnz;
        uint32_t *heavy = degp;                      // degp is consumed by the scan above
        unsigned *nheavy = reinterpret_cast<unsigned *>(w0 ? w0 : (uint32_t *)cub_tmp);
        (void)w1;
        GSW_CUDA(cudaMemsetAsync(nheavy, 0, 4, s));
        k_permute_rows_pairs<<<grid_for((long long)n * 32, g->sms), kBlock, 0, s>>>(noff, off, col, perm, inv, n, ka, va,
                                                                                   heavy, nheavy);
        k_permute_heavy<<<g->sms * 2, kBlock, 0, s>>>(noff, off, col, perm, inv, ka, va, heavy, nheavy);
        GSW_CUDA(cudaGetLastError());
        GSW_CUDA(cudaMemcpyAsync(off, noff, (size_t)(n + 1) * 4, cudaMemcpyDeviceToDevice, s));
        cub::DoubleBuffer<uint32_t> kd(ka, kb2), vd(va, vb2);
        cb = cub_bytes;
        GSW_CUDA(cub::DeviceRadixSort::SortPairs(cub_tmp, cb, kd, vd, (int)nnz, 0, key_end_bit(n) - 32, s));
        GSW_CUDA(cudaMemcpyAsync(col, vd.Current(), (size_t)nnz * 4, cudaMemcpyDeviceToDevice, s));
        return GSW_OK;
    }
    k_permute_rows_keys<<<grid_for((long long)n * 32, g->sms), kBlock, 0, s>>>(noff, off, col, w, perm, inv, n, k0, w0);
    GSW_CUDA(cudaGetLastError());
    GSW_CUDA(cudaMemcpyAsync(off, noff, (size_t)(n + 1) * 4, cudaMemcpyDeviceToDevice, s));
    if (nnz == 0) return GSW_OK;
    cb = cub_bytes;
    cub::DoubleBuffer<unsigned long long> kb(k0, k1);
    if (w) {
        cub::DoubleBuffer<uint32_t> vb(w0, w1);
        GSW_CUDA(cub::DeviceRadixSort::SortPairs(cub_tmp, cb, kb, vb, (int)nnz, 0, key_end_bit(n), s));
        GSW_CUDA(cudaMemcpyAsync(w, vb.Current(), (size_t)nnz * 4, cudaMemcpyDeviceToDevice, s));
    } else {
        GSW_CUDA(cub::DeviceRadixSort::SortKeys(cub_tmp, cb, kb, (int)nnz, 0, key_end_bit(n), s));
    }
    k_key_cols<<<grid_for(nnz, g->sms), kBlock, 0, s>>>(kb.Current(), nnz, col);
    GSW_CUDA(cudaGetLastError());
    return GSW_OK;
}

gsw_status relabel_graph(gsw_graph g, uint32_t *perm, uint32_t *inv, char *tmp, size_t tmp_bytes) {
    const int n = g->g.n;
    const int64_t nnz = g->g.nnz;
    const int has_w = g->g.w != nullptr;
    if (tmp_bytes < relabel_temp_bytes(n, nnz, has_w)) { set_error("relabel: scratch too small"); return GSW_ENOMEM; }
    Workspace t{tmp, tmp_bytes, 0};
    uint32_t *deg = (uint32_t *)t.take((size_t)n * 4), *ids = (uint32_t *)t.take((size_t)n * 4);
    uint32_t *degs = (uint32_t *)t.take((size_t)n * 4), *noff = (uint32_t *)t.take((size_t)(n + 1) * 4);
    const size_t m = (size_t)std::max<int64_t>(nnz, 1);
    unsigned long long *k0 = (unsigned long long *)t.take(m * 8), *k1 = (unsigned long long *)t.take(m * 8);
    uint32_t *w0 = has_w ? (uint32_t *)t.take(m * 4) : nullptr, *w1 = has_w ? (uint32_t *)t.take(m * 4) : nullptr;
    size_t cub_bytes = tmp_bytes - t.used - 512;
    void *cub_tmp = t.take(cub_bytes);
    cudaStream_t s = g->stream;
    k_deg_iota<<<grid_for(n, g->sms), kBlock, 0, s>>>(g->g.off, n, deg, ids);
    size_t cb = cub_bytes;
    GSW_CUDA(cub::DeviceRadixSort::SortPairsDescending(cub_tmp, cb, deg, degs, ids, perm, n, 0, 32, s));
    k_invert<<<grid_for(n, g->sms), kBlock, 0, s>>>(perm, n, inv);
    GSW_CUDA(cudaGetLastError());
    gsw_status st = relabel_csr(g, (uint32_t *)g->g.off, (int32_t *)g->g.col, (uint32_t *)g->g.w, perm, inv, degs,
                                noff, k0, k1, w0, w1, cub_tmp, cub_bytes);
    if (st != GSW_OK) return st;
    if (!g->symmetric) {
        st = relabel_csr(g, (uint32_t *)g->g.in_off, (int32_t *)g->g.in_col, (uint32_t *)g->g.in_w, perm, inv, degs,
                         noff, k0, k1, w0, w1, cub_tmp, cub_bytes);
        if (st != GSW_OK) return st;
    }
    g->g.perm = perm;
    g->g.inv = inv;
    return GSW_OK;
}

gsw_status validate_graph(gsw_graph g) {
    unsigned *bad = (unsigned *)g->scratch;
    GSW_CUDA(cudaMemsetAsync(bad, 0, 4, g->stream));
    k_validate<<<grid_for(std::max<long long>(g->g.n, g->g.nnz), g->sms), kBlock, 0, g->stream>>>(
        g->g.off, g->g.col, g->g.n, g->g.nnz, bad);
    if (!g->symmetric)
        k_validate<<<grid_for(std::max<long long>(g->g.n, g->g.nnz), g->sms), kBlock, 0, g->stream>>>(
            g->g.in_off, g->g.in_col, g->g.n, g->g.nnz, bad);
    GSW_CUDA(cudaGetLastError());
    unsigned hb = 0;
    GSW_CUDA(cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, g->stream));
    GSW_CUDA(cudaStreamSynchronize(g->stream));
    if (hb & 1u) { set_error("row offsets are not monotone"); return GSW_EINVAL; }
    if (hb & 2u) { set_error("column index out of range"); return GSW_EINVAL; }
    return GSW_OK;
}

gsw_status build_first_nbr(gsw_graph g, int32_t *first) {
    k_first_nbr<<<grid_for(g->g.n, g->sms), kBlock, 0, g->stream>>>(g->g.in_off, g->g.in_col, g->g.n, first);
    GSW_CUDA(cudaGetLastError());
    g->g.in_first = first;
    return GSW_OK;
}

}  // namespace gsw
