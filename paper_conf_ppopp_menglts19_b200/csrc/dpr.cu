// dpr.cu -- Delta-PageRank ([19]; Fig. 3 "Iteration No. of Delta-PR"), the
// SURVEY F2 row.  Unlike the power iteration of pr.cu, only vertices whose unpropagated residual
// exceeds eps are active, so the active set shrinks over the run and direction switching matters
// ("the push mode outperforms the pull mode when the active vertices decrease").
// Reading R16, identical to oracle.c orc_dpr:
//   delta_0 = (1-d)/N, r_0 = 0;   A_t = { v : delta_t(v) > eps },  r(v) += delta_t(v) on A_t,
//   delta_{t+1}(w) = [w not in A_t] delta_t(w) + sum_{v in A_t, v->w} d delta_t(v)/deg_out(v).
// eps = tol (1-d)/N bounds the result: 0 <= x - r and ||x - r||_1 <= tol (x = fixed point).
//
// One iteration = three stream-ordered kernels, no host round trip:
//   Filter  k_dpr_filter  one pass over N: delta += acc, acc = 0, activation, rank update, the
//                         contribution c(v) = d delta/deg (0 when inactive), block-aggregated
//                         enqueue of A_t, Va/Ea of A_t (Table 1 features) -> cnt[t]
//   Expand  k_dpr_push    fp64 atomicAdd of c(u) into acc of u's targets, for queued u
//           k_dpr_pull    acc(w) = sum of c over in-neighbours (atomics only for heavy rows)
//           both in four edge-balanced tiers: a lane per tiny row, 8-lane groups for short
//           rows, a warp per mid row, 1024-edge warp chunks of heavy rows (table built on the
//           device at run start, no host round trip)
// The selector (pull iff Ea > nnz - Ea, "the pull mode is preferable ... when the number of the
// active edges is greater than that of inactive edges") is evaluated on the device by
// both expand kernels from cnt[t]; the one not chosen returns at once.  The host polls the active
// count once per batch of iterations, one batch behind the stream; kernels after the empty
// iteration are no-ops.
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <vector>

#include "common.cuh"
#include "internal.h"

namespace gsw {

namespace {

constexpr int kDprBlock = 256;
constexpr int kBatch = 4;          // iterations enqueued between two host polls (at least)
constexpr int kBatchMax = 32;      // ... and at most
constexpr int kFilterChunk = 4;    // vertices per thread per block round of the filter
constexpr uint32_t kChunk = 1024;  // heavy-row chunk (edges per warp task)
constexpr uint32_t kHeavy = 128;   // rows above this many edges become chunk tasks: after the
                                   // degree-ordered relabeling the mid rows sit together, and 32
                                   // of them serialised on one warp were the tail of small graphs
constexpr uint32_t kSmall = 64;    // rows up to this many edges go to an 8-lane group
constexpr uint32_t kTiny = 8;      // rows up to this many edges are finished by one lane
static_assert(kChunk % kHeavy == 0 && kChunk / kHeavy == 8, "k_dpr_chunks capacity bound");
struct Chunk;

struct DprCnt {                    // per-iteration record, zeroed at run start
    unsigned long long va, ea;
    int dir, pad0;
    unsigned long long pad1;
};

struct DprArgs {
    int n;
    uint32_t nnz;
    const uint32_t *off;       // out-edges (push, deg_out)
    const int32_t *col;
    const uint32_t *in_off;    // in-edges (pull)
    const int32_t *in_col;
    double d, eps;
    double *r, *delta, *acc, *c;
    int32_t *q;
    unsigned *qlen;            // per iteration (max_iters entries)
    DprCnt *cnt;
    int force_dir;
    unsigned pull_k;                     // pull iff Ea * pull_k > nnz (2: the paper's Ea > Eia)
    const Chunk *chunk_out, *chunk_in;   // heavy-row chunk tables (push: out-rows, pull: in-rows)
    const unsigned *nchunk_out, *nchunk_in;   // their lengths (device counters, k_dpr_chunks)
};

__global__ void k_dpr_init(DprArgs a) {
    const double base = (1.0 - a.d) / (double)a.n;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < a.n; v += (long long)gridDim.x * blockDim.x) {
        a.r[v] = 0.0;
        a.delta[v] = base;
        a.acc[v] = 0.0;
    }
}

__device__ __forceinline__ bool dpr_done(const DprArgs &a, int t) { return t > 0 && a.cnt[t - 1].va == 0; }

__global__ void __launch_bounds__(kDprBlock) k_dpr_filter(DprArgs a, int t) {
    if (dpr_done(a, t)) return;
    constexpr int W = kDprBlock / 32;
    __shared__ unsigned s_off[kFilterChunk][W];
    __shared__ unsigned s_base;
    __shared__ unsigned long long s_ea[W];
    __shared__ unsigned s_va[W];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    unsigned long long ea = 0;
    unsigned va = 0;
    const long long chunk = (long long)kDprBlock * kFilterChunk;
    for (long long c0 = blockIdx.x * chunk; c0 < a.n; c0 += gridDim.x * chunk) {
        unsigned m[kFilterChunk];
        double dl[kFilterChunk];
        uint32_t deg[kFilterChunk];
        // all loads of the round first (4 independent vertices in flight per thread)
#pragma unroll
        for (int k = 0; k < kFilterChunk; ++k) {
            const long long v = c0 + k * kDprBlock + threadIdx.x;
            dl[k] = 0.0;
            deg[k] = 0;
            if (v < a.n) {
                dl[k] = a.delta[v] + a.acc[v];
                deg[k] = __ldg(a.off + v + 1) - __ldg(a.off + v);
            }
        }
#pragma unroll
        for (int k = 0; k < kFilterChunk; ++k) {
            const long long v = c0 + k * kDprBlock + threadIdx.x;
            bool act = false;
            if (v < a.n) {
                a.acc[v] = 0.0;
                double cv = 0.0;
                if (dl[k] > a.eps) {
                    act = true;
                    a.r[v] += dl[k];
                    a.delta[v] = 0.0;
                    if (deg[k]) cv = a.d * dl[k] / (double)deg[k];
                    ea += deg[k];
                    ++va;
                } else {
                    a.delta[v] = dl[k];
                }
                a.c[v] = cv;
            }
            m[k] = __ballot_sync(0xffffffffu, act);
            if (lane == 0) s_off[k][w] = __popc(m[k]);
        }
        __syncthreads();
        if (threadIdx.x == 0) {   // exclusive scan over (k, w) and one queue reservation per round
            unsigned s = 0;
            for (int k = 0; k < kFilterChunk; ++k)
                for (int j = 0; j < W; ++j) { unsigned x = s_off[k][j]; s_off[k][j] = s; s += x; }
            s_base = s ? atomicAdd(a.qlen + t, s) : 0u;
        }
        __syncthreads();
#pragma unroll
        for (int k = 0; k < kFilterChunk; ++k)
            if (m[k] >> lane & 1u)
                a.q[s_base + s_off[k][w] + __popc(m[k] & lanemask_lt())] = (int32_t)(c0 + k * kDprBlock + threadIdx.x);
        __syncthreads();
    }
    for (int o = 16; o; o >>= 1) {
        ea += __shfl_xor_sync(0xffffffffu, ea, o);
        va += __shfl_xor_sync(0xffffffffu, va, o);
    }
    if (lane == 0) { s_ea[w] = ea; s_va[w] = va; }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long E = 0, V = 0;
        for (int j = 0; j < W; ++j) { E += s_ea[j]; V += s_va[j]; }
        if (V) { atomicAdd(&a.cnt[t].va, V); atomicAdd(&a.cnt[t].ea, E); }
    }
}

// 1 = push, 2 = pull (GSW_PUSH / GSW_PULL)
__device__ __forceinline__ int dpr_dir(const DprArgs &a, const DprCnt &c) {
    if (a.force_dir) return a.force_dir;
    return c.ea * a.pull_k > (unsigned long long)a.nnz ? GSW_PULL : GSW_PUSH;
}

// Edge-balanced tiers shared by push and pull (Delta-PR):
//   heavy rows (deg > kHeavy): cut into kChunk-edge chunks at run start (host-built table), one
//     warp per chunk, partial results by fp64 atomics -- a 163K-edge R-MAT hub no longer runs on
//     one warp for milliseconds;
//   mid rows (kSmall < deg <= kHeavy): one warp, 4 loads in flight per lane;
//   short rows (deg <= kSmall): an 8-lane group per row, 4 rows per warp.
struct Chunk {
    int row;
    uint32_t beg, end;
};

// push a mid row u (whole warp): acc[v] += cu for every out-edge
__device__ __forceinline__ void push_range(const DprArgs &a, uint32_t j, uint32_t e, double cu, int stride) {
    for (; j + 3 * stride < e; j += 4 * stride) {
        const int v0 = __ldg(a.col + j), v1 = __ldg(a.col + j + stride), v2 = __ldg(a.col + j + 2 * stride),
                  v3 = __ldg(a.col + j + 3 * stride);
        atomicAdd(a.acc + v0, cu); atomicAdd(a.acc + v1, cu); atomicAdd(a.acc + v2, cu); atomicAdd(a.acc + v3, cu);
    }
    for (; j < e; j += stride) atomicAdd(a.acc + __ldg(a.col + j), cu);
}

__device__ __forceinline__ double pull_range(const DprArgs &a, uint32_t j, uint32_t e, int stride) {
    double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
    for (; j + 3 * stride < e; j += 4 * stride) {
        const int u0 = __ldg(a.in_col + j), u1 = __ldg(a.in_col + j + stride), u2 = __ldg(a.in_col + j + 2 * stride),
                  u3 = __ldg(a.in_col + j + 3 * stride);
        s0 += a.c[u0]; s1 += a.c[u1]; s2 += a.c[u2]; s3 += a.c[u3];
    }
    for (; j < e; j += stride) s0 += a.c[__ldg(a.in_col + j)];
    return (s0 + s1) + (s2 + s3);
}

// Rows of one 32-row warp batch, one row per lane: tiny rows (deg <= kTiny) are finished by
// their own lane, short rows by 8-lane groups (4 at a time, __fns picks each group's row), mid
// rows by the whole warp; heavy rows are skipped (chunk tasks).  Op: push or pull body.
template <class Op>
__device__ __forceinline__ void row_tiers(const Op &op, bool valid, uint32_t b, uint32_t e) {
    const int lane = threadIdx.x & 31, sub = lane >> 3, sl = lane & 7;
    const uint32_t deg = e - b;
    const bool live = valid && op.live();
    if (live && deg <= kTiny) op.tiny(b, e);
    unsigned sm = __ballot_sync(0xffffffffu, live && deg > kTiny && deg <= kSmall);
    while (sm) {
        const unsigned k = __fns(sm, 0, sub + 1);
        const int src = k < 32 ? (int)k : lane;
        const uint32_t bb = __shfl_sync(0xffffffffu, b, src), ee = __shfl_sync(0xffffffffu, e, src);
        op.group(src, k < 32, bb, ee, sl);
        for (int i = 0; i < 4 && sm; ++i) sm &= sm - 1;
    }
    unsigned mid = __ballot_sync(0xffffffffu, live && deg > kSmall && deg <= kHeavy);
    while (mid) {
        const int k = __ffs(mid) - 1;
        mid &= mid - 1;
        const uint32_t bb = __shfl_sync(0xffffffffu, b, k), ee = __shfl_sync(0xffffffffu, e, k);
        op.warp(k, bb, ee, lane);
    }
}

struct PushOp {
    const DprArgs &a;
    double cu;
    __device__ bool live() const { return cu != 0.0; }
    __device__ void tiny(uint32_t b, uint32_t e) const { for (uint32_t j = b; j < e; ++j) atomicAdd(a.acc + __ldg(a.col + j), cu); }
    __device__ void group(int src, bool on, uint32_t b, uint32_t e, int sl) const {
        const double c = __shfl_sync(0xffffffffu, cu, src);
        if (on) push_range(a, b + sl, e, c, 8);
    }
    __device__ void warp(int src, uint32_t b, uint32_t e, int lane) const {
        const double c = __shfl_sync(0xffffffffu, cu, src);
        push_range(a, b + lane, e, c, 32);
    }
};

struct PullOp {
    const DprArgs &a;
    unsigned v0;
    __device__ bool live() const { return true; }
    __device__ void tiny(uint32_t b, uint32_t e) const {
        double s = 0.0;
        for (uint32_t j = b; j < e; ++j) s += a.c[__ldg(a.in_col + j)];
        a.acc[v0 + (threadIdx.x & 31)] = s;
    }
    __device__ void group(int src, bool on, uint32_t b, uint32_t e, int sl) const {
        double s = on ? pull_range(a, b + sl, e, 8) : 0.0;
        s += __shfl_xor_sync(0xffffffffu, s, 4);
        s += __shfl_xor_sync(0xffffffffu, s, 2);
        s += __shfl_xor_sync(0xffffffffu, s, 1);
        if (on && sl == 0) a.acc[v0 + src] = s;
    }
    __device__ void warp(int src, uint32_t b, uint32_t e, int lane) const {
        double m = pull_range(a, b + lane, e, 32);
        for (int o = 16; o; o >>= 1) m += __shfl_xor_sync(0xffffffffu, m, o);
        if (lane == 0) a.acc[v0 + src] = m;
    }
};

__global__ void __launch_bounds__(kDprBlock) k_dpr_push(DprArgs a, int t) {
    const DprCnt cn = a.cnt[t];
    if (cn.va == 0 || dpr_dir(a, cn) != GSW_PUSH) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.cnt[t].dir = GSW_PUSH;
    const unsigned qn = a.qlen[t];
    const int lane = threadIdx.x & 31;
    const unsigned gw = blockIdx.x * (kDprBlock / 32) + (threadIdx.x >> 5);
    const unsigned nw = gridDim.x * (kDprBlock / 32);
    // heavy chunks (inactive rows have c = 0 and return at once)
    const unsigned nch = *a.nchunk_out;
    for (unsigned k = gw; k < nch; k += nw) {
        const Chunk ch = a.chunk_out[k];
        const double cu = a.c[ch.row];
        if (cu != 0.0) push_range(a, ch.beg + lane, ch.end, cu, 32);
    }
    // queued vertices, 32 per warp batch
    for (unsigned i0 = gw * 32; i0 < qn; i0 += nw * 32) {
        const unsigned i = i0 + lane;
        uint32_t b = 0, e = 0;
        double cu = 0.0;
        if (i < qn) {
            const int u = a.q[i];
            cu = a.c[u];
            b = __ldg(a.off + u); e = __ldg(a.off + u + 1);
        }
        row_tiers(PushOp{a, cu}, i < qn, b, e);
    }
}

__global__ void __launch_bounds__(kDprBlock) k_dpr_pull(DprArgs a, int t) {
    const DprCnt cn = a.cnt[t];
    if (cn.va == 0 || dpr_dir(a, cn) != GSW_PULL) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.cnt[t].dir = GSW_PULL;
    const int lane = threadIdx.x & 31;
    const unsigned gw = blockIdx.x * (kDprBlock / 32) + (threadIdx.x >> 5);
    const unsigned nw = gridDim.x * (kDprBlock / 32);
    // heavy chunks: partial sums into acc (zeroed by the filter)
    const unsigned nch = *a.nchunk_in;
    for (unsigned k = gw; k < nch; k += nw) {
        const Chunk ch = a.chunk_in[k];
        double s = pull_range(a, ch.beg + lane, ch.end, 32);
        for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0 && s != 0.0) atomicAdd(a.acc + ch.row, s);
    }
    for (unsigned v0 = gw * 32; v0 < (unsigned)a.n; v0 += nw * 32) {
        const unsigned v = v0 + lane;
        uint32_t b = 0, e = 0;
        if (v < (unsigned)a.n) { b = __ldg(a.in_off + v); e = __ldg(a.in_off + v + 1); }
        row_tiers(PullOp{a, v0}, v < (unsigned)a.n, b, e);
    }
}

// heavy-row chunk table (run start, on the device): every row with more than kHeavy edges
// reserves ceil(deg / kChunk) slots with one atomic and writes its (row, begin, end) chunks.  The
// order of the chunks is irrelevant (their partial sums meet in fp64 atomics), so no scan is
// needed.  A heavy row has deg > kHeavy = kChunk / 8, so the table holds at most nnz / kHeavy
// entries (the capacity the workspace reserves, scratch_bytes_for).
__global__ void k_dpr_chunks(const uint32_t *off, int n, Chunk *tab, unsigned *cnt) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
        const uint32_t b = off[v], e = off[v + 1];
        if (e - b > kHeavy) {
            const unsigned k = (e - b + kChunk - 1) / kChunk;
            const unsigned i = atomicAdd(cnt, k);
            for (unsigned j = 0; j < k; ++j) {
                const uint32_t cb = b + j * kChunk;
                tab[i + j] = Chunk{(int)v, cb, min(e, cb + kChunk)};
            }
        }
    }
}

__global__ void k_dpr_out(const double *r, const uint32_t *perm, int n, double *out) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        out[perm ? perm[v] : v] = r[v];
}

// one full wave: SMs x resident blocks of this kernel (a second partial wave of a grid-stride
// kernel would leave most SMs idle during its tail); cached per (kernel, device)
int wave_grid(const void *k, int device, int sms) {
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    const auto key = std::make_pair(k, device);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, kDprBlock, 0) != cudaSuccess || nb < 1) {
        cudaGetLastError();
        nb = 1;
    }
    return cache[key] = sms * nb;
}

}  // namespace

gsw_status run_dpr(gsw_graph g, double damping, double tol, int32_t max_iters, double *rank, gsw_run_stats *st) {
    const int n = g->g.n;
    if (!rank) { set_error("gsw_dpr: rank is NULL"); return GSW_EINVAL; }
    if (max_iters < 1 || max_iters > kDprMaxIters) { set_error("gsw_dpr: max_iters must be in [1, 65536]"); return GSW_EINVAL; }
    if (!(damping >= 0.0 && damping < 1.0)) { set_error("gsw_dpr: damping must be in [0,1)"); return GSW_EINVAL; }
    if (!(tol >= 0.0 && tol < 1e300)) { set_error("gsw_dpr: tol must be finite and >= 0"); return GSW_EINVAL; }
    const int fdir = g->forced.direction;
    if (fdir != GSW_AUTO && fdir != GSW_PUSH && fdir != GSW_PULL) { set_error("gsw_dpr: bad forced direction"); return GSW_EUNSUPPORTED; }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(rank) == 1;
    DprArgs a{};
    a.n = n;
    a.nnz = g->g.nnz;
    a.off = g->g.off; a.col = g->g.col;
    a.in_off = g->g.in_off; a.in_col = g->g.in_col;
    a.d = damping;
    a.eps = tol * (1.0 - damping) / (double)n;
    a.force_dir = fdir;
    {   // GSW_DPR_PULL_K: calibration knob for the direction split (default 2)
        const char *e = std::getenv("GSW_DPR_PULL_K");
        a.pull_k = (e && *e && std::atoi(e) > 0) ? (unsigned)std::atoi(e) : 2u;
    }
    a.r = (double *)ws.take((size_t)n * 8);
    a.delta = (double *)ws.take((size_t)n * 8);
    a.acc = (double *)ws.take((size_t)n * 8);
    a.c = (double *)ws.take((size_t)n * 8);
    a.q = (int32_t *)ws.take((size_t)n * 4);
    a.qlen = (unsigned *)ws.take((size_t)max_iters * 4);
    a.cnt = (DprCnt *)ws.take((size_t)max_iters * sizeof(DprCnt));
    double *out = dev_out ? rank : (double *)ws.take((size_t)n * 8);
    if (!a.r || !a.delta || !a.acc || !a.c || !a.q || !a.qlen || !a.cnt || !out) { set_error("gsw_dpr: workspace too small"); return GSW_ENOMEM; }
    cudaStream_t s = g->stream;
    if (!g->poll) GSW_CUDA(cudaHostAlloc((void **)&g->poll, 2 * sizeof(unsigned long long), cudaHostAllocDefault));
    const int grid = g->sms * 8;
    const int g_filter = wave_grid((const void *)k_dpr_filter, g->device, g->sms);
    const int g_push = wave_grid((const void *)k_dpr_push, g->device, g->sms);
    const int g_pull = wave_grid((const void *)k_dpr_pull, g->device, g->sms);
    // heavy-row chunk tables: capacity nnz / kHeavy + 1 each (see k_dpr_chunks)
    const size_t ccap = (size_t)a.nnz / kHeavy + 1;
    const bool same_in = a.in_off == a.off && a.in_col == a.col;
    unsigned *ccnt = (unsigned *)ws.take(256);
    Chunk *tab_out = (Chunk *)ws.take(ccap * sizeof(Chunk));
    Chunk *tab_in = same_in ? tab_out : (Chunk *)ws.take(ccap * sizeof(Chunk));
    if (!ccnt || !tab_out || !tab_in) { set_error("gsw_dpr: workspace too small"); return GSW_ENOMEM; }
    a.chunk_out = tab_out; a.nchunk_out = ccnt;
    a.chunk_in = tab_in; a.nchunk_in = same_in ? ccnt : ccnt + 1;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemsetAsync(ccnt, 0, 8, s));
    k_dpr_chunks<<<grid, kDprBlock, 0, s>>>(a.off, n, tab_out, ccnt);
    if (!same_in) k_dpr_chunks<<<grid, kDprBlock, 0, s>>>(a.in_off, n, tab_in, ccnt + 1);
    GSW_CUDA(cudaGetLastError());
    GSW_CUDA(cudaMemsetAsync(a.qlen, 0, (size_t)max_iters * 4, s));
    GSW_CUDA(cudaMemsetAsync(a.cnt, 0, (size_t)max_iters * sizeof(DprCnt), s));
    k_dpr_init<<<grid, kDprBlock, 0, s>>>(a);
    GSW_CUDA(cudaGetLastError());
    // Pipelined termination poll: batch b is enqueued (with an async copy of its last active
    // count into pinned memory and an event) BEFORE the host waits on batch b-1's event, so the
    // stream never drains while the host decides.  Batches grow with t (clamp(t/4, 4, 32)), so at
    // most one batch of no-op kernels runs past the empty iteration.
    unsigned long long *hva = g->poll;   // 2 pinned slots (one per in-flight batch), owned by the handle
    cudaEvent_t evb[2] = {nullptr, nullptr};
    GSW_CUDA(cudaEventCreateWithFlags(&evb[0], cudaEventDisableTiming));
    GSW_CUDA(cudaEventCreateWithFlags(&evb[1], cudaEventDisableTiming));
    auto poll_fail = [&](cudaError_t e, const char *what) {
        cudaEventDestroy(evb[0]);
        cudaEventDestroy(evb[1]);
        return cuda_fail(e, what);
    };
    int t = 0, b = 0;
    bool done = false;
    while (!done) {
        {
            const int t1 = std::min(max_iters, t + std::min(kBatchMax, std::max(kBatch, t / 4)));
            for (; t < t1; ++t) {
                k_dpr_filter<<<g_filter, kDprBlock, 0, s>>>(a, t);
                k_dpr_push<<<g_push, kDprBlock, 0, s>>>(a, t);
                k_dpr_pull<<<g_pull, kDprBlock, 0, s>>>(a, t);
            }
            cudaError_t e = cudaGetLastError();
            if (e == cudaSuccess) e = cudaMemcpyAsync(&hva[b & 1], &a.cnt[t - 1].va, 8, cudaMemcpyDeviceToHost, s);
            if (e == cudaSuccess) e = cudaEventRecord(evb[b & 1], s);
            if (e != cudaSuccess) return poll_fail(e, "gsw_dpr: batch enqueue");
            ++b;
        }
        if (b >= 2 || t >= max_iters) {
            // check the previous batch (or, when no more can be enqueued, the last one)
            const int chk = (t >= max_iters) ? (b - 1) : (b - 2);
            const int slot = chk & 1;
            if (cudaError_t e = cudaEventSynchronize(evb[slot])) return poll_fail(e, "gsw_dpr: batch poll");
            done = hva[slot] == 0 || t >= max_iters;
        }
    }
    cudaEventDestroy(evb[0]);
    cudaEventDestroy(evb[1]);
    const int launched = t;
    k_dpr_out<<<grid, kDprBlock, 0, s>>>(a.r, g->g.perm, n, out);
    GSW_CUDA(cudaGetLastError());
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank, out, (size_t)n * 8, cudaMemcpyDeviceToHost, s));
    std::vector<DprCnt> h((size_t)launched);
    GSW_CUDA(cudaMemcpyAsync(h.data(), a.cnt, sizeof(DprCnt) * (size_t)launched, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        int it = 0;
        while (it < launched && h[it].va) ++it;
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        long long edges = 0, bytes = 0;
        const long long N = n, E = a.nnz;
        for (int i = 0; i < it; ++i) {
            const long long Va = (long long)h[i].va, Ea = (long long)h[i].ea;
            const bool pull = h[i].dir == GSW_PULL;
            const long long ed = pull ? E : Ea;
            edges += ed;
            // DESIGN.md section 6, Delta-PR, counted per SURVEY 8(d) D0 (compulsory DRAM only):
            // filter 40 B/vertex (delta r/w, acc r/w, c write: fp64 streams) + 20 B per active
            // vertex (rank r/w, queue); push 8 B/active vertex (row offsets) + 4 B per column;
            // pull 4 B/row (offsets) + 8 B/row (acc write) + 4 B per in-edge column.  Gathers of
            // c[] and the atomics into acc[] are probes of L2-resident state (D0) and not counted.
            bytes += 40 * N + 20 * Va + (pull ? 12 * N + 4 * E : 8 * Va + 4 * Ea);
            if (st->records && i < st->max_records) {
                gsw_iter_record &rec = st->records[i];
                rec = gsw_iter_record{};
                rec.iteration = i;
                rec.direction = h[i].dir;
                rec.format = GSW_QUEUE;
                rec.load_balance = GSW_LB_WM;
                rec.fusion = GSW_STANDALONE;
                rec.Va = Va; rec.Ea = Ea;
                rec.Via = N - Va; rec.Eia = E - Ea;
                rec.edges = ed;
                rec.ctas = pull ? g_pull : g_push;
            }
        }
        st->iterations = it;
        st->gpu_ms = ms;
        st->edges_touched = edges;
        st->bytes_alg = bytes;
    }
    return GSW_OK;
}

}  // namespace gsw
