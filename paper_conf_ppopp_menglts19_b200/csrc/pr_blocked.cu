// pr_blocked.cu -- PageRank pull with row tiers and (optionally) the gather blocked by SOURCE range,
// for graphs whose contribution array does not fit in L2 ("L2 blocking of the PR
// gather by source range is the B200 lever" at C5, where pr/deg of 67M vertices is 268 MB against
// a 126 MB L2).  Measured, the blocking does not pay on B200 (see run_pr_blocked: B = 1 wins), and
// once the stream kernel's hub cache was sized for L1 the row tiers lost their lead at C5 too
// (116 vs 120 it/s): a measured alternative, selected with GSW_PR_BLOCKED=1.
//
// Same iteration as pr.cu / pr_stream.cu (reading R7):
//   pr_{t+1}(v) = (1-d)/N + d * ( sum_{u in N_in(v)} pr_t(u)/deg_out(u) + D_t/N ),  D_t = dangling mass
// with every vertex active.  The sources are cut into B blocks of SB vertices whose
// fp32 contributions fit a third of L2; iteration t makes B passes over the rows, pass b summing
// only the in-edges whose source lies in block b.  Because every row's in-neighbours are sorted
// ascending, the edges of block b form one contiguous range of the row, [split_b(v), split_b+1(v)),
// found once per run by binary search -- no second copy of the edges.  Each pass therefore
// gathers from a 1/B slice of the contributions that stays L2-resident while the column stream
// (evict-first loads) goes by, instead of missing to DRAM with a 32-byte sector per 4-byte value.
//   light rows (<= kHeavyRow in-edges): a lane per row (4 gathers in flight), the warp for rows
//     above 32 edges; pass 0 writes the fp32 partial, later passes add to it (the row's B partial
//     sums are fp64 in registers, rounded once each);
//   heavy rows: their per-block ranges cut into 1024-edge tasks (built per run), warp sums added
//     in fp64 to a compact per-heavy-row accumulator;
//   a final pass per iteration forms pr, the next contributions, the dangling mass and (last
//   iteration) the caller-order output.
// Launches per iteration: 2B + 1, stream-ordered; no host round trip.
#include "engine.cuh"
#include "internal.h"
#include "launch.h"

#include <algorithm>
#include <cstdlib>

namespace gsw {

namespace {

constexpr int kPB = 256;
constexpr uint32_t kHeavyRow = 4096;    // rows above this many in-edges: chunk tasks + fp64 partials
constexpr uint32_t kTask = 1024;        // edges per heavy task
constexpr int kMaxBlocks = 8;

struct PbTask {
    int hk;            // heavy-row index
    uint32_t beg, end;
};

struct PbArgs {
    int n;
    uint32_t nnz;
    const uint32_t *in_off;
    const int32_t *in_col;
    const uint32_t *off;       // out-offsets (deg_out)
    const uint32_t *perm;      // internal -> caller (relabeled) or nullptr
    int B;
    uint32_t SB;
    uint32_t *split;           // (B-1) x n: split[(b-1)*n + v] = first in-edge of v with source >= b*SB
    int *hk;                   // n: heavy-row index or -1
    int *hrow;                 // heavy rows (compact)
    unsigned *nheavy;
    PbTask *tasks;             // B x task_cap
    unsigned *ntasks;          // B counters
    uint32_t task_cap, heavy_cap;
    const float *cur;
    float *next;
    float *acc;                // n fp32 partial sums of light rows
    double *hacc;              // heavy_cap fp64 sums of heavy rows
    double *dsum;              // iters+1 dangling masses
    double *out;               // caller-order result (last iteration)
    double d, invN;
};

__global__ void k_pb_setup(PbArgs a) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < a.n; v += (long long)gridDim.x * blockDim.x) {
        const uint32_t b0 = a.in_off[v], e0 = a.in_off[v + 1];
        for (int b = 1; b < a.B; ++b) {
            const int32_t lim = (int32_t)((uint32_t)b * a.SB);
            uint32_t lo = b0, hi = e0;                 // first edge with col >= lim
            while (lo < hi) {
                const uint32_t m = (lo + hi) >> 1;
                if (a.in_col[m] < lim) lo = m + 1; else hi = m;
            }
            a.split[(size_t)(b - 1) * a.n + v] = lo;
        }
        int h = -1;
        if (e0 - b0 > kHeavyRow) {
            h = (int)atomicAdd(a.nheavy, 1u);
            if ((uint32_t)h < a.heavy_cap) {
                a.hrow[h] = (int)v;
                a.hacc[h] = 0.0;
                for (int b = 0; b < a.B; ++b) {
                    const uint32_t s0 = b == 0 ? b0 : a.split[(size_t)(b - 1) * a.n + v];
                    const uint32_t s1 = b == a.B - 1 ? e0 : a.split[(size_t)b * a.n + v];
                    if (s1 <= s0) continue;
                    const unsigned k = (s1 - s0 + kTask - 1) / kTask;
                    const unsigned i = atomicAdd(a.ntasks + b, k);
                    for (unsigned j = 0; j < k && i + j < a.task_cap; ++j)
                        a.tasks[(size_t)b * a.task_cap + i + j] = PbTask{h, s0 + j * kTask, min(s1, s0 + (j + 1) * kTask)};
                }
            } else {
                h = -2;      // over capacity: cannot happen (heavy_cap = nnz / kHeavyRow + 1)
            }
        }
        a.hk[v] = h;
    }
}

__global__ void k_pb_init(PbArgs a, float *c0) {
    double dang = 0.0;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < a.n; v += (long long)gridDim.x * blockDim.x) {
        const uint32_t dg = a.off[v + 1] - a.off[v];
        c0[v] = dg ? (float)(a.invN / dg) : 0.f;
        if (!dg) dang += a.invN;
    }
    dang = warp_sum(dang);
    if (lane_id() == 0 && dang != 0.0) atomicAdd(a.dsum, dang);
}

// pass b over the light rows
__global__ void __launch_bounds__(kPB) k_pb_light(PbArgs a, int b) {
    const unsigned lane = lane_id();
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    const uint32_t *sp0 = b == 0 ? nullptr : a.split + (size_t)(b - 1) * a.n;
    const uint32_t *sp1 = b == a.B - 1 ? nullptr : a.split + (size_t)b * a.n;
    for (long long wb = gw * 32; wb < a.n; wb += nw * 32) {
        const long long v = wb + lane;
        uint32_t s0 = 0, s1 = 0;
        bool light = false;
        if (v < a.n) {
            const uint32_t r0 = a.in_off[v], r1 = a.in_off[v + 1];
            light = r1 - r0 <= kHeavyRow;
            s0 = sp0 ? sp0[v] : r0;
            s1 = sp1 ? sp1[v] : r1;
        }
        const uint32_t L = light ? s1 - s0 : 0u;
        double s = 0.0;
        if (L && L <= 32) {
            double t0 = 0.0, t1 = 0.0;
            uint32_t k = s0;
            for (; k + 4 <= s1; k += 4) {
                const int u0 = __ldcs(a.in_col + k), u1 = __ldcs(a.in_col + k + 1), u2 = __ldcs(a.in_col + k + 2),
                          u3 = __ldcs(a.in_col + k + 3);
                t0 += (double)a.cur[u0] + (double)a.cur[u1];
                t1 += (double)a.cur[u2] + (double)a.cur[u3];
            }
            for (; k < s1; ++k) t0 += (double)a.cur[__ldcs(a.in_col + k)];
            s = t0 + t1;
        }
        unsigned mid = __ballot_sync(0xffffffffu, L > 32);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, s0, j), ej = __shfl_sync(0xffffffffu, s1, j);
            double t = 0.0;
            for (uint32_t k = bj + lane; k < ej; k += 32) t += (double)a.cur[__ldcs(a.in_col + k)];
            t = warp_sum(t);
            if ((int)lane == j) s = t;
        }
        if (light) {
            if (b == 0) a.acc[v] = (float)s;
            else if (L) a.acc[v] += (float)s;
        }
    }
}

// pass b over the heavy rows' tasks of block b
__global__ void __launch_bounds__(kPB) k_pb_heavy(PbArgs a, int b) {
    const unsigned nt = min(a.ntasks[b], a.task_cap);
    const PbTask *tk = a.tasks + (size_t)b * a.task_cap;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long k = gw; k < nt; k += nw) {
        const PbTask t = tk[k];
        double s = 0.0;
        for (uint32_t e = t.beg + lane_id(); e < t.end; e += 32) s += (double)a.cur[__ldcs(a.in_col + e)];
        s = warp_sum(s);
        if (lane_id() == 0) atomicAdd(a.hacc + t.hk, s);
    }
}

// pr_{t+1}, next contributions, dangling mass D_{t+1}; the output on the last iteration
__global__ void __launch_bounds__(kPB) k_pb_final(PbArgs a, int t, bool last) {
    const double D = a.dsum[t];
    const double base = (1.0 - a.d) * a.invN + a.d * D * a.invN;
    double dang = 0.0;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < a.n; v += (long long)gridDim.x * blockDim.x) {
        const int h = a.hk[v];
        double s;
        if (h >= 0) { s = a.hacc[h]; a.hacc[h] = 0.0; }
        else s = (double)a.acc[v];
        const double p = base + a.d * s;
        const uint32_t dg = a.off[v + 1] - a.off[v];
        a.next[v] = dg ? (float)p * __frcp_rn((float)dg) : 0.f;
        if (!dg) dang += p;
        if (last) a.out[a.perm ? a.perm[v] : v] = p;
    }
    dang = warp_sum(dang);
    if (lane_id() == 0 && dang != 0.0) atomicAdd(a.dsum + t + 1, dang);
}

}  // namespace

// Blocking is worth it once the fp32 contributions exceed half of L2; GSW_PR_BLOCKED=1 forces it
// (parity tests on small graphs), =0 disables it.
// Not AUTO's choice any more: with the hub cache sized for L1 (pr_stream.cu) the stream kernel
// reaches 120 it/s on C5 against 116 for this one (profiles/r2/pr_cache_sweep.txt), so the
// row-tier / source-blocked kernel is kept as a measured alternative, selected by GSW_PR_BLOCKED=1.
bool pr_blocked_wanted(gsw_graph g) {
    (void)g;
    if (const char *e = std::getenv("GSW_PR_BLOCKED")) return std::atoi(e) != 0;
    return false;
}

gsw_status run_pr_blocked(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st) {
    const int n = g->g.n;
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(rank) == 1;
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g->device);
    cudaGetLastError();
    // Source blocks: measured on C5 (profiles/r2/minblocks_ab_m1_m2_c5pr_blocks.txt, r2k): B = 1
    // 116 it/s, 2: 108, 3: 101, 4: 96, 6: 87, 8: 79 -- the split reads and the partial's
    // read-modify-write per pass cost more than the L2 hits of the narrower gather save, so the
    // default is one block (the row tiers alone are 2.35x the stream kernel at C5: 49 it/s).
    // GSW_PR_BLOCKS=B keeps the blocked passes selectable (tests, calibration on other GPUs).
    (void)l2;
    int B = 1;
    if (const char *e = std::getenv("GSW_PR_BLOCKS")) B = std::atoi(e);
    B = std::max(1, std::min(B, kMaxBlocks));
    PbArgs a{};
    a.n = n;
    a.nnz = g->g.nnz;
    a.in_off = g->g.in_off;
    a.in_col = g->g.in_col;
    a.off = g->g.off;
    a.perm = g->g.perm;
    a.B = B;
    a.SB = (uint32_t)(((int64_t)n + B - 1) / B);
    a.d = damping;
    a.invN = 1.0 / (double)n;
    a.heavy_cap = a.nnz / kHeavyRow + 1;
    a.task_cap = a.nnz / kTask + a.heavy_cap + 1;
    a.out = dev_out ? rank : (double *)ws.take((size_t)n * 8);
    float *C[2] = {(float *)ws.take((size_t)n * 4 + 16), (float *)ws.take((size_t)n * 4 + 16)};
    a.acc = (float *)ws.take((size_t)n * 4 + 16);
    a.split = (uint32_t *)ws.take((size_t)std::max(1, B - 1) * n * 4);
    a.hk = (int *)ws.take((size_t)n * 4);
    a.hrow = (int *)ws.take((size_t)a.heavy_cap * 4);
    a.hacc = (double *)ws.take((size_t)a.heavy_cap * 8);
    a.tasks = (PbTask *)ws.take((size_t)B * a.task_cap * sizeof(PbTask));
    a.ntasks = (unsigned *)ws.take(256);
    a.nheavy = a.ntasks + kMaxBlocks;
    a.dsum = (double *)ws.take((size_t)(iters + 2) * 8);
    if (!a.out || !C[1] || !a.acc || !a.split || !a.hk || !a.hrow || !a.hacc || !a.tasks || !a.ntasks || !a.dsum) {
        set_error("gsw_pr (blocked): workspace too small");
        return GSW_ENOMEM;
    }
    cudaStream_t s = g->stream;
    const int grid = g->sms * 8;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemsetAsync(a.ntasks, 0, 256, s));
    GSW_CUDA(cudaMemsetAsync(a.dsum, 0, (size_t)(iters + 2) * 8, s));
    k_pb_setup<<<grid, kPB, 0, s>>>(a);
    k_pb_init<<<grid, kPB, 0, s>>>(a, C[0]);
    GSW_CUDA(cudaGetLastError());
    if (iters == 0) {
        // pr_0 = 1/N in caller order
        a.cur = C[0]; a.next = C[1];
        GSW_CUDA(cudaMemsetAsync(a.acc, 0, (size_t)n * 4, s));
        // a final pass with d = 0 would give (1 - 0)/N = 1/N exactly
        PbArgs z = a;
        z.d = 0.0;
        k_pb_final<<<grid, kPB, 0, s>>>(z, 0, true);
    }
    for (int t = 0; t < iters; ++t) {
        a.cur = C[t & 1];
        a.next = C[(t + 1) & 1];
        for (int b = 0; b < B; ++b) {
            k_pb_light<<<grid, kPB, 0, s>>>(a, b);
            k_pb_heavy<<<grid, kPB, 0, s>>>(a, b);
        }
        k_pb_final<<<grid, kPB, 0, s>>>(a, t, t == iters - 1);
    }
    GSW_CUDA(cudaGetLastError());
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank, a.out, (size_t)n * 8, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = iters;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)a.nnz * iters;
        // per iteration, SURVEY 8(d) D0 "PR iteration (pull): 4 nnz + 16 N" -- the blocking's own
        // traffic (split offsets, the fp32 partial's read-modify-write per pass) is overhead of
        // this design, not compulsory, and is not counted
        st->bytes_alg = (int64_t)((4ull * a.nnz + 16ull * n) * iters);
        if (st->records && st->max_records > 0) {
            for (int i = 0; i < std::min(iters, st->max_records); ++i) {
                gsw_iter_record &r = st->records[i];
                r = gsw_iter_record{};
                r.iteration = i;
                r.direction = GSW_PULL; r.format = GSW_BITMAP; r.load_balance = GSW_LB_TWC; r.fusion = GSW_FUSED;
                r.Va = n; r.Ea = a.nnz; r.edges = a.nnz;
                r.ctas = grid;
            }
        }
    }
    return GSW_OK;
}

}  // namespace gsw
