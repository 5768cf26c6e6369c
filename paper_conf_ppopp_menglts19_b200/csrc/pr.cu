// pr.cu -- PageRank power iteration (PAPER.md:264 [11]; "all the vertices and edges are active in
// each iteration") with the dangling-mass convention of DESIGN.md reading R7:
//   pr_0 = 1/N;  D_t = sum_{deg_out(u)=0} pr_t(u)
//   pr_{t+1}(v) = (1-d)/N + d * ( sum_{u in N_in(v)} pr_t(u)/deg_out(u) + D_t/N )
// State per iteration: contrib_t(u) = pr_t(u)/deg_out(u) (fp64, 0 for dangling u) and D_t.
// Expand = pull (reduction over in-edges; owner mappings finish pr_{t+1}(v) in the same pass) or
// push (fp64 atomicAdd of contrib into an accumulator, then an epilogue pass).  Accumulation is
// fp64 throughout.  The paper's format/fusion patterns do not apply (every vertex is active).
#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"
#include "lb_reduce.cuh"

namespace gsw {

struct PrArgs {
    DevGraph g;
    double damping;
    int iters;
    double *out;          // final ranks (device)
    double *contrib[2];   // pr/deg_out, double buffered
    double *sum;          // accumulator for edge-parallel pull / push (zero between iterations)
    double *dsum;         // dangling mass D_t, iters+1 entries
    uint32_t *scan;
    unsigned *heavy_cnt;
    unsigned *heavy, *hblk;   // tiered pull: heavy rows and their block prefix
    RunCommon rc;
};

// epilogue shared by owner flushes and the accumulator pass
struct PrEpi {
    const uint32_t *off;
    const uint32_t *perm;   // relabeled graphs: out is in caller order
    double *out;
    double *cnext;
    double base, d;
    bool last;
    __device__ __forceinline__ void finish(int v, double s, double &dang) const {
        double p = base + d * s;
        uint32_t dg = __ldg(off + v + 1) - __ldg(off + v);
        if (last) out[perm ? perm[v] : v] = p;
        cnext[v] = dg ? p / (double)dg : 0.0;
        if (!dg) dang += p;
    }
};

struct PrPullOp {
    const double *contrib;
    double *sum;
    PrEpi epi;
    bool owner;                                   // THREAD/TWC: every flush carries a whole row
    using Probe = double;
    using Acc = double;
    static constexpr bool kFlushEmpty = true;     // vertices without in-edges still get pr_{t+1}
    static __device__ __forceinline__ Acc identity() { return 0.0; }
    static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a + b; }
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const { return contrib[u]; }
    __device__ __forceinline__ Acc val(int, uint32_t, int, Probe p) const { return p; }
    __device__ __forceinline__ void flush(int v, Acc s, bool exclusive, LocalCnt &c) const {
        if (owner && exclusive) epi.finish(v, s, c.facc);
        else if (s != 0.0) atomicAdd(sum + v, s);       // accumulator epilogue finishes v
    }
};

struct PrPushOp {
    const double *contrib;
    double *sum;
    using Probe = double;
    using Tok = int;
    using Aux = int;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int u, uint32_t, int) const { return contrib[u]; }
    __device__ __forceinline__ Tok act(int, uint32_t, int v, Probe p) const {
        if (p != 0.0) atomicAdd(sum + v, p);
        return 0;
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int, Tok) const { return 0; }
    __device__ __forceinline__ bool commit(int, uint32_t, int, Tok, Aux, LocalCnt &) const { return false; }
};

// ---------------------------------------------------------------- B200 tiered pull (TWC)
// lb_reduce.cuh lbr_tiered: rows < 32 warp-segmented, 32..1023 one warp per row, >= 1024 cut into
// 1024-edge blocks shared by the whole grid; their partial sums land in `sum` (fp64 atomics) and are
// finished after a grid barrier (phase B below).
__device__ __forceinline__ double warp_row_sum(const double *contrib, const int32_t *col, uint32_t b, uint32_t e,
                                               unsigned long long &edges) {
    const unsigned lane = lane_id();
    double s = 0.0;
    for (uint32_t k0 = b; k0 < e; k0 += 128) {
        int y[4];
        double c[4];
#pragma unroll
        for (int h = 0; h < 4; ++h) { uint32_t k = k0 + 32 * h + lane; y[h] = k < e ? __ldg(col + k) : -1; }
#pragma unroll
        for (int h = 0; h < 4; ++h) c[h] = y[h] >= 0 ? contrib[y[h]] : 0.0;
#pragma unroll
        for (int h = 0; h < 4; ++h) { s += c[h]; edges += y[h] >= 0; }
    }
    return warp_sum(s);
}

// phase A: heavy blocks (atomics into sum) + light/medium rows finished in place
__device__ __noinline__ LocalCnt pr_pull_tiered_a(const PrPullOp op, const Adj g, const Tiers tiers, int n) {
    LocalCnt cnt;
    const unsigned lane = lane_id();
    const long long NW = gwarps();
    // grid tier: kHeavy-edge blocks of heavy rows
    const unsigned nblk = tiers.nheavy ? tiers.hblk[tiers.nheavy] : 0u;
    for (long long blk = gwarp(); blk < nblk; blk += NW) {
        // row r: last r with hblk[r] <= blk
        unsigned lo = 0, hi = tiers.nheavy - 1;
        while (lo < hi) { unsigned mid = (lo + hi + 1) >> 1; if (tiers.hblk[mid] <= blk) lo = mid; else hi = mid - 1; }
        const unsigned v = tiers.heavy[lo];
        const uint32_t rb = __ldg(g.off + v), re = __ldg(g.off + v + 1);
        const uint32_t b = rb + (uint32_t)(blk - tiers.hblk[lo]) * kHeavy, e = min(re, b + kHeavy);
        double s = warp_row_sum(op.contrib, g.col, b, e, cnt.edges);
        if (lane == 0) atomicAdd(op.sum + v, s);
    }
    // light and medium rows: a warp takes 32 consecutive vertices
    for (long long wb = gwarp() * 32; wb < n; wb += NW * 32) {
        const int x = wb + lane < n ? (int)(wb + lane) : -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        const double r = warp_seg_rows(op, g, x, b, d < 32u ? d : 0u, cnt);
        if (x >= 0 && d < 32u) op.epi.finish(x, r, cnt.facc);
        unsigned med = __ballot_sync(0xffffffffu, x >= 0 && d >= 32u && d < kHeavy);
        while (med) {
            const int j = __ffs(med) - 1;
            med &= med - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), dj = __shfl_sync(0xffffffffu, d, j);
            const double s = warp_row_sum(op.contrib, g.col, bj, bj + dj, cnt.edges);
            if ((int)lane == j) op.epi.finish(x, s, cnt.facc);
        }
    }
    return cnt;
}

// phase B (after a grid barrier): finish the heavy rows from their accumulated block sums
__device__ __forceinline__ void pr_pull_tiered_b(const PrPullOp &op, const Tiers &tiers, LocalCnt &cnt) {
    for (long long i = gtid(); i < tiers.nheavy; i += gthreads()) {
        const unsigned v = tiers.heavy[i];
        const double s = op.sum[v];
        op.sum[v] = 0.0;
        op.epi.finish((int)v, s, cnt.facc);
    }
}

__device__ __forceinline__ DevCfg select_pr(const Features &f, const gsw_config &force) {
    DevCfg c = select_traversal(f, force);
    // every vertex and edge is active: pull (atomic-free); the AUTO choice (pull + STRICT) is
    // dispatched to pr_stream.cu by run_pr, so this kernel only runs forced combinations
    if (force.load_balance == GSW_AUTO) c.lb = GSW_LB_TWC;
    c.fmt = GSW_BITMAP;
    c.fused = GSW_FUSED;
    return c;
}

union PrSmem {
    LbSmem push;
    LbRedSmem pull;
};

__device__ __forceinline__ void flush_dangling(double v, double *dst) {
    __shared__ double s[kWarps];
    v = warp_sum(v);
    __syncthreads();
    if (lane_id() == 0) s[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int i = 0; i < kWarps; ++i) t += s[i];
        if (t != 0.0) atomicAdd(dst, t);
    }
}

__global__ void __launch_bounds__(kBlock, kMinBlocksPr) pr_kernel(PrArgs a) {
    __shared__ PrSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n;
    const double N = (double)n, d = a.damping;
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};

    // ---- init: pr_0 = 1/N -> contrib_0, D_0
    double dang = 0.0;
    for (long long v = gtid(); v < n; v += gthreads()) {
        uint32_t dg = __ldg(a.g.off + v + 1) - __ldg(a.g.off + v);
        a.contrib[0][v] = dg ? (1.0 / N) / (double)dg : 0.0;
        a.sum[v] = 0.0;
        if (!dg) dang += 1.0 / N;
        if (a.iters == 0) a.out[v] = 1.0 / N;         // uniform: order-free
    }
    for (long long i = gtid(); i <= a.iters; i += gthreads()) a.dsum[i] = 0.0;
    if (is_book()) *a.heavy_cnt = 0u;
    grid_sync(bar, epoch);
    flush_dangling(dang, a.dsum);
    // heavy-row table of the tiered pull (rows >= kHeavy in-edges): list, then block prefix
    Tiers tiers{a.heavy, a.hblk, 0u};
    tiered_build_p1(adj_in, n, tiers, a.heavy_cnt);
    grid_sync(bar, epoch);
    tiers.nheavy = cta_read_u32(a.heavy_cnt);
    tiered_build_p2(adj_in, tiers, red);
    grid_sync(bar, epoch);

    Book book;
    Features f = rc.base;
    f.Va = n; f.Ea = (long long)a.g.nnz; f.Via = 0; f.Eia = 0;
    f.maxd = 0; f.mind = 0;
    int t = 0;
    for (; t < a.iters; ++t) {
        if (is_book()) {
            book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
            if (t > 0) {
                book.bytes += 4ull * a.g.nnz + 20ull * n;
                book.edges += a.g.nnz;
                if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)a.g.nnz;
            }
        }
        f.iter = t;
        const DevCfg c = select_pr(f, rc.force);
        write_record(rc, t, c, f, 0u);
        if (is_book()) reset_cnt(rc.cnt + ((t + 2) % 3));
        __shared__ double sD;
        if (threadIdx.x == 0) sD = *(volatile const double *)(a.dsum + t);
        __syncthreads();
        const double D = sD;
        const PrEpi epi{a.g.off, a.g.perm, a.out, a.contrib[(t + 1) & 1], (1.0 - d) / N + d * D / N, d, t == a.iters - 1};
        const double *cur = a.contrib[t & 1];
        if (is_book()) book_expand(book);
        LocalCnt lc;
        bool owner = false;
        if (c.dir == GSW_PULL && c.lb == GSW_LB_TWC) {
            const PrPullOp op{cur, a.sum, epi, true};
            lc = pr_pull_tiered_a(op, adj_in, tiers, n);
            grid_sync(bar, epoch);
            pr_pull_tiered_b(op, tiers, lc);
            owner = true;
        } else if (c.dir == GSW_PULL) {
            owner = c.lb == GSW_LB_THREAD || c.lb == GSW_LB_WM;
            const PrPullOp op{cur, a.sum, epi, owner};
            lc = run_lb_reduce(c.lb, AllSrc{(unsigned)n}, adj_in, op, sm.pull, red, bar, epoch, rc.partial, a.scan);
        } else {
            const PrPushOp op{cur, a.sum};
            lc = run_lb(c.lb, AllSrc{(unsigned)n}, adj_out, op, sm.push, red, bar, epoch, rc.partial, a.scan);
        }
        if (!owner) {
            // accumulator epilogue: pr_{t+1} from the summed contributions
            grid_sync(bar, epoch);
            for (long long v = gtid(); v < n; v += gthreads()) {
                double s = a.sum[v];
                a.sum[v] = 0.0;
                epi.finish((int)v, s, lc.facc);
            }
        }
        flush_dangling(lc.facc, a.dsum + t + 1);
        grid_sync(bar, epoch);
    }
    if (is_book()) {
        if (t > 0) {
            book.bytes += 4ull * a.g.nnz + 20ull * n;
            book.edges += a.g.nnz;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)a.g.nnz;
        }
        book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
        book_finish(book, rc, t);
    }
}

gsw_status run_pr_stream(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st);
gsw_status run_pr_blocked(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st);
bool pr_blocked_wanted(gsw_graph g);

gsw_status run_pr(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st) {
    const int n = g->g.n;
    if (!rank) { set_error("gsw_pr: rank is NULL"); return GSW_EINVAL; }
    if (iters < 0 || iters > kMaxHist - 2) { set_error("gsw_pr: iters out of range"); return GSW_EINVAL; }
    if (!(damping >= 0.0 && damping <= 1.0)) { set_error("gsw_pr: damping must be in [0,1]"); return GSW_EINVAL; }
    // Every iteration of PR has the same features (Va = N, Ea = nnz), so select_pr's decision is the
    // same for all of them and is taken here once: pull + STRICT runs the edge-tiled stream kernel
    // (pr_stream.cu); every other forced combination runs pr_kernel below.
    {
        const gsw_config &fc = g->forced;
        const int dir = fc.direction != GSW_AUTO ? fc.direction : GSW_PULL;
        const int lb = fc.load_balance != GSW_AUTO ? fc.load_balance : GSW_LB_STRICT;
        // AUTO on graphs whose contributions overflow L2: the source-blocked gather (pr_blocked.cu)
        if (fc.direction == GSW_AUTO && fc.load_balance == GSW_AUTO && pr_blocked_wanted(g))
            return run_pr_blocked(g, damping, iters, rank, st);
        if (dir == GSW_PULL && lb == GSW_LB_STRICT) return run_pr_stream(g, damping, iters, rank, st);
    }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(rank) == 1;
    PrArgs a{};
    a.g = g->g;
    a.damping = damping;
    a.iters = iters;
    a.out = dev_out ? rank : (double *)ws.take((size_t)n * 8);
    a.contrib[0] = (double *)ws.take((size_t)n * 8);
    a.contrib[1] = (double *)ws.take((size_t)n * 8);
    a.sum = (double *)ws.take((size_t)n * 8);
    a.dsum = (double *)ws.take((size_t)(iters + 1) * 8);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    const size_t nh = std::min<size_t>((size_t)n, (size_t)g->g.nnz / kHeavy + 1);
    a.heavy = (unsigned *)ws.take(nh * 4);
    a.hblk = (unsigned *)ws.take((nh + 1) * 4);
    a.heavy_cnt = (unsigned *)ws.take(256);
    LaunchInfo li;
    gsw_status s = prepare_common(g, ws, (const void *)pr_kernel, a.rc, li, kMinBlocksPr);
    if (s != GSW_OK) return s;
    if (!a.out || !a.contrib[1] || !a.sum || !a.dsum || !a.scan || !a.heavy || !a.hblk || !a.heavy_cnt) { set_error("workspace too small"); return GSW_ENOMEM; }
    void *args[] = {&a};
    s = launch_persistent(g, (const void *)pr_kernel, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank, a.out, (size_t)n * 8, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
