// bc.cu -- betweenness centrality (Brandes [10], PAPER.md:265-266 [47]; generalised push/pull for
// BC) on the persistent Filter/Expand engine, all sources in one launch.
// Per source s:
//   forward : level-synchronous BFS that also counts shortest paths sigma (exact u64):
//             push  -- claim v with atomicCAS(depth, -1, l+1); sigma[v] += sigma[u] for every
//                      frontier u with depth[v] == l+1 (compAtomic);
//             pull  -- for unvisited v: sigma[v] = sum of sigma[u] over in-neighbours at level l
//                      (comp, a reduction; no early exit, every parent counts);
//             the visited vertices are appended level by level to the stack S (Filter output).
//   backward: for l = L-1 .. 1, for v in S_l: delta[v] = sigma[v] * sum over successors w
//             (depth[w] == l+1) of omega[w], omega[w] = (1 + delta[w]) / sigma[w];
//             bc[v] += delta[v].  Always pull (atomic-free reduction per vertex).
// bc is unnormalised: sum over the given sources, no halving for undirected graphs.
#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"
#include "lb_reduce.cuh"

namespace gsw {

struct BcArgs {
    DevGraph g;
    const unsigned *iso;
    const int *sources;   // device copy
    int nsrc;
    double *bc;           // internal order
    double *out;          // caller order (relabeled graphs), else nullptr
    int *depth;
    unsigned long long *sigma;
    double *omega;        // (1 + delta) / sigma
    double *dacc;         // accumulator for edge-parallel backward mappings
    unsigned *V;          // visited map (pull workload)
    int *S;               // BFS stack: vertices in level order
    unsigned *lvl_off;    // level boundaries in S (per source, reused)
    uint32_t *scan;
    unsigned *err;        // sigma overflow flag
    unsigned *heavy[2], *hblk[2], *heavy_cnt;   // tiered reductions: [0] in-edges, [1] out-edges
    RunCommon rc;
};

#ifndef GSW_BC_COND
#define GSW_BC_COND 1   // gather sigma / omega only for the edges whose depth matches (A/B knob)
#endif

struct BcProbe { int dv; unsigned su_lo, su_hi; };

// forward push
struct BcPushOp {
    int *depth;
    unsigned long long *sigma;
    unsigned *V;
    const uint32_t *off;
    int lvl1;
    CtaQueue S;
    struct Tok { int old; unsigned su_lo, su_hi; };
    using Probe = BcProbe;
    using Aux = uint2;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int u, uint32_t, int v) const {
        unsigned long long su = sigma[u];          // final: u is on level l
        return BcProbe{depth[v], (unsigned)su, (unsigned)(su >> 32)};
    }
    __device__ __forceinline__ Tok act(int, uint32_t, int v, Probe p) const {
        return Tok{p.dv == -1 ? atomicCAS(depth + v, -1, lvl1) : p.dv, p.su_lo, p.su_hi};
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int v, Tok t) const {
        return t.old == -1 ? make_uint2(__ldg(off + v), __ldg(off + v + 1)) : make_uint2(0u, 0u);
    }
    __device__ __forceinline__ bool commit(int, uint32_t, int v, Tok t, Aux d, LocalCnt &c) const {
        const bool won = t.old == -1;
        if (won || t.old == lvl1) atomicAdd(sigma + v, ((unsigned long long)t.su_hi << 32) | t.su_lo);
        if (won) {
            c.add_vertex(d.y - d.x);
            atomicOr(V + (v >> 5), 1u << (v & 31));
        }
        if (won) S.push(v);
        return false;
    }
};

// forward pull (reduction): sigma[v] = sum of sigma[u] over in-neighbours u at level l
struct BcPullOp {
    int *depth;
    unsigned long long *sigma;
    unsigned *V;
    const uint32_t *off;
    int lvl;
    CtaQueue S;
    using Probe = BcProbe;
    using Acc = unsigned long long;
    static constexpr bool kFlushEmpty = false;
    static __device__ __forceinline__ Acc identity() { return 0ull; }
    static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a + b; }
    // skip vertices settled BEFORE this level only: a vertex claimed during this phase (depth
    // l+1) must keep accumulating sigma from the rest of its parents (hub rows are split across
    // warps by the tiered mapping)
    __device__ __forceinline__ bool skip(int v) const {
        const int d = depth[v];
        return d >= 0 && d <= lvl;
    }
#if GSW_BC_COND
    // depth[u] first; sigma[u] (8 B) only for the parents on level lvl -- most scanned in-edges
    // of the wide pull levels are not parents, and the two gathers per edge were the level's cost
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const { return BcProbe{depth[u], 0u, 0u}; }
    __device__ __forceinline__ Acc val(int, uint32_t, int u, Probe p) const {
        return p.dv == lvl ? sigma[u] : 0ull;
    }
#else
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const {
        unsigned long long su = sigma[u];
        return BcProbe{depth[u], (unsigned)su, (unsigned)(su >> 32)};
    }
    __device__ __forceinline__ Acc val(int, uint32_t, int, Probe p) const {
        return p.dv == lvl ? (((unsigned long long)p.su_hi << 32) | p.su_lo) : 0ull;
    }
#endif
    __device__ __forceinline__ void flush(int v, Acc s, bool exclusive, LocalCnt &c) const {
        if (s == 0ull) return;
        bool won;
        if (exclusive) { depth[v] = lvl + 1; sigma[v] = s; won = true; }
        else { atomicAdd(sigma + v, s); won = atomicCAS(depth + v, -1, lvl + 1) == -1; }
        if (won) {
            atomicOr(V + (v >> 5), 1u << (v & 31));
            c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
            S.push(v);
        }
    }
};

// backward (reduction over successors): acc(v) = sum over w with depth[w] == l+1 of omega[w]
struct BcBackOp {
    const int *depth;
    const unsigned long long *sigma;
    double *omega;
    double *bc;
    double *dacc;
    int lvl;
    bool owner;
    bool by_level;        // items are all vertices; only those on level lvl take part
#if GSW_BC_COND
    using Probe = int;    // depth[w]; omega[w] is gathered in val() only for the successors
#else
    using Probe = double;
#endif
    using Acc = double;
    static constexpr bool kFlushEmpty = true;
    static __device__ __forceinline__ Acc identity() { return 0.0; }
    static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a + b; }
    __device__ __forceinline__ bool skip(int v) const { return by_level && depth[v] != lvl; }
#if GSW_BC_COND
    __device__ __forceinline__ Probe probe(int, uint32_t, int w) const { return depth[w]; }
    __device__ __forceinline__ Acc val(int, uint32_t, int w, Probe p) const { return p == lvl + 1 ? omega[w] : 0.0; }
#else
    __device__ __forceinline__ Probe probe(int, uint32_t, int w) const {
        const int dw = depth[w];
        const double ow = omega[w];                // issued together with depth[w]
        return dw == lvl + 1 ? ow : 0.0;
    }
    __device__ __forceinline__ Acc val(int, uint32_t, int, Probe p) const { return p; }
#endif
    __device__ __forceinline__ void finish(int v, double a) const {
        double sv = (double)sigma[v];
        double dv = sv * a;
        omega[v] = (1.0 + dv) / sv;
        bc[v] += dv;
    }
    __device__ __forceinline__ void flush(int v, Acc a, bool exclusive, LocalCnt &) const {
        if (owner && exclusive) finish(v, a);
        else if (a != 0.0) atomicAdd(dacc + v, a);
    }
};

union BcSmem {
    LbSmem push;
    LbRedSmem pull;
};

__global__ void __launch_bounds__(kBlock, kMinBlocksBc) bc_kernel(BcArgs a) {
    __shared__ BcSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    __shared__ CtaQStore qs;              // staged appends to the BFS stack S
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5;
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};

    for (long long v = gtid(); v < n; v += gthreads()) a.bc[v] = 0.0;
    if (is_book()) { a.heavy_cnt[0] = 0u; a.heavy_cnt[32] = 0u; }
    cta_queue_reset(qs);
    grid_sync(bar, epoch);
    // heavy-row tables of the tiered reductions (forward pull: in-edges, backward: out-edges)
    const bool sym = a.g.in_off == a.g.off;
    Tiers tin{a.heavy[0], a.hblk[0], 0u}, tout{a.heavy[1], a.hblk[1], 0u};
    tiered_build_p1(adj_in, n, tin, a.heavy_cnt);
    if (!sym) tiered_build_p1(adj_out, n, tout, a.heavy_cnt + 32);
    grid_sync(bar, epoch);
    tin.nheavy = cta_read_u32(a.heavy_cnt);
    tiered_build_p2(adj_in, tin, red);
    if (sym) tout = tin;
    else {
        tout.nheavy = cta_read_u32(a.heavy_cnt + 32);
        tiered_build_p2(adj_out, tout, red);
    }
    grid_sync(bar, epoch);
    Book book;
    Features f = rc.base;
    int t = 0;                          // global iteration counter (records)
    for (int k = 0; k < a.nsrc; ++k) {
        const int src = map_in(a.g.inv, a.sources[k]);
        // ---- per-source init
        for (long long v = gtid(); v < n; v += gthreads()) {
            a.depth[v] = v == src ? 0 : -1;
            a.sigma[v] = v == src ? 1ull : 0ull;
            a.omega[v] = 0.0;
            a.dacc[v] = 0.0;
        }
        for (long long w = gtid(); w < W; w += gthreads()) {
            unsigned x = a.iso[w];
            if (w == (src >> 5)) x |= 1u << (src & 31);
            a.V[w] = x;
        }
        const unsigned dsrc = __ldg(a.g.off + src + 1) - __ldg(a.g.off + src);
        if (is_book()) {
            for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + ((t + i) % 3));
            IterCnt *c0 = rc.cnt + (t % 3);
            c0->va = 1; c0->ea = dsrc; c0->maxd = dsrc; c0->mind = dsrc;
            a.S[0] = src;
            a.lvl_off[0] = 0; a.lvl_off[1] = 1;
        }
        grid_sync(bar, epoch);
        // ---- forward
        long long Via = (long long)n - 1, Eia = (long long)a.g.nnz - dsrc;
        int L = 0;                      // levels
        unsigned send = 1;              // |S| so far
        for (int lvl = 0;; ++lvl, ++t) {
            IterCnt *cur = rc.cnt + (t % 3), *nxt = rc.cnt + ((t + 1) % 3);
            if (is_book()) book_start(book, rc, t, nxt);
            const CntView cv = cta_read_cnt(cur);
            if (is_book() && t > 0) {
                book.edges += cv.edges;
                book.bytes += 16ull * cv.va + 12ull * cv.edges;
                if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)cv.edges;
            }
            if (cv.va == 0) { L = lvl; break; }
            if (lvl > 0) { Via -= (long long)cv.va; Eia -= (long long)cv.ea; }
            f.Va = (long long)cv.va; f.Ea = (long long)cv.ea; f.Via = Via; f.Eia = Eia;
            f.maxd = cv.maxd; f.mind = cv.mind; f.iter = t;
            hist_features(cv, f);
            DevCfg c = select_traversal(f, rc.force);
            if (c.dir == GSW_PULL && rc.force.load_balance == GSW_AUTO) c.lb = GSW_LB_TWC;
            write_record(rc, t, c, f, 0u);
            if (is_book()) reset_cnt(rc.cnt + ((t + 2) % 3));
            const unsigned lbeg = send - (unsigned)cv.va;          // level lvl occupies S[lbeg, send)
            if (is_book()) book_expand(book);
            LocalCnt lc;
            // next level is appended at S[send ...); its counter lives in the next slot's qlen
            const CtaQueue sq = cta_queue(qs, a.S + send, &nxt->qlen);
            if (c.dir == GSW_PUSH) {
                const BcPushOp op{a.depth, a.sigma, a.V, a.g.off, lvl + 1, sq};
                lc = run_lb(c.lb, QueueSrc{a.S + lbeg, (unsigned)cv.va}, adj_out, op, sm.push, red, bar, epoch,
                            rc.partial, a.scan);
            } else {
                const BcPullOp op{a.depth, a.sigma, a.V, a.g.off, lvl, sq};
                if (c.lb == GSW_LB_TWC)
                    lc = lbr_tiered(op, adj_in, tin, n);      // B200 TWC (skip = visited)
                else
                    lc = run_lb_reduce(c.lb, BitmapSrc{a.V, (unsigned)n, 0u}, adj_in, op, sm.pull, red, bar, epoch,
                                       rc.partial, a.scan);
            }
            cta_queue_flush(qs, a.S + send, &nxt->qlen);
            flush_counts(lc, nxt);
            grid_sync(bar, epoch);
            // the next level's size is its Va (read at the top of the next iteration)
            __shared__ unsigned s_next;
            if (threadIdx.x == 0) s_next = *(volatile unsigned *)&nxt->va;
            __syncthreads();
            send += s_next;
            if (is_book() && lvl + 2 < kMaxHist) a.lvl_off[lvl + 2] = send;
            __syncthreads();
        }
        // ---- backward: levels L-1 .. 1
        unsigned hi = send;
        for (int lvl = L - 1; lvl >= 1; --lvl, ++t) {
            // level lvl occupies S[lo, hi): lo = hi - |level| (level sizes recomputed from depth)
            __shared__ unsigned s_lo;
            if (threadIdx.x == 0) s_lo = a.lvl_off[lvl];
            __syncthreads();
            const unsigned lo = s_lo;
            __syncthreads();
            if (is_book()) {
                book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
                book_expand(book);
                if (t < kMaxHist) {
                    gsw_iter_record r{};
                    r.iteration = t; r.direction = GSW_PULL; r.format = GSW_QUEUE;
                    r.load_balance = rc.force.load_balance ? rc.force.load_balance : GSW_LB_TWC;
                    r.fusion = GSW_FUSED; r.Va = hi - lo;
                    rc.rec[t] = r;
                }
            }
            const int lb = rc.force.load_balance ? rc.force.load_balance : GSW_LB_TWC;
            const bool owner = lb == GSW_LB_THREAD || lb == GSW_LB_TWC || lb == GSW_LB_WM;
            LocalCnt lc;
            if (lb == GSW_LB_TWC) {
                // B200 TWC over every vertex of the level (skip others); hub rows are reduced by the
                // grid tier into dacc and finished after a barrier
                const BcBackOp op{a.depth, a.sigma, a.omega, a.bc, a.dacc, lvl, true, true};
                lc = lbr_tiered(op, adj_out, tout, n);
                grid_sync(bar, epoch);
                for (long long i = gtid(); i < tout.nheavy; i += gthreads()) {
                    const int v = (int)tout.heavy[i];
                    if (a.depth[v] != lvl) continue;
                    const double s = a.dacc[v];
                    a.dacc[v] = 0.0;
                    op.finish(v, s);
                }
            } else {
            const BcBackOp op{a.depth, a.sigma, a.omega, a.bc, a.dacc, lvl, owner, false};
            lc = run_lb_reduce(lb, QueueSrc{a.S + lo, hi - lo}, adj_out, op, sm.pull, red, bar, epoch,
                               rc.partial, a.scan);
            if (!owner) {
                grid_sync(bar, epoch);
                for (long long i = gtid(); i < hi - lo; i += gthreads()) {
                    int v = a.S[lo + i];
                    double s = a.dacc[v];
                    a.dacc[v] = 0.0;
                    op.finish(v, s);
                }
            }
            }
            flush_counts(lc, rc.cnt + ((t + 1) % 3));
            grid_sync(bar, epoch);
            if (is_book()) {
                // backward edges: read from the slot just flushed (plain load after the barrier)
                unsigned long long e = rc.cnt[(t + 1) % 3].edges;
                book.edges += e;
                book.bytes += 4ull * e + 24ull * (hi - lo);
                if (t < kMaxHist) rc.rec[t].edges = (long long)e;
                reset_cnt(rc.cnt + ((t + 1) % 3));
            }
            hi = lo;
        }
        // sigma overflow check (exactness of the u64 path counts)
        for (long long v = gtid(); v < n; v += gthreads())
            if (a.sigma[v] >> 63) atomicOr(a.err, 1u);
        grid_sync(bar, epoch);
    }
    if (a.out) gather_out(a.out, a.bc, a.g.inv, n);
    if (is_book()) book_finish(book, rc, t);
}

gsw_status run_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc_out, gsw_run_stats *st) {
    const int n = g->g.n, W = (n + 31) / 32;
    if (!bc_out) { set_error("gsw_bc: bc is NULL"); return GSW_EINVAL; }
    if (nsrc < 0 || (nsrc > 0 && !sources)) { set_error("gsw_bc: bad sources"); return GSW_EINVAL; }
    if (is_device_ptr(sources) == 1) { set_error("gsw_bc: sources must be a host array"); return GSW_EINVAL; }
    for (int i = 0; i < nsrc; ++i)
        if (sources[i] < 0 || sources[i] >= n) { set_error("gsw_bc: source out of range"); return GSW_EINVAL; }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(bc_out) == 1;
    BcArgs a{};
    a.g = g->g;
    a.iso = g->iso;
    a.nsrc = nsrc;
    const bool relabeled = g->g.inv != nullptr;
    a.bc = (dev_out && !relabeled) ? bc_out : (double *)ws.take((size_t)n * 8);
    a.out = relabeled ? (dev_out ? bc_out : (double *)ws.take((size_t)n * 8)) : nullptr;
    a.depth = (int *)ws.take((size_t)n * 4);
    a.sigma = (unsigned long long *)ws.take((size_t)n * 8);
    a.omega = (double *)ws.take((size_t)n * 8);
    a.dacc = (double *)ws.take((size_t)n * 8);
    a.V = (unsigned *)ws.take((size_t)W * 4);
    a.S = (int *)ws.take((size_t)n * 4);
    a.lvl_off = (unsigned *)ws.take((size_t)kMaxHist * 4);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    a.err = (unsigned *)ws.take(256);
    const size_t nh = std::min<size_t>((size_t)n, (size_t)g->g.nnz / kHeavy + 1);
    for (int i = 0; i < 2; ++i) {
        a.heavy[i] = (unsigned *)ws.take(nh * 4);
        a.hblk[i] = (unsigned *)ws.take((nh + 1) * 4);
    }
    a.heavy_cnt = (unsigned *)ws.take(256);
    int *dsrc = (int *)ws.take((size_t)std::max(nsrc, 1) * 4);
    a.sources = dsrc;
    LaunchInfo li;
    gsw_status s = prepare_common(g, ws, (const void *)bc_kernel, a.rc, li, kMinBlocksBc);
    if (s != GSW_OK) return s;
    if (!a.bc || !a.depth || !a.sigma || !a.omega || !a.dacc || !a.V || !a.S || !a.lvl_off || !a.scan || !a.err || !dsrc ||
        !a.heavy[1] || !a.hblk[1] || !a.heavy_cnt) {
        set_error("workspace too small");
        return GSW_ENOMEM;
    }
    if (nsrc > 0) GSW_CUDA(cudaMemcpyAsync(dsrc, sources, (size_t)nsrc * 4, cudaMemcpyHostToDevice, g->stream));
    GSW_CUDA(cudaMemsetAsync(a.err, 0, 4, g->stream));
    void *args[] = {&a};
    s = launch_persistent(g, (const void *)bc_kernel, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out)
        GSW_CUDA(cudaMemcpyAsync(bc_out, relabeled ? a.out : a.bc, (size_t)n * 8, cudaMemcpyDeviceToHost, g->stream));
    s = finish_run(g, a.rc, li, st);
    if (s != GSW_OK) return s;
    unsigned herr = 0;
    GSW_CUDA(cudaMemcpy(&herr, a.err, 4, cudaMemcpyDeviceToHost));
    if (herr) { set_error("gsw_bc: a shortest-path count exceeded 2^63"); return GSW_EOVERFLOW; }
    return GSW_OK;
}

}  // namespace gsw
