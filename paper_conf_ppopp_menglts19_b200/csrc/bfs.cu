// bfs.cu -- BFS as GSWITCH Filter + Expand iterations (BFS functors Fig. 11,
// P:860-883) in one persistent cooperative kernel.  Every iteration t:
//   Inspector : read Va/Ea of the active set (counted by whoever activated the vertices), update
//               Via/Eia (Table 1), history times
//   Selector  : select_traversal() -> direction, LB, format, fusion
//   Filter    : materialise AS_t in the selected format unless the fused Expand of t-1 already
//               did (P5); standalone = regenerate from vertex status depth==t
//   Expand    : push (atomic claim = compAtomic) or pull (first active in-neighbour = comp, with
//               early exit, "edge skipping" Fig. 2) under the selected load balance
// Status (Fig. 11 filter): Active = depth==t, Inactive = depth<0 (not in the visited map),
// Fixed = visited earlier.  compAtomic = atomicExch in the paper is applied only to
// Inactive targets (reading R3): an atomicOr test-and-set on the visited bitmap.
#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"

namespace gsw {

enum { MAT_NONE = 0, MAT_QUEUE = 1, MAT_SQUEUE = 2, MAT_BITMAP = 3 };

struct BfsArgs {
    DevGraph g;
    const unsigned *iso;
    int src;
    int *depth;
    unsigned *V;          // visited map (isolated + padding bits pre-set)
    unsigned *fb[3];      // frontier bitmaps, ring of 3
    int *q[2];            // active-set queues, double buffered
    int *iq;              // inactive queue (pull workload in queue formats)
    uint32_t *scan;       // STRICT degree scan
    long long iso_count;
    RunCommon rc;
};

union TravSmem {
    TwcSmem twc;
    CmSmem cm;
    StrictSmem strict;
};

template <class Src, class Op>
__device__ __forceinline__ void run_lb(int lb, const Src &src, const Adj &adj, Op &op, LocalCnt &cnt, TravSmem &sm,
                                       uint32_t *red, const GridBarrier &bar, unsigned &epoch, uint32_t *partial,
                                       uint32_t *scan) {
    switch (lb) {
    case GSW_LB_THREAD: lb_thread(src, adj, op, cnt); break;
    case GSW_LB_TWC: lb_twc(src, adj, op, cnt, &sm.twc); break;
    case GSW_LB_WM: lb_wm(src, adj, op, cnt); break;
    case GSW_LB_CM: lb_cm(src, adj, op, cnt, &sm.cm); break;
    default: {
        strict_scan_p1(src, adj, partial, red);
        grid_sync(bar, epoch);
        uint32_t total = strict_scan_p2(src, adj, partial, scan, red);
        grid_sync(bar, epoch);
        lb_strict(src, adj, op, cnt, scan, total, &sm.strict);
    }
    }
}

// push: for active u and out-neighbour v, claim v if Inactive (compAtomic), depth[v] = lvl+1
struct BfsPushOp {
    int *depth;
    unsigned *V;
    const uint32_t *off;
    int lvl1;
    bool fused;
    int *nq;
    unsigned *nqlen;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ bool edge(int, uint32_t, int v, LocalCnt &c) const {
        bool won = false;
        if (!test_bit(V, v)) won = claim_bit(V, v);
        if (won) {
            depth[v] = lvl1;
            c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
        }
        if (fused) warp_append(nq, nqlen, won, v);
        return false;
    }
};

// pull: for inactive v, scan in-neighbours u; the first Active u gives depth[v] = lvl+1 (comp)
struct BfsPullOp {
    int *depth;
    unsigned *V;
    const uint32_t *off;      // out-offsets (degree of the newly activated vertex)
    const unsigned *fb;       // active-set bitmap, or nullptr -> test depth[u] == lvl
    int lvl;
    bool fused;
    unsigned *nfb;
    static constexpr bool kEarlyExit = true;
    __device__ __forceinline__ bool skip(int v) const { return test_bit_relaxed(V, v); }
    __device__ __forceinline__ bool edge(int v, uint32_t, int u, LocalCnt &c) const {
        bool act = fb ? test_bit(fb, u) : (depth[u] == lvl);
        if (!act) return false;
        if (claim_bit(V, v)) {
            depth[v] = lvl + 1;
            c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
            if (fused) atomicOr(nfb + (v >> 5), 1u << (v & 31));
        }
        return true;
    }
};

__global__ void __launch_bounds__(kBlock, kMinBlocks) bfs_kernel(BfsArgs a) {
    __shared__ TravSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5, src = a.src;
    int *depth = a.depth;
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};

    // ---- init: depth, visited map, frontier bitmaps, counters, AS_0 = {src}
    for (long long v = gtid(); v < n; v += gthreads()) depth[v] = (v == src) ? 0 : -1;
    for (long long w = gtid(); w < W; w += gthreads()) {
        unsigned x = a.iso[w];
        if (w == (src >> 5)) x |= 1u << (src & 31);
        a.V[w] = x;
        a.fb[0][w] = 0u; a.fb[1][w] = 0u; a.fb[2][w] = 0u;
    }
    const unsigned dsrc = a.g.off[src + 1] - a.g.off[src];
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
        rc.cnt[0].va = 1; rc.cnt[0].ea = dsrc; rc.cnt[0].maxd = dsrc; rc.cnt[0].mind = dsrc; rc.cnt[0].qlen = 1;
        a.q[0][0] = src;
    }
    grid_sync(bar, epoch);

    long long Via = (long long)n - 1, Eia = (long long)a.g.nnz - dsrc;
    int mat = MAT_SQUEUE;
    bool dirty[3] = {false, false, false};
    Features f = rc.base;
    int prev_dir = GSW_PUSH;
    long long prev_va = 0, prev_via = 0;
    int t = 0;
    for (;; ++t) {
        stamp_iteration_start(rc, t);
        IterCnt *cur = rc.cnt + (t % 3), *nxt = rc.cnt + ((t + 1) % 3);
        unsigned long long va, ea, edges_prev;
        unsigned maxd, mind, qlen;
        read_cnt(cur, va, ea, maxd, mind, qlen, edges_prev);
        if (blockIdx.x == 0 && threadIdx.x == 0 && t > 0) {
            // algorithmic bytes of iteration t-1 (DESIGN.md roofline model D0)
            unsigned long long b = prev_dir == GSW_PUSH
                ? 12ull * prev_va + 4ull * edges_prev + 8ull * va
                : (unsigned long long)n / 4 + 8ull * (unsigned long long)max(0LL, prev_via - a.iso_count) +
                      4ull * edges_prev + 4ull * va;
            rc.ctl->bytes_alg += b;
            rc.ctl->edges_total += edges_prev;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)edges_prev;
        }
        if (va == 0) break;
        if (t > 0) { Via -= (long long)va; Eia -= (long long)ea; }
        f.Va = (long long)va; f.Ea = (long long)ea; f.Via = Via; f.Eia = Eia;
        f.maxd = maxd; f.mind = mind; f.iter = t;
        read_hist(rc, t, f);
        DevCfg c = select_traversal(f, rc.force);
        write_record(rc, t, c, f, 0u);
        if (blockIdx.x == 0 && threadIdx.x == 0) reset_cnt(rc.cnt + ((t + 2) % 3));
        const int b2 = (t + 2) % 3;
        if (dirty[b2]) { clear_words(a.fb[b2], W); dirty[b2] = false; }

        // ---------------- Filter
        const bool push = c.dir == GSW_PUSH;
        int need;
        if (push) need = c.fmt == GSW_BITMAP ? MAT_BITMAP : (c.fmt == GSW_QUEUE ? MAT_QUEUE : MAT_SQUEUE);
        else need = c.fmt == GSW_BITMAP ? MAT_BITMAP : MAT_NONE;
        int *qa = a.q[t & 1];
        unsigned *fbt = a.fb[t % 3];
        bool filtered = false;
        const int lvl = t;
        auto is_active = [&](int v) { return depth[v] == lvl; };
        if (need == MAT_BITMAP && mat != MAT_BITMAP) {
            if (mat == MAT_QUEUE || mat == MAT_SQUEUE) bm_from_q(fbt, qa, qlen);
            else bm_from_pred(fbt, n, is_active);
            dirty[t % 3] = true;
            mat = MAT_BITMAP;
            filtered = true;
        } else if (need == MAT_QUEUE && mat != MAT_QUEUE && mat != MAT_SQUEUE) {
            if (mat == MAT_BITMAP) q_from_bm(qa, &cur->qlen, fbt, W, 0u);
            else q_from_pred(qa, &cur->qlen, n, is_active);
            mat = MAT_QUEUE;
            filtered = true;
        } else if (need == MAT_SQUEUE && mat != MAT_SQUEUE) {
            if (mat != MAT_BITMAP) {
                if (mat == MAT_QUEUE) bm_from_q(fbt, qa, qlen);
                else bm_from_pred(fbt, n, is_active);
                dirty[t % 3] = true;
                grid_sync(bar, epoch);
            }
            sq_from_bm_p1(fbt, W, 0u, rc.partial, red);
            grid_sync(bar, epoch);
            sq_from_bm_p2(qa, &cur->qlen, fbt, W, 0u, rc.partial, red);
            mat = MAT_SQUEUE;
            filtered = true;
        }
        if (!push && c.fmt != GSW_BITMAP) {               // inactive workload as a queue
            if (c.fmt == GSW_QUEUE) {
                q_from_bm(a.iq, &cur->iqlen, a.V, W, ~0u);
            } else {
                sq_from_bm_p1(a.V, W, ~0u, rc.partial, red);
                grid_sync(bar, epoch);
                sq_from_bm_p2(a.iq, &cur->iqlen, a.V, W, ~0u, rc.partial, red);
            }
            filtered = true;
        }
        if (filtered) grid_sync(bar, epoch);
        stamp_expand_start(rc);

        // ---------------- Expand
        LocalCnt lc;
        const bool fused = c.fused == GSW_FUSED;
        if (push) {
            BfsPushOp op{depth, a.V, a.g.off, t + 1, fused, a.q[(t + 1) & 1], &nxt->qlen};
            if (mat == MAT_BITMAP) {
                BitmapSrc s{fbt, (unsigned)n, 1u};
                run_lb(c.lb, s, adj_out, op, lc, sm, red, bar, epoch, rc.partial, a.scan);
            } else {
                QueueSrc s{qa, ld_relaxed(&cur->qlen)};
                run_lb(c.lb, s, adj_out, op, lc, sm, red, bar, epoch, rc.partial, a.scan);
            }
        } else {
            BfsPullOp op{depth, a.V, a.g.off, c.fmt == GSW_BITMAP ? fbt : nullptr, t, fused, a.fb[(t + 1) % 3]};
            if (c.fmt == GSW_BITMAP) {
                BitmapSrc s{a.V, (unsigned)n, 0u};
                run_lb(c.lb, s, adj_in, op, lc, sm, red, bar, epoch, rc.partial, a.scan);
            } else {
                QueueSrc s{a.iq, ld_relaxed(&cur->iqlen)};
                run_lb(c.lb, s, adj_in, op, lc, sm, red, bar, epoch, rc.partial, a.scan);
            }
            if (fused) dirty[(t + 1) % 3] = true;
        }
        flush_counts(lc, nxt);
        grid_sync(bar, epoch);
        mat = fused ? (push ? MAT_QUEUE : MAT_BITMAP) : MAT_NONE;
        prev_dir = c.dir;
        prev_va = (long long)va;
        prev_via = Via;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) rc.ctl->iters = (unsigned)t;
}

gsw_status run_bfs(gsw_graph g, int32_t source, int32_t *depth_out, gsw_run_stats *st) {
    const int n = g->g.n, W = (n + 31) / 32;
    if (!depth_out) { set_error("gsw_bfs: depth is NULL"); return GSW_EINVAL; }
    if (source < 0 || source >= n) { set_error("gsw_bfs: source out of range"); return GSW_EINVAL; }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(depth_out) == 1;
    BfsArgs a{};
    a.g = g->g;
    a.iso = g->iso;
    a.src = source;
    a.depth = dev_out ? depth_out : (int *)ws.take((size_t)n * 4);
    a.V = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 3; ++i) a.fb[i] = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 2; ++i) a.q[i] = (int *)ws.take((size_t)n * 4);
    a.iq = (int *)ws.take((size_t)n * 4);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    a.iso_count = g->attrs.isolated;
    LaunchInfo li;
    gsw_status s = prepare_common(g, ws, (const void *)bfs_kernel, a.rc, li);
    if (s != GSW_OK) return s;
    if (!a.depth || !a.V || !a.fb[2] || !a.q[1] || !a.iq || !a.scan) { set_error("workspace too small"); return GSW_ENOMEM; }
    void *args[] = {&a};
    s = launch_persistent(g, (const void *)bfs_kernel, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(depth_out, a.depth, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
