// lb_reduce.cuh -- the load-balance candidates of Pattern 3 for Expands whose
// per-vertex update is a reduction over its edges (pull "via a reduction operation"):
// CC min-label, PageRank sums, SSSP relaxation minimum, BC dependency sums.
//   RedOp interface:
//     using Probe, Acc (Acc is a 64-bit POD: unsigned long long or double)
//     static Acc identity(); static Acc combine(Acc, Acc)
//     bool  skip(int x)
//     Probe probe(int x, uint32 e, int y)       the load(s) of edge e = (x, y)
//     Acc   val(int x, uint32 e, int y, Probe)  the edge's contribution (identity to ignore it)
//     void  flush(int x, Acc a, bool exclusive, LocalCnt&)   apply the reduced value to x;
//           exclusive = this call carries the reduction of ALL of x's edges (owner mappings), else
//           a partial that must be combined atomically (edge-parallel mappings: seg_reduce)
//   THREAD, TWC (thread/warp/CTA tiers) and WM own whole rows and flush once per row (the TWC
//   thread tier and WM reduce short rows with a warp-segmented scan); CM and STRICT split rows
//   across threads and flush partials (STRICT merges runs of the same row first).
#pragma once
#include "engine.cuh"
#include "lb.cuh"

namespace gsw {

template <class T>
__device__ __forceinline__ T shfl_xor_any(T v, int o) {
    return __shfl_xor_sync(0xffffffffu, v, o);
}

template <class Op>
__device__ __forceinline__ typename Op::Acc warp_combine(typename Op::Acc a) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a = Op::combine(a, shfl_xor_any(a, o));
    return a;
}

// ------------------------------------------------------------------ warp-segmented row batch
// A warp reduces the rows of its 32 lanes (lane r owns row x_r with edges [b_r, b_r + d_r)) edge-
// parallel: the warp walks the concatenated edge list 64 edges at a time (two 32-edge chunks in
// flight), each lane loads one edge per chunk, a 5-step segmented shuffle scan sums runs of the
// same row, and lane r collects its row's run total.  All lanes stay busy regardless of the degree
// mix (the per-thread serial loop idles lanes on skewed short rows).  Returns lane r's row total.
template <class Op>
__device__ __forceinline__ typename Op::Acc warp_seg_rows(const Op &op, const Adj &g, int x, uint32_t b, uint32_t d,
                                                          LocalCnt &cnt) {
    using Acc = typename Op::Acc;
    const unsigned lane = lane_id();
    const uint32_t incl = warp_incl_scan(d);
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    const uint32_t excl = incl - d;
    Acc acc = Op::identity();
    for (uint32_t k0 = 0; k0 < total; k0 += 64) {
        uint32_t kk[2];
        unsigned jj[2];
        int xs[2], ys[2];
        uint32_t es[2];
        bool ok[2];
        typename Op::Probe p[2];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            kk[h] = k0 + 32 * h + lane;
            unsigned lo = 0, hi = 31;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                unsigned mid = (lo + hi) >> 1;
                uint32_t v = __shfl_sync(0xffffffffu, incl, mid);
                if (v > kk[h]) hi = mid; else lo = mid + 1;
            }
            jj[h] = lo;
            xs[h] = __shfl_sync(0xffffffffu, x, lo);
            const uint32_t bb = __shfl_sync(0xffffffffu, b, lo), ex = __shfl_sync(0xffffffffu, excl, lo);
            es[h] = bb + (kk[h] - ex);
            ok[h] = kk[h] < total;
        }
#pragma unroll
        for (int h = 0; h < 2; ++h) ys[h] = ok[h] ? __ldg(g.col + es[h]) : 0;
#pragma unroll
        for (int h = 0; h < 2; ++h) if (ok[h]) p[h] = op.probe(xs[h], es[h], ys[h]);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            Acc v = ok[h] ? op.val(xs[h], es[h], ys[h], p[h]) : Op::identity();
            if (ok[h]) cnt.edges++;
            // segmented inclusive scan over runs of equal row index
#pragma unroll
            for (int s = 1; s < 32; s <<= 1) {
                Acc o = __shfl_up_sync(0xffffffffu, v, s);
                unsigned oj = __shfl_up_sync(0xffffffffu, jj[h], s);
                if (lane >= (unsigned)s && oj == jj[h]) v = Op::combine(v, o);
            }
            // row `lane` collects the run that ends inside this chunk
            const uint32_t c0 = k0 + 32 * h, c1 = min(c0 + 32, total);
            const uint32_t lo = max(excl, c0), hi = min(incl, c1);
            const unsigned src = hi > lo ? hi - 1 - c0 : 0u;
            Acc tv = __shfl_sync(0xffffffffu, v, src);
            if (hi > lo) acc = Op::combine(acc, tv);
        }
    }
    return acc;
}

// ------------------------------------------------------------------ THREAD (owner, ILP cursors)
template <class Src, class Op>
__device__ __noinline__ LocalCnt lbr_thread(const Src src, const Adj g, Op op) {
    LocalCnt cnt;
    using Acc = typename Op::Acc;
    const unsigned sz = src.size();
    const long long T = gthreads();
    for (long long base = gtid(); base < sz; base += kIlp * T) {
        int x[kIlp];
        uint32_t e[kIlp], end[kIlp];
        Acc acc[kIlp];
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            long long i = base + j * T;
            int v = i < sz ? src.get((unsigned)i) : -1;
            if (v >= 0 && op.skip(v)) v = -1;
            x[j] = v;
            acc[j] = Op::identity();
        }
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            e[j] = x[j] >= 0 ? __ldg(g.off + x[j]) : 0u;
            end[j] = x[j] >= 0 ? __ldg(g.off + x[j] + 1) : 0u;
        }
        for (;;) {
            bool ok[kIlp], any = false;
#pragma unroll
            for (int j = 0; j < kIlp; ++j) { ok[j] = e[j] < end[j]; any |= ok[j]; }
            if (!any) break;
            int y[kIlp];
            typename Op::Probe p[kIlp];
#pragma unroll
            for (int j = 0; j < kIlp; ++j) y[j] = ok[j] ? __ldg(g.col + e[j]) : 0;
#pragma unroll
            for (int j = 0; j < kIlp; ++j) if (ok[j]) p[j] = op.probe(x[j], e[j], y[j]);
#pragma unroll
            for (int j = 0; j < kIlp; ++j)
                if (ok[j]) { cnt.edges++; acc[j] = Op::combine(acc[j], op.val(x[j], e[j], y[j], p[j])); ++e[j]; }
        }
#pragma unroll
        for (int j = 0; j < kIlp; ++j) if (x[j] >= 0) op.flush(x[j], acc[j], true, cnt);
    }
    return cnt;
}

// ------------------------------------------------------------------ TWC (owner tiers)
struct TwcRedSmem {
    TwcElect el;                     // lb.cuh: race-free CTA-tier election
    unsigned long long part[kWarps];
};
template <class Src, class Op>
__device__ __noinline__ LocalCnt lbr_twc(const Src src, const Adj g, Op op, TwcRedSmem *sm) {
    LocalCnt cnt;
    using Acc = typename Op::Acc;
    static_assert(sizeof(Acc) == 8, "64-bit accumulators");
    const unsigned sz = src.size();
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    constexpr int kTile = kBlock * kIlp;
    unsigned round = 0;
    for (long long base = (long long)blockIdx.x * kTile; base < sz; base += (long long)gridDim.x * kTile) {
        int x[kIlp];
        uint32_t b[kIlp], e[kIlp];
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            long long i = base + j * kBlock + threadIdx.x;
            int v = i < sz ? src.get((unsigned)i) : -1;
            if (v >= 0 && op.skip(v)) v = -1;
            x[j] = v;
        }
        uint32_t d0[kIlp];
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            b[j] = x[j] >= 0 ? __ldg(g.off + x[j]) : 0u;
            e[j] = x[j] >= 0 ? __ldg(g.off + x[j] + 1) : 0u;
            d0[j] = e[j] - b[j];
        }
        // CTA tier: degree >= blockDim
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            for (;;) {
                int xx;
                uint32_t bb, ee;
                if (!twc_elect(sm->el, round, x[j], b[j], e[j], xx, bb, ee)) break;
                Acc a = Op::identity();
                for (uint32_t k0 = bb; k0 < ee; k0 += 2 * kBlock) {
                    uint32_t k[2] = {k0 + threadIdx.x, k0 + kBlock + threadIdx.x};
                    int y[2];
                    typename Op::Probe p[2];
#pragma unroll
                    for (int h = 0; h < 2; ++h) y[h] = k[h] < ee ? __ldg(g.col + k[h]) : 0;
#pragma unroll
                    for (int h = 0; h < 2; ++h) if (k[h] < ee) p[h] = op.probe(xx, k[h], y[h]);
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (k[h] < ee) { cnt.edges++; a = Op::combine(a, op.val(xx, k[h], y[h], p[h])); }
                }
                a = warp_combine<Op>(a);
                if (lane == 0) sm->part[wid] = *reinterpret_cast<unsigned long long *>(&a);
                __syncthreads();
                if (threadIdx.x == 0) {
                    Acc t = Op::identity();
                    for (int w = 0; w < kWarps; ++w) t = Op::combine(t, *reinterpret_cast<Acc *>(&sm->part[w]));
                    op.flush(xx, t, true, cnt);
                }
                __syncthreads();
            }
        }
        // warp tier: 32 <= degree < blockDim
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            for (;;) {
                unsigned m = __ballot_sync(0xffffffffu, e[j] - b[j] >= 32u);
                if (!m) break;
                const int leader = __ffs(m) - 1;
                const int xx = __shfl_sync(0xffffffffu, x[j], leader);
                const uint32_t bb = __shfl_sync(0xffffffffu, b[j], leader), ee = __shfl_sync(0xffffffffu, e[j], leader);
                if ((int)lane == leader) e[j] = b[j];
                Acc a = Op::identity();
                for (uint32_t k0 = bb; k0 < ee; k0 += 64) {
                    uint32_t k[2] = {k0 + lane, k0 + 32 + lane};
                    int y[2];
                    typename Op::Probe p[2];
#pragma unroll
                    for (int h = 0; h < 2; ++h) y[h] = k[h] < ee ? __ldg(g.col + k[h]) : 0;
#pragma unroll
                    for (int h = 0; h < 2; ++h) if (k[h] < ee) p[h] = op.probe(xx, k[h], y[h]);
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (k[h] < ee) { cnt.edges++; a = Op::combine(a, op.val(xx, k[h], y[h], p[h])); }
                }
                a = warp_combine<Op>(a);
                if ((int)lane == leader) op.flush(xx, a, true, cnt);
            }
        }
        // thread tier (degree < 32): the warp reduces its lanes' short rows edge-parallel
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            const bool own = x[j] >= 0 && d0[j] < 32u;
            const Acc r = warp_seg_rows(op, g, x[j], b[j], own ? d0[j] : 0u, cnt);
            if (own && (d0[j] > 0u || Op::kFlushEmpty)) op.flush(x[j], r, true, cnt);
        }
    }
    return cnt;
}

// ------------------------------------------------------------------ WM / CM / STRICT (edge-parallel)
template <class Op, int K>
__device__ __forceinline__ void red_edges(const Op &op, const Adj &g, const int (&x)[K], const uint32_t (&e)[K],
                                          const bool (&ok)[K], LocalCnt &cnt) {
    int y[K];
    typename Op::Probe p[K];
#pragma unroll
    for (int j = 0; j < K; ++j) y[j] = ok[j] ? __ldg(g.col + e[j]) : 0;
#pragma unroll
    for (int j = 0; j < K; ++j) if (ok[j]) p[j] = op.probe(x[j], e[j], y[j]);
#pragma unroll
    for (int j = 0; j < K; ++j)
        if (ok[j]) { cnt.edges++; op.flush(x[j], op.val(x[j], e[j], y[j], p[j]), false, cnt); }
}

template <class Src, class Op>
__device__ __noinline__ LocalCnt lbr_wm(const Src src, const Adj g, Op op) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    const unsigned lane = lane_id();
    for (long long wb = gwarp() * 32; wb < sz; wb += gwarps() * 32) {
        long long i = wb + lane;
        int x = i < sz ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        // WM: the warp's 32 consecutive rows, warpsize edges at a time, log2(32)-step
        // search for each edge's row -- reduced per row and flushed by the row's lane
        const typename Op::Acc r = warp_seg_rows(op, g, x, b, d, cnt);
        (void)lane;
        if (x >= 0 && (d > 0 || Op::kFlushEmpty)) op.flush(x, r, true, cnt);
    }
    return cnt;
}

template <class Src, class Op>
__device__ __noinline__ LocalCnt lbr_cm(const Src src, const Adj g, Op op, CmSmem *sm) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    for (long long cb = (long long)blockIdx.x * kBlock; cb < sz; cb += (long long)gridDim.x * kBlock) {
        long long i = cb + threadIdx.x;
        int x = i < sz ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        if (Op::kFlushEmpty && x >= 0 && d == 0) op.flush(x, Op::identity(), true, cnt);
        uint32_t total;
        uint32_t excl = block_excl_scan(d, sm->scan_tmp, &total);
        sm->excl[threadIdx.x] = excl;
        sm->beg[threadIdx.x] = b;
        sm->x[threadIdx.x] = x;
        __syncthreads();
        for (uint32_t k0 = 0; k0 < total; k0 += 2 * kBlock) {
            int xs[2];
            uint32_t es[2];
            bool ok[2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                uint32_t k = k0 + h * kBlock + threadIdx.x;
                ok[h] = k < total;
                xs[h] = -1; es[h] = 0;
                if (ok[h]) {
                    unsigned lo = 0, hi = kBlock - 1;
                    while (lo < hi) {
                        unsigned mid = (lo + hi + 1) >> 1;
                        if (sm->excl[mid] <= k) lo = mid; else hi = mid - 1;
                    }
                    xs[h] = sm->x[lo];
                    es[h] = sm->beg[lo] + (k - sm->excl[lo]);
                }
            }
            red_edges<Op, 2>(op, g, xs, es, ok, cnt);
        }
        __syncthreads();
    }
    return cnt;
}

// STRICT: merge-path tiles (lb.cuh); each thread's kStrictVT consecutive diagonals are reduced
// locally per row (seg_reduce) and flushed at row changes.
template <class Src, class Op>
__device__ __noinline__ LocalCnt lbr_strict(const Src src, const Adj g, Op op, const uint32_t *scan, uint32_t total,
                                            StrictSmem *sm) {
    LocalCnt cnt;
    using Acc = typename Op::Acc;
    const unsigned sz = src.size();
    const unsigned long long D = (unsigned long long)sz + total;
    const unsigned long long ntiles = (D + kStrictTile - 1) / kStrictTile;
    for (unsigned long long t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const unsigned long long d0 = t * kStrictTile, d1 = min(D, d0 + kStrictTile);
        if (threadIdx.x == 0) sm->i0 = merge_path(scan, sz, total, d0);
        if (threadIdx.x == 32) sm->i1 = merge_path(scan, sz, total, d1);
        __syncthreads();
        const int i0 = sm->i0, i1 = sm->i1;
        const int ni = min(i1 + 1, (int)sz) - i0;
        for (int j = threadIdx.x; j <= ni; j += kBlock) sm->scan[j] = scan[i0 + j];
        for (int j = threadIdx.x; j < ni; j += kBlock) {
            int x = src.get(i0 + j);
            if (x >= 0 && op.skip(x)) x = -1;
            sm->x[j] = x;
            sm->beg[j] = x >= 0 ? __ldg(g.off + x) : 0u;
        }
        __syncthreads();
        const unsigned long long dd0 = min(d1, d0 + (unsigned long long)threadIdx.x * kStrictVT);
        const unsigned long long dd1 = min(d1, dd0 + kStrictVT);
        long long lo = dd0 > total ? (long long)(dd0 - total) - i0 : 0;
        if (lo < 0) lo = 0;
        long long hi = (long long)min((unsigned long long)sz, dd0) - i0;
        if (hi > ni) hi = ni;
        while (lo < hi) {
            long long mid = (lo + hi) >> 1;
            if ((unsigned long long)sm->scan[mid + 1] <= dd0 - 1 - (unsigned long long)(mid + i0)) lo = mid + 1;
            else hi = mid;
        }
        long long ii = lo;
        unsigned long long k = dd0 - (unsigned long long)(ii + i0);
        int xs[kStrictVT];
        uint32_t es[kStrictVT];
        bool ok[kStrictVT];
        long long item[kStrictVT];
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) {
            ok[s] = false; xs[s] = -1; es[s] = 0; item[s] = -1;
            unsigned long long dd = dd0 + s;
            if (dd < dd1) {
                if (ii < ni && (unsigned long long)sm->scan[ii + 1] <= k) {
                    // item ii ends at this diagonal; an empty item is flushed by its merge step
                    if (Op::kFlushEmpty && sm->scan[ii + 1] == sm->scan[ii] && sm->x[ii] >= 0)
                        op.flush(sm->x[ii], Op::identity(), true, cnt);
                    ++ii;
                } else {
                    int x = sm->x[ii];
                    xs[s] = x; item[s] = ii;
                    es[s] = sm->beg[ii] + (uint32_t)(k - sm->scan[ii]);
                    ok[s] = x >= 0;
                    ++k;
                }
            }
        }
        int y[kStrictVT];
        typename Op::Probe p[kStrictVT];
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) y[s] = ok[s] ? __ldg(g.col + es[s]) : 0;
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) if (ok[s]) p[s] = op.probe(xs[s], es[s], y[s]);
        Acc run = Op::identity();
        long long run_item = -1;
        int run_x = -1;
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) {
            if (!ok[s]) continue;
            cnt.edges++;
            if (item[s] != run_item) {
                if (run_item >= 0) op.flush(run_x, run, false, cnt);
                run = Op::identity(); run_item = item[s]; run_x = xs[s];
            }
            run = Op::combine(run, op.val(xs[s], es[s], y[s], p[s]));
        }
        if (run_item >= 0) op.flush(run_x, run, false, cnt);
        __syncthreads();
    }
    return cnt;
}

union LbRedSmem {
    TwcRedSmem twc;
    CmSmem cm;
    StrictSmem strict;
};

template <class Src, class Op>
__device__ __forceinline__ LocalCnt run_lb_reduce(int lb, const Src &src, const Adj &adj, const Op &op,
                                                  LbRedSmem &sm, uint32_t *red, const GridBarrier &bar,
                                                  unsigned &epoch, uint32_t *partial, uint32_t *scan) {
    switch (lb) {
    case GSW_LB_THREAD: return lbr_thread(src, adj, op);
    case GSW_LB_TWC: return lbr_twc(src, adj, op, &sm.twc);
    case GSW_LB_WM: return lbr_wm(src, adj, op);
    case GSW_LB_CM: return lbr_cm(src, adj, op, &sm.cm);
    default: {
        strict_scan_p1(src, adj, partial, red);
        grid_sync(bar, epoch);
        uint32_t total = strict_scan_p2(src, adj, partial, scan, red);
        grid_sync(bar, epoch);
        return lbr_strict(src, adj, op, scan, total, &sm.strict);
    }
    }
}

}  // namespace gsw

// ------------------------------------------------------------------ B200 tiered reduction (TWC)
// TWC re-tiered for B200 for reductions over a STATIC item set (every vertex, or every
// non-isolated vertex): rows < 32 edges -> warp-segmented scan (32 rows per warp); 32..kHeavy-1 ->
// one warp per row with 4 loads in flight per lane; >= kHeavy -> kHeavy-edge blocks shared by all
// warps of the grid, each flushed as a partial (exclusive = false).  Ops whose partial flush
// accumulates into a side buffer finish those rows after a grid barrier (tiered_finish).  The
// heavy-row table is built once per run (tiered_build, two phases).
namespace gsw {

constexpr uint32_t kHeavy = 1024;

struct Tiers {
    unsigned *heavy;        // heavy row ids
    unsigned *hblk;         // exclusive prefix of ceil(d/kHeavy) over heavy rows, hblk[nheavy] = total
    unsigned nheavy;
};

// phase 1 (all CTAs): list heavy rows (in-degree >= kHeavy) with warp-aggregated appends
__device__ __forceinline__ void tiered_build_p1(const Adj g, int n, Tiers t, unsigned *count) {
    q_from_pred((int *)t.heavy, count, n, [&](int v) { return __ldg(g.off + v + 1) - __ldg(g.off + v) >= kHeavy; });
}
// phase 2 (after a grid barrier; CTA 0 scans, the others return): block prefix
__device__ __forceinline__ void tiered_build_p2(const Adj g, Tiers t, uint32_t *red) {
    if (blockIdx.x != 0) return;
    uint32_t base = 0;
    for (unsigned t0 = 0; t0 < t.nheavy; t0 += kBlock) {
        const unsigned i = t0 + threadIdx.x;
        uint32_t c = 0;
        if (i < t.nheavy) {
            const unsigned v = t.heavy[i];
            c = (__ldg(g.off + v + 1) - __ldg(g.off + v) + kHeavy - 1) / kHeavy;
        }
        uint32_t tot;
        const uint32_t ex = block_excl_scan(c, red, &tot);
        if (i < t.nheavy) t.hblk[i] = base + ex;
        base += tot;
    }
    if (threadIdx.x == 0) t.hblk[t.nheavy] = base;
}

// one warp reduces the edges [b, e) of row x (4 loads in flight per lane)
template <class Op>
__device__ __forceinline__ typename Op::Acc warp_row_reduce(const Op &op, const Adj &g, int x, uint32_t b, uint32_t e,
                                                            unsigned long long &edges) {
    using Acc = typename Op::Acc;
    const unsigned lane = lane_id();
    Acc a = Op::identity();
    for (uint32_t k0 = b; k0 < e; k0 += 128) {
        int y[4];
        typename Op::Probe p[4];
#pragma unroll
        for (int h = 0; h < 4; ++h) { const uint32_t k = k0 + 32 * h + lane; y[h] = k < e ? __ldg(g.col + k) : -1; }
#pragma unroll
        for (int h = 0; h < 4; ++h) if (y[h] >= 0) p[h] = op.probe(x, k0 + 32 * h + lane, y[h]);
#pragma unroll
        for (int h = 0; h < 4; ++h)
            if (y[h] >= 0) { a = Op::combine(a, op.val(x, k0 + 32 * h + lane, y[h], p[h])); edges++; }
    }
    return warp_combine<Op>(a);
}

// items: vertices v in [0, n) with !skip(v) (isolated rows reduce to the identity)
template <class Op>
__device__ __noinline__ LocalCnt lbr_tiered(const Op op, const Adj g, const Tiers tiers, int n) {
    LocalCnt cnt;
    const unsigned lane = lane_id();
    const long long NW = gwarps();
    // grid tier
    const unsigned nblk = tiers.nheavy ? tiers.hblk[tiers.nheavy] : 0u;
    for (long long blk = gwarp(); blk < nblk; blk += NW) {
        unsigned lo = 0, hi = tiers.nheavy - 1;
        while (lo < hi) { const unsigned mid = (lo + hi + 1) >> 1; if (tiers.hblk[mid] <= blk) lo = mid; else hi = mid - 1; }
        const int v = (int)tiers.heavy[lo];
        if (op.skip(v)) continue;
        const uint32_t rb = __ldg(g.off + v), re = __ldg(g.off + v + 1);
        const uint32_t b = rb + (uint32_t)(blk - tiers.hblk[lo]) * kHeavy, e = min(re, b + kHeavy);
        const typename Op::Acc s = warp_row_reduce(op, g, v, b, e, cnt.edges);
        if (lane == 0) op.flush(v, s, false, cnt);
    }
    // light and medium rows: a warp takes 32 consecutive vertices
    for (long long wb = gwarp() * 32; wb < n; wb += NW * 32) {
        int x = wb + lane < n ? (int)(wb + lane) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        const typename Op::Acc r = warp_seg_rows(op, g, x, b, d < 32u ? d : 0u, cnt);
        if (x >= 0 && d < 32u && (d > 0u || Op::kFlushEmpty)) op.flush(x, r, true, cnt);
        unsigned med = __ballot_sync(0xffffffffu, x >= 0 && d >= 32u && d < kHeavy);
        while (med) {
            const int j = __ffs(med) - 1;
            med &= med - 1;
            const int xj = __shfl_sync(0xffffffffu, x, j);
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), dj = __shfl_sync(0xffffffffu, d, j);
            const typename Op::Acc s = warp_row_reduce(op, g, xj, bj, bj + dj, cnt.edges);
            if ((int)lane == j) op.flush(x, s, true, cnt);
        }
    }
    return cnt;
}

}  // namespace gsw
