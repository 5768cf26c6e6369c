// lb.cuh -- Pattern 3, load balance (Fig. 6): how (item, edge) work of an
// Expand is mapped onto threads.  Every strategy is a device function used inside a persistent
// kernel phase, templated on
//   Src : the active set in its format (Pattern 2): size() item slots, get(i) -> vertex or -1
//   Op  : the algorithm's per-edge operation (emit + comp/compAtomic), split in two
//         so that several edges' loads are in flight per thread (memory-level parallelism):
//           bool  skip(int x)                          x needs no (more) work (pull early exit)
//           Probe probe(int x, uint32 e, int y)        the dependent load(s) of edge e=(x,y)
//           bool  apply(int x, uint32 e, int y, Probe, LocalCnt&)  update; true = x done
//           static constexpr bool kEarlyExit           stop scanning x once apply returned true
// Candidates:
//   THREAD : one thread per item, serial edge loop (the naive mapping the north_star lists);
//            kIlp independent items per thread are advanced in lock-step
//   TWC    : degree-binned thread / warp / CTA mapping (B40C [41])
//   WM     : a warp takes 32 consecutive items, 32-edge chunks, log2(32)-step search
//   CM     : a CTA takes blockDim items, blockDim-edge chunks, log2(blockDim) search
//   STRICT : equal (items+edges) per tile via merge-path over the degree scan ([13])
#pragma once
#include "common.cuh"
#include "gsw.h"

namespace gsw {

constexpr int kIlp = 4;

struct QueueSrc {
    const int *q;
    unsigned len;
    __device__ __forceinline__ unsigned size() const { return len; }
    __device__ __forceinline__ int get(unsigned i) const { return q[i]; }
};
// bitmap source: slot i is vertex i if its bit equals `want` (want=1: active set bitmap;
// want=0: the zero bits of the visited map = the inactive workload of pull)
struct BitmapSrc {
    const unsigned *bits;
    unsigned n;
    unsigned want;
    __device__ __forceinline__ unsigned size() const { return n; }
    __device__ __forceinline__ int get(unsigned i) const {
        return (((bits[i >> 5] >> (i & 31)) & 1u) == want) ? (int)i : -1;
    }
};
// every vertex is an item (dense workloads: PR, CC/SSSP pull over all vertices)
struct AllSrc {
    unsigned n;
    __device__ __forceinline__ unsigned size() const { return n; }
    __device__ __forceinline__ int get(unsigned i) const { return (int)i; }
};

struct Adj {
    const uint32_t *off;
    const int32_t *col;
};

// Process up to K edges (x[j], e[j]) (valid when ok[j]) in five stages, each issued for all K
// edges before the next consumes its results, so a thread keeps K independent memory chains in
// flight instead of waiting on one dependent round trip per edge:
//   1 y   = col[e]                       (adjacency load)
//   2 p   = op.probe(x, e, y)            (status load of the other endpoint)
//   3 tok = op.act(x, e, y, p)           (decision; may issue an atomic whose result is in tok)
//   4 aux = op.aux(x, e, y, tok)         (loads needed only by winners, e.g. a degree)
//   5 stop = op.commit(x, e, y, tok, aux, cnt)   (plain stores, counters; true = x done)
template <int K, class Op>
__device__ __forceinline__ void edge_batch(const Op &op, const Adj &g, const int (&x)[K], const uint32_t (&e)[K],
                                           const bool (&ok)[K], bool (&stop)[K], LocalCnt &cnt) {
    int y[K];
    typename Op::Probe p[K];
    typename Op::Tok tk[K];
    typename Op::Aux ax[K];
#pragma unroll
    for (int j = 0; j < K; ++j) y[j] = ok[j] ? __ldg(g.col + e[j]) : 0;
#pragma unroll
    for (int j = 0; j < K; ++j) if (ok[j]) p[j] = op.probe(x[j], e[j], y[j]);
#pragma unroll
    for (int j = 0; j < K; ++j) if (ok[j]) tk[j] = op.act(x[j], e[j], y[j], p[j]);
#pragma unroll
    for (int j = 0; j < K; ++j) if (ok[j]) ax[j] = op.aux(x[j], e[j], y[j], tk[j]);
#pragma unroll
    for (int j = 0; j < K; ++j) {
        stop[j] = false;
        if (ok[j]) { cnt.edges++; stop[j] = op.commit(x[j], e[j], y[j], tk[j], ax[j], cnt); }
    }
}

// ------------------------------------------------------------------ THREAD
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_thread(const Src src, const Adj g, Op op) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    const long long T = gthreads();
    for (long long base = gtid(); base < sz; base += kIlp * T) {
        int x[kIlp];
        uint32_t e[kIlp], end[kIlp];
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            long long i = base + j * T;
            int v = i < sz ? src.get((unsigned)i) : -1;
            if (v >= 0 && op.skip(v)) v = -1;
            x[j] = v;
        }
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            e[j] = x[j] >= 0 ? __ldg(g.off + x[j]) : 0u;
            end[j] = x[j] >= 0 ? __ldg(g.off + x[j] + 1) : 0u;
        }
        for (;;) {
            bool ok[kIlp], stop[kIlp], any = false;
#pragma unroll
            for (int j = 0; j < kIlp; ++j) { ok[j] = e[j] < end[j]; any |= ok[j]; }
            if (!any) break;
            edge_batch<kIlp>(op, g, x, e, ok, stop, cnt);
#pragma unroll
            for (int j = 0; j < kIlp; ++j)
                if (ok[j]) e[j] = (Op::kEarlyExit && stop[j]) ? end[j] : e[j] + 1;
        }
    }
    return cnt;
}

// ------------------------------------------------------------------ TWC
// CTA-tier election of TWC (a row with degree >= blockDim is expanded by the whole CTA).  Every
// warp publishes its ballot of big rows and its first candidate (row, begin, end) into the half
// of a double buffer selected by the round's parity; after one barrier every thread picks the
// lowest warp with a candidate.  A half is rewritten two rounds later, after the intervening
// round's barrier, so no reset store (and no write-write race between candidates) is needed --
// the single "owner" word with a reset store raced under compute-sanitizer racecheck (round 2).
struct TwcElect {
    unsigned ball[2][kWarps];
    int cx[2][kWarps];
    uint32_t cb[2][kWarps], ce[2][kWarps];
};
// returns true with (xx, bb, ee) of the elected row, consuming it in its owner thread
__device__ __forceinline__ bool twc_elect(TwcElect &el, unsigned &round, int x, uint32_t &b, uint32_t e, int &xx,
                                          uint32_t &bb, uint32_t &ee) {
    const int h = round & 1;
    ++round;
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    const bool big = e - b >= (uint32_t)kBlock;
    const unsigned m = __ballot_sync(0xffffffffu, big);
    if (m && (int)lane == __ffs(m) - 1) { el.cx[h][wid] = x; el.cb[h][wid] = b; el.ce[h][wid] = e; }
    if (lane == 0) el.ball[h][wid] = m;
    __syncthreads();
    int w = -1;
#pragma unroll
    for (int k = kWarps - 1; k >= 0; --k) if (el.ball[h][k]) w = k;
    if (w < 0) return false;
    xx = el.cx[h][w]; bb = el.cb[h][w]; ee = el.ce[h][w];
    if ((int)wid == w && (int)lane == __ffs(el.ball[h][w]) - 1) b = e;    // consumed by its owner
    return true;
}
struct TwcSmem {
    TwcElect el;
};
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_twc(const Src src, const Adj g, Op op, TwcSmem *sm) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    const unsigned lane = lane_id();
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
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            b[j] = x[j] >= 0 ? __ldg(g.off + x[j]) : 0u;
            e[j] = x[j] >= 0 ? __ldg(g.off + x[j] + 1) : 0u;
        }
        // CTA tier: degree >= blockDim
#pragma unroll
        for (int j = 0; j < kIlp; ++j) {
            for (;;) {
                int xx;
                uint32_t bb, ee;
                if (!twc_elect(sm->el, round, x[j], b[j], e[j], xx, bb, ee)) break;
                for (uint32_t k0 = bb; k0 < ee; k0 += 2 * kBlock) {
                    int xs[2] = {xx, xx};
                    uint32_t ks[2] = {k0 + threadIdx.x, k0 + kBlock + threadIdx.x};
                    bool ok[2] = {ks[0] < ee, ks[1] < ee}, stop[2];
                    edge_batch<2>(op, g, xs, ks, ok, stop, cnt);
                    if (Op::kEarlyExit) { if (__syncthreads_or(stop[0] | stop[1])) break; }
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
                int leader = __ffs(m) - 1;
                const int xx = __shfl_sync(0xffffffffu, x[j], leader);
                const uint32_t bb = __shfl_sync(0xffffffffu, b[j], leader), ee = __shfl_sync(0xffffffffu, e[j], leader);
                if ((int)lane == leader) e[j] = b[j];
                for (uint32_t k0 = bb; k0 < ee; k0 += 64) {
                    int xs[2] = {xx, xx};
                    uint32_t ks[2] = {k0 + lane, k0 + 32 + lane};
                    bool ok[2] = {ks[0] < ee, ks[1] < ee}, stop[2];
                    edge_batch<2>(op, g, xs, ks, ok, stop, cnt);
                    if (Op::kEarlyExit) { if (__any_sync(0xffffffffu, stop[0] | stop[1])) break; }
                }
            }
        }
        // thread tier: degree < 32, kIlp items advanced in lock-step
        for (;;) {
            bool ok[kIlp], stop[kIlp], any = false;
#pragma unroll
            for (int j = 0; j < kIlp; ++j) { ok[j] = b[j] < e[j]; any |= ok[j]; }
            if (!any) break;
            edge_batch<kIlp>(op, g, x, b, ok, stop, cnt);
#pragma unroll
            for (int j = 0; j < kIlp; ++j)
                if (ok[j]) b[j] = (Op::kEarlyExit && stop[j]) ? e[j] : b[j] + 1;
        }
    }
    return cnt;
}

// ------------------------------------------------------------------ WM
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_wm(const Src src, const Adj g, Op op) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    const unsigned lane = lane_id();
    // items per warp: up to warpsize; fewer when the active set cannot fill every warp
    // of the grid, so that small frontiers are spread over all SMs (one edge per lane)
    const long long NW = gwarps();
    const unsigned ipw = (unsigned)max(1LL, min(32LL, ((long long)sz + NW - 1) / NW));
    for (long long wb = gwarp() * ipw; wb < sz; wb += NW * ipw) {
        long long i = wb + lane;
        int x = (lane < ipw && i < sz) ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        const uint32_t incl = warp_incl_scan(d);
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        const uint32_t excl = incl - d;
        for (uint32_t k0 = 0; k0 < total; k0 += 64) {
            int xs[2];
            uint32_t es[2];
            bool ok[2], stop[2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                uint32_t k = k0 + 32 * h + lane;
                // owner lane: first lane with incl > k  (log2(32) = 5 steps)
                unsigned lo = 0, hi = 31;
#pragma unroll
                for (int s = 0; s < 5; ++s) {
                    unsigned mid = (lo + hi) >> 1;
                    uint32_t v = __shfl_sync(0xffffffffu, incl, mid);
                    if (v > k) hi = mid; else lo = mid + 1;
                }
                xs[h] = __shfl_sync(0xffffffffu, x, lo);
                uint32_t bb = __shfl_sync(0xffffffffu, b, lo), ex = __shfl_sync(0xffffffffu, excl, lo);
                es[h] = bb + (k - ex);
                ok[h] = k < total && !(Op::kEarlyExit && op.skip(xs[h]));
            }
            edge_batch<2>(op, g, xs, es, ok, stop, cnt);
        }
    }
    return cnt;
}

// ------------------------------------------------------------------ CM
struct CmSmem {
    uint32_t excl[kBlock + 1];
    uint32_t beg[kBlock];
    int x[kBlock];
    uint32_t scan_tmp[kWarps + 1];
};
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_cm(const Src src, const Adj g, Op op, CmSmem *sm) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    for (long long cb = (long long)blockIdx.x * kBlock; cb < sz; cb += (long long)gridDim.x * kBlock) {
        long long i = cb + threadIdx.x;
        int x = i < sz ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        uint32_t total;
        uint32_t excl = block_excl_scan(d, sm->scan_tmp, &total);
        sm->excl[threadIdx.x] = excl;
        sm->beg[threadIdx.x] = b;
        sm->x[threadIdx.x] = x;
        __syncthreads();
        for (uint32_t k0 = 0; k0 < total; k0 += 2 * kBlock) {
            int xs[2];
            uint32_t es[2];
            bool ok[2], stop[2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                uint32_t k = k0 + h * kBlock + threadIdx.x;
                ok[h] = k < total;
                xs[h] = -1; es[h] = 0;
                if (ok[h]) {
                    // last item j with excl_j <= k  (log2(blockDim) steps)
                    unsigned lo = 0, hi = kBlock - 1;
                    while (lo < hi) {
                        unsigned mid = (lo + hi + 1) >> 1;
                        if (sm->excl[mid] <= k) lo = mid; else hi = mid - 1;
                    }
                    xs[h] = sm->x[lo];
                    es[h] = sm->beg[lo] + (k - sm->excl[lo]);
                    ok[h] = !(Op::kEarlyExit && op.skip(xs[h]));
                }
            }
            edge_batch<2>(op, g, xs, es, ok, stop, cnt);
        }
        __syncthreads();
    }
    return cnt;
}

// ------------------------------------------------------------------ STRICT (merge path)
// Needs the exclusive scan of item degrees in `scan` (size()+1 entries, scan[size()] = total),
// produced by strict_scan_* below (two grid-barrier phases).
constexpr int kStrictVT = 7;
constexpr int kStrictTile = kBlock * kStrictVT;
struct StrictSmem {
    uint32_t scan[kStrictTile + 2];
    int x[kStrictTile + 1];
    uint32_t beg[kStrictTile + 1];
    int i0, i1;
};

// phase 1: per-CTA degree sums over contiguous item chunks -> partial[blockIdx]
template <class Src>
__device__ void strict_scan_p1(const Src &src, const Adj &g, uint32_t *partial, uint32_t *red) {
    unsigned sz = src.size();
    unsigned chunk = (sz + gridDim.x - 1) / gridDim.x;
    unsigned lo = blockIdx.x * chunk, hi = min(sz, lo + chunk);
    uint32_t s = 0;
    for (unsigned i = lo + threadIdx.x; i < hi; i += kBlock) {
        int x = src.get(i);
        if (x >= 0) s += __ldg(g.off + x + 1) - __ldg(g.off + x);
    }
    s = block_sum(s, red);
    if (threadIdx.x == 0) partial[blockIdx.x] = s;
}
// phase 2: exclusive scan written to scan[0..sz], returns the total
template <class Src>
__device__ uint32_t strict_scan_p2(const Src &src, const Adj &g, const uint32_t *partial, uint32_t *scan,
                                   uint32_t *red) {
    unsigned sz = src.size();
    unsigned chunk = (sz + gridDim.x - 1) / gridDim.x;
    unsigned lo = blockIdx.x * chunk, hi = min(sz, lo + chunk);
    uint32_t before = 0, all = 0;
    for (unsigned j = threadIdx.x; j < gridDim.x; j += kBlock) {
        uint32_t p = ((volatile const uint32_t *)partial)[j];
        all += p;
        if (j < blockIdx.x) before += p;
    }
    before = block_sum(before, red);
    all = block_sum(all, red);
    uint32_t base = before;
    for (unsigned t0 = lo; t0 < hi; t0 += kBlock) {
        unsigned i = t0 + threadIdx.x;
        uint32_t d = 0;
        if (i < hi) { int x = src.get(i); if (x >= 0) d = __ldg(g.off + x + 1) - __ldg(g.off + x); }
        uint32_t tot;
        uint32_t ex = block_excl_scan(d, red, &tot);
        if (i < hi) scan[i] = base + ex;
        base += tot;
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) scan[sz] = all;
    return all;
}

// number of items fully consumed at merge-path diagonal d (A = item ends scan[1..], B = edges)
__device__ __forceinline__ unsigned merge_path(const uint32_t *scan, unsigned sz, uint32_t total, unsigned long long d) {
    long long lo = d > total ? (long long)(d - total) : 0;
    long long hi = d < sz ? (long long)d : (long long)sz;
    while (lo < hi) {
        long long mid = (lo + hi) >> 1;
        if ((unsigned long long)scan[mid + 1] <= d - 1 - (unsigned long long)mid) lo = mid + 1; else hi = mid;
    }
    return (unsigned)lo;
}

// phase 3: process tiles of kStrictTile diagonals; every tile gets an equal share of items+edges.
// Each thread walks kStrictVT consecutive diagonals in shared memory first, then issues all of
// their edge loads together.
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_strict(const Src src, const Adj g, Op op, const uint32_t *scan,
                          uint32_t total, StrictSmem *sm) {
    LocalCnt cnt;
    const unsigned sz = src.size();
    const unsigned long long D = (unsigned long long)sz + total;
    const unsigned long long ntiles = (D + kStrictTile - 1) / kStrictTile;
    for (unsigned long long t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const unsigned long long d0 = t * kStrictTile, d1 = min(D, d0 + kStrictTile);
        if (threadIdx.x == 0) sm->i0 = merge_path(scan, sz, total, d0);
        if (threadIdx.x == 32) sm->i1 = merge_path(scan, sz, total, d1);
        __syncthreads();
        const int i0 = sm->i0, i1 = sm->i1;
        const int ni = min(i1 + 1, (int)sz) - i0;              // items touched by this tile
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
        // local merge path: items consumed at dd0, searched in [max(0,dd0-total)-i0, min(sz,dd0)-i0]
        long long lo = dd0 > total ? (long long)(dd0 - total) - i0 : 0;
        if (lo < 0) lo = 0;
        long long hi = (long long)min((unsigned long long)sz, dd0) - i0;
        if (hi > ni) hi = ni;
        while (lo < hi) {
            long long mid = (lo + hi) >> 1;
            if ((unsigned long long)sm->scan[mid + 1] <= dd0 - 1 - (unsigned long long)(mid + i0)) lo = mid + 1;
            else hi = mid;
        }
        long long ii = lo;                                      // local item index
        unsigned long long k = dd0 - (unsigned long long)(ii + i0);  // global edge index
        int xs[kStrictVT];
        uint32_t es[kStrictVT];
        bool ok[kStrictVT], stop[kStrictVT];
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) {
            ok[s] = false; xs[s] = -1; es[s] = 0;
            unsigned long long dd = dd0 + s;
            if (dd < dd1) {
                if (ii < ni && (unsigned long long)sm->scan[ii + 1] <= k) {
                    ++ii;                                       // item ends: consume it
                } else {
                    int x = sm->x[ii];
                    xs[s] = x;
                    es[s] = sm->beg[ii] + (uint32_t)(k - sm->scan[ii]);
                    ok[s] = x >= 0 && !(Op::kEarlyExit && op.skip(x));
                    ++k;
                }
            }
        }
        edge_batch<kStrictVT>(op, g, xs, es, ok, stop, cnt);
        __syncthreads();
    }
    return cnt;
}

}  // namespace gsw

namespace gsw {

// STRICT for small active sets (<= kStrictTile items, e.g. a few hubs): every CTA scans the item
// degrees itself in shared memory (no grid-wide scan, no grid barriers) and the diagonals per
// thread shrink so that the edges spread over every thread of the grid (one edge per thread when
// the frontier is tiny but the edges are many).
template <class Src, class Op>
__device__ __noinline__ LocalCnt lb_strict_small(const Src src, const Adj g, Op op, StrictSmem *sm) {
    LocalCnt cnt;
    __shared__ uint32_t red[kWarps + 1];
    const unsigned sz = src.size();
    uint32_t base = 0;
    for (unsigned t0 = 0; t0 < sz; t0 += kBlock) {
        const unsigned i = t0 + threadIdx.x;
        int x = i < sz ? src.get(i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        const uint32_t b = x >= 0 ? __ldg(g.off + x) : 0u;
        const uint32_t d = x >= 0 ? __ldg(g.off + x + 1) - b : 0u;
        uint32_t tot;
        const uint32_t ex = block_excl_scan(d, red, &tot);
        if (i < sz) { sm->scan[i] = base + ex; sm->x[i] = x; sm->beg[i] = b; }
        base += tot;
    }
    const uint32_t total = base;
    if (threadIdx.x == 0) sm->scan[sz] = total;
    __syncthreads();
    const unsigned long long D = (unsigned long long)sz + total;
    const unsigned long long per = ((unsigned long long)gridDim.x * kBlock);
    const unsigned vt = (unsigned)max(1ull, min((unsigned long long)kStrictVT, (D + per - 1) / per));
    const unsigned long long tile = (unsigned long long)kBlock * vt;
    const unsigned long long ntiles = (D + tile - 1) / tile;
    for (unsigned long long t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const unsigned long long dd0 = min(D, t * tile + (unsigned long long)threadIdx.x * vt);
        const unsigned long long dd1 = min(D, dd0 + vt);
        // items consumed at dd0: merge path over the whole (shared-memory) scan
        long long lo = dd0 > total ? (long long)(dd0 - total) : 0;
        long long hi = (long long)min((unsigned long long)sz, dd0);
        while (lo < hi) {
            const long long mid = (lo + hi) >> 1;
            if ((unsigned long long)sm->scan[mid + 1] <= dd0 - 1 - (unsigned long long)mid) lo = mid + 1; else hi = mid;
        }
        long long ii = lo;
        unsigned long long k = dd0 - (unsigned long long)ii;
        int xs[kStrictVT];
        uint32_t es[kStrictVT];
        bool ok[kStrictVT], stop[kStrictVT];
#pragma unroll
        for (int s = 0; s < kStrictVT; ++s) {
            ok[s] = false; xs[s] = -1; es[s] = 0;
            const unsigned long long dd = dd0 + s;
            if (dd < dd1) {
                if (ii < (long long)sz && (unsigned long long)sm->scan[ii + 1] <= k) {
                    ++ii;
                } else {
                    const int x = sm->x[ii];
                    xs[s] = x;
                    es[s] = sm->beg[ii] + (uint32_t)(k - sm->scan[ii]);
                    ok[s] = x >= 0 && !(Op::kEarlyExit && op.skip(x));
                    ++k;
                }
            }
        }
        edge_batch<kStrictVT>(op, g, xs, es, ok, stop, cnt);
    }
    __syncthreads();
    return cnt;
}

union LbSmem {
    TwcSmem twc;
    CmSmem cm;
    StrictSmem strict;
};

// Dispatch the selected load-balance candidate (Fig. 13: one Expand variant per iteration).
// STRICT adds its two scan phases, each closed by a grid barrier.
template <class Src, class Op>
__device__ __forceinline__ LocalCnt run_lb(int lb, const Src &src, const Adj &adj, const Op &op, LbSmem &sm,
                                           uint32_t *red, const GridBarrier &bar, unsigned &epoch,
                                           uint32_t *partial, uint32_t *scan) {
    switch (lb) {
    case GSW_LB_THREAD: return lb_thread(src, adj, op);
    case GSW_LB_TWC: return lb_twc(src, adj, op, &sm.twc);
    case GSW_LB_WM: return lb_wm(src, adj, op);
    case GSW_LB_CM: return lb_cm(src, adj, op, &sm.cm);
    default: {
        if (src.size() <= (unsigned)kStrictTile) return lb_strict_small(src, adj, op, &sm.strict);
        strict_scan_p1(src, adj, partial, red);
        grid_sync(bar, epoch);
        uint32_t total = strict_scan_p2(src, adj, partial, scan, red);
        grid_sync(bar, epoch);
        return lb_strict(src, adj, op, scan, total, &sm.strict);
    }
    }
}

}  // namespace gsw
