// lb.cuh -- Pattern 3, load balance (Fig. 6): how (item, edge) work of an
// Expand is mapped onto threads.  Every strategy is a device function used inside a persistent
// kernel phase, templated on
//   Src : the active set in its format (Pattern 2): size() item slots, get(i) -> vertex or -1
//   Op  : the algorithm's per-edge operation (emit + comp/compAtomic)
//         bool skip(int x)                      -- x needs no (more) work (pull early exit)
//         bool edge(int x, uint32 e, int y, LocalCnt&) -- process edge e=(x,y); true = x done
//         static constexpr bool kEarlyExit       -- stop scanning x after edge() returned true
// Candidates:
//   THREAD : one thread per item, serial edge loop (the naive mapping the north_star lists)
//   TWC    : degree-binned thread / warp / CTA mapping (B40C [41])
//   WM     : a warp takes 32 consecutive items, 32-edge chunks, log2(32)-step search
//   CM     : a CTA takes blockDim items, blockDim-edge chunks, log2(blockDim) search
//   STRICT : equal (items+edges) per tile via merge-path over the degree scan ([13])
#pragma once
#include "common.cuh"

namespace gsw {

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

// ------------------------------------------------------------------ THREAD
template <class Src, class Op>
__device__ void lb_thread(const Src &src, const Adj &g, Op &op, LocalCnt &cnt) {
    unsigned sz = src.size();
    for (long long i = gtid(); i < sz; i += gthreads()) {
        int x = src.get((unsigned)i);
        if (x < 0 || op.skip(x)) continue;
        uint32_t b = __ldg(g.off + x), e = __ldg(g.off + x + 1);
        for (uint32_t k = b; k < e; ++k) {
            cnt.edges++;
            if (op.edge(x, k, __ldg(g.col + k), cnt) && Op::kEarlyExit) break;
        }
    }
}

// ------------------------------------------------------------------ TWC
struct TwcSmem {
    int owner, x, stop;
    uint32_t b, e;
};
template <class Src, class Op>
__device__ void lb_twc(const Src &src, const Adj &g, Op &op, LocalCnt &cnt, TwcSmem *sm) {
    unsigned sz = src.size();
    const unsigned lane = lane_id();
    for (long long base = (long long)blockIdx.x * kBlock; base < sz; base += (long long)gridDim.x * kBlock) {
        long long i = base + threadIdx.x;
        int x = i < sz ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, e = 0;
        if (x >= 0) { b = __ldg(g.off + x); e = __ldg(g.off + x + 1); }
        uint32_t d = e - b;
        // CTA tier: degree >= blockDim
        for (;;) {
            if (threadIdx.x == 0) sm->owner = -1;
            __syncthreads();
            if (d >= (uint32_t)kBlock) sm->owner = threadIdx.x;
            __syncthreads();
            int owner = sm->owner;
            if (owner < 0) break;
            if ((int)threadIdx.x == owner) { sm->x = x; sm->b = b; sm->e = e; d = 0; }
            __syncthreads();
            int xx = sm->x;
            uint32_t bb = sm->b, ee = sm->e;
            for (uint32_t k0 = bb; k0 < ee; k0 += kBlock) {
                uint32_t k = k0 + threadIdx.x;
                bool stop = false;
                if (k < ee) { cnt.edges++; stop = op.edge(xx, k, __ldg(g.col + k), cnt); }
                if (Op::kEarlyExit) { if (__syncthreads_or(stop)) break; }
            }
            __syncthreads();
        }
        // warp tier: 32 <= degree < blockDim
        for (;;) {
            unsigned m = __ballot_sync(0xffffffffu, d >= 32u);
            if (!m) break;
            int leader = __ffs(m) - 1;
            int xx = __shfl_sync(0xffffffffu, x, leader);
            uint32_t bb = __shfl_sync(0xffffffffu, b, leader), ee = __shfl_sync(0xffffffffu, e, leader);
            if ((int)lane == leader) d = 0;
            for (uint32_t k0 = bb; k0 < ee; k0 += 32) {
                uint32_t k = k0 + lane;
                bool stop = false;
                if (k < ee) { cnt.edges++; stop = op.edge(xx, k, __ldg(g.col + k), cnt); }
                if (Op::kEarlyExit) { if (__any_sync(0xffffffffu, stop)) break; }
            }
        }
        // thread tier: degree < 32
        if (d > 0) {
            for (uint32_t k = b; k < e; ++k) {
                cnt.edges++;
                if (op.edge(x, k, __ldg(g.col + k), cnt) && Op::kEarlyExit) break;
            }
        }
    }
}

// ------------------------------------------------------------------ WM
template <class Src, class Op>
__device__ void lb_wm(const Src &src, const Adj &g, Op &op, LocalCnt &cnt) {
    unsigned sz = src.size();
    const unsigned lane = lane_id();
    for (long long wb = gwarp() * 32; wb < sz; wb += gwarps() * 32) {
        long long i = wb + lane;
        int x = i < sz ? src.get((unsigned)i) : -1;
        if (x >= 0 && op.skip(x)) x = -1;
        uint32_t b = 0, d = 0;
        if (x >= 0) { b = __ldg(g.off + x); d = __ldg(g.off + x + 1) - b; }
        uint32_t incl = warp_incl_scan(d);
        uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        uint32_t excl = incl - d;
        for (uint32_t k0 = 0; k0 < total; k0 += 32) {
            uint32_t k = k0 + lane;
            // owner lane j: first lane with incl_j > k  (binary search, log2(32) = 5 steps)
            unsigned lo = 0, hi = 31;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                unsigned mid = (lo + hi) >> 1;
                uint32_t v = __shfl_sync(0xffffffffu, incl, mid);
                if (v > k) hi = mid; else lo = mid + 1;
            }
            int xx = __shfl_sync(0xffffffffu, x, lo);
            uint32_t bb = __shfl_sync(0xffffffffu, b, lo), ex = __shfl_sync(0xffffffffu, excl, lo);
            if (k < total && !op.skip(xx)) {
                uint32_t e = bb + (k - ex);
                cnt.edges++;
                op.edge(xx, e, __ldg(g.col + e), cnt);
            }
        }
    }
}

// ------------------------------------------------------------------ CM
struct CmSmem {
    uint32_t excl[kBlock + 1];
    uint32_t beg[kBlock];
    int x[kBlock];
    uint32_t scan_tmp[kWarps + 1];
};
template <class Src, class Op>
__device__ void lb_cm(const Src &src, const Adj &g, Op &op, LocalCnt &cnt, CmSmem *sm) {
    unsigned sz = src.size();
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
        for (uint32_t k0 = 0; k0 < total; k0 += kBlock) {
            uint32_t k = k0 + threadIdx.x;
            if (k < total) {
                // last item j with excl_j <= k  (log2(blockDim) steps)
                unsigned lo = 0, hi = kBlock - 1;
                while (lo < hi) {
                    unsigned mid = (lo + hi + 1) >> 1;
                    if (sm->excl[mid] <= k) lo = mid; else hi = mid - 1;
                }
                int xx = sm->x[lo];
                if (!op.skip(xx)) {
                    uint32_t e = sm->beg[lo] + (k - sm->excl[lo]);
                    cnt.edges++;
                    op.edge(xx, e, __ldg(g.col + e), cnt);
                }
            }
        }
        __syncthreads();
    }
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

// phase 3: process tiles of kStrictTile diagonals; every tile gets an equal share of items+edges
template <class Src, class Op>
__device__ void lb_strict(const Src &src, const Adj &g, Op &op, LocalCnt &cnt, const uint32_t *scan,
                          uint32_t total, StrictSmem *sm) {
    unsigned sz = src.size();
    unsigned long long D = (unsigned long long)sz + total;
    unsigned long long ntiles = (D + kStrictTile - 1) / kStrictTile;
    for (unsigned long long t = blockIdx.x; t < ntiles; t += gridDim.x) {
        unsigned long long d0 = t * kStrictTile, d1 = min(D, d0 + kStrictTile);
        if (threadIdx.x == 0) sm->i0 = merge_path(scan, sz, total, d0);
        if (threadIdx.x == 32) sm->i1 = merge_path(scan, sz, total, d1);
        __syncthreads();
        int i0 = sm->i0, i1 = sm->i1;
        int ni = min(i1 + 1, (int)sz) - i0;              // items touched by this tile
        for (int j = threadIdx.x; j <= ni; j += kBlock) sm->scan[j] = scan[i0 + j];
        for (int j = threadIdx.x; j < ni; j += kBlock) {
            int x = src.get(i0 + j);
            if (x >= 0 && op.skip(x)) x = -1;
            sm->x[j] = x;
            sm->beg[j] = x >= 0 ? __ldg(g.off + x) : 0u;
        }
        __syncthreads();
        // this thread's diagonals [dd0, dd1) -> local merge path within the tile
        unsigned long long dd0 = min(d1, d0 + (unsigned long long)threadIdx.x * kStrictVT);
        unsigned long long dd1 = min(d1, dd0 + kStrictVT);
        // items consumed at dd0 (search in smem, relative to i0)
        unsigned long long k_lo = dd0 - i0;                 // not used directly; binary search below
        (void)k_lo;
        long long lo = 0, hi = ni;
        {
            // global item index i in [i0, i0+ni]; condition scan[i+1] <= dd0-1-i
            long long l = dd0 > total ? (long long)(dd0 - total) - i0 : 0;
            if (l < 0) l = 0;
            long long h = (long long)min((unsigned long long)sz, dd0) - i0;
            if (h > ni) h = ni;
            lo = l; hi = h;
            while (lo < hi) {
                long long mid = (lo + hi) >> 1;
                if ((unsigned long long)sm->scan[mid + 1] <= dd0 - 1 - (unsigned long long)(mid + i0)) lo = mid + 1; else hi = mid;
            }
        }
        long long ii = lo;                                    // local item index
        unsigned long long k = dd0 - (unsigned long long)(ii + i0);  // global edge index
        for (unsigned long long dd = dd0; dd < dd1; ++dd) {
            if (ii < ni && (unsigned long long)sm->scan[ii + 1] <= k) { ++ii; continue; }   // item ends
            // edge k belongs to item ii
            int x = sm->x[ii];
            if (x >= 0 && !op.skip(x)) {
                uint32_t e = sm->beg[ii] + (uint32_t)(k - sm->scan[ii]);
                cnt.edges++;
                op.edge(x, e, __ldg(g.col + e), cnt);
            }
            ++k;
        }
        __syncthreads();
    }
}

}  // namespace gsw
