// engine.cuh -- the device-resident iteration engine: control block, history/records, and the
// Filter-side active-set builders of Pattern 2 (Fig. 4):
//   bitmap        : one bit per vertex, no scan, idle threads on sparse sets
//   unsorted queue: compact ids in any order, warp-aggregated atomics
//   sorted queue  : compact ids ascending via a scan of bitmap words
#pragma once
#include <cstddef>
#include "common.cuh"
#include "gsw.h"
#include "select.cuh"

namespace gsw {

constexpr int kMaxHist = 1 << 16;   // iterations with stored history / records
// CTA-resident (solo) tier thresholds: an iteration runs on CTA 0 alone when its active set has
// at most kSoloV vertices and kSoloE edges (and the selector picked fused push on a queue).
// Calibrated on B200 (tools/solo_sweep.py, tools/round_stats.py): a solo
// level costs ~2.7 us at 1 vertex and ~9 us at 300 vertices, a grid level ~13 us.
constexpr long long kSoloE = 2048;
constexpr long long kSoloV = 512;
constexpr long long kSoloESssp = 512;     // SSSP's near/far rounds (re-calibrated in round 2)
constexpr long long kSoloVSssp = 256;

struct Hist {
    float tf, te, Tf, Te;
};

struct Ctl {
    unsigned arrive, spare, err, iters;   // arrive: the grid barrier's word (flip-bit protocol)
    unsigned long long edges_total, bytes_alg;
    unsigned long long t_start, t_phase, t_expand;   // kernel entry, loop start, output start (%globaltimer)
    float sum_tf, sum_te;
    unsigned stop;
    unsigned pad;
    unsigned long long t_end;                        // kernel end (GSW_PHASES=1 prints the split)
};

struct RunCommon {
    Ctl *ctl;
    IterCnt *cnt;            // ring of 3
    Hist *hist;              // kMaxHist
    gsw_iter_record *rec;    // kMaxHist
    uint32_t *partial;       // gridDim entries (+1)
    gsw_config force;
    Features base;           // dataset attributes (runtime fields filled per iteration)
    struct TeamPub *pub;     // loop state handed from CTA 0 to the parked CTAs (solo tier)
    long long solo_e, solo_v;  // solo-tier thresholds on Ea / Va (0 disables the tier)
    int cluster;             // nonzero: launched as one thread-block cluster (grid barrier = barrier.cluster)
    int team_k;              // > 1: launched in clusters of team_k CTAs; cluster 0 runs the team tier
    long long team_e;        // team-tier threshold on Ea (capacity is checked separately)
};

// Loop state CTA 0 hands to the parked CTAs when a solo episode ends:
// written by thread 0 of CTA 0 before the releasing grid barrier, read after it.
struct alignas(16) TeamPub {
    long long t, Via, Eia;
    unsigned long long va, ea;
    int mat, dirty, done, qlen;
    int dir, fmt, lb, step, fused, pad;
    unsigned long long aux[8];   // algorithm-specific (SSSP: theta, floor, |F|, ...)
};
__device__ __forceinline__ void pub_read(const TeamPub *g, TeamPub &out) {
    __shared__ TeamPub s;
    __syncthreads();
    if (threadIdx.x == 0) s = *g;   // plain loads after the barrier's acquire (L1 invalidated)
    __syncthreads();
    out = s;
    __syncthreads();
}

__device__ __forceinline__ GridBarrier make_bar(const RunCommon &rc) {
    return GridBarrier{&rc.ctl->arrive, &rc.ctl->err, rc.cluster};
}

// Per-run bookkeeping of CTA 0 / thread 0, kept in registers so that nothing on the critical
// path between two grid barriers waits for a global read-modify-write.
struct Book {
    uint64_t t_start = 0, t_expand = 0;
    float sum_tf = 0.f, sum_te = 0.f;
    unsigned long long bytes = 0, edges = 0;
};
__device__ __forceinline__ bool is_book() { return blockIdx.x == 0 && threadIdx.x == 0; }

// Start of iteration t (CTA 0 / thread 0): close the timing of iteration t-1 (Filter = start ->
// expand stamp, Expand = expand stamp -> now) and publish it as history features through the
// counter slot `carry` that every CTA reads at iteration t+1 (lag 2, identical in all CTAs).
__device__ __forceinline__ float4 book_start(Book &b, const RunCommon &rc, int t, IterCnt *carry) {
    uint64_t now = globaltimer();
    float4 h = make_float4(0.f, 0.f, 0.f, 0.f);
    if (t >= 1) {
        float tf = (float)(b.t_expand - b.t_start) * 1e-3f;
        float te = (float)(now - b.t_expand) * 1e-3f;
        b.sum_tf += tf; b.sum_te += te;
        h = make_float4(tf, te, b.sum_tf / (float)t, b.sum_te / (float)t);
        carry->tf = h.x; carry->te = h.y; carry->Tf = h.z; carry->Te = h.w;
        if (t - 1 < kMaxHist) { rc.rec[t - 1].filter_us = tf; rc.rec[t - 1].expand_us = te; }
    }
    b.t_start = now;
    b.t_expand = now;
    return h;   // the history features iteration t+1 will read from `carry`
}
__device__ __forceinline__ void book_expand(Book &b) { b.t_expand = globaltimer(); }
__device__ __forceinline__ void book_finish(const Book &b, const RunCommon &rc, int iters) {
    rc.ctl->bytes_alg = b.bytes;
    rc.ctl->edges_total = b.edges;
    rc.ctl->iters = (unsigned)iters;
}
__device__ __forceinline__ void hist_features(const CntView &v, Features &f) {
    f.tf = v.tf; f.te = v.te; f.Tf = v.Tf; f.Te = v.Te;
}

__device__ __forceinline__ void write_record(const RunCommon &rc, int t, const DevCfg &c, const Features &f,
                                             unsigned theta) {
    if (blockIdx.x == 0 && threadIdx.x == 0 && t < kMaxHist) {
        // five 16-byte stores straight from registers (a gsw_iter_record temporary went through
        // the stack: local-memory round trips on the critical path of every level)
        static_assert(sizeof(gsw_iter_record) == 80 && offsetof(gsw_iter_record, Va) == 24 &&
                      offsetof(gsw_iter_record, theta) == 64, "record layout");
        int4 *p = reinterpret_cast<int4 *>(rc.rec + t);
        p[0] = make_int4(t, c.dir, c.fmt, c.lb);
        p[1] = make_int4(c.step, c.fused, (int)(unsigned long long)f.Va, (int)((unsigned long long)f.Va >> 32));
        p[2] = make_int4((int)(unsigned long long)f.Ea, (int)((unsigned long long)f.Ea >> 32),
                         (int)(unsigned long long)f.Via, (int)((unsigned long long)f.Via >> 32));
        p[3] = make_int4((int)(unsigned long long)f.Eia, (int)((unsigned long long)f.Eia >> 32), 0, 0);
        p[4] = make_int4((int)theta, 0, 0, (int)gridDim.x);
    }
}

// ------------------------------------------------------------------ caller-order output
// internal ids are degree-ordered (graph.cu relabel): out[j] = in[inv[j]] for caller ids j
// Batched: each thread issues kG index loads, then kG value loads, then kG stores, so one
// dependent (inv -> in) round trip covers kG elements (the plain loop was latency-bound: ~28
// serial round trips per thread at C3, ~25 us).
template <class T>
__device__ __forceinline__ void gather_out(T *__restrict__ out, const T *__restrict__ in,
                                           const uint32_t *__restrict__ inv, int n) {
    constexpr int kG = 8;
    const long long T0 = gtid(), NT = gthreads();
    for (long long base = T0; base < n; base += kG * NT) {
        uint32_t ix[kG];
        T val[kG];
#pragma unroll
        for (int k = 0; k < kG; ++k) {
            const long long j = base + k * NT;
            ix[k] = j < n ? __ldg(inv + j) : 0u;
        }
#pragma unroll
        for (int k = 0; k < kG; ++k) {
            const long long j = base + k * NT;
            if (j < n) val[k] = in[ix[k]];
        }
#pragma unroll
        for (int k = 0; k < kG; ++k) {
            const long long j = base + k * NT;
            if (j < n) out[j] = val[k];
        }
    }
}
__device__ __forceinline__ int map_in(const uint32_t *inv, int v) { return inv ? (int)inv[v] : v; }

// ------------------------------------------------------------------ active-set builders
// bitmap from a per-vertex predicate: one warp per 32-vertex word, ballot, one store
template <class Pred>
__device__ inline void bm_from_pred(unsigned *bm, int n, Pred pred) {
    int W = (n + 31) >> 5;
    for (long long w = gwarp(); w < W; w += gwarps()) {
        int v = (int)(w * 32 + lane_id());
        bool b = v < n && pred(v);
        unsigned m = __ballot_sync(0xffffffffu, b);
        if (lane_id() == 0) bm[w] = m;
    }
}
// unsorted queue from a per-vertex predicate (ascending within a warp, warps in any order)
template <class Pred>
__device__ inline void q_from_pred(int *q, unsigned *len, int n, Pred pred) {
    int W = (n + 31) >> 5;
    for (long long w = gwarp(); w < W; w += gwarps()) {
        int v = (int)(w * 32 + lane_id());
        bool b = v < n && pred(v);
        unsigned m = __ballot_sync(0xffffffffu, b);
        if (!m) continue;
        unsigned base = 0;
        if (lane_id() == 0) base = atomicAdd(len, (unsigned)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (b) q[base + __popc(m & lanemask_lt())] = v;
    }
}
// unsorted queue from bitmap words (word ^ flip; flip=~0 takes the zero bits)
__device__ inline void q_from_bm(int *q, unsigned *len, const unsigned *bm, int W, unsigned flip) {
    for (long long w0 = gwarp() * 32; w0 < W; w0 += gwarps() * 32) {
        long long w = w0 + lane_id();
        unsigned word = w < W ? (bm[w] ^ flip) : 0u;
        unsigned c = __popc(word);
        unsigned inc = warp_incl_scan(c);
        unsigned tot = __shfl_sync(0xffffffffu, inc, 31);
        if (!tot) continue;
        unsigned base = 0;
        if (lane_id() == 31) base = atomicAdd(len, tot);
        base = __shfl_sync(0xffffffffu, base, 31);
        unsigned pos = base + inc - c;
        while (word) {
            int b = __ffs(word) - 1;
            word &= word - 1;
            q[pos++] = (int)(w * 32 + b);
        }
    }
}
// sorted queue from bitmap words, pass 1: per-CTA popcount of a contiguous word range
__device__ inline void sq_from_bm_p1(const unsigned *bm, int W, unsigned flip, uint32_t *partial, uint32_t *red) {
    unsigned chunk = (W + gridDim.x - 1) / gridDim.x;
    unsigned lo = blockIdx.x * chunk, hi = min((unsigned)W, lo + chunk);
    uint32_t s = 0;
    for (unsigned w = lo + threadIdx.x; w < hi; w += kBlock) s += __popc(bm[w] ^ flip);
    s = block_sum(s, red);
    if (threadIdx.x == 0) partial[blockIdx.x] = s;
}
// pass 2 (after a grid barrier): scatter ids in ascending order; the last CTA stores the length
__device__ inline void sq_from_bm_p2(int *q, unsigned *len, const unsigned *bm, int W, unsigned flip,
                              const uint32_t *partial, uint32_t *red) {
    unsigned chunk = (W + gridDim.x - 1) / gridDim.x;
    unsigned lo = blockIdx.x * chunk, hi = min((unsigned)W, lo + chunk);
    uint32_t before = 0;
    for (unsigned j = threadIdx.x; j < blockIdx.x; j += kBlock) before += ((volatile const uint32_t *)partial)[j];
    before = block_sum(before, red);
    uint32_t base = before;
    for (unsigned t0 = lo; t0 < hi; t0 += kBlock) {
        unsigned w = t0 + threadIdx.x;
        unsigned word = w < hi ? (bm[w] ^ flip) : 0u;
        uint32_t tot;
        uint32_t ex = block_excl_scan((uint32_t)__popc(word), red, &tot);
        uint32_t pos = base + ex;
        while (word) {
            int b = __ffs(word) - 1;
            word &= word - 1;
            q[pos++] = (int)(w * 32 + b);
        }
        base += tot;
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) *len = base;
}
__device__ inline void bm_from_q(unsigned *bm, const int *q, unsigned len) {
    for (long long i = gtid(); i < len; i += gthreads()) {
        int v = q[i];
        atomicOr(bm + (v >> 5), 1u << (v & 31));
    }
}
__device__ inline void clear_words(unsigned *bm, int W) {
    for (long long w = gtid(); w < W; w += gthreads()) bm[w] = 0u;
}
__device__ inline void copy_words(unsigned *dst, const unsigned *src, int W) {
    for (long long w = gtid(); w < W; w += gthreads()) dst[w] = src[w];
}

}  // namespace gsw
