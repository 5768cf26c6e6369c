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
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include <cooperative_groups.h>

#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"
#include "bfs_pull.cuh"

namespace gsw {
namespace cg = cooperative_groups;

enum { MAT_NONE = 0, MAT_QUEUE = 1, MAT_SQUEUE = 2, MAT_BITMAP = 3 };

// GSW_PULL_PROF=1 (diagnostic builds only): per-warp entry/exit %globaltimer of the list pull of
// every level, summarised on stderr after each run (where a pull level's time goes: the slowest
// warps vs the median)
#ifndef GSW_PULL_PROF
#define GSW_PULL_PROF 0
#endif
#if GSW_PULL_PROF
__device__ unsigned long long g_pull_prof[8][16384][2];
#endif
// GSW_TEAM_PROF=1 (diagnostic builds only): per-phase %globaltimer sums of the team tier's levels
// (CTA 0 and CTA k-1, thread 0), printed on stderr after each run
#ifndef GSW_TEAM_PROF
#define GSW_TEAM_PROF 0
#endif

#if GSW_TEAM_PROF
__device__ unsigned long long g_team_prof[2][10];
__device__ unsigned long long g_team_late[16];
#define TEAM_STAMP(i) do { if (tid == 0) { const unsigned long long nw = globaltimer(); \
    tp_acc[i] += nw - tp_last; tp_last = nw; } } while (0)
#else
#define TEAM_STAMP(i) do { } while (0)
#endif

struct BfsArgs {
    DevGraph g;
    const unsigned *iso;
    const unsigned *iso_c;    // isolated bitmap in caller order (relabeled graphs)
    int n_init;           // depth entries initialised: all n, or the non-isolated prefix after relabeling
    int src;              // caller id
    int *depth;           // internal order
    int *out;             // caller order (relabeled graphs), else nullptr
    int scatter;          // caller-order output: -1 at init, then scatter the reached depths (vs gather)
    unsigned *V;          // visited map (isolated + padding bits pre-set)
    unsigned *fb[3];      // frontier bitmaps, ring of 3
    int *q[2];            // active-set queues, double buffered
    int *iq;              // inactive queue (pull workload in queue formats)
    uint32_t *scan;       // STRICT degree scan
    long long iso_count;
    RunCommon rc;
};

// Five-stage edge op (lb.cuh edge_batch): probe -> act (atomic issued, result kept raw) -> aux
// (degree of a winner) -> commit.  Tok carries the raw atomicOr result; ~0u means "not claimed".
struct ClaimTok {
    unsigned old;
    unsigned flag;   // push: unused; pull: target is active (stop scanning)
};

// push: for active u and out-neighbour v, claim v if Inactive (compAtomic), depth[v] = lvl+1
struct BfsPushOp {
    int *depth;
    unsigned *V;
    const uint32_t *off;
    int lvl1;
    int fused;                // 0 standalone, 1 fused -> append to queue, 2 fused -> mark bitmap
    CtaQueue nq;              // CTA-staged append to the next queue
    unsigned *nfb;
    using Probe = unsigned;
    using Tok = ClaimTok;
    using Aux = uint2;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int, uint32_t, int v) const { return V[v >> 5]; }
    __device__ __forceinline__ Tok act(int, uint32_t, int v, Probe p) const {
        unsigned bit = 1u << (v & 31);
        return ClaimTok{(p & bit) ? ~0u : atomicOr(V + (v >> 5), bit), 0u};
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int v, Tok t) const {
        bool won = !((t.old >> (v & 31)) & 1u);
        return won ? make_uint2(__ldg(off + v), __ldg(off + v + 1)) : make_uint2(0u, 0u);
    }
    __device__ __forceinline__ bool commit(int, uint32_t, int v, Tok t, Aux d, LocalCnt &c) const {
        bool won = !((t.old >> (v & 31)) & 1u);
        if (won) {
            depth[v] = lvl1;
            c.add_vertex(d.y - d.x);
            if (fused == 2) atomicOr(nfb + (v >> 5), 1u << (v & 31));
            else if (fused == 1) nq.push(v);
        }
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
    using Probe = unsigned;
    using Tok = ClaimTok;
    using Aux = uint2;
    static constexpr bool kEarlyExit = true;
    __device__ __forceinline__ bool skip(int v) const { return test_bit_relaxed(V, v); }
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const {
        return fb ? fb[u >> 5] : (unsigned)depth[u];
    }
    __device__ __forceinline__ Tok act(int v, uint32_t, int u, Probe p) const {
        bool in = fb ? ((p >> (u & 31)) & 1u) : ((int)p == lvl);
        return ClaimTok{in ? atomicOr(V + (v >> 5), 1u << (v & 31)) : ~0u, in ? 1u : 0u};
    }
    __device__ __forceinline__ Aux aux(int v, uint32_t, int, Tok t) const {
        bool won = !((t.old >> (v & 31)) & 1u);
        return won ? make_uint2(__ldg(off + v), __ldg(off + v + 1)) : make_uint2(0u, 0u);
    }
    __device__ __forceinline__ bool commit(int v, uint32_t, int, Tok t, Aux d, LocalCnt &c) const {
        bool won = !((t.old >> (v & 31)) & 1u);
        if (won) {
            depth[v] = lvl + 1;
            c.add_vertex(d.y - d.x);
            if (fused) atomicOr(nfb + (v >> 5), 1u << (v & 31));
        }
        return t.flag != 0u;
    }
};

// Pull over the visited map with word ownership (the THREAD candidate on the bitmap format):
// warp w owns 32-vertex words of V, lane = vertex, so claiming needs no atomics -- the warp
// ballots its hits and stores V[w] | hits and the next-frontier word itself.  Each warp keeps
// kPullWords words in flight, each lane one independent (col -> frontier-bit) chain per word.
constexpr int kPullWords = 4;
__device__ __noinline__ LocalCnt bfs_pull_words(const unsigned *__restrict__ fb, unsigned *__restrict__ V,
                                                int *__restrict__ depth, const uint32_t *__restrict__ in_off,
                                                const int32_t *__restrict__ in_col,
                                                const uint32_t *__restrict__ out_off, bool symmetric, int lvl,
                                                unsigned *__restrict__ nfb, int n) {
    LocalCnt cnt;
    const int W = (n + 31) >> 5;
    const unsigned lane = lane_id();
    const long long NW = gwarps();
    for (long long wb = gwarp(); wb < W; wb += kPullWords * NW) {
        unsigned vis[kPullWords];
        uint32_t e[kPullWords], end[kPullWords], beg[kPullWords];
        bool alive[kPullWords], found[kPullWords];
#pragma unroll
        for (int j = 0; j < kPullWords; ++j) {
            long long w = wb + j * NW;
            vis[j] = w < W ? V[w] : ~0u;                      // warp-uniform address: one request
        }
#pragma unroll
        for (int j = 0; j < kPullWords; ++j) {
            int v = (int)((wb + j * NW) * 32 + lane);
            alive[j] = !((vis[j] >> lane) & 1u);
            found[j] = false;
            beg[j] = e[j] = alive[j] ? __ldg(in_off + v) : 0u;
            end[j] = alive[j] ? __ldg(in_off + v + 1) : 0u;
            alive[j] = alive[j] && e[j] < end[j];
        }
        for (;;) {
            bool any = false;
#pragma unroll
            for (int j = 0; j < kPullWords; ++j) any |= alive[j];
            if (!__any_sync(0xffffffffu, any)) break;
            int y[kPullWords];
            unsigned p[kPullWords];
#pragma unroll
            for (int j = 0; j < kPullWords; ++j) y[j] = alive[j] ? __ldg(in_col + e[j]) : 0;
#pragma unroll
            for (int j = 0; j < kPullWords; ++j) p[j] = alive[j] ? fb[y[j] >> 5] : 0u;
#pragma unroll
            for (int j = 0; j < kPullWords; ++j) {
                if (!alive[j]) continue;
                cnt.edges++;
                if ((p[j] >> (y[j] & 31)) & 1u) { found[j] = true; alive[j] = false; }
                else if (++e[j] >= end[j]) alive[j] = false;
            }
        }
#pragma unroll
        for (int j = 0; j < kPullWords; ++j) {
            long long w = wb + j * NW;
            unsigned hits = __ballot_sync(0xffffffffu, found[j]);
            if (hits && lane == 0) {
                V[w] = vis[j] | hits;
                if (nfb) nfb[w] = hits;
            }
            if (found[j]) {
                int v = (int)(w * 32 + lane);
                depth[v] = lvl + 1;
                cnt.add_vertex(symmetric ? end[j] - beg[j] : __ldg(out_off + v + 1) - __ldg(out_off + v));
            }
        }
    }
    return cnt;
}

// ---------------------------------------------------------------- CTA-resident tier (solo)
// On road-like graphs and in the first/last levels of scale-free ones the active set is a few
// hundred vertices: one grid-wide iteration then costs ~8-13 us of barrier and dependent L2/HBM
// round trips (queue -> offsets -> columns -> probe -> claim -> degree -> counters -> barrier),
// almost none of it work.  While the selector keeps choosing fused push and the level stays
// below (solo_v vertices, solo_e edges), CTA 0 runs the levels alone with the frontier, its
// offsets, degrees and degree scan in shared memory; the other CTAs park at one grid barrier.
// Per level the dependent global chain is two round trips: the column loads, then the claim
// (atomicOr on the visited map) issued together with a speculative load of the target's offsets,
// so a winner enters the next frontier with its row already known.  The edges of a level are
// split evenly over the 256 threads by a merge-path search on the degree scan.  The selector
// still runs every level on the same features and the records mark these iterations ctas = 1.
constexpr int kSQ = 768;       // solo frontier capacity (vertices of one level); sized so that
                               // SoloSmem fits inside LbSmem (the kernel's smem, hence its L1 share, is unchanged)
constexpr int kSoloK = 4;      // edges in flight per thread
struct SoloSmem {
    int q[2][kSQ];
    uint32_t beg[2][kSQ];
    uint32_t scan[2][kSQ + 1];     // degrees, then their exclusive scan
    unsigned qn[2];
    unsigned long long ea;
    unsigned maxd, mind;
    int go;
    uint32_t red[kWarps + 1];
    unsigned long long book_raw[(sizeof(Book) + 7) / 8];   // CTA 0 / thread 0's Book during the episode
    long long prev_va;
};
union BfsSmem {
    LbSmem lb;
    SoloSmem solo;
};
static_assert(sizeof(SoloSmem) <= sizeof(LbSmem), "the solo tier must not grow the kernel's shared memory");

// Runs levels t, t+1, ... on the calling CTA (CTA 0) until the selector or the size limits end
// the episode; returns with AS_t (t = first level NOT run) in a.q[t & 1], its counters in
// rc.cnt[t % 3] and the loop state in rc.pub.  Called by all threads of CTA 0.
// Everything is passed by value (the kernel's bookkeeping travels through ss.book / ss.prev_va):
// taking the address of the kernel's locals would pin them to local memory for the whole run.
__device__ __noinline__ void bfs_solo(const BfsArgs &a, SoloSmem &ss, int t, long long Via, long long Eia,
                                      const Features fbase, unsigned qn0) {
    float4 hist = make_float4(0.f, 0.f, 0.f, 0.f);   // history features of the next level (thread 0)
    Book &book = *reinterpret_cast<Book *>(ss.book_raw);   // thread 0 only
    long long &prev_va = ss.prev_va;                  // thread 0 only
    const RunCommon &rc = a.rc;
    const unsigned tid = threadIdx.x;
    const uint32_t *__restrict__ off = a.g.off;
    const int32_t *__restrict__ col = a.g.col;
    unsigned *V = a.V;
    int *depth = a.depth;
    const long long sv = rc.solo_v < (long long)kSQ ? rc.solo_v : (long long)kSQ, se = rc.solo_e;
    // AS_t0 from the grid's queue (qn0 <= kSQ), with its offsets
    for (unsigned i0 = tid; i0 < qn0; i0 += kBlock * 4) {
        int u[4];
        uint32_t b[4], e[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) u[k] = i0 + k * kBlock < qn0 ? a.q[t & 1][i0 + k * kBlock] : -1;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            b[k] = u[k] >= 0 ? __ldg(off + u[k]) : 0u;
            e[k] = u[k] >= 0 ? __ldg(off + u[k] + 1) : 0u;
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            if (u[k] < 0) continue;
            const unsigned i = i0 + k * kBlock;
            ss.q[0][i] = u[k]; ss.beg[0][i] = b[k]; ss.scan[0][i] = e[k] - b[k];
        }
    }
    int cur = 0;
    unsigned qn = qn0;
    bool first = true;
    unsigned long long E_prev = 0, Ea = 0;
    unsigned mxd = 0, mnd = 0;
    for (;;) {
        // (A) features of AS_t: degrees are in shared memory (spilled entries: global queue)
        if (tid == 0) { ss.ea = 0ull; ss.maxd = 0u; ss.mind = 0xffffffffu; }
        __syncthreads();
        {
            const int *gq = a.q[t & 1];
            unsigned long long lea = 0;
            unsigned lmx = 0, lmn = 0xffffffffu;
            for (unsigned i = tid; i < qn; i += kBlock) {
                unsigned d;
                if (i < (unsigned)kSQ) d = ss.scan[cur][i];
                else { const int u = gq[i]; d = __ldg(off + u + 1) - __ldg(off + u); }
                lea += d;
                lmx = d > lmx ? d : lmx;
                lmn = d < lmn ? d : lmn;
            }
            lea = warp_sum(lea);
            lmx = warp_max(lmx);
            lmn = warp_min(lmn);
            if (lane_id() == 0 && lea) {
                atomicAdd(&ss.ea, lea);
                atomicMax(&ss.maxd, lmx);
                atomicMin(&ss.mind, lmn);
            }
        }
        __syncthreads();
        Ea = ss.ea; mxd = ss.maxd; mnd = ss.mind;
        // (B) the selector on AS_t's features: continue solo only for fused push on a small set
        if (tid == 0) {
            int go = first ? 1 : 0;
            if (!first && qn > 0) {
                Features f = fbase;
                f.Va = (long long)qn; f.Ea = (long long)Ea; f.Via = Via - (long long)qn; f.Eia = Eia - (long long)Ea;
                f.maxd = mxd; f.mind = mnd; f.iter = t;
                f.tf = hist.x; f.te = hist.y; f.Tf = hist.z; f.Te = hist.w;
                DevCfg c = select_traversal(f, rc.force);
                if (c.dir == GSW_PUSH && c.fused == GSW_FUSED && (long long)qn <= sv && (long long)Ea <= se) {
                    go = 1;
                    c.fmt = GSW_QUEUE;
                    book.bytes += 12ull * (unsigned long long)prev_va + 4ull * E_prev + 8ull * qn;
                    book.edges += E_prev;
                    if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)E_prev;
                    // history carried to iteration t+1 (book_start's lag-2 protocol, kept in registers)
                    hist = book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
                    write_record(rc, t, c, f, 0u);
                    reset_cnt(rc.cnt + ((t + 2) % 3));
                }
            }
            if (first) {       // the main loop's book_start(t) wrote the history of t+1
                const IterCnt *cs = rc.cnt + ((t + 1) % 3);
                hist = make_float4(cs->tf, cs->te, cs->Tf, cs->Te);
            }
            if (go && t < kMaxHist) rc.rec[t].ctas = 1;
            ss.go = go;
            ss.qn[cur ^ 1] = 0u;
        }
        __syncthreads();
        if (!ss.go) break;
        if (!first) { Via -= (long long)qn; Eia -= (long long)Ea; }
        // (C) exclusive scan of the degrees (consecutive entries per thread)
        {
            const unsigned per = (qn + kBlock - 1) / kBlock, i0 = tid * per;
            uint32_t loc = 0;
            for (unsigned k = 0; k < per; ++k)
                if (i0 + k < qn) loc += ss.scan[cur][i0 + k];
            uint32_t tot;
            uint32_t ex = block_excl_scan(loc, ss.red, &tot);
            for (unsigned k = 0; k < per; ++k) {
                if (i0 + k < qn) { const uint32_t d = ss.scan[cur][i0 + k]; ss.scan[cur][i0 + k] = ex; ex += d; }
            }
            if (tid == 0) ss.scan[cur][qn] = tot;
            __syncthreads();
        }
        if (tid == 0) book_expand(book);
        // (D) Expand: thread tid takes edges [lo, hi) of the level.  Round trip 1: columns;
        // round trip 2: claim (atomicOr on V) + the target's offsets, loaded speculatively
        {
            const unsigned E = (unsigned)Ea;
            const int nx = cur ^ 1;
            int *gqn = a.q[(t + 1) & 1];
            const uint32_t *scan = ss.scan[cur], *beg = ss.beg[cur];
            const unsigned lo = (unsigned)(((unsigned long long)E * tid) / kBlock);
            const unsigned hi = (unsigned)(((unsigned long long)E * (tid + 1)) / kBlock);
            // every lane of a warp runs the warp's maximum number of batches, so the claim
            // commits can be warp-aggregated (one shared atomic per warp and batch)
            const unsigned mine = hi > lo ? (hi - lo + kSoloK - 1) / kSoloK : 0u;
            const unsigned nb = __reduce_max_sync(0xffffffffu, mine);
            unsigned i = 0, j = lo;
            if (lo < hi) {
                unsigned L = 0, R = qn;
                while (R - L > 1) {
                    const unsigned m = (L + R) >> 1;
                    if (scan[m] <= lo) L = m; else R = m;
                }
                i = L;
            }
            for (unsigned bt = 0; bt < nb; ++bt) {
                int v[kSoloK];
#pragma unroll
                for (int k = 0; k < kSoloK; ++k) {
                    v[k] = -1;
                    if (j < hi) {
                        while (scan[i + 1] <= j) ++i;
                        v[k] = __ldg(col + beg[i] + (j - scan[i]));
                        ++j;
                    }
                }
                unsigned old[kSoloK];
                uint32_t vb[kSoloK], ve[kSoloK];
#pragma unroll
                for (int k = 0; k < kSoloK; ++k) {
                    old[k] = v[k] >= 0 ? atomicOr(V + (v[k] >> 5), 1u << (v[k] & 31)) : 0xffffffffu;
                    vb[k] = v[k] >= 0 ? __ldg(off + v[k]) : 0u;
                    ve[k] = v[k] >= 0 ? __ldg(off + v[k] + 1) : 0u;
                }
#pragma unroll
                for (int k = 0; k < kSoloK; ++k) {
                    const bool won = v[k] >= 0 && !((old[k] >> (v[k] & 31)) & 1u);
                    const unsigned m = __ballot_sync(0xffffffffu, won);
                    if (!m) continue;
                    unsigned base = 0;
                    if (lane_id() == (unsigned)(__ffs(m) - 1)) base = atomicAdd(&ss.qn[nx], (unsigned)__popc(m));
                    base = __shfl_sync(0xffffffffu, base, __ffs(m) - 1);
                    if (won) {
                        depth[v[k]] = t + 1;
                        const unsigned p = base + __popc(m & lanemask_lt());
                        if (p < (unsigned)kSQ) { ss.q[nx][p] = v[k]; ss.beg[nx][p] = vb[k]; ss.scan[nx][p] = ve[k] - vb[k]; }
                        else gqn[p] = v[k];
                    }
                }
            }
            __syncthreads();
            E_prev = E;
            if (tid == 0) prev_va = (long long)qn;
            qn = ss.qn[nx];
            cur = nx;
            ++t;
            first = false;
        }
    }
    // hand AS_t to the grid: the queue (smem part; the spill is already in place), its counters
    // in slot t % 3 (plus the edges of level t-1, accounted by the main loop), the loop state
    {
        int *gq = a.q[t & 1];
        const unsigned m = qn < (unsigned)kSQ ? qn : (unsigned)kSQ;
        for (unsigned i = tid; i < m; i += kBlock) gq[i] = ss.q[cur][i];
        if (tid == 0) {
            IterCnt *c = rc.cnt + (t % 3);
            c->va = qn; c->ea = Ea; c->maxd = mxd; c->mind = mnd; c->qlen = qn; c->edges = E_prev;
            TeamPub p{};
            p.t = t; p.Via = Via; p.Eia = Eia;
            *rc.pub = p;
        }
    }
}

// ---------------------------------------------------------------- cluster tier (team)
// The solo tier's per-level cost grows by ~2.3 ns per edge on its single SM (C2, tools/round_stats.py:
// 2.9 us at one vertex, 9 us at ~700 vertices): one SM issues about one scattered L1/L2 request
// per clock, so a 1,000-4,000-edge level is throughput-bound on that SM while the grid path pays
// its fixed ~7 us of barrier and dependent round trips.  On road-like graphs the persistent
// kernel is launched as thread-block clusters of k CTAs (one per SM) and the k CTAs of cluster 0
// run the small levels together; the other clusters park at one grid barrier as in the solo tier.
//   * each team CTA keeps its part of the frontier (vertex, row begin, degree) in its own shared
//     memory, triple-buffered by level;
//   * per level, one hardware cluster barrier: every CTA publishes (|part|, sum/max/min degree)
//     and reads all k records through distributed shared memory (one DSMEM round trip), so every
//     CTA evaluates the same Inspector totals and the same selector decision; CTA 0's history
//     features travel in its record;
//   * CTA r expands vertices [V r/k, V (r+1)/k) of the concatenated frontier, read from the
//     owners' shared memory (DSMEM), with the solo tier's merge-path edge split, column loads and
//     claim + speculative offsets round trips; winners append to the claiming CTA's own part;
//   * capacity is checked before a level is run (max degree x ceil(V/k) <= kTQ), so no CTA can
//     overflow its part; a level that does not fit ends the episode and the parts are handed
//     back to the grid as one queue.
constexpr int kTQ = 512;       // frontier part per team CTA
constexpr int kTeamMax = 16;   // cluster size limit (non-portable 16)
struct TeamRec {
    unsigned qn, maxd, mind, pad;
    unsigned long long ea;
    float4 hist;               // CTA 0 only: history features of this level (lag-2 protocol)
#if GSW_TEAM_PROF
    unsigned long long t_arr;
#endif
};
struct TeamSmem {
    int q[3][kTQ];
    uint32_t beg[3][kTQ];
    uint16_t deg[3][kTQ];          // saturated at 65535 (a level with such a vertex fails the capacity check)
    uint32_t sbeg[kTQ];
    uint32_t sscan[kTQ + 1];
    TeamRec rec[2];
    unsigned cq[kTeamMax + 1];     // prefix of the parts' sizes
    unsigned long long ea;
    unsigned maxd, mind, qn_next;
    int go;
    float4 hist;
    unsigned wmx[kWarps], wmn[kWarps];
    unsigned long long wsum[kWarps];
    uint32_t red[kWarps + 1];
    unsigned long long book_raw[(sizeof(Book) + 7) / 8];
    long long prev_va;
};
static_assert(sizeof(TeamSmem) <= sizeof(BfsSmem), "the team tier must not grow the kernel's shared memory");

// Runs levels t, t+1, ... on the k CTAs of cluster 0 until the selector or the capacity check
// ends the episode; returns with AS_t in a.q[t & 1] (parts concatenated in CTA order), its
// counters in rc.cnt[t % 3] and the loop state in rc.pub (written by CTA 0).  Called by all
// threads of CTAs 0..k-1 (cluster 0), which all see the same totals and take the same decisions.
#ifndef GSW_TEAM_INLINE
#define GSW_TEAM_INLINE 0
#endif
#if GSW_TEAM_INLINE
__device__ __forceinline__
#else
__device__ __noinline__
#endif
void bfs_team(const BfsArgs &a, TeamSmem &ts, int t, long long Via, long long Eia,
                                      const Features fbase, unsigned qn0, int k) {
    cg::cluster_group cl = cg::this_cluster();
    const unsigned tid = threadIdx.x, r = blockIdx.x;
    const bool book0 = r == 0 && tid == 0;
    Book &book = *reinterpret_cast<Book *>(ts.book_raw);   // CTA 0 / thread 0 only
    long long &prev_va = ts.prev_va;
    const RunCommon &rc = a.rc;
    const uint32_t *__restrict__ off = a.g.off;
    const int32_t *__restrict__ col = a.g.col;
    unsigned *V = a.V;
    int *depth = a.depth;
    const long long se = rc.solo_e;
    // AS_t0: my share of the grid's queue, with offsets
    unsigned qn_l;
    {
        const unsigned s0 = (unsigned)((unsigned long long)qn0 * r / k);
        qn_l = (unsigned)((unsigned long long)qn0 * (r + 1) / k) - s0;
        const int *gq = a.q[t & 1] + s0;
        for (unsigned i0 = tid; i0 < qn_l; i0 += kBlock * 4) {
            int u[4];
            uint32_t b[4], e[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) u[j] = i0 + j * kBlock < qn_l ? gq[i0 + j * kBlock] : -1;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                b[j] = u[j] >= 0 ? __ldg(off + u[j]) : 0u;
                e[j] = u[j] >= 0 ? __ldg(off + u[j] + 1) : 0u;
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if (u[j] < 0) continue;
                const unsigned i = i0 + j * kBlock;
                ts.q[0][i] = u[j]; ts.beg[0][i] = b[j]; ts.deg[0][i] = (uint16_t)min(e[j] - b[j], 65535u);
            }
        }
    }
    float4 hist = make_float4(0.f, 0.f, 0.f, 0.f);   // CTA 0 / thread 0: history of the next level
    if (book0) {      // the main loop's book_start(t) wrote the history of t+1
        const IterCnt *cs = rc.cnt + ((t + 1) % 3);
        hist = make_float4(cs->tf, cs->te, cs->Tf, cs->Te);
    }
    int cur = 0, par = 0;
    bool first = true;
    unsigned long long E_prev = 0, Ea = 0;
    unsigned mxd = 0, mnd = 0, qn = 0;
#if GSW_TEAM_PROF
    unsigned long long tp_last = globaltimer(), tp_acc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    unsigned long long tp_late = 0;
#endif
    for (;;) {
        // (A) my part's features -> my record
        __syncthreads();
        TEAM_STAMP(0);
        {
            unsigned long long lea = 0;
            unsigned lmx = 0, lmn = 0xffffffffu;
            for (unsigned i = tid; i < qn_l; i += kBlock) {
                const unsigned d = ts.deg[cur][i];
                lea += d;
                lmx = d > lmx ? d : lmx;
                lmn = d < lmn ? d : lmn;
            }
            lea = warp_sum(lea);
            lmx = warp_max(lmx);
            lmn = warp_min(lmn);
            const unsigned w = tid >> 5;
            if (lane_id() == 0) { ts.wsum[w] = lea; ts.wmx[w] = lmx; ts.wmn[w] = lmn; }
            __syncthreads();
            if (tid == 0) {
                for (int i = 1; i < kWarps; ++i) {
                    lea += ts.wsum[i];
                    lmx = max(lmx, ts.wmx[i]);
                    lmn = min(lmn, ts.wmn[i]);
                }
                TeamRec &m = ts.rec[par];
                m.qn = qn_l; m.maxd = lmx; m.mind = lmn; m.ea = lea; m.hist = hist;
#if GSW_TEAM_PROF
                m.t_arr = globaltimer();
#endif
            }
        }
        TEAM_STAMP(1);
        cluster_barrier();
        TEAM_STAMP(2);
        // (B) every part's record (warp 0: lane c reads CTA c) -> totals and the parts' prefix
        if (tid < 32) {
            const unsigned c = tid;
            unsigned cqn = 0, cmx = 0, cmn = 0xffffffffu;
            unsigned long long cea = 0;
            float4 h = make_float4(0.f, 0.f, 0.f, 0.f);
            if (c < (unsigned)k) {
                const TeamRec *rm = cl.map_shared_rank(&ts.rec[par], c);
                cqn = rm->qn; cmx = rm->maxd; cmn = rm->mind; cea = rm->ea;
                if (c == 0) h = rm->hist;
            }
#if GSW_TEAM_PROF
            {
                const unsigned long long ta = c < (unsigned)k ? cl.map_shared_rank(&ts.rec[par], c)->t_arr : ~0ull;
                unsigned long long mn = ta;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) { const unsigned long long x = __shfl_xor_sync(0xffffffffu, mn, o); mn = x < mn ? x : mn; }
                if (r == 0 && c < (unsigned)k) tp_late += ta - mn;
                if (r == 0 && c == 0) TEAM_STAMP(9);
            }
#endif
            const unsigned inc = warp_incl_scan(cqn);
            if (c < (unsigned)k) ts.cq[c + 1] = inc;
            cea = warp_sum(cea);
            cmx = warp_max(cmx);
            cmn = warp_min(cmn);
            if (c == 0) {
                ts.cq[0] = 0u;
                ts.ea = cea; ts.maxd = cmx; ts.mind = cmn;
                ts.hist = h;
            }
        }
        __syncthreads();
        TEAM_STAMP(3);
        qn = ts.cq[k];
        Ea = ts.ea; mxd = ts.maxd; mnd = ts.mind;
        // (C) the selector on AS_t's totals (identical inputs in every team CTA)
        if (tid == 0) {
            int go = first ? 1 : 0;
            if (!first && qn > 0) {
                Features f = fbase;
                f.Va = (long long)qn; f.Ea = (long long)Ea; f.Via = Via - (long long)qn; f.Eia = Eia - (long long)Ea;
                f.maxd = mxd; f.mind = mnd; f.iter = t;
                const float4 h = ts.hist;
                f.tf = h.x; f.te = h.y; f.Tf = h.z; f.Te = h.w;
                DevCfg c = select_traversal(f, rc.force);
                const unsigned per = (qn + (unsigned)k - 1) / (unsigned)k;
                const bool fits = per <= (unsigned)kTQ && (unsigned long long)mxd * per <= (unsigned long long)kTQ;
                if (c.dir == GSW_PUSH && c.fused == GSW_FUSED && fits && (long long)Ea <= se) {
                    go = 1;
                    if (r == 0) {
                        c.fmt = GSW_QUEUE;
                        book.bytes += 12ull * (unsigned long long)prev_va + 4ull * E_prev + 8ull * qn;
                        book.edges += E_prev;
                        if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)E_prev;
                        hist = book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
                        write_record(rc, t, c, f, 0u);
                        reset_cnt(rc.cnt + ((t + 2) % 3));
                    }
                }
            }
            if (go && r == 0 && t < kMaxHist) rc.rec[t].ctas = k;
            ts.go = go;
            ts.qn_next = 0u;
        }
        __syncthreads();
        TEAM_STAMP(4);
        if (!ts.go) break;
        if (!first) { Via -= (long long)qn; Eia -= (long long)Ea; }
        // (D) my slice [qn r/k, qn (r+1)/k) of the concatenated frontier, from its owners (DSMEM)
        const unsigned vs = (unsigned)((unsigned long long)qn * r / k);
        const unsigned m = (unsigned)((unsigned long long)qn * (r + 1) / k) - vs;
        for (unsigned i = tid; i < m; i += kBlock) {
            const unsigned idx = vs + i;
            unsigned lo = 0, hi = (unsigned)k;          // owner c: cq[c] <= idx < cq[c + 1]
            while (hi - lo > 1) {
                const unsigned mid = (lo + hi) >> 1;
                if (ts.cq[mid] <= idx) lo = mid; else hi = mid;
            }
            const unsigned j = idx - ts.cq[lo];
            const uint32_t *rb = cl.map_shared_rank(&ts.beg[cur][0], lo);
            const uint16_t *rd = cl.map_shared_rank(&ts.deg[cur][0], lo);
            ts.sbeg[i] = rb[j];
            ts.sscan[i] = rd[j];
        }
        __syncthreads();
        TEAM_STAMP(5);
        // exclusive scan of the slice's degrees (consecutive entries per thread)
        unsigned Em;
        {
            const unsigned per = (m + kBlock - 1) / kBlock, i0 = tid * per;
            uint32_t loc = 0;
            for (unsigned j = 0; j < per; ++j)
                if (i0 + j < m) loc += ts.sscan[i0 + j];
            uint32_t tot;
            uint32_t ex = block_excl_scan(loc, ts.red, &tot);
            for (unsigned j = 0; j < per; ++j) {
                if (i0 + j < m) { const uint32_t d = ts.sscan[i0 + j]; ts.sscan[i0 + j] = ex; ex += d; }
            }
            if (tid == 0) ts.sscan[m] = tot;
            Em = tot;
            __syncthreads();
        }
        TEAM_STAMP(6);
        if (book0) book_expand(book);
        // (E) Expand my slice's edges: columns, then claim + the winner's offsets (as bfs_solo)
        const int nx = cur == 2 ? 0 : cur + 1;
        {
            const uint32_t *scan = ts.sscan, *beg = ts.sbeg;
            const unsigned lo = (unsigned)(((unsigned long long)Em * tid) / kBlock);
            const unsigned hi = (unsigned)(((unsigned long long)Em * (tid + 1)) / kBlock);
            const unsigned mine = hi > lo ? (hi - lo + kSoloK - 1) / kSoloK : 0u;
            const unsigned nb = __reduce_max_sync(0xffffffffu, mine);
            unsigned i = 0, j = lo;
            if (lo < hi) {
                unsigned L = 0, R = m;
                while (R - L > 1) {
                    const unsigned mid = (L + R) >> 1;
                    if (scan[mid] <= lo) L = mid; else R = mid;
                }
                i = L;
            }
            for (unsigned bt = 0; bt < nb; ++bt) {
                int v[kSoloK];
#pragma unroll
                for (int q = 0; q < kSoloK; ++q) {
                    v[q] = -1;
                    if (j < hi) {
                        while (scan[i + 1] <= j) ++i;
                        v[q] = __ldg(col + beg[i] + (j - scan[i]));
                        ++j;
                    }
                }
                unsigned old[kSoloK];
                uint32_t vb[kSoloK], ve[kSoloK];
#pragma unroll
                for (int q = 0; q < kSoloK; ++q) {
                    old[q] = v[q] >= 0 ? atomicOr(V + (v[q] >> 5), 1u << (v[q] & 31)) : 0xffffffffu;
                    vb[q] = v[q] >= 0 ? __ldg(off + v[q]) : 0u;
                    ve[q] = v[q] >= 0 ? __ldg(off + v[q] + 1) : 0u;
                }
#pragma unroll
                for (int q = 0; q < kSoloK; ++q) {
                    const bool won = v[q] >= 0 && !((old[q] >> (v[q] & 31)) & 1u);
                    const unsigned mk = __ballot_sync(0xffffffffu, won);
                    if (!mk) continue;
                    unsigned base = 0;
                    if (lane_id() == (unsigned)(__ffs(mk) - 1)) base = atomicAdd(&ts.qn_next, (unsigned)__popc(mk));
                    base = __shfl_sync(0xffffffffu, base, __ffs(mk) - 1);
                    if (won) {
                        depth[v[q]] = t + 1;
                        const unsigned p = base + __popc(mk & lanemask_lt());
                        if (p < (unsigned)kTQ) { ts.q[nx][p] = v[q]; ts.beg[nx][p] = vb[q]; ts.deg[nx][p] = (uint16_t)min(ve[q] - vb[q], 65535u); }
                        else atomicExch(&rc.ctl->err, 0x7E0u);   // impossible by the capacity check
                    }
                }
            }
        }
        __syncthreads();
        TEAM_STAMP(7);
#if GSW_TEAM_PROF
        if (tid == 0) tp_acc[8] += 1;
#endif
        E_prev = Ea;
        if (book0) prev_va = (long long)qn;
        qn_l = ts.qn_next;
        cur = nx;
        par ^= 1;
        ++t;
        first = false;
    }
    // hand AS_t to the grid: my part at cq[r] of the queue; CTA 0 writes the counters and the state
    {
        int *gq = a.q[t & 1] + ts.cq[r];
        for (unsigned i = tid; i < qn_l; i += kBlock) gq[i] = ts.q[cur][i];
        if (book0) {
            IterCnt *c = rc.cnt + (t % 3);
            c->va = qn; c->ea = Ea; c->maxd = mxd; c->mind = mnd; c->qlen = qn; c->edges = E_prev;
            TeamPub p{};
            p.t = t; p.Via = Via; p.Eia = Eia;
            *rc.pub = p;
        }
    }
#if GSW_TEAM_PROF
    if (tid == 0 && (r == 0 || r == (unsigned)k - 1))
        for (int i = 0; i < 10; ++i) atomicAdd(&g_team_prof[r == 0 ? 0 : 1][i], tp_acc[i]);
    if (r == 0 && tid < (unsigned)k) atomicAdd(&g_team_late[tid], tp_late);
#endif
    // nobody may reuse this shared memory (aliased with the grid path's) while a peer could still
    // be reading it through DSMEM
    cluster_barrier();
}

template <int kResident>
__global__ void __launch_bounds__(kBlock, kResident) bfs_kernel(const __grid_constant__ BfsArgs a) {
    __shared__ BfsSmem bsm;
    LbSmem &sm = bsm.lb;
    __shared__ CtaQStore qs;
    __shared__ uint32_t red[kWarps + 1];
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5, src = map_in(a.g.inv, a.src);
    int *depth = a.depth;
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};

    if (is_book()) rc.ctl->t_start = globaltimer();
    // ---- init: depth, visited map, frontier bitmaps, counters, AS_0 = {src}
    // (relabeled symmetric graphs: the isolated vertices are the internal tail and never leave -1;
    // their depth entries are not written, the caller-order output takes -1 from iso_c)
    for (long long v = gtid(); v < a.n_init; v += gthreads()) depth[v] = (v == src) ? 0 : -1;
    if (gtid() == 0) depth[src] = 0;
    if (a.out && a.scatter)
        for (long long j = gtid(); j < n; j += gthreads()) a.out[j] = -1;
    for (long long w = gtid(); w < W; w += gthreads()) {
        unsigned x = a.iso[w];
        if (w == (src >> 5)) x |= 1u << (src & 31);
        a.V[w] = x;
        a.fb[0][w] = 0u; a.fb[1][w] = 0u; a.fb[2][w] = 0u;
    }
    const unsigned dsrc = __ldg(a.g.off + src + 1) - __ldg(a.g.off + src);
    if (is_book()) {
        for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
        rc.cnt[0].va = 1; rc.cnt[0].ea = dsrc; rc.cnt[0].maxd = dsrc; rc.cnt[0].mind = dsrc; rc.cnt[0].qlen = 1;
        a.q[0][0] = src;
    }
    cta_queue_reset(qs);
    const bool all_auto = rc.force.direction == GSW_AUTO && rc.force.format == GSW_AUTO &&
                          rc.force.load_balance == GSW_AUTO && rc.force.fusion == GSW_AUTO;
    const int team_k = rc.team_k;
    const bool solo_allowed = (rc.solo_e > 0 || team_k > 1) && all_auto;
    bool last_small = false;
    long long Via = (long long)n - 1, Eia = (long long)a.g.nnz - dsrc;
    int mat = MAT_SQUEUE;
    bool dirty[3] = {false, false, false};
    Features f = rc.base;
    int prev_dir = GSW_PUSH;
    long long prev_va = 0, prev_via = 0;
    int t = 0;
    // CTA 0 / thread 0's run bookkeeping lives in shared memory: as a spilled local it was
    // re-fetched from L2 after every grid barrier (the barrier's acquire invalidates L1), a
    // dependent round trip on every level's critical path (C2 SSSP 42.6 -> 41.7 ms)
    __shared__ Book book_s;
    if (threadIdx.x == 0) book_s = Book();
    Book &book = book_s;
    grid_sync(bar, epoch);
    if (is_book()) rc.ctl->t_phase = globaltimer();
    for (;; ++t) {
        IterCnt *cur = rc.cnt + (t % 3), *nxt = rc.cnt + ((t + 1) % 3);
        if (is_book()) book_start(book, rc, t, nxt);
        const CntView cv = cta_read_cnt(cur);       // one L2 round trip per CTA per iteration
        const unsigned long long va = cv.va, ea = cv.ea;
        if (is_book() && t > 0) {
            // algorithmic bytes of iteration t-1 (DESIGN.md roofline model D0)
            book.bytes += prev_dir == GSW_PUSH
                ? 12ull * prev_va + 4ull * cv.edges + 8ull * va
                : (unsigned long long)n / 4 + 8ull * (unsigned long long)max(0LL, prev_via - a.iso_count) +
                      4ull * cv.edges + 4ull * va;
            book.edges += cv.edges;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)cv.edges;
        }
        if (va == 0) break;
        if (t > 0) { Via -= (long long)va; Eia -= (long long)ea; }
        f.Va = (long long)va; f.Ea = (long long)ea; f.Via = Via; f.Eia = Eia;
        f.maxd = cv.maxd; f.mind = cv.mind; f.iter = t;
        hist_features(cv, f);
        const DevCfg c = select_traversal(f, rc.force);
        write_record(rc, t, c, f, 0u);
        if (is_book()) reset_cnt(rc.cnt + ((t + 2) % 3));
        // CTA-resident tier: CTA 0 runs the levels alone while the frontier stays tiny
        // (entered only after two consecutive small levels: a one-level episode costs more in
        // park/wake and hand-back than it saves, measured on C1/C3)
        // (cluster launch: the team tier of cluster 0 takes the place of the solo CTA, sized by the
        // capacity of its parts instead of the solo thresholds)
        const unsigned long long per = (va + (unsigned)team_k - 1) / (unsigned)team_k;
        const bool small = team_k > 1
            ? (va > 0 && per <= (unsigned long long)kTQ && (unsigned long long)cv.maxd * per <= (unsigned long long)kTQ &&
               (long long)ea <= rc.team_e)
            : ((long long)ea <= rc.solo_e && (long long)va <= rc.solo_v && va <= (unsigned long long)kSQ);
        const bool solo = solo_allowed && small && last_small && c.dir == GSW_PUSH && c.fused == GSW_FUSED &&
                          (mat == MAT_QUEUE || mat == MAT_SQUEUE);
        last_small = small;
        if (solo && team_k > 1) {
            TeamSmem &tsm = *reinterpret_cast<TeamSmem *>(&bsm);
            if ((int)blockIdx.x < team_k) {
                if (is_book()) { *reinterpret_cast<Book *>(tsm.book_raw) = book; tsm.prev_va = prev_va; }
                bfs_team(a, tsm, t, Via, Eia, f, cv.qlen, team_k);
                if (is_book()) { book = *reinterpret_cast<const Book *>(tsm.book_raw); prev_va = tsm.prev_va; }
                prev_dir = GSW_PUSH;
                grid_sync(bar, epoch);
            } else {
                grid_park(bar, epoch);
            }
            TeamPub p;
            pub_read(rc.pub, p);
            t = (int)p.t; Via = p.Via; Eia = p.Eia;
            mat = MAT_QUEUE;
            if (dirty[0] || dirty[1] || dirty[2]) {
                for (int i = 0; i < 3; ++i) if (dirty[i]) { clear_words(a.fb[i], W); dirty[i] = false; }
                grid_sync(bar, epoch);
            }
            --t;
            continue;
        }
        if (solo) {
            if (blockIdx.x == 0) {
                if (threadIdx.x == 0) { *reinterpret_cast<Book *>(bsm.solo.book_raw) = book; bsm.solo.prev_va = prev_va; }
                bfs_solo(a, bsm.solo, t, Via, Eia, f, cv.qlen);
                if (threadIdx.x == 0) { book = *reinterpret_cast<const Book *>(bsm.solo.book_raw); prev_va = bsm.solo.prev_va; }
                prev_dir = GSW_PUSH;
                grid_sync(bar, epoch);
            } else {
                grid_park(bar, epoch);
            }
            TeamPub p;
            pub_read(rc.pub, p);
            t = (int)p.t; Via = p.Via; Eia = p.Eia;
            mat = MAT_QUEUE;
            if (dirty[0] || dirty[1] || dirty[2]) {          // the grid's next Filter expects clean maps
                for (int i = 0; i < 3; ++i) if (dirty[i]) { clear_words(a.fb[i], W); dirty[i] = false; }
                grid_sync(bar, epoch);
            }
            --t;
            continue;
        }
        const int b2 = (t + 2) % 3;
        if (dirty[b2]) { clear_words(a.fb[b2], W); dirty[b2] = false; }

        // ---------------- Filter: materialise AS_t in the selected format
        const bool push = c.dir == GSW_PUSH;
        int need;
        if (push) need = c.fmt == GSW_BITMAP ? MAT_BITMAP : (c.fmt == GSW_QUEUE ? MAT_QUEUE : MAT_SQUEUE);
        else need = c.fmt == GSW_BITMAP ? MAT_BITMAP : MAT_NONE;
        int *qa = a.q[t & 1];
        unsigned *fbt = a.fb[t % 3];
        bool filtered = false, qlen_changed = false;
        const int lvl = t;
        auto is_active = [&](int v) { return depth[v] == lvl; };
        if (need == MAT_BITMAP && mat != MAT_BITMAP) {
            if (mat == MAT_QUEUE || mat == MAT_SQUEUE) bm_from_q(fbt, qa, cv.qlen);
            else bm_from_pred(fbt, n, is_active);
            dirty[t % 3] = true;
            mat = MAT_BITMAP;
            filtered = true;
        } else if (need == MAT_QUEUE && mat != MAT_QUEUE && mat != MAT_SQUEUE) {
            if (mat == MAT_BITMAP) q_from_bm(qa, &cur->qlen, fbt, W, 0u);
            else q_from_pred(qa, &cur->qlen, n, is_active);
            mat = MAT_QUEUE;
            filtered = qlen_changed = true;
        } else if (need == MAT_SQUEUE && mat != MAT_SQUEUE) {
            if (mat != MAT_BITMAP) {
                if (mat == MAT_QUEUE) bm_from_q(fbt, qa, cv.qlen);
                else bm_from_pred(fbt, n, is_active);
                dirty[t % 3] = true;
                grid_sync(bar, epoch);
            }
            sq_from_bm_p1(fbt, W, 0u, rc.partial, red);
            grid_sync(bar, epoch);
            sq_from_bm_p2(qa, &cur->qlen, fbt, W, 0u, rc.partial, red);
            mat = MAT_SQUEUE;
            filtered = qlen_changed = true;
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
        if (is_book()) book_expand(book);

        // ---------------- Expand
        LocalCnt lc;
        const bool fused = c.fused == GSW_FUSED;
        // fused push writes the next active set directly ("write u to AS directly"):
        // as a warp-aggregated queue append when the claims are few, as bitmap marking (the
        // paper's duplicate-tolerant technique) when a single queue counter would be
        // the contended address
        const bool mark_bitmap = (long long)ea > (long long)(n >> 6);
        const bool next_bitmap = !push || mark_bitmap;
        if (push) {
            const BfsPushOp op{depth, a.V, a.g.off, t + 1, fused ? (mark_bitmap ? 2 : 1) : 0,
                               cta_queue(qs, a.q[(t + 1) & 1], &nxt->qlen), a.fb[(t + 1) % 3]};
            if (fused && mark_bitmap) dirty[(t + 1) % 3] = true;
            if (mat == MAT_BITMAP) {
                lc = run_lb(c.lb, BitmapSrc{fbt, (unsigned)n, 1u}, adj_out, op, sm, red, bar, epoch, rc.partial, a.scan);
            } else {
                const unsigned ql = qlen_changed ? cta_read_u32(&cur->qlen) : cv.qlen;
                lc = run_lb(c.lb, QueueSrc{qa, ql}, adj_out, op, sm, red, bar, epoch, rc.partial, a.scan);
            }
        } else {
            const BfsPullOp op{depth, a.V, a.g.off, c.fmt == GSW_BITMAP ? fbt : nullptr, t, fused, a.fb[(t + 1) % 3]};
            if (c.fmt == GSW_BITMAP && c.lb == GSW_LB_THREAD) {
                static_assert(sizeof(LbSmem) >= sizeof(int) * (kPullList + kPullWordsPerWarp) * kWarps, "pull lists live in the LB smem");
#if GSW_PULL_PROF
                const unsigned long long p0 = globaltimer();
#endif
                lc = bfs_pull_list(fbt, a.V, depth, a.g.in_off, a.g.in_col, a.g.in_first, a.g.off, a.g.in_off == a.g.off, t,
                                   fused ? a.fb[(t + 1) % 3] : nullptr, n, reinterpret_cast<int *>(&sm));
#if GSW_PULL_PROF
                if (t < 8 && lane_id() == 0) {
                    const long long w = gwarp();
                    if (w < 16384) { g_pull_prof[t][w][0] = p0; g_pull_prof[t][w][1] = globaltimer(); }
                }
#endif
            } else if (c.fmt == GSW_BITMAP) {
                lc = run_lb(c.lb, BitmapSrc{a.V, (unsigned)n, 0u}, adj_in, op, sm, red, bar, epoch, rc.partial, a.scan);
            } else {
                lc = run_lb(c.lb, QueueSrc{a.iq, cta_read_u32(&cur->iqlen)}, adj_in, op, sm, red, bar, epoch,
                            rc.partial, a.scan);
            }
            if (fused) dirty[(t + 1) % 3] = true;
        }
        if (push && fused && !mark_bitmap) cta_queue_flush(qs, a.q[(t + 1) & 1], &nxt->qlen);
        flush_counts(lc, nxt);
        grid_sync(bar, epoch);
        mat = fused ? (next_bitmap ? MAT_BITMAP : MAT_QUEUE) : MAT_NONE;
        prev_dir = c.dir;
        prev_va = (long long)va;
        prev_via = Via;
    }
    if (is_book()) rc.ctl->t_expand = globaltimer();
    if (a.out && a.scatter) {
        // caller order by scattering: coalesced reads of depth and perm over the non-isolated
        // prefix, a fire-and-forget store for every reached vertex (the output was -1 from init)
        constexpr int kG = 8;
        const long long T0 = gtid(), NT = gthreads();
        for (long long base = T0; base < a.n_init; base += kG * NT) {
            int dv[kG];
            uint32_t pv[kG];
#pragma unroll
            for (int k = 0; k < kG; ++k) {
                const long long v = base + k * NT;
                dv[k] = v < a.n_init ? depth[v] : -1;
                pv[k] = v < a.n_init ? __ldg(a.g.perm + v) : 0u;
            }
#pragma unroll
            for (int k = 0; k < kG; ++k)
                if (dv[k] >= 0) a.out[pv[k]] = dv[k];
        }
        if (gtid() == 0) a.out[a.src] = 0;          // the source may be an isolated vertex (tail)
    } else if (a.out) {
        // caller order: isolated vertices (iso_c) are -1 without touching depth (their entries were
        // never initialised); the others gather depth[inv[j]], kG loads in flight per thread
        constexpr int kG = 8;
        const long long T0 = gtid(), NT = gthreads();
        for (long long base = T0; base < n; base += kG * NT) {
            int ix[kG], val[kG];
            unsigned isw[kG];
#pragma unroll
            for (int k = 0; k < kG; ++k) {          // independent loads: the isolated word and inv[j]
                const long long j = base + k * NT;
                isw[k] = j < n ? __ldg(a.iso_c + (j >> 5)) : ~0u;
                ix[k] = j < n ? (int)__ldg(a.g.inv + j) : -1;
            }
#pragma unroll
            for (int k = 0; k < kG; ++k) {
                const long long j = base + k * NT;
                const bool iso = ((isw[k] >> (j & 31)) & 1u) && j != a.src;
                val[k] = (ix[k] >= 0 && !iso) ? depth[ix[k]] : -1;
            }
#pragma unroll
            for (int k = 0; k < kG; ++k) {
                const long long j = base + k * NT;
                if (j < n) a.out[j] = val[k];
            }
        }
    }
    if (is_book()) { book_finish(book, rc, t); rc.ctl->t_end = globaltimer(); }
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
    a.iso_c = g->iso_caller;
    a.src = source;
    const bool relabeled = g->g.inv != nullptr;
    // relabeled (degree-descending) symmetric graphs keep their isolated vertices as the internal
    // tail [n - isolated, n): only the prefix needs depth = -1 (the output reads iso_c for the rest)
    a.n_init = (relabeled && g->symmetric && g->iso_caller) ? (int)(n - g->attrs.isolated) : n;
    a.depth = (dev_out && !relabeled) ? depth_out : (int *)ws.take((size_t)n * 4);
    a.out = relabeled ? (dev_out ? depth_out : (int *)ws.take((size_t)n * 4)) : nullptr;
    // scatter measured faster on C3 (0.1556 vs 0.1594 ms per root, profiles/r2/bfs_output_scatter_ab.txt)
    // but only while the caller-order array stays in L2: at C5 (268 MB) the scattered 4-byte stores
    // become DRAM read-modify-writes (single-GPU BFS 653 -> 466 GTEPS), so it is used up to 8M vertices
    a.scatter = std::getenv("GSW_BFS_SCATTER") ? std::atoi(std::getenv("GSW_BFS_SCATTER")) : (n <= (1 << 23) ? 1 : 0);
    a.V = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 3; ++i) a.fb[i] = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 2; ++i) a.q[i] = (int *)ws.take((size_t)n * 4);
    a.iq = (int *)ws.take((size_t)n * 4);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    a.iso_count = g->attrs.isolated;
    LaunchInfo li;
    // Residency per graph shape (profiles/r2/minblocks_ab_*, ab_m4.txt): road-like graphs (mean
    // degree below 8: thousands of tiny levels) run one CTA per SM, the cheapest grid barrier (C2
    // 28 ms vs 31 ms at 2/SM); scale-free graphs keep kMinBlocksBfs (C3: 0.150 ms at 2/SM vs 0.174
    // at 4/SM, 0.23 at 1/SM), except very large ones (2^24+ vertices), whose levels are long enough
    // that the extra warps hiding gather latency outweigh the dearer barrier (C5: 1.05 / 2.21 ms per
    // root at 4/SM vs 1.29 / 3.09 ms at 2/SM).
    const bool fixed = std::getenv("GSW_MINB_BFS_FIXED") != nullptr;
    const bool roadlike = g->attrs.dbar < 8.0 && kMinBlocksBfs >= 2 && !fixed;
    const bool huge = !roadlike && n >= (1ll << 24) && kMinBlocksBfs == 2 && !fixed;
    const void *kern = roadlike ? (const void *)bfs_kernel<1>
                       : huge   ? (const void *)bfs_kernel<4>
                                : (const void *)bfs_kernel<kMinBlocksBfs>;
    gsw_status s = prepare_common(g, ws, kern, a.rc, li, roadlike ? 1 : huge ? 4 : kMinBlocksBfs);
    if (s != GSW_OK) return s;
    // road-like graphs: clustered launch, cluster 0 runs the small levels as a team
    if (roadlike) setup_team(g, kern, a.rc, li);
    // BFS selector: hand-set rules (default) or the learned trees (GSW_SELECTOR=trees)
    if (const char *sel = std::getenv("GSW_SELECTOR")) a.rc.base.selector = std::strcmp(sel, "trees") == 0 ? 1 : 0;
    if (!a.depth || !a.V || !a.fb[2] || !a.q[1] || !a.iq || !a.scan) { set_error("workspace too small"); return GSW_ENOMEM; }
    void *args[] = {&a};
    s = launch_persistent(g, kern, args, li);
    if (s != GSW_OK) return s;
#if GSW_PULL_PROF
    {
        static unsigned long long h[8][16384][2];
        GSW_CUDA(cudaStreamSynchronize(g->stream));
        GSW_CUDA(cudaMemcpyFromSymbol(h, g_pull_prof, sizeof(h)));
        const int nw = li.grid * (kBlock / 32);
        for (int lv = 0; lv < 8; ++lv) {
            std::vector<double> d;
            unsigned long long lo = ~0ull, hi = 0;
            for (int w = 0; w < nw && w < 16384; ++w) {
                if (!h[lv][w][0] || h[lv][w][1] < h[lv][w][0]) continue;
                d.push_back((double)(h[lv][w][1] - h[lv][w][0]) * 1e-3);
                lo = std::min(lo, h[lv][w][0]); hi = std::max(hi, h[lv][w][1]);
            }
            if (d.empty()) continue;
            std::sort(d.begin(), d.end());
            std::fprintf(stderr, "pull level %d: warps %zu span %.2f us  warp us: min %.2f p50 %.2f p90 %.2f p99 %.2f max %.2f\n",
                         lv, d.size(), (hi - lo) * 1e-3, d.front(), d[d.size() / 2], d[d.size() * 9 / 10],
                         d[d.size() * 99 / 100], d.back());
        }
        static const unsigned long long z[8][16384][2] = {};
        GSW_CUDA(cudaMemcpyToSymbol(g_pull_prof, z, sizeof(z)));
    }
#endif
#if GSW_TEAM_PROF
    {
        unsigned long long h[2][10];
        GSW_CUDA(cudaStreamSynchronize(g->stream));
        GSW_CUDA(cudaMemcpyFromSymbol(h, g_team_prof, sizeof(h)));
        static const char *nm[10] = {"loop/start", "A features", "cluster barrier", "B records", "C selector",
                                    "D slice copy", "scan", "E expand", "-", "B first reads"};
        unsigned long long late[16];
        GSW_CUDA(cudaMemcpyFromSymbol(late, g_team_late, sizeof(late)));
        if (h[0][8]) {
            std::fprintf(stderr, "team arrival lateness per CTA (us):");
            for (int c = 0; c < 16; ++c) std::fprintf(stderr, " %.2f", (double)late[c] * 1e-3 / (double)h[0][8]);
            std::fprintf(stderr, "\n");
        }
        static const unsigned long long zl[16] = {};
        GSW_CUDA(cudaMemcpyToSymbol(g_team_late, zl, sizeof(zl)));
        for (int c = 0; c < 2; ++c) {
            if (!h[c][8]) continue;
            std::fprintf(stderr, "team prof CTA %s: %llu levels;", c ? "k-1" : "0", h[c][8]);
            for (int i = 0; i < 10; ++i) if (i != 8) std::fprintf(stderr, " %s %.2f us", nm[i], (double)h[c][i] * 1e-3 / (double)h[c][8]);
            std::fprintf(stderr, "\n");
        }
        static const unsigned long long z[2][10] = {};
        GSW_CUDA(cudaMemcpyToSymbol(g_team_prof, z, sizeof(z)));
    }
#endif
    if (!dev_out)
        GSW_CUDA(cudaMemcpyAsync(depth_out, relabeled ? a.out : a.depth, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
