// sssp.cu -- single-source shortest paths with GSWITCH's stepping pattern (P4, PAPER.md:548-556,
// 646-666; footnote 2 P:411-413) on the persistent Filter/Expand engine.
// Ordered, label-correcting near/far scheme (reading R5/R7):
//   - the active (near) set N_t = vertices improved in round t-1 with dist < theta;
//   - improved vertices with dist >= theta go to the far set F (deferred);
//   - Expand relaxes every edge out of N_t: nd = dist[u] + w(u,v); atomicMin(dist[v], nd)
//     (compAtomic, push) or dist[v] = min over near in-neighbours (comp, pull reduction);
//   - when N_t is empty, theta advances and F is split: dist < theta -> N, the rest stays in F;
//   - terminate when N and F are empty.
// Stepping candidates for the threshold theta (gsw_config.stepping):
//   AUTO (dynamic stepping): per round, compare the active edges with the previous round's: grown
//   by more than 35% -> Increase (theta += delta0), shrunk by more than 35% -> Decrease
//   (theta -= delta0/2, never below the last split point), otherwise Remain (law 1;
//   alternative readings selectable with GSW_SSSP_LAW for calibration);
//   INCREASE / DECREASE / REMAIN pin that per-round decision; STATIC = delta-stepping with a fixed
//   step (theta moves only at splits); UNORDERED = Bellman-Ford (theta = infinity).
// delta0 = gsw_config.delta0, or c*wbar/dbar with c = 32 (reading R6b).
// Any schedule reaches the exact distances (they are the unique fixpoint); only speed differs.
#include <cstdlib>

#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"
#include "lb_reduce.cuh"

namespace gsw {

enum { SM_NONE = 0, SM_QUEUE = 1, SM_SQUEUE = 2, SM_BITMAP = 3 };
enum { ST_DYNAMIC = 0, ST_STATIC = 1, ST_UNORDERED = 2, ST_INC = 3, ST_DEC = 4, ST_REMAIN = 5 };
// Law 1 (the literal reading of P:651-654, "if the number of edges increases or decreases by some
// margin, we increase or decrease the priority threshold accordingly") measured best: C2 SSSP
// 62.7 ms vs 87.1 ms for law 0 and 79.6 ms for static delta (tools/sssp_law_sweep.py, DESIGN R7).
constexpr int kDefaultLaw = 1;

struct SplitCnt {
    unsigned long long va, ea;
    unsigned qlen, kept, minf, pad;
};

struct SsspArgs {
    DevGraph g;
    int src;              // caller id
    unsigned *dist;       // internal order
    unsigned *out;        // caller order (relabeled graphs), else nullptr
    unsigned *nb[3];      // near-set bitmaps (ring of 3); also the claim map of the next near set
    int *q[2];            // near queues
    unsigned *chg;        // "improved this round" status flags (standalone filter)
    unsigned *farbit;     // far-set membership
    int *fq[2];           // far queues
    unsigned *flen;       // far queue append counters [2]
    SplitCnt *split;      // [2]
    uint32_t *scan;
    unsigned delta0;
    int mode;
    int law;              // dynamic-stepping control law (R7); GSW_SSSP_LAW overrides
    RunCommon rc;
};

struct SsTok { unsigned old, nd; };
struct SsAux { unsigned nclaim, fclaim; uint32_t d0, d1; };

// classify an improved vertex: near (claim the next near map) or far (claim the far map)
struct SsClassify {
    unsigned *nnb;
    unsigned *farbit;
    unsigned theta;
    bool fused;
    unsigned *chg;
};

// push: relax (u, v): nd = dist[u] + w; atomicMin(dist[v], nd)
struct SsspPushOp {
    unsigned *dist;
    const uint32_t *w;
    const uint32_t *off;
    SsClassify cl;
    bool use_q;           // next near set as a queue (fused, few claims) or bitmap marking only
    CtaQueue nq;          // CTA-staged appends (common.cuh)
    CtaQueue fq;
    using Probe = uint2;  // (dist[u] + w(u,v), dist[v])
    using Tok = SsTok;
    using Aux = SsAux;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int u, uint32_t e, int v) const {
        return make_uint2(dist[u] + __ldg(w + e), dist[v]);
    }
    __device__ __forceinline__ Tok act(int, uint32_t, int v, Probe p) const {
        return SsTok{p.x < p.y ? atomicMin(dist + v, p.x) : 0u, p.x < p.y ? p.x : 0xffffffffu};
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int v, Tok t) const {
        SsAux a{~0u, ~0u, 0u, 0u};
        if (!(t.nd < t.old)) return a;
        const unsigned bit = 1u << (v & 31);
        if (!cl.fused) { atomicOr(cl.chg + (v >> 5), bit); return a; }
        if (t.nd < cl.theta) {
            a.nclaim = atomicOr(cl.nnb + (v >> 5), bit);
            a.d0 = __ldg(off + v); a.d1 = __ldg(off + v + 1);
        } else {
            a.fclaim = atomicOr(cl.farbit + (v >> 5), bit);
        }
        return a;
    }
    __device__ __forceinline__ bool commit(int, uint32_t, int v, Tok, Aux a, LocalCnt &c) const {
        const unsigned bit = 1u << (v & 31);
        const bool nw = !(a.nclaim & bit), fw = !(a.fclaim & bit);
        if (nw) {
            c.add_vertex(a.d1 - a.d0);
            if (use_q) nq.push(v);
        }
        if (fw) {
            c.aux++;
            fq.push(v);
        }
        return false;
    }
};

// pull: dist[v] = min(dist[v], min over near in-neighbours u of dist[u] + w(u,v))
struct SsspPullOp {
    unsigned *dist;
    const uint32_t *w;        // in-edge weights
    const unsigned *nbt;      // near set N_t
    const uint32_t *off;      // out-offsets
    SsClassify cl;
    CtaQueue fq;
    using Probe = uint2;      // (near word of u, dist[u])
    using Acc = unsigned long long;
    static constexpr bool kFlushEmpty = false;
    static __device__ __forceinline__ Acc identity() { return 0xffffffffull; }
    static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a < b ? a : b; }
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const { return make_uint2(nbt[u >> 5], dist[u]); }
    __device__ __forceinline__ Acc val(int, uint32_t e, int u, Probe p) const {
        return ((p.x >> (u & 31)) & 1u) ? (Acc)p.y + (Acc)__ldg(w + e) : identity();
    }
    __device__ __forceinline__ void flush(int v, Acc m, bool exclusive, LocalCnt &c) const {
        if (m >= 0xffffffffull) return;
        const unsigned nd = (unsigned)m;
        unsigned old;
        if (exclusive) { old = dist[v]; if (nd < old) dist[v] = nd; }
        else old = atomicMin(dist + v, nd);
        if (!(nd < old)) return;
        const unsigned bit = 1u << (v & 31);
        if (!cl.fused) { atomicOr(cl.chg + (v >> 5), bit); return; }
        if (nd < cl.theta) {
            if (!(atomicOr(cl.nnb + (v >> 5), bit) & bit)) c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
        } else if (!(atomicOr(cl.farbit + (v >> 5), bit) & bit)) {
            c.aux++;
            fq.push(v);
        }
    }
};

__device__ __forceinline__ DevCfg select_sssp(const Features &f, const gsw_config &force) {
    DevCfg c = select_traversal(f, force);
    if (c.dir == GSW_PULL && force.load_balance == GSW_AUTO) c.lb = GSW_LB_TWC;   // reduction: owner tiers
    return c;
}


// ---------------------------------------------------------------- CTA-resident tier (solo)
// The BFS tier of bfs.cu applied to the near/far rounds: while the
// selector keeps fused push and the near set stays below (solo_v vertices, solo_e edges) with a
// far set of at most kSSQ entries, CTA 0 runs the rounds alone -- near set, offsets, degree scan
// and dist[u] in shared memory, the stepping law evaluated per round exactly as in the grid loop,
// far-set splits done in place -- and the other CTAs park at one grid barrier.  Per round the
// dependent chain is: columns + weights, atomicMin on dist[v] issued with a speculative load of
// v's offsets, then the near / far claim.  The near claim map is cleared after each round by
// the CTA itself (it holds exactly the pushed vertices).
constexpr int kSSQ = 512;
struct SsSoloSmem {
    int q[2][kSSQ];
    uint32_t beg[2][kSSQ];
    uint32_t scan[2][kSSQ + 1];
    unsigned du[kSSQ];
    unsigned qn[2];
    unsigned long long ea;
    unsigned maxd, mind, minf;
    int go;
    uint32_t red[kWarps + 1];
    unsigned long long book_raw[(sizeof(Book) + 7) / 8];
    unsigned long long prev_va;
};
struct SsLoop {
    unsigned long long theta, floor_t, flen, prev_ea;
    int fcur, nsplit;
};

// warp-aggregated append of (v, beg, deg) to a shared near queue.  A round may claim more
// vertices than the shared queue holds (up to one per relaxed edge): entries p >= kSSQ spill to
// the same position of the grid's queue `spill` (the queue of the round being built), exactly as
// the BFS tier does (bfs.cu); such a round ends the episode, because the selector check (B)
// requires qn <= kSSQ to continue, and the hand-back leaves the spilled part in place.
__device__ __forceinline__ void solo_push(SsSoloSmem &ss, int nx, bool pred, int v, uint32_t b, uint32_t d,
                                          int *spill) {
    const unsigned act = __activemask();
    const unsigned m = __ballot_sync(act, pred);
    if (!m) return;
    const int leader = __ffs(m) - 1;
    unsigned base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(&ss.qn[nx], (unsigned)__popc(m));
    base = __shfl_sync(act, base, leader);
    if (pred) {
        const unsigned p = base + __popc(m & lanemask_lt());
        if (p < (unsigned)kSSQ) { ss.q[nx][p] = v; ss.beg[nx][p] = b; ss.scan[nx][p] = d; }
        else spill[p] = v;
    }
}

// Runs rounds t, t+1, ... on CTA 0 (all its threads); hands back the near set of the first round
// NOT run in a.q[t & 1] with its counters in rc.cnt[t % 3] and the loop state in rc.pub.
__device__ __noinline__ void sssp_solo(const SsspArgs &a, SsSoloSmem &ss, int t, SsLoop L, const Features fbase,
                                       unsigned qn0, DevCfg c0) {
    const RunCommon &rc = a.rc;
    const unsigned tid = threadIdx.x;
    const uint32_t *__restrict__ off = a.g.off;
    const int32_t *__restrict__ col = a.g.col;
    const uint32_t *__restrict__ wt = a.g.w;
    unsigned *dist = a.dist;
    const int n = a.g.n;
    Book &book = *reinterpret_cast<Book *>(ss.book_raw);
    const long long sv = rc.solo_v < (long long)kSSQ ? rc.solo_v : (long long)kSSQ, se = rc.solo_e;
    const unsigned long long kInf = 0xffffffffull, d0 = a.delta0;
    unsigned *nnb = a.nb[(t + 1) % 3];            // near claim map of every solo round (cleaned each round)
    for (unsigned i = tid; i < qn0; i += kBlock) {
        const int u = a.q[t & 1][i];
        const uint32_t b = __ldg(off + u), e = __ldg(off + u + 1);
        ss.q[0][i] = u; ss.beg[0][i] = b; ss.scan[0][i] = e - b;
    }
    int cur = 0;
    unsigned qn = qn0;
    bool first = true;
    unsigned long long E_prev = 0, Ea = 0;
    unsigned mxd = 0, mnd = 0;
    float4 hist = make_float4(0.f, 0.f, 0.f, 0.f);
    bool done_run = false;
    for (;;) {
        __syncthreads();
        // (S) near set empty: advance theta and split the far set (in place while it is small)
        while (qn == 0 && !first) {
            if (L.flen == 0) { done_run = true; break; }
            if (L.flen > (unsigned long long)kSSQ) break;                      // the grid splits big sets
            L.theta += d0;
            L.floor_t = L.theta;
            const int fsrc = L.fcur, fdst = L.fcur ^ 1;
            const unsigned Lf = (unsigned)L.flen;
            if (tid == 0) { ss.qn[cur] = 0u; ss.minf = 0xffffffffu; }
            __syncthreads();
            for (unsigned i = tid; i < Lf; i += kBlock) {
                const int v = __ldcg(a.fq[fsrc] + i);
                const unsigned dv = __ldcg(dist + v);
                const bool near = (unsigned long long)dv < L.theta;
                uint32_t b = 0, e = 0;
                if (near) {
                    atomicAnd(a.farbit + (v >> 5), ~(1u << (v & 31)));
                    b = __ldg(off + v); e = __ldg(off + v + 1);
                } else {
                    a.fq[fdst][atomicAdd(a.flen + fdst, 1u)] = v;
                    atomicMin(&ss.minf, dv);
                }
                solo_push(ss, cur, near, v, b, e - b, a.q[t & 1]);
            }
            __syncthreads();
            qn = ss.qn[cur];
            L.flen = Lf - qn;
            if (tid == 0) a.flen[fsrc] = 0u;
            L.fcur = fdst;
            L.nsplit++;
            if (qn == 0 && ss.minf != 0xffffffffu && (unsigned long long)ss.minf + 1 > L.theta + d0)
                L.theta = (unsigned long long)ss.minf + 1 - d0;               // jump over empty buckets
            __syncthreads();
        }
        if (done_run || qn == 0) {
            if (!first) break;
        }
        // (A) features of N_t and dist[u] of its vertices
        if (tid == 0) { ss.ea = 0ull; ss.maxd = 0u; ss.mind = 0xffffffffu; }
        __syncthreads();
        {
            unsigned long long lea = 0;
            unsigned lmx = 0, lmn = 0xffffffffu;
            const int *gq = a.q[t & 1];
            for (unsigned i = tid; i < qn; i += kBlock) {
                unsigned d;
                if (i < (unsigned)kSSQ) {
                    d = ss.scan[cur][i];
                    ss.du[i] = __ldcg(dist + ss.q[cur][i]);   // L2: atomicMin updates bypass this SM's L1
                } else {                                       // spilled entry: the episode ends here
                    const int u = gq[i];
                    d = __ldg(off + u + 1) - __ldg(off + u);
                }
                lea += d; lmx = d > lmx ? d : lmx; lmn = d < lmn ? d : lmn;
            }
            lea = warp_sum(lea); lmx = warp_max(lmx); lmn = warp_min(lmn);
            if (lane_id() == 0 && lea) { atomicAdd(&ss.ea, lea); atomicMax(&ss.maxd, lmx); atomicMin(&ss.mind, lmn); }
        }
        __syncthreads();
        Ea = ss.ea; mxd = ss.maxd; mnd = ss.mind;
        // (B) selector + stepping law on N_t (thread 0), same rules as the grid loop
        if (tid == 0) {
            int go = first ? 1 : 0;
            DevCfg c = c0;
            if (!first && qn > 0) {
                Features f = fbase;
                f.Va = (long long)qn; f.Ea = (long long)Ea; f.Via = (long long)n - f.Va; f.Eia = (long long)a.g.nnz - f.Ea;
                f.maxd = mxd; f.mind = mnd; f.iter = t;
                f.tf = hist.x; f.te = hist.y; f.Tf = hist.z; f.Te = hist.w;
                c = select_sssp(f, rc.force);
                if (c.dir == GSW_PUSH && c.fused == GSW_FUSED && (long long)qn <= sv && (long long)Ea <= se) {
                    go = 1;
                    int step = GSW_STEP_REMAIN;
                    if (t > 0 && L.prev_ea > 0) {
                        const double e = (double)Ea, ep = (double)L.prev_ea, lo = (double)gridDim.x * blockDim.x;
                        const bool drop = e < 0.65 * ep, grow = e > 1.35 * ep;
                        switch (a.law) {
                        case 1: step = grow ? GSW_STEP_INCREASE : (drop ? GSW_STEP_DECREASE : GSW_STEP_REMAIN); break;
                        case 2: step = e < lo ? GSW_STEP_INCREASE : (e > 8.0 * lo ? GSW_STEP_DECREASE : GSW_STEP_REMAIN); break;
                        case 3: step = (drop && e < lo) ? GSW_STEP_INCREASE : (grow ? GSW_STEP_DECREASE : GSW_STEP_REMAIN); break;
                        default: step = drop ? GSW_STEP_INCREASE : (grow ? GSW_STEP_DECREASE : GSW_STEP_REMAIN);
                        }
                    }
                    if (step == GSW_STEP_INCREASE) L.theta = min(kInf, L.theta + d0);
                    else if (step == GSW_STEP_DECREASE) L.theta = max(L.floor_t, L.theta > d0 / 2 ? L.theta - d0 / 2 : 0ull);
                    c.step = step;
                    L.prev_ea = Ea;
                    book.bytes += 12ull * ss.prev_va + 8ull * E_prev + 8ull * qn;
                    book.edges += E_prev;
                    if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)E_prev;
                    hist = book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
                    write_record(rc, t, c, f, (unsigned)min(L.theta, kInf));
                    reset_cnt(rc.cnt + ((t + 2) % 3));
                }
            }
            if (first) {
                const IterCnt *cs = rc.cnt + ((t + 1) % 3);
                hist = make_float4(cs->tf, cs->te, cs->Tf, cs->Te);
            }
            if (go && t < kMaxHist) rc.rec[t].ctas = 1;
            ss.go = go;
            ss.qn[cur ^ 1] = 0u;
            ss.minf = (unsigned)L.theta;            // broadcast theta (< 2^32 while rounds remain finite)
            ss.red[kWarps] = (unsigned)(L.theta >> 32);
        }
        __syncthreads();
        // every thread needs the same loop state: thread 0 evaluated the law, broadcast it
        L.theta = ((unsigned long long)ss.red[kWarps] << 32) | ss.minf;
        if (!ss.go) break;
        L.prev_ea = Ea;
        // (C) exclusive scan of the degrees
        {
            const unsigned per = (qn + kBlock - 1) / kBlock, i0 = tid * per;
            uint32_t loc = 0;
            for (unsigned k = 0; k < per; ++k) if (i0 + k < qn) loc += ss.scan[cur][i0 + k];
            uint32_t tot;
            uint32_t ex = block_excl_scan(loc, ss.red, &tot);
            for (unsigned k = 0; k < per; ++k)
                if (i0 + k < qn) { const uint32_t d = ss.scan[cur][i0 + k]; ss.scan[cur][i0 + k] = ex; ex += d; }
            if (tid == 0) ss.scan[cur][qn] = tot;
            __syncthreads();
        }
        if (tid == 0) book_expand(book);
        // (D) relax: columns + weights, atomicMin with the target's offsets, then near/far claim
        {
            const unsigned E = (unsigned)Ea;
            const int nx = cur ^ 1;
            const uint32_t *scan = ss.scan[cur], *beg = ss.beg[cur];
            const unsigned lo = (unsigned)(((unsigned long long)E * tid) / kBlock);
            const unsigned hi = (unsigned)(((unsigned long long)E * (tid + 1)) / kBlock);
            const unsigned mine = hi > lo ? (hi - lo + 3) / 4 : 0u;
            const unsigned nb = __reduce_max_sync(0xffffffffu, mine);
            unsigned i = 0, j = lo;
            if (lo < hi) {
                unsigned Lq = 0, R = qn;
                while (R - Lq > 1) { const unsigned m = (Lq + R) >> 1; if (scan[m] <= lo) Lq = m; else R = m; }
                i = Lq;
            }
            const unsigned long long th = L.theta;
            for (unsigned bt = 0; bt < nb; ++bt) {
                int v[4];
                unsigned nd[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    v[k] = -1; nd[k] = 0;
                    if (j < hi) {
                        while (scan[i + 1] <= j) ++i;
                        const uint32_t e = beg[i] + (j - scan[i]);
                        v[k] = __ldg(col + e);
                        nd[k] = ss.du[i] + __ldg(wt + e);
                        ++j;
                    }
                }
                unsigned old[4];
                uint32_t vb[4], ve[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    old[k] = v[k] >= 0 ? atomicMin(dist + v[k], nd[k]) : 0u;
                    vb[k] = v[k] >= 0 ? __ldg(off + v[k]) : 0u;
                    ve[k] = v[k] >= 0 ? __ldg(off + v[k] + 1) : 0u;
                }
                unsigned cl[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    cl[k] = 0xffffffffu;
                    if (v[k] >= 0 && nd[k] < old[k]) {
                        const unsigned bit = 1u << (v[k] & 31);
                        cl[k] = (unsigned long long)nd[k] < th ? atomicOr(nnb + (v[k] >> 5), bit)
                                                                : atomicOr(a.farbit + (v[k] >> 5), bit);
                    }
                }
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const bool won = cl[k] != 0xffffffffu && !((cl[k] >> (v[k] & 31)) & 1u);
                    const bool near = won && (unsigned long long)nd[k] < th;
                    solo_push(ss, nx, near, v[k], vb[k], ve[k] - vb[k], a.q[(t + 1) & 1]);
                    if (won && !near) a.fq[L.fcur][atomicAdd(a.flen + L.fcur, 1u)] = v[k];
                }
            }
            __syncthreads();
            // far appends of this round, then clean the near claim map (it holds exactly N_{t+1})
            const unsigned nq = ss.qn[nx];
            const int *gqn = a.q[(t + 1) & 1];
            for (unsigned k = tid; k < nq; k += kBlock)
                atomicAnd(nnb + ((k < (unsigned)kSSQ ? ss.q[nx][k] : __ldcg(gqn + k)) >> 5), 0u);
            __threadfence();
            __syncthreads();
            L.flen = *(volatile unsigned *)(a.flen + L.fcur);
            E_prev = E;
            if (tid == 0) ss.prev_va = qn;
            qn = nq;
            cur = nx;
            ++t;
            first = false;
        }
    }
    // hand N_t back to the grid
    {
        int *gq = a.q[t & 1];
        const unsigned m = qn < (unsigned)kSSQ ? qn : (unsigned)kSSQ;   // entries >= kSSQ were spilled in place
        for (unsigned k = tid; k < m; k += kBlock) gq[k] = ss.q[cur][k];
        if (tid == 0) {
            IterCnt *cc = rc.cnt + (t % 3);
            cc->va = qn; cc->ea = qn ? Ea : 0; cc->maxd = mxd; cc->mind = mnd; cc->qlen = qn; cc->edges = E_prev;
            cc->aux0 = 0u;
            TeamPub p{};
            p.t = t;
            p.aux[0] = L.theta; p.aux[1] = L.floor_t; p.aux[2] = L.flen; p.aux[3] = L.prev_ea;
            p.aux[4] = (unsigned long long)L.fcur; p.aux[5] = (unsigned long long)L.nsplit;
            *rc.pub = p;
        }
    }
}

union SsSmem {
    LbSmem push;
    LbRedSmem pull;
    SsSoloSmem solo;
};
static_assert(sizeof(SsSoloSmem) <= sizeof(LbSmem), "the solo tier must not grow the kernel's shared memory");

template <int kResident>
__global__ void __launch_bounds__(kBlock, kResident) sssp_kernel(const __grid_constant__ SsspArgs a) {
    __shared__ SsSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    __shared__ CtaQStore qs0, qs1;        // staged appends: near queue, far queue
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5, src = map_in(a.g.inv, a.src);
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};
    unsigned *dist = a.dist;

    // ---- init
    for (long long v = gtid(); v < n; v += gthreads()) dist[v] = (v == src) ? 0u : 0xffffffffu;
    for (long long w = gtid(); w < W; w += gthreads()) {
        a.nb[0][w] = 0u; a.nb[1][w] = 0u; a.nb[2][w] = 0u;
        a.chg[w] = 0u; a.farbit[w] = 0u;
    }
    const unsigned dsrc = __ldg(a.g.off + src + 1) - __ldg(a.g.off + src);
    if (is_book()) {
        for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
        rc.cnt[0].va = 1; rc.cnt[0].ea = dsrc; rc.cnt[0].maxd = dsrc; rc.cnt[0].mind = dsrc; rc.cnt[0].qlen = 1;
        a.q[0][0] = src;
        a.flen[0] = 0u; a.flen[1] = 0u;
        for (int i = 0; i < 2; ++i) { a.split[i] = SplitCnt{0ull, 0ull, 0u, 0u, 0xffffffffu, 0u}; }
    }
    cta_queue_reset(qs0);
    cta_queue_reset(qs1);
    grid_sync(bar, epoch);

    // CTA 0 / thread 0's run bookkeeping lives in shared memory: as a spilled local it was
    // re-fetched from L2 after every grid barrier (the barrier's acquire invalidates L1), a
    // dependent round trip on every level's critical path (C2 SSSP 42.6 -> 41.7 ms)
    __shared__ Book book_s;
    if (threadIdx.x == 0) book_s = Book();
    Book &book = book_s;
    Features f = rc.base;
    const unsigned long long kInf = 0xffffffffull;
    const unsigned d0 = a.delta0;
    unsigned long long theta = a.mode == ST_UNORDERED ? kInf : (unsigned long long)d0;
    unsigned long long floor_t = 0;
    unsigned long long flen = 0;          // |F| (identical in every thread)
    int fcur = 0;                         // far queue buffer receiving appends
    int nsplit = 0;
    unsigned long long prev_ea = 0;
    int mat = SM_SQUEUE;
    bool dirty[3] = {false, false, false};
    int prev_dir = GSW_PUSH;
    unsigned long long prev_va = 0;
    const bool solo_allowed = rc.solo_e > 0 && a.mode == ST_DYNAMIC && rc.force.direction == GSW_AUTO &&
                              rc.force.format == GSW_AUTO && rc.force.load_balance == GSW_AUTO &&
                              rc.force.fusion == GSW_AUTO && rc.force.stepping == GSW_AUTO;
    bool last_small = false;
    int t = 0;
    for (;; ++t) {
        IterCnt *cur = rc.cnt + (t % 3), *nxt = rc.cnt + ((t + 1) % 3);
        if (is_book()) book_start(book, rc, t, nxt);
        CntView cv = cta_read_cnt(cur);
        flen += cv.aux0;
        if (is_book() && t > 0) {
            book.bytes += 12ull * prev_va + 8ull * cv.edges + 8ull * cv.va +
                          (prev_dir == GSW_PULL ? 4ull * n + n / 8 : 0ull);
            book.edges += cv.edges;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)cv.edges;
        }
        // ---- near set empty: advance theta and split the far set (Filter of the far queue)
        while (cv.va == 0 && flen > 0) {
            SplitCnt *sp = a.split + (nsplit & 1);
            theta = theta + d0;
            floor_t = theta;
            const int fsrc = fcur, fdst = fcur ^ 1;
            // everything appended to fq[fsrc] so far: flen entries
            const unsigned L = (unsigned)flen;
            LocalCnt lc;
            unsigned lmin = 0xffffffffu;
            int *qa = a.q[t & 1];
            const CtaQueue qn = cta_queue(qs0, qa, &sp->qlen), qk = cta_queue(qs1, a.fq[fdst], a.flen + fdst);
            for (long long i = gtid(); i < L; i += gthreads()) {
                const int v = a.fq[fsrc][i];
                const unsigned dv = dist[v];
                if ((unsigned long long)dv < theta) {
                    atomicAnd(a.farbit + (v >> 5), ~(1u << (v & 31)));
                    lc.add_vertex(__ldg(a.g.off + v + 1) - __ldg(a.g.off + v));
                    qn.push(v);
                } else {
                    qk.push(v);
                    lc.aux++;
                    lmin = min(lmin, dv);
                }
            }
            cta_queue_flush(qs0, qa, &sp->qlen);
            cta_queue_flush(qs1, a.fq[fdst], a.flen + fdst);
            // per-CTA reduction into the split counters
            {
                unsigned long long va = block_sum(lc.va, (unsigned long long *)sm.push.cm.excl);
                unsigned long long ea = block_sum(lc.ea, (unsigned long long *)sm.push.cm.excl);
                unsigned kept = block_sum(lc.aux, red);
                unsigned mn = warp_min(lmin);
                __shared__ unsigned smin[kWarps];
                if (lane_id() == 0) smin[threadIdx.x >> 5] = mn;
                __syncthreads();
                if (threadIdx.x == 0) {
                    for (int i = 0; i < kWarps; ++i) mn = min(mn, smin[i]);
                    if (va) { atomicAdd(&sp->va, va); atomicAdd(&sp->ea, ea); }
                    if (kept) atomicAdd(&sp->kept, kept);
                    if (mn != 0xffffffffu) atomicMin(&sp->minf, mn);
                }
            }
            grid_sync(bar, epoch);
            __shared__ SplitCnt ssp;
            if (threadIdx.x == 0) {
                // plain loads after the barrier's acquire (L1 invalidated)
                ssp.va = sp->va; ssp.ea = sp->ea; ssp.qlen = sp->qlen; ssp.kept = sp->kept; ssp.minf = sp->minf;
            }
            __syncthreads();
            const SplitCnt r = ssp;
            __syncthreads();
            if (is_book()) {
                a.flen[fsrc] = 0u;                                   // drained buffer
                a.split[(nsplit + 1) & 1] = SplitCnt{0ull, 0ull, 0u, 0u, 0xffffffffu, 0u};
            }
            nsplit++;
            fcur = fdst;
            flen = r.kept;
            cv.va = r.va; cv.ea = r.ea; cv.qlen = r.qlen;
            cv.maxd = 0; cv.mind = 0;
            mat = SM_QUEUE;
            if (r.va == 0 && r.minf != 0xffffffffu && (unsigned long long)r.minf + 1 > theta + d0)
                theta = (unsigned long long)r.minf + 1 - d0;              // jump over empty buckets
        }
        if (cv.va == 0) break;
        f.Va = (long long)cv.va; f.Ea = (long long)cv.ea;
        f.Via = (long long)n - f.Va; f.Eia = (long long)a.g.nnz - f.Ea;
        f.maxd = cv.maxd; f.mind = cv.mind; f.iter = t;
        hist_features(cv, f);
        DevCfg c = select_sssp(f, rc.force);
        // ---- P4 stepping decision for this round
        int step = GSW_STEP_REMAIN;
        if (a.mode == ST_DYNAMIC && t > 0 && prev_ea > 0) {
            const double e = (double)cv.ea, ep = (double)prev_ea, lo = (double)gthreads();
            const bool drop = e < 0.65 * ep, grow = e > 1.35 * ep;
            switch (a.law) {
            case 1:  // literal: threshold follows the edge trend
                step = grow ? GSW_STEP_INCREASE : (drop ? GSW_STEP_DECREASE : GSW_STEP_REMAIN);
                break;
            case 2:  // absolute (Fig. 12(e)): raise while the round is latency-bound, lower when wasteful
                step = e < lo ? GSW_STEP_INCREASE : (e > 8.0 * lo ? GSW_STEP_DECREASE : GSW_STEP_REMAIN);
                break;
            case 3:  // relative 35% rule, raising only while latency-bound
                step = (drop && e < lo) ? GSW_STEP_INCREASE : (grow ? GSW_STEP_DECREASE : GSW_STEP_REMAIN);
                break;
            default: // inverse: refill a draining band, brake an exploding one
                step = drop ? GSW_STEP_INCREASE : (grow ? GSW_STEP_DECREASE : GSW_STEP_REMAIN);
            }
        } else if (a.mode == ST_INC) step = GSW_STEP_INCREASE;
        else if (a.mode == ST_DEC) step = GSW_STEP_DECREASE;
        if (a.mode != ST_UNORDERED && a.mode != ST_STATIC) {
            if (step == GSW_STEP_INCREASE) theta = min(kInf, theta + d0);
            else if (step == GSW_STEP_DECREASE) theta = max(floor_t, theta > d0 / 2 ? theta - d0 / 2 : 0ull);
        }
        c.step = a.mode == ST_STATIC ? GSW_STEP_STATIC : (a.mode == ST_UNORDERED ? GSW_STEP_UNORDERED : step);
        prev_ea = cv.ea;
        const unsigned th = (unsigned)min(theta, kInf);
        write_record(rc, t, c, f, th);
        if (is_book()) reset_cnt(rc.cnt + ((t + 2) % 3));
        // CTA-resident tier (see sssp_solo): entered after two consecutive small rounds
        {
            const bool small = (long long)cv.ea <= rc.solo_e && (long long)cv.va <= rc.solo_v &&
                               cv.va <= (unsigned long long)kSSQ && flen <= (unsigned long long)kSSQ;
            const bool solo = solo_allowed && small && last_small && c.dir == GSW_PUSH && c.fused == GSW_FUSED &&
                              mat == SM_QUEUE;
            last_small = small;
            if (solo) {
                if (blockIdx.x == 0) {
                    if (threadIdx.x == 0) { *reinterpret_cast<Book *>(sm.solo.book_raw) = book; sm.solo.prev_va = prev_va; }
                    sssp_solo(a, sm.solo, t, SsLoop{theta, floor_t, flen, prev_ea, fcur, nsplit}, f, cv.qlen, c);
                    if (threadIdx.x == 0) { book = *reinterpret_cast<const Book *>(sm.solo.book_raw); prev_va = sm.solo.prev_va; }
                    prev_dir = GSW_PUSH;
                    grid_sync(bar, epoch);
                } else {
                    grid_park(bar, epoch);
                }
                TeamPub p;
                pub_read(rc.pub, p);
                t = (int)p.t;
                theta = p.aux[0]; floor_t = p.aux[1]; flen = p.aux[2]; prev_ea = p.aux[3];
                fcur = (int)p.aux[4]; nsplit = (int)p.aux[5];
                mat = SM_QUEUE;
                if (dirty[0] || dirty[1] || dirty[2]) {      // the solo claim map is already clean
                    for (int i = 0; i < 3; ++i) if (dirty[i]) { clear_words(a.nb[i], W); dirty[i] = false; }
                    grid_sync(bar, epoch);
                }
                --t;
                continue;
            }
        }
        const int b2 = (t + 2) % 3;
        if (dirty[b2]) { clear_words(a.nb[b2], W); dirty[b2] = false; }

        // ---------------- Filter: materialise N_t in the selected format
        const bool push = c.dir == GSW_PUSH;
        int need;
        if (push) need = c.fmt == GSW_BITMAP ? SM_BITMAP : (c.fmt == GSW_QUEUE ? SM_QUEUE : SM_SQUEUE);
        else need = SM_BITMAP;                     // pull tests membership in N_t
        int *qa = a.q[t & 1];
        unsigned *nbt = a.nb[t % 3];
        bool filtered = false, qlen_changed = false;
        if (need == SM_BITMAP && mat != SM_BITMAP) {
            bm_from_q(nbt, qa, cv.qlen);
            dirty[t % 3] = true;
            mat = SM_BITMAP;
            filtered = true;
        } else if (need == SM_QUEUE && mat == SM_BITMAP) {
            q_from_bm(qa, &cur->qlen, nbt, W, 0u);
            mat = SM_QUEUE;
            filtered = qlen_changed = true;
        } else if (need == SM_SQUEUE && mat != SM_SQUEUE) {
            if (mat != SM_BITMAP) {
                bm_from_q(nbt, qa, cv.qlen);
                dirty[t % 3] = true;
                grid_sync(bar, epoch);
            }
            sq_from_bm_p1(nbt, W, 0u, rc.partial, red);
            grid_sync(bar, epoch);
            sq_from_bm_p2(qa, &cur->qlen, nbt, W, 0u, rc.partial, red);
            mat = SM_SQUEUE;
            filtered = qlen_changed = true;
        }
        if (filtered) grid_sync(bar, epoch);
        if (is_book()) book_expand(book);

        // ---------------- Expand
        const bool fused = c.fused == GSW_FUSED;
        unsigned *nnb = a.nb[(t + 1) % 3];
        const SsClassify cl{nnb, a.farbit, th, fused, a.chg};
        const bool use_q = push && fused && (long long)cv.ea <= (long long)(n >> 6);
        LocalCnt lc;
        if (push) {
            const SsspPushOp op{dist, a.g.w, a.g.off, cl, use_q, cta_queue(qs0, a.q[(t + 1) & 1], &nxt->qlen),
                                cta_queue(qs1, a.fq[fcur], a.flen + fcur)};
            if (mat == SM_BITMAP) {
                lc = run_lb(c.lb, BitmapSrc{nbt, (unsigned)n, 1u}, adj_out, op, sm.push, red, bar, epoch, rc.partial, a.scan);
            } else {
                const unsigned ql = qlen_changed ? cta_read_u32(&cur->qlen) : cv.qlen;
                lc = run_lb(c.lb, QueueSrc{qa, ql}, adj_out, op, sm.push, red, bar, epoch, rc.partial, a.scan);
            }
        } else {
            const SsspPullOp op{dist, a.g.in_w, nbt, a.g.off, cl, cta_queue(qs1, a.fq[fcur], a.flen + fcur)};
            lc = run_lb_reduce(c.lb, AllSrc{(unsigned)n}, adj_in, op, sm.pull, red, bar, epoch, rc.partial, a.scan);
        }
        dirty[(t + 1) % 3] = true;
        if (fused) {
            cta_queue_flush(qs0, a.q[(t + 1) & 1], &nxt->qlen);
            cta_queue_flush(qs1, a.fq[fcur], a.flen + fcur);
            flush_counts(lc, nxt);
            grid_sync(bar, epoch);
            mat = use_q ? SM_QUEUE : SM_BITMAP;
        } else {
            // standalone Filter: classify the improved vertices of this round
            LocalCnt ec;
            ec.edges = lc.edges;
            grid_sync(bar, epoch);
            const CtaQueue qf = cta_queue(qs1, a.fq[fcur], a.flen + fcur);
            for (long long w = gwarp(); w < W; w += gwarps()) {
                const unsigned m = a.chg[w];
                const int v = (int)(w * 32 + lane_id());
                bool near = false, far = false;
                if ((m >> lane_id()) & 1u) {
                    if ((unsigned long long)dist[v] < theta) {
                        near = true;
                        ec.add_vertex(__ldg(a.g.off + v + 1) - __ldg(a.g.off + v));
                    } else {
                        far = !(atomicOr(a.farbit + w, 1u << lane_id()) & (1u << lane_id()));
                    }
                }
                const unsigned nm = __ballot_sync(0xffffffffu, near);
                if (lane_id() == 0) { nnb[w] = nm; a.chg[w] = 0u; }
                if (far) ec.aux++;
                if (far) qf.push(v);
            }
            cta_queue_flush(qs1, a.fq[fcur], a.flen + fcur);
            flush_counts(ec, nxt);
            grid_sync(bar, epoch);
            mat = SM_BITMAP;
        }
        prev_dir = c.dir;
        prev_va = cv.va;
    }
    if (a.out) gather_out(a.out, dist, a.g.inv, n);
    if (is_book()) book_finish(book, rc, t);
}

gsw_status run_sssp(gsw_graph g, int32_t source, uint32_t *dist_out, gsw_run_stats *st) {
    const int n = g->g.n, W = (n + 31) / 32;
    if (!dist_out) { set_error("gsw_sssp: dist is NULL"); return GSW_EINVAL; }
    if (source < 0 || source >= n) { set_error("gsw_sssp: source out of range"); return GSW_EINVAL; }
    if (!g->g.w) { set_error("gsw_sssp: the graph has no weights"); return GSW_EINVAL; }
    if ((double)g->attrs.maxw * (double)(n - 1) >= 4294967295.0) {
        set_error("gsw_sssp: max_w * (n-1) does not fit the 32-bit distance type");
        return GSW_EOVERFLOW;
    }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(dist_out) == 1;
    SsspArgs a{};
    a.g = g->g;
    a.src = source;
    const bool relabeled = g->g.inv != nullptr;
    a.dist = (dev_out && !relabeled) ? dist_out : (unsigned *)ws.take((size_t)n * 4);
    a.out = relabeled ? (dev_out ? dist_out : (unsigned *)ws.take((size_t)n * 4)) : nullptr;
    for (int i = 0; i < 3; ++i) a.nb[i] = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 2; ++i) a.q[i] = (int *)ws.take((size_t)n * 4);
    for (int i = 0; i < 2; ++i) a.fq[i] = (int *)ws.take((size_t)n * 4);
    a.chg = (unsigned *)ws.take((size_t)W * 4);
    a.farbit = (unsigned *)ws.take((size_t)W * 4);
    a.flen = (unsigned *)ws.take(64);
    a.split = (SplitCnt *)ws.take(2 * sizeof(SplitCnt));
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    // P4 stepping mode and the static step delta0 = c*wbar/dbar (c = 32)
    const gsw_config &fc = g->forced;
    double dbar = g->attrs.dbar > 0 ? g->attrs.dbar : 1.0;
    double d0 = fc.delta0 ? (double)fc.delta0 : 32.0 * g->attrs.wbar / dbar;
    a.delta0 = (unsigned)std::max(1.0, std::min(d0, 2147483647.0));
    switch (fc.stepping) {
    case GSW_STEP_STATIC: a.mode = ST_STATIC; break;
    case GSW_STEP_UNORDERED: a.mode = ST_UNORDERED; break;
    case GSW_STEP_INCREASE: a.mode = ST_INC; break;
    case GSW_STEP_DECREASE: a.mode = ST_DEC; break;
    case GSW_STEP_REMAIN: a.mode = ST_REMAIN; break;
    default: a.mode = ST_DYNAMIC;
    }
    a.law = kDefaultLaw;
    if (const char *law = getenv("GSW_SSSP_LAW")) a.law = atoi(law);
    LaunchInfo li;
    // Residency per graph shape (profiles/r2/minblocks_ab_*): on road-like graphs (mean degree
    // below 8: every round is a few hundred to a few thousand vertices) one CTA per SM gives the
    // cheapest grid barrier (C2 43 ms vs 46 ms at 2/SM); scale-free graphs keep kMinBlocksSssp.
    const bool roadlike = g->attrs.dbar < 8.0 && kMinBlocksSssp >= 2 && !std::getenv("GSW_MINB_SSSP_FIXED");
    const void *kern = roadlike ? (const void *)sssp_kernel<1> : (const void *)sssp_kernel<kMinBlocksSssp>;
    gsw_status s = prepare_common(g, ws, kern, a.rc, li, roadlike ? 1 : kMinBlocksSssp);
    if (s != GSW_OK) return s;
    // SSSP's own solo thresholds (profiles/r2/solo_sweep_r2.txt, 2 CTAs/SM build): C2 45.2 ms at
    // (512 edges, 256 vertices) vs 46.6 ms at BFS's (2,048, 512) and 45.4 ms with the tier off
    if (!std::getenv("GSW_SOLO_E")) a.rc.solo_e = kSoloESssp;
    if (!std::getenv("GSW_SOLO_V")) a.rc.solo_v = kSoloVSssp;
    if (!a.dist || !a.nb[2] || !a.q[1] || !a.fq[1] || !a.chg || !a.farbit || !a.flen || !a.split || !a.scan) {
        set_error("workspace too small");
        return GSW_ENOMEM;
    }
    void *args[] = {&a};
    s = launch_persistent(g, kern, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out)
        GSW_CUDA(cudaMemcpyAsync(dist_out, relabeled ? a.out : a.dist, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
