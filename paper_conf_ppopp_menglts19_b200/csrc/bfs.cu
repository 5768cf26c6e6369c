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
    int src;              // caller id
    int *depth;           // internal order
    int *out;             // caller order (relabeled graphs), else nullptr
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

// Pull over the unvisited vertices of 16 visited-map words per warp (the THREAD candidate on the
// bitmap format, B200 version).  Pass 1: every unvisited vertex probes its first in-neighbour
// through the coalesced in_first array (after relabeling, the highest-degree neighbour -- the
// likeliest frontier member), which settles most vertices of the big middle level without the
// random col access.  Pass 2: the misses are compacted into shared memory and every lane runs
// kPullCur independent cursors over them, from their second edge;
// a cursor that finishes (frontier parent found, or row exhausted) immediately refills from the
// list, so a lane's time is the SUM of its scan lengths spread over kPullCur chains rather than
// the maximum over a warp.  Each vertex has exactly one owner lane, so its visited / next-frontier
// bits are set with fire-and-forget atomicOr (no returned value, no dependent round trip).
constexpr int kPullCur = 4;
constexpr int kPullWordsPerWarp = 16;
constexpr int kPullList = kPullWordsPerWarp * 32;
__device__ __noinline__ LocalCnt bfs_pull_list(const unsigned *__restrict__ fb, unsigned *__restrict__ V,
                                               int *__restrict__ depth, const uint32_t *__restrict__ in_off,
                                               const int32_t *__restrict__ in_col, const int32_t *__restrict__ in_first,
                                               const uint32_t *__restrict__ out_off, bool symmetric, int lvl,
                                               unsigned *__restrict__ nfb, int n, int *lists) {
    LocalCnt cnt;
    const int W = (n + 31) >> 5;
    const unsigned lane = lane_id();
    int *list = lists + (threadIdx.x >> 5) * (kPullList + kPullWordsPerWarp);
    unsigned *found_bits = reinterpret_cast<unsigned *>(list + kPullList);
    for (long long chunk = gwarp(); chunk * kPullWordsPerWarp < W; chunk += gwarps()) {
        const long long w0 = chunk * kPullWordsPerWarp;
        unsigned word = 0, orig = ~0u;
        if (lane < (unsigned)kPullWordsPerWarp && w0 + lane < W) {
            orig = V[w0 + lane];
            word = ~orig;                                   // padding bits are set in V
            found_bits[lane] = 0u;
        }
        // pass 1: probe the first in-neighbour (the highest-degree one) of every unvisited vertex,
        // coalesced through in_first, 4 words in flight; a miss with more edges joins the list
        unsigned total = 0;                                  // warp-uniform list length
        unsigned nz = __ballot_sync(0xffffffffu, word != 0u);  // words with unvisited vertices
#pragma unroll 1
        while (nz) {
            int y[4], vv[4], kk[4];
            uint32_t b[4], en[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                kk[j] = nz ? __ffs(nz) - 1 : -1;              // warp-uniform
                nz &= nz - 1u;
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const unsigned wm = __shfl_sync(0xffffffffu, word, kk[j] < 0 ? 0 : kk[j]);
                vv[j] = (int)((w0 + kk[j]) * 32 + lane);
                const bool act = kk[j] >= 0 && ((wm >> lane) & 1u);   // padding bits are set in V: vv < n
                y[j] = act ? __ldg(in_first + vv[j]) : -2;
                b[j] = act ? __ldg(in_off + vv[j]) : 0u;
                en[j] = act ? __ldg(in_off + vv[j] + 1) : 0u;
            }
            unsigned p[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) p[j] = y[j] >= 0 ? fb[y[j] >> 5] : 0u;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const bool hit = y[j] >= 0 && ((p[j] >> (y[j] & 31)) & 1u);
                if (y[j] >= 0) cnt.edges++;
                if (hit) {
                    depth[vv[j]] = lvl + 1;
                    cnt.add_vertex(symmetric ? en[j] - b[j] : __ldg(out_off + vv[j] + 1) - __ldg(out_off + vv[j]));
                }
                const unsigned hm = __ballot_sync(0xffffffffu, hit);
                if (lane == 0 && kk[j] >= 0) found_bits[kk[j]] = hm;
                const bool miss = y[j] >= 0 && !hit && en[j] - b[j] > 1u;
                const unsigned mm = __ballot_sync(0xffffffffu, miss);
                if (miss) list[total + __popc(mm & lanemask_lt())] = vv[j];
                total += __popc(mm);
            }
        }
        __syncwarp();
        // pass 2: cursors over the misses, from their second edge
        int v[kPullCur];
        uint32_t e[kPullCur], end[kPullCur], beg[kPullCur];
        unsigned next = lane;
#pragma unroll
        for (int j = 0; j < kPullCur; ++j) {
            v[j] = next < total ? list[next] : -1;
            next += 32;
        }
#pragma unroll
        for (int j = 0; j < kPullCur; ++j) {
            beg[j] = v[j] >= 0 ? __ldg(in_off + v[j]) : 0u;
            e[j] = beg[j] + 1;
            end[j] = v[j] >= 0 ? __ldg(in_off + v[j] + 1) : 0u;
        }
        for (;;) {
            bool any = false;
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) any |= v[j] >= 0;
            if (!any) break;
            int y[kPullCur];
            unsigned p[kPullCur];
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) y[j] = (v[j] >= 0 && e[j] < end[j]) ? __ldg(in_col + e[j]) : -1;
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) p[j] = y[j] >= 0 ? fb[y[j] >> 5] : 0u;
            int nv[kPullCur];
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) {
                nv[j] = v[j];
                if (v[j] < 0) continue;
                bool done = false;
                if (y[j] >= 0) {
                    cnt.edges++;
                    if ((p[j] >> (y[j] & 31)) & 1u) {
                        const int x = v[j];
                        depth[x] = lvl + 1;
                        atomicOr(found_bits + ((x >> 5) - w0), 1u << (x & 31));   // shared memory
                        cnt.add_vertex(symmetric ? end[j] - beg[j] : __ldg(out_off + x + 1) - __ldg(out_off + x));
                        done = true;
                    } else if (++e[j] >= end[j]) {
                        done = true;
                    }
                } else {
                    done = true;                     // empty row
                }
                if (done) { nv[j] = next < total ? list[next] : -1; next += 32; }
            }
            // refill: offsets of the newly taken entries
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) {
                if (nv[j] != v[j]) {
                    v[j] = nv[j];
                    beg[j] = v[j] >= 0 ? __ldg(in_off + v[j]) : 0u;
                    e[j] = beg[j] + 1;
                    end[j] = v[j] >= 0 ? __ldg(in_off + v[j] + 1) : 0u;
                }
            }
        }
        __syncwarp();
        // the warp owns its chunk's words: one store each for the visited map and AS_{t+1}
        if (lane < (unsigned)kPullWordsPerWarp && w0 + lane < W) {
            const unsigned fbits = found_bits[lane];
            if (fbits) V[w0 + lane] = orig | fbits;
            if (nfb) nfb[w0 + lane] = fbits;
        }
        __syncwarp();
    }
    return cnt;
}

__global__ void __launch_bounds__(kBlock, kMinBlocks) bfs_kernel(BfsArgs a) {
    __shared__ LbSmem sm;
    __shared__ CtaQStore qs;
    __shared__ uint32_t red[kWarps + 1];
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5, src = map_in(a.g.inv, a.src);
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
    const unsigned dsrc = __ldg(a.g.off + src + 1) - __ldg(a.g.off + src);
    if (is_book()) {
        for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
        rc.cnt[0].va = 1; rc.cnt[0].ea = dsrc; rc.cnt[0].maxd = dsrc; rc.cnt[0].mind = dsrc; rc.cnt[0].qlen = 1;
        a.q[0][0] = src;
    }
    cta_queue_reset(qs);
    grid_sync(bar, epoch);

    Book book;
    long long Via = (long long)n - 1, Eia = (long long)a.g.nnz - dsrc;
    int mat = MAT_SQUEUE;
    bool dirty[3] = {false, false, false};
    Features f = rc.base;
    int prev_dir = GSW_PUSH;
    long long prev_va = 0, prev_via = 0;
    int t = 0;
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
                lc = bfs_pull_list(fbt, a.V, depth, a.g.in_off, a.g.in_col, a.g.in_first, a.g.off, a.g.in_off == a.g.off, t,
                                   fused ? a.fb[(t + 1) % 3] : nullptr, n, reinterpret_cast<int *>(&sm));
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
    if (a.out) gather_out(a.out, depth, a.g.inv, n);
    if (is_book()) book_finish(book, rc, t);
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
    const bool relabeled = g->g.inv != nullptr;
    a.depth = (dev_out && !relabeled) ? depth_out : (int *)ws.take((size_t)n * 4);
    a.out = relabeled ? (dev_out ? depth_out : (int *)ws.take((size_t)n * 4)) : nullptr;
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
    if (!dev_out)
        GSW_CUDA(cudaMemcpyAsync(depth_out, relabeled ? a.out : a.depth, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
