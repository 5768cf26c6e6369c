// cc.cu -- connected components ("edge-centric") as min-label
// propagation in GSWITCH's Filter/Expand form (reading R8): label[v] starts at v; the
// active set is the vertices whose label changed in the previous iteration; Expand propagates
// labels either by push (compAtomic = atomicMin on the neighbour) or by pull (comp = min over the
// active in-neighbours, an atomic-free reduction for owner mappings).  The fixpoint is
// label[v] = min vertex id of v's component.  Terminates when no label changed.
//   Filter: fused  -> Expand marks changed vertices in the next active-set bitmap
//           standalone -> a Filter pass compares label with its value at the iteration start
#include <algorithm>
#include <cstdlib>

#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"
#include "lb_reduce.cuh"

namespace gsw {

constexpr int kCcSwitchIters = 12;   // label-propagation iterations before the switch to hooking (C1-C4 converge in <= 6)

struct CcArgs {
    DevGraph g;
    const unsigned *iso;
    int *label;           // internal order, values are caller ids
    int *out;             // caller order (relabeled graphs), else nullptr
    unsigned *chg;        // per-vertex "label changed" status flags (standalone filter)
    unsigned *fb[3];      // active-set bitmaps, ring of 3
    int *q;               // active-set queue (push in queue formats)
    uint32_t *scan;
    long long iso_count;
    unsigned *heavy, *hblk, *heavy_cnt;   // tiered pull (lb_reduce.cuh lbr_tiered)
    int max_iters;        // > 0: stop after this many iterations and raise *unfinished (run_cc's switch)
    unsigned *unfinished;
    RunCommon rc;
};

struct CcPushTok { unsigned old; int lu; };
struct CcPushAux { unsigned claim; uint32_t d0, d1; };

// push: for active u, every neighbour v gets atomicMin(label[v], label[u])
struct CcPushOp {
    int *label;
    const uint32_t *off;
    bool fused;
    unsigned *nfb;
    using Probe = int2;          // (label[u], label[v])
    using Tok = CcPushTok;
    using Aux = CcPushAux;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int u, uint32_t, int v) const { return make_int2(label[u], label[v]); }
    __device__ __forceinline__ Tok act(int, uint32_t, int v, Probe p) const {
        return CcPushTok{p.x < p.y ? (unsigned)atomicMin(label + v, p.x) : 0x80000000u, p.x};
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int v, Tok t) const {
        bool improved = t.old != 0x80000000u && t.lu < (int)t.old;
        if (!improved) return CcPushAux{~0u, 0u, 0u};
        unsigned bit = 1u << (v & 31);
        if (!fused) { atomicOr(nfb + (v >> 5), bit); return CcPushAux{~0u, 0u, 0u}; }   // status flag only
        unsigned c = atomicOr(nfb + (v >> 5), bit);
        return CcPushAux{c, __ldg(off + v), __ldg(off + v + 1)};
    }
    __device__ __forceinline__ bool commit(int, uint32_t, int v, Tok, Aux a, LocalCnt &c) const {
        if (fused && !((a.claim >> (v & 31)) & 1u)) c.add_vertex(a.d1 - a.d0);
        return false;
    }
};

// pull: label[v] = min(label[v], min over active in-neighbours u of label[u]), then the
// pointer-jumping shortcut label[v] = min(that, label[x]) with x the vertex whose id is that label
// (Soman et al. [53]; R17): labels are ids of same-component vertices and
// never exceed their own vertex's id, so the fixpoint (the component's minimum id) is unchanged
// and long label chains collapse in fewer iterations -- on the R-MAT configs it did not cut the 4
// iterations and cost the extra loads, so it is built only with GSW_CC_JUMP=1.
#ifndef GSW_CC_JUMP
#define GSW_CC_JUMP 0       // measured: C3 still 4 iterations, 1.95 vs 2.16 ms with it (profiles/r2/pr_ept_cc_jump_ab.txt)
#endif
struct CcPullOp {
    int *label;
    const uint32_t *inv;         // caller id -> internal id (labels are caller ids), or nullptr
    const unsigned *fb;          // active set
    const uint32_t *off;         // out-offsets (degree of a changed vertex)
    bool fused;
    unsigned *nfb;
    // The min over ALL in-neighbours equals the min over the active ones combined with label[v]
    // (inactive labels were already propagated; min is idempotent), so pull gathers labels only:
    // one random load per edge instead of two (the active-set probe).
    using Probe = unsigned;      // label[u]
    using Acc = unsigned long long;
    static constexpr bool kFlushEmpty = false;
    static __device__ __forceinline__ Acc identity() { return 0x7fffffffull; }
    static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a < b ? a : b; }
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int, uint32_t, int u) const { return (unsigned)label[u]; }
    __device__ __forceinline__ Acc val(int, uint32_t, int, Probe p) const { return (Acc)p; }
    __device__ __forceinline__ void flush(int v, Acc m, bool exclusive, LocalCnt &c) const {
        if (m == identity()) return;
        int mi = (int)m;
#if GSW_CC_JUMP
        if (mi < label[v]) {
            const int x = inv ? (int)__ldg(inv + mi) : mi;
            const int lx = label[x];
            mi = lx < mi ? lx : mi;
        }
#endif
        unsigned bit = 1u << (v & 31);
        if (exclusive) {
            if (mi < label[v]) {
                label[v] = mi;
                atomicOr(nfb + (v >> 5), bit);
                if (fused) c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
            }
        } else {
            int old = atomicMin(label + v, mi);
            if (mi < old) {
                if (!fused) atomicOr(nfb + (v >> 5), bit);
                else if (!(atomicOr(nfb + (v >> 5), bit) & bit)) c.add_vertex(__ldg(off + v + 1) - __ldg(off + v));
            }
        }
    }
};

__device__ __forceinline__ DevCfg select_cc(const Features &f, const gsw_config &force) {
    // Direction (P1) for min-label propagation: unlike BFS there is no "inactive" set that pull
    // could skip -- a CC pull iteration reduces over every non-isolated row (all 2M entries) while
    // push touches only the Ea out-edges of the changed vertices.  Measured on C3 (B200): pull
    // 730 us per iteration, push ~25 us per million active edges, so the split is pull <=> Ea > 2M/4
    // (the BFS rule's Ea*16 > Eia flipped C3's third iteration between 140 us and 730 us).
    gsw_config fc = force;
    if (fc.direction == GSW_AUTO) fc.direction = ((float)f.Ea * 4.f > 2.f * f.M) ? GSW_PULL : GSW_PUSH;
    DevCfg c = select_traversal(f, fc);
    // the pull workload is every non-isolated vertex: reduce with the owner mappings
    if (c.dir == GSW_PULL && force.load_balance == GSW_AUTO) c.lb = GSW_LB_TWC;
    return c;
}

union CcSmem {
    LbSmem push;
    LbRedSmem pull;
};

__global__ void __launch_bounds__(kBlock, kMinBlocksCc) cc_kernel(CcArgs a) {
    __shared__ CcSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n, W = (n + 31) >> 5;
    const Adj adj_out{a.g.off, a.g.col}, adj_in{a.g.in_off, a.g.in_col};

    // ---- init: label = id, AS_0 = every non-isolated vertex
    // labels are CALLER ids so that the fixpoint is the minimum caller id of each component
    for (long long v = gtid(); v < n; v += gthreads()) a.label[v] = a.g.perm ? (int)a.g.perm[v] : (int)v;
    for (long long w = gtid(); w < W; w += gthreads()) {
        unsigned valid = (w == W - 1 && (n & 31)) ? ((1u << (n & 31)) - 1u) : ~0u;
        a.fb[0][w] = ~a.iso[w] & valid;
        a.fb[1][w] = 0u; a.fb[2][w] = 0u;
        a.chg[w] = 0u;
    }
    if (is_book()) {
        for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
        rc.cnt[0].va = (unsigned long long)(n - a.iso_count);
        rc.cnt[0].ea = a.g.nnz;
        rc.cnt[0].maxd = 0; rc.cnt[0].mind = 0;
        *a.heavy_cnt = 0u;
        *a.unfinished = 0u;
    }
    grid_sync(bar, epoch);
    Tiers tiers{a.heavy, a.hblk, 0u};
    tiered_build_p1(adj_in, n, tiers, a.heavy_cnt);
    grid_sync(bar, epoch);
    tiers.nheavy = cta_read_u32(a.heavy_cnt);
    tiered_build_p2(adj_in, tiers, red);
    grid_sync(bar, epoch);

    Book book;
    Features f = rc.base;
    bool dirty[3] = {true, false, false};
    int prev_dir = GSW_PULL;
    unsigned long long prev_va = 0;
    int t = 0;
    for (;; ++t) {
        IterCnt *cur = rc.cnt + (t % 3), *nxt = rc.cnt + ((t + 1) % 3);
        if (is_book()) book_start(book, rc, t, nxt);
        const CntView cv = cta_read_cnt(cur);
        if (is_book() && t > 0) {
            book.bytes += 12ull * prev_va + 4ull * cv.edges + (prev_dir == GSW_PULL ? 4ull * n + n / 8 : 0ull);
            book.edges += cv.edges;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)cv.edges;
        }
        if (cv.va == 0) break;
        if (a.max_iters > 0 && t >= a.max_iters) {          // high diameter: hand over to hooking
            if (is_book()) *a.unfinished = 1u;
            break;
        }
        f.Va = (long long)cv.va; f.Ea = (long long)cv.ea;
        f.Via = (long long)n - f.Va; f.Eia = (long long)a.g.nnz - f.Ea;
        f.maxd = cv.maxd; f.mind = cv.mind; f.iter = t;
        hist_features(cv, f);
        const DevCfg c = select_cc(f, rc.force);
        write_record(rc, t, c, f, 0u);
        if (is_book()) reset_cnt(rc.cnt + ((t + 2) % 3));
        const int b2 = (t + 2) % 3;
        if (dirty[b2]) { clear_words(a.fb[b2], W); dirty[b2] = false; }
        unsigned *fbt = a.fb[t % 3];
        const bool push = c.dir == GSW_PUSH;
        const bool fused = c.fused == GSW_FUSED;
        unsigned *nfb = a.fb[(t + 1) % 3];

        // ---------------- Filter: AS_t is a bitmap; queue formats compact it for push
        unsigned qlen = 0;
        if (push && c.fmt != GSW_BITMAP) {
            if (c.fmt == GSW_QUEUE) {
                q_from_bm(a.q, &cur->qlen, fbt, W, 0u);
            } else {
                sq_from_bm_p1(fbt, W, 0u, rc.partial, red);
                grid_sync(bar, epoch);
                sq_from_bm_p2(a.q, &cur->qlen, fbt, W, 0u, rc.partial, red);
            }
            grid_sync(bar, epoch);
            qlen = cta_read_u32(&cur->qlen);
        }
        if (is_book()) book_expand(book);

        // ---------------- Expand
        // fused: Expand claims changed vertices straight into AS_{t+1} (counting the winners);
        // standalone: Expand only raises the per-vertex "changed" status flag
        unsigned *mark = fused ? nfb : a.chg;
        LocalCnt lc;
        if (push) {
            const CcPushOp op{a.label, a.g.off, fused, mark};
            if (c.fmt == GSW_BITMAP)
                lc = run_lb(c.lb, BitmapSrc{fbt, (unsigned)n, 1u}, adj_out, op, sm.push, red, bar, epoch, rc.partial, a.scan);
            else
                lc = run_lb(c.lb, QueueSrc{a.q, qlen}, adj_out, op, sm.push, red, bar, epoch, rc.partial, a.scan);
        } else {
            const CcPullOp op{a.label, a.g.inv, fbt, a.g.off, fused, mark};
            if (c.lb == GSW_LB_TWC)
                lc = lbr_tiered(op, adj_in, tiers, n);          // B200 TWC: warp-seg / warp / grid tiers
            else
                lc = run_lb_reduce(c.lb, BitmapSrc{a.iso, (unsigned)n, 0u}, adj_in, op, sm.pull, red, bar, epoch,
                                   rc.partial, a.scan);
        }
        dirty[(t + 1) % 3] = true;
        if (fused) {
            flush_counts(lc, nxt);
            grid_sync(bar, epoch);
        } else {
            // standalone Filter: generate AS_{t+1} from the vertex status flags
            LocalCnt ec;
            ec.edges = lc.edges;
            grid_sync(bar, epoch);
            for (long long w = gwarp(); w < W; w += gwarps()) {
                unsigned m = a.chg[w];                     // warp-uniform word
                int v = (int)(w * 32 + lane_id());
                if ((m >> lane_id()) & 1u) ec.add_vertex(__ldg(a.g.off + v + 1) - __ldg(a.g.off + v));
                if (lane_id() == 0) { nfb[w] = m; a.chg[w] = 0u; }
            }
            flush_counts(ec, nxt);
            grid_sync(bar, epoch);
        }
        prev_dir = c.dir;
        prev_va = cv.va;
    }
    if (a.out) gather_out(a.out, a.label, a.g.inv, n);
    if (is_book()) book_finish(book, rc, t);
}

gsw_status run_cc(gsw_graph g, int32_t *label_out, gsw_run_stats *st) {
    const int n = g->g.n, W = (n + 31) / 32;
    if (!label_out) { set_error("gsw_cc: label is NULL"); return GSW_EINVAL; }
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(label_out) == 1;
    CcArgs a{};
    a.g = g->g;
    a.iso = g->iso;
    const bool relabeled = g->g.inv != nullptr;
    a.label = (dev_out && !relabeled) ? label_out : (int *)ws.take((size_t)n * 4);
    a.out = relabeled ? (dev_out ? label_out : (int *)ws.take((size_t)n * 4)) : nullptr;
    a.chg = (unsigned *)ws.take((size_t)W * 4);
    for (int i = 0; i < 3; ++i) a.fb[i] = (unsigned *)ws.take((size_t)W * 4);
    a.q = (int *)ws.take((size_t)n * 4);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    a.iso_count = g->attrs.isolated;
    const size_t nh = std::min<size_t>((size_t)n, (size_t)g->g.nnz / kHeavy + 1);
    a.heavy = (unsigned *)ws.take(nh * 4);
    a.hblk = (unsigned *)ws.take((nh + 1) * 4);
    a.heavy_cnt = (unsigned *)ws.take(256);
    a.unfinished = a.heavy_cnt + 32;
    // Algorithm switch of the autotuned run (CC): label propagation needs about as
    // many iterations as the graph's diameter (C2: 4,013, 244 ms); when it is still running after
    // GSW_CC_SWITCH (default 12) iterations, its labels seed the hooking + pointer-jumping CC
    // (cc_hook.cu), which converges in a few sweeps.  Forced variants never switch.
    const gsw_config &fc = g->forced;
    const bool all_auto = fc.direction == GSW_AUTO && fc.format == GSW_AUTO && fc.load_balance == GSW_AUTO &&
                          fc.fusion == GSW_AUTO;
    const char *sw = std::getenv("GSW_CC_SWITCH");
    a.max_iters = all_auto ? (sw ? std::atoi(sw) : kCcSwitchIters) : 0;
    LaunchInfo li;
    gsw_status s = prepare_common(g, ws, (const void *)cc_kernel, a.rc, li, kMinBlocksCc);
    if (s != GSW_OK) return s;
    if (!a.label || !a.chg || !a.fb[2] || !a.q || !a.scan || !a.heavy || !a.hblk || !a.heavy_cnt) { set_error("workspace too small"); return GSW_ENOMEM; }
    void *args[] = {&a};
    s = launch_persistent(g, (const void *)cc_kernel, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out)
        GSW_CUDA(cudaMemcpyAsync(label_out, relabeled ? a.out : a.label, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    if ((s = finish_run(g, a.rc, li, st)) != GSW_OK) return s;
    if (a.max_iters <= 0) return GSW_OK;
    unsigned unfinished = 0;
    GSW_CUDA(cudaMemcpy(&unfinished, a.unfinished, 4, cudaMemcpyDeviceToHost));
    if (!unfinished) return GSW_OK;
    // hand over: the hooking run continues from a.label and appends its records
    gsw_run_stats h{};
    if (st) {
        const int used = std::min(st->iterations, st->max_records);
        h.records = st->records ? st->records + used : nullptr;
        h.max_records = st->records ? std::max(0, st->max_records - used) : 0;
    }
    if ((s = run_cc_hook_seeded(g, label_out, st ? &h : nullptr, a.label, ws.used)) != GSW_OK) return s;
    if (st) {
        for (int i = 0; i < std::min(h.iterations, h.max_records); ++i) h.records[i].iteration += st->iterations;
        st->iterations += h.iterations;
        st->gpu_ms += h.gpu_ms;
        st->edges_touched += h.edges_touched;
        st->bytes_alg += h.bytes_alg;
    }
    return GSW_OK;
}

}  // namespace gsw
