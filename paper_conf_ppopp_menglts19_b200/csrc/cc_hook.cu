// cc_hook.cu -- connected components by hooking + pointer jumping, the edge-centric GPU CC the
// paper compares against (Soman et al. [53], reading Q8 "hooking is
// NEXT"), on the same persistent engine and Expand load-balance patterns as the GSWITCH CC.
//
// Every vertex v holds a parent pointer P[v], packed as (key(p) << 32 | p) where p is an
// internal id and key(p) its caller id, so that unsigned 64-bit order is caller-id order.
// Iteration t (until no hook succeeds):
//   hook    : for every edge (x, y) with P[x] != P[y] (different trees after the last
//             compression), atomicMin(P[hi], lo) with lo < hi the two packed roots -- the tree
//             whose root has the larger key is hung below the other root.  Concurrent hooks of one
//             root keep the smallest; an edge whose hook lost is seen again next iteration.
//   compress: P[v] <- the root of v's tree (pointer jumping to the fixpoint P[r] == r).
// A component's minimum-key vertex is never hooked (nothing is smaller), so at the fixpoint every
// vertex points at it: label[v] = key(P[v]) = the minimum caller id of v's component, the same
// output as gsw_cc.  Symmetric graphs scan each undirected edge once (the y > x direction).
#include "engine.cuh"
#include "internal.h"
#include "launch.h"
#include "lb.cuh"

namespace gsw {

// Resident CTAs per SM (A/B knob).  With 24-byte tokens (two packed 64-bit pointers + the
// pre-check value per edge in flight) the sweep spilled and the spill stores reached DRAM (ncu:
// 11 GB written in an 8.5 ms C3 run, profiles/r2/ncu_cc_hook_c3.md); with the 16-byte token below,
// 4 CTAs/SM measured best (C3 7.65 ms vs 10.4 at 2/SM; C4 9.0 vs 12.5; profiles/r2/cc_hook_minb_ab.txt)
#ifndef GSW_HOOK_MINB
#define GSW_HOOK_MINB 4
#endif
constexpr int kMinBlocksCcHook = GSW_HOOK_MINB;

#ifndef GSW_HOOK_PRECHECK
#define GSW_HOOK_PRECHECK 1     // read the larger root's pointer before the atomic (A/B knob)
#endif

struct CcHookArgs {
    DevGraph g;
    bool sym;                 // symmetric CSR: hook each undirected edge from one side only
    unsigned long long *P;    // packed parent pointers (internal order)
    int *out;                 // labels, caller order
    uint32_t *scan;           // STRICT degree scan
    const int *seed;          // optional start labels (internal order, caller-id values, each a
                              // vertex of v's component with key <= v's): gsw_cc's switch (cc.cu)
    RunCommon rc;
};

__device__ __forceinline__ unsigned long long hk_pack(const uint32_t *perm, unsigned v) {
    return ((unsigned long long)(perm ? perm[v] : v) << 32) | v;
}

// hook: the Expand edge op (lb.cuh edge_batch stages: probe = both trees' roots, act = the hook)
// Stages: probe loads both endpoints' pointers; act loads the current pointer of the larger root
// (another edge may already have hooked it below something at least as small -- then the atomic
// is skipped, which removes most of the contended atomics on hub roots in the first sweep); aux
// issues the hook.
// keys are unique (caller ids), so comparing packed pointers is comparing their keys: the token
// keeps 32-bit halves (16 bytes per edge in flight instead of 24)
struct HookTok {
    unsigned lo_key, lo_id, hi_id, cur_key;
};
struct HookOp {
    unsigned long long *P;
    bool sym;
    using Probe = ulonglong2;
    using Tok = HookTok;
    using Aux = unsigned;
    static constexpr bool kEarlyExit = false;
    __device__ __forceinline__ bool skip(int) const { return false; }
    __device__ __forceinline__ Probe probe(int x, uint32_t, int y) const {
        if (sym && y <= x) return make_ulonglong2(0ull, 0ull);          // the other direction hooks it
        return make_ulonglong2(P[x], P[y]);
    }
    __device__ __forceinline__ Tok act(int, uint32_t, int, Probe p) const {
        if (p.x == p.y) return HookTok{0u, 0u, 0u, 0u};
        const unsigned long long lo = p.x < p.y ? p.x : p.y, hi = p.x < p.y ? p.y : p.x;
#if GSW_HOOK_PRECHECK
        const unsigned ck = (unsigned)(P[(unsigned)hi] >> 32);
#else
        const unsigned ck = 0xffffffffu;
#endif
        return HookTok{(unsigned)(lo >> 32), (unsigned)lo, (unsigned)hi, ck};
    }
    __device__ __forceinline__ Aux aux(int, uint32_t, int, Tok t) const {
        if (t.cur_key <= t.lo_key) return 0u;                          // equal roots, or already lower
        const unsigned long long lo = ((unsigned long long)t.lo_key << 32) | t.lo_id;
        return atomicMin(P + t.hi_id, lo) > lo ? 1u : 0u;
    }
    __device__ __forceinline__ bool commit(int, uint32_t, int, Tok, Aux h, LocalCnt &c) const {
        c.aux += h;
        return false;
    }
};

__global__ void __launch_bounds__(kBlock, kMinBlocksCcHook) cc_hook_kernel(const __grid_constant__ CcHookArgs a) {
    __shared__ LbSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n;
    const Adj adj{a.g.off, a.g.col};
    unsigned long long *P = a.P;

    if (a.seed) {
        // start from a labeling: v points at the vertex whose caller id is its label (the forest
        // stays acyclic: keys never increase along a pointer), then compress, so that every
        // pointer names a root when the first hook sweep starts (what termination relies on)
        for (long long v = gtid(); v < n; v += gthreads()) {
            const unsigned c = (unsigned)a.seed[v];
            P[v] = ((unsigned long long)c << 32) | (a.g.inv ? __ldg(a.g.inv + c) : c);
        }
        grid_sync(bar, epoch);
        for (long long v = gtid(); v < n; v += gthreads()) {
            unsigned long long p = P[v], q = P[(unsigned)p];
            while (q != p) { p = q; q = P[(unsigned)p]; }
            P[v] = p;
        }
    } else {
        for (long long v = gtid(); v < n; v += gthreads()) P[v] = hk_pack(a.g.perm, (unsigned)v);
    }
    if (is_book()) for (int i = 0; i < 3; ++i) reset_cnt(rc.cnt + i);
    grid_sync(bar, epoch);

    // AUTO: one thread per vertex on graphs with a narrow degree range (road-like: C2 0.49 ms vs
    // 1.15 ms for STRICT), the equal-edges STRICT tiles on skewed ones (C3 19.6 ms vs 114 ms for
    // TWC: hub rows would serialise on their thread / CTA); profiles/r2/cc_hook_perf.txt
    const int lb = rc.force.load_balance != GSW_AUTO ? rc.force.load_balance
                   : (rc.base.rd <= 16.f ? GSW_LB_THREAD : GSW_LB_STRICT);
    Book book;
    int t = 0;
    for (;; ++t) {
        IterCnt *cur = rc.cnt + (t % 3);
        if (is_book()) {
            book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
            reset_cnt(rc.cnt + ((t + 1) % 3));
            book_expand(book);
        }
        // ---- hook over every edge (Expand, all vertices active, P:479-481 style dense sweep)
        LocalCnt lc = run_lb(lb, AllSrc{(unsigned)n}, adj, HookOp{P, a.sym}, sm, red, bar, epoch, rc.partial, a.scan);
        flush_counts(lc, cur);
        grid_sync(bar, epoch);
        // ---- compress: pointer jumping to the root
        for (long long v = gtid(); v < n; v += gthreads()) {
            const unsigned long long p0 = P[v];
            unsigned long long p = p0, q = P[(unsigned)p];
            while (q != p) { p = q; q = P[(unsigned)p]; }
            if (p != p0) P[v] = p;
        }
        grid_sync(bar, epoch);
        const CntView cv = cta_read_cnt(cur);
        if (is_book()) {
            if (t < kMaxHist) {
                gsw_iter_record r{};
                r.iteration = t;
                r.direction = GSW_PUSH; r.format = GSW_BITMAP; r.load_balance = lb;
                r.stepping = GSW_AUTO; r.fusion = GSW_STANDALONE;
                r.Va = (long long)cv.aux0;              // successful hooks
                r.Ea = (long long)a.g.nnz; r.Via = 0; r.Eia = 0;
                r.edges = (long long)cv.edges;
                r.ctas = (int32_t)gridDim.x;
                rc.rec[t] = r;
            }
            // D0 bytes: columns + offsets of the sweep, P read by compress and written back
            book.bytes += 4ull * cv.edges + 4ull * (unsigned long long)n + 16ull * (unsigned long long)n;
            book.edges += cv.edges;
        }
        if (cv.aux0 == 0) break;
    }
    // labels in caller order: out[j] = key(root of inv[j])
    for (long long j = gtid(); j < n; j += gthreads()) {
        const unsigned v = a.g.inv ? __ldg(a.g.inv + j) : (unsigned)j;
        a.out[j] = (int)(P[v] >> 32);
    }
    if (is_book()) {
        book_start(book, rc, t + 1, rc.cnt + ((t + 2) % 3));   // closes the last iteration's times
        book_finish(book, rc, t + 1);
    }
}

gsw_status run_cc_hook(gsw_graph g, int32_t *label_out, gsw_run_stats *st) {
    return run_cc_hook_seeded(g, label_out, st, nullptr, 0);
}

gsw_status run_cc_hook_seeded(gsw_graph g, int32_t *label_out, gsw_run_stats *st, const int *seed, size_t ws_used) {
    const int n = g->g.n;
    if (!label_out) { set_error("gsw_cc_hook: label is NULL"); return GSW_EINVAL; }
    const int lbf = g->forced.load_balance;
    if (lbf != GSW_AUTO && (lbf < GSW_LB_THREAD || lbf > GSW_LB_STRICT)) {
        set_error("gsw_cc_hook: unknown forced load balance");
        return GSW_EUNSUPPORTED;
    }
    Workspace ws{g->scratch, g->scratch_bytes, ws_used};     // ws_used: keep the seed's region
    const bool dev_out = is_device_ptr(label_out) == 1;
    CcHookArgs a{};
    a.g = g->g;
    a.sym = g->symmetric;
    a.seed = seed;
    a.P = (unsigned long long *)ws.take((size_t)n * 8);
    a.out = dev_out ? label_out : (int *)ws.take((size_t)n * 4);
    a.scan = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    LaunchInfo li;
    gsw_status s = prepare_common(g, ws, (const void *)cc_hook_kernel, a.rc, li, kMinBlocksCcHook);
    if (s != GSW_OK) return s;
    if (!a.P || !a.out || !a.scan) { set_error("workspace too small"); return GSW_ENOMEM; }
    void *args[] = {&a};
    s = launch_persistent(g, (const void *)cc_hook_kernel, args, li);
    if (s != GSW_OK) return s;
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(label_out, a.out, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
