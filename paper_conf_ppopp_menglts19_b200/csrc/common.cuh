// common.cuh -- device building blocks shared by every algorithm of the library.
//
// The whole per-iteration loop of GSWITCH (Inspector -> Selector -> Executor, PAPER.md:805-844,
// Fig. 10) runs inside ONE persistent cooperative kernel per run.  Phases of an iteration are
// separated by a software grid barrier (below) instead of kernel boundaries, so there is no host
// round trip per iteration (the paper's 58-120 us feature copy, disappears).
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace gsw {

constexpr int kBlock = 256;           // threads per CTA of every persistent kernel
constexpr int kWarps = kBlock / 32;

// ------------------------------------------------------------------ memory-order helpers
__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_relaxed(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ int ld_relaxed_s32(const int *p) {
    int v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ------------------------------------------------------------------ grid barrier
// One arrival word with the flip-bit protocol of grid_sync below (every CTA adds to the same
// counter; the waiters poll for the flip of its top bit).  Co-residency of all CTAs is guaranteed
// by cudaLaunchCooperativeKernel.  A spin longer than kBarrierTimeoutNs sets an error code and
// traps, so a bug becomes a launch failure rather than a hung GPU.
struct GridBarrier {
    unsigned *arrive;
    unsigned *err;
    int cluster;      // nonzero: the whole grid is ONE thread-block cluster (cluster tier)
};

// Hardware cluster barrier with release/acquire at cluster scope: orders the global and shared
// memory operations of every thread of the cluster (ptxas emits the L1 invalidation the acquire
// needs), so when the grid is a single cluster it replaces the software grid barrier.
__device__ __forceinline__ void cluster_barrier() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
constexpr uint64_t kBarrierTimeoutNs = 20ull * 1000 * 1000 * 1000;
#ifndef GSW_BAR_SC
#define GSW_BAR_SC 0
#endif

// Flip-bit barrier (the cooperative-groups scheme): CTA 0 adds 2^31 - (gridDim - 1), every other
// CTA adds 1, so the counter's top bit flips exactly when the last CTA arrives; waiters poll the
// word until they see the flip.  One atomic per CTA and no separate publish store by the last
// arriver (tools/micro_barrier.cu on B200, 592 CTAs: 1.61 us vs 1.85 us for the acq_rel
// counter + generation-word form).  The counter must be 0 when the kernel starts (prepare_common).
__device__ __forceinline__ unsigned ld_volatile_u32(const unsigned *p) {
    unsigned v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// Release before the arrival, acquire after the flip is seen: fence.acq_rel.gpu on both sides
// (GSW_BAR_SC=1: __threadfence, i.e. the sequentially consistent MEMBAR.SC.GPU, A/B knob).
__device__ __forceinline__ void bar_fence() {
#if GSW_BAR_SC
    __threadfence();
#else
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
}
__device__ __forceinline__ void grid_sync(const GridBarrier &b, unsigned &epoch) {
#ifndef GSW_NO_CLUSTER_BAR
    if (b.cluster) { cluster_barrier(); epoch += 1; return; }
#endif
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned add = blockIdx.x == 0 ? 0x80000000u - (gridDim.x - 1u) : 1u;
        bar_fence();
        const unsigned old = atomicAdd(b.arrive, add);
        uint64_t t0 = 0;
        unsigned spins = 0;
        while (((old ^ ld_volatile_u32(b.arrive)) & 0x80000000u) == 0u) {
            if (((++spins) & 1023u) == 0) {
                const uint64_t now = globaltimer();
                if (t0 == 0) t0 = now;
                else if (now - t0 > kBarrierTimeoutNs) { atomicExch(b.err, 0xBA4u); __trap(); }
            }
        }
        bar_fence();
    }
    epoch += 1;
    __syncthreads();
}

// Grid barrier for CTAs parked while CTA 0 runs a solo episode (engine.cuh):
// same protocol as grid_sync, but the wait sleeps between polls so the parked CTAs do not steal
// issue slots from CTA 0's SM or keep invalidating its L1 with acquire loads.
__device__ __forceinline__ void grid_park(const GridBarrier &b, unsigned &epoch) {
#ifndef GSW_NO_CLUSTER_BAR
    if (b.cluster) { cluster_barrier(); epoch += 1; return; }
#endif
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned add = blockIdx.x == 0 ? 0x80000000u - (gridDim.x - 1u) : 1u;
        bar_fence();
        const unsigned old = atomicAdd(b.arrive, add);
        const uint64_t t0 = globaltimer();
        unsigned spins = 0;
        while (((old ^ ld_volatile_u32(b.arrive)) & 0x80000000u) == 0u) {
            __nanosleep(200);
            if (((++spins) & 255u) == 0 && globaltimer() - t0 > kBarrierTimeoutNs) {
                atomicExch(b.err, 0xBA5u);
                __trap();
            }
        }
        bar_fence();
    }
    epoch += 1;
    __syncthreads();
}

// ------------------------------------------------------------------ warp / block reductions
template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
template <typename T>
__device__ __forceinline__ T warp_max(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) { T x = __shfl_xor_sync(0xffffffffu, v, o); v = x > v ? x : v; }
    return v;
}
template <typename T>
__device__ __forceinline__ T warp_min(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) { T x = __shfl_xor_sync(0xffffffffu, v, o); v = x < v ? x : v; }
    return v;
}
// inclusive warp scan
template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
    unsigned l = lane_id();
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T x = __shfl_up_sync(0xffffffffu, v, o);
        if (l >= (unsigned)o) v += x;
    }
    return v;
}

// Block-wide exclusive scan of one value per thread (kBlock threads).  Returns the exclusive
// prefix; *total gets the block sum.  Uses `sm` (>= kWarps+1 entries).  Contains __syncthreads.
template <typename T>
__device__ __forceinline__ T block_excl_scan(T v, T *sm, T *total) {
    T inc = warp_incl_scan(v);
    unsigned w = threadIdx.x >> 5, l = lane_id();
    __syncthreads();
    if (l == 31) sm[w] = inc;
    __syncthreads();
    if (w == 0) {
        T s = l < (unsigned)kWarps ? sm[l] : T(0);
        T si = warp_incl_scan(s);
        if (l < (unsigned)kWarps) sm[l] = si - s;
        if (l == kWarps - 1) sm[kWarps] = si;
    }
    __syncthreads();
    T res = sm[w] + inc - v;
    *total = sm[kWarps];
    return res;
}

// Block-wide sum (all threads get the result).  Contains __syncthreads.
template <typename T>
__device__ __forceinline__ T block_sum(T v, T *sm) {
    v = warp_sum(v);
    unsigned w = threadIdx.x >> 5, l = lane_id();
    __syncthreads();
    if (l == 0) sm[w] = v;
    __syncthreads();
    T s = l < (unsigned)kWarps ? sm[l] : T(0);
    s = warp_sum(s);
    return s;
}

// ------------------------------------------------------------------ bitmaps
__device__ __forceinline__ bool test_bit(const unsigned *bm, int v) {
    return (bm[v >> 5] >> (v & 31)) & 1u;
}
__device__ __forceinline__ bool test_bit_relaxed(const unsigned *bm, int v) {
    return (ld_relaxed(bm + (v >> 5)) >> (v & 31)) & 1u;
}
// atomic test-and-set; returns true if this call set the bit (0 -> 1 winner)
__device__ __forceinline__ bool claim_bit(unsigned *bm, int v) {
    unsigned bit = 1u << (v & 31);
    unsigned old = atomicOr(bm + (v >> 5), bit);
    return !(old & bit);
}

// ------------------------------------------------------------------ warp-aggregated append
// Append `v` to q[*len] for every calling lane with pred true; one atomicAdd per warp.
// Safe under divergence: aggregates over the currently converged lanes.
__device__ __forceinline__ void warp_append(int *q, unsigned *len, bool pred, int v) {
    unsigned active = __activemask();
    unsigned m = __ballot_sync(active, pred);
    if (m == 0) return;
    int leader = __ffs(active) - 1;
    unsigned base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(len, (unsigned)__popc(m));
    base = __shfl_sync(active, base, leader);
    if (pred) q[base + __popc(m & lanemask_lt())] = v;
}

// ------------------------------------------------------------------ CTA-staged queue append
// Fused Expands append activated vertices to the next queue from divergent code.  A single global
// counter serialises at one L2 address (1K appending warps cost ~50 us on B200, measured), so
// appends go to a per-CTA shared-memory buffer through shared atomics and the CTA publishes them
// with ONE global atomicAdd when the phase ends (cta_queue_flush, called by all threads).  A full
// buffer spills directly to the global queue.
constexpr int kCtaQ = 2048;
struct CtaQueue {
    int *buf;          // shared memory, kCtaQ entries
    unsigned *count;   // shared memory
    int *gq;           // global queue
    unsigned *glen;    // global length counter
    __device__ __forceinline__ void push(int v) const {
        unsigned i = atomicAdd(count, 1u);
        if (i < (unsigned)kCtaQ) buf[i] = v;
        else gq[atomicAdd(glen, 1u)] = v;
    }
};
// shared storage of one staged queue
struct CtaQStore {
    int buf[kCtaQ];
    unsigned count;
    unsigned base;
};
__device__ __forceinline__ CtaQueue cta_queue(CtaQStore &s, int *gq, unsigned *glen) {
    return CtaQueue{s.buf, &s.count, gq, glen};
}
__device__ __forceinline__ void cta_queue_reset(CtaQStore &s) {
    if (threadIdx.x == 0) s.count = 0u;
    __syncthreads();
}
// publish the CTA's staged entries: one global atomicAdd, then a coalesced copy
__device__ __forceinline__ void cta_queue_flush(CtaQStore &s, int *gq, unsigned *glen) {
    __syncthreads();
    const unsigned n = min(s.count, (unsigned)kCtaQ);
    if (threadIdx.x == 0) s.base = n ? atomicAdd(glen, n) : 0u;
    __syncthreads();
    const unsigned base = s.base;
    for (unsigned i = threadIdx.x; i < n; i += blockDim.x) gq[base + i] = s.buf[i];
    __syncthreads();
    if (threadIdx.x == 0) s.count = 0u;
    __syncthreads();
}

// ------------------------------------------------------------------ per-iteration counters
// Runtime characteristics of the NEXT active set, accumulated by whoever activates a vertex
// (Table 1): Va, Ea, max/min degree; plus edges scanned by this iteration's Expand.
struct alignas(128) IterCnt {
    unsigned long long va, ea, edges;
    unsigned maxd, mind;
    unsigned qlen;          // length of the queue materialised for this active set (if any)
    unsigned iqlen;         // length of the inactive (pull workload) queue, if built
    float tf, te, Tf, Te;   // history features carried to the iteration that reads this slot
    unsigned aux0, aux1;    // algorithm-specific control words (SSSP: far-set length / min)
};

// After a grid barrier every CTA needs the same few control words.  Reading them from every warp
// of ~600 CTAs serialises ~20K requests on one L2 line (~10 us/iteration measured on B200); instead
// thread 0 of each CTA reads once and broadcasts through shared memory.
struct CntView {
    unsigned long long va, ea, edges;
    unsigned maxd, mind, qlen, iqlen;
    float tf, te, Tf, Te;
    unsigned aux0, aux1;
};
__device__ __forceinline__ unsigned long long ld_relaxed64_nc(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ unsigned ld_relaxed_nc(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ CntView cta_read_cnt(const IterCnt *c) {
    __shared__ CntView s;
    __syncthreads();
    if (threadIdx.x == 0) {
        // Plain (vectorisable, pipelined) loads: this always follows a grid barrier whose acquire
        // invalidated this SM's L1 (CCTL.IVALL), so they observe every write released before it.
        // (11 separate ld.relaxed.gpu here cost ~5 us per iteration.)
        const uint4 *p = reinterpret_cast<const uint4 *>(c);
        uint4 a = p[0], b = p[1], d = p[2], e = p[3];
        CntView v;
        v.va = ((unsigned long long)a.y << 32) | a.x;
        v.ea = ((unsigned long long)a.w << 32) | a.z;
        v.edges = ((unsigned long long)b.y << 32) | b.x;
        v.maxd = b.z; v.mind = b.w;
        v.qlen = d.x; v.iqlen = d.y;
        v.tf = __uint_as_float(d.z); v.te = __uint_as_float(d.w);
        v.Tf = __uint_as_float(e.x); v.Te = __uint_as_float(e.y);
        v.aux0 = e.z; v.aux1 = e.w;
        s = v;
    }
    __syncthreads();
    return s;
}
__device__ __forceinline__ unsigned cta_read_u32(const unsigned *p) {
    __shared__ unsigned s;
    __syncthreads();
    if (threadIdx.x == 0) s = *(volatile const unsigned *)p;
    __syncthreads();
    return s;
}

struct LocalCnt {
    unsigned long long va = 0, ea = 0, edges = 0;
    unsigned maxd = 0, mind = 0xffffffffu;
    double facc = 0.0;          // algorithm-specific fp64 side sum (PR dangling mass)
    unsigned aux = 0;           // algorithm-specific count (SSSP far-set appends) -> IterCnt::aux0
    __device__ __forceinline__ void add_vertex(unsigned deg) {
        va += 1; ea += deg;
        maxd = deg > maxd ? deg : maxd;
        mind = deg < mind ? deg : mind;
    }
};

// Reduce a thread's counters over the CTA and add them to the global slot (one atomic each per
// CTA).  Must be called by all threads of the CTA.
__device__ __forceinline__ void flush_counts(LocalCnt &c, IterCnt *dst) {
    // most CTAs have nothing to report in small iterations: one barrier decides
    if (!__syncthreads_or(c.va != 0 || c.edges != 0 || c.aux != 0)) { c = LocalCnt(); return; }
    __shared__ unsigned long long s64[kWarps][3];
    __shared__ unsigned s32[kWarps][2];
    unsigned long long va = warp_sum(c.va), ea = warp_sum(c.ea), ed = warp_sum(c.edges);
    unsigned mx = warp_max(c.maxd), mn = warp_min(c.mind), ax = warp_sum(c.aux);
    unsigned w = threadIdx.x >> 5;
    __shared__ unsigned sax[kWarps];
    if (lane_id() == 0) { s64[w][0] = va; s64[w][1] = ea; s64[w][2] = ed; s32[w][0] = mx; s32[w][1] = mn; sax[w] = ax; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < kWarps; ++i) {
            va += s64[i][0]; ea += s64[i][1]; ed += s64[i][2]; ax += sax[i];
            mx = s32[i][0] > mx ? s32[i][0] : mx;
            mn = s32[i][1] < mn ? s32[i][1] : mn;
        }
        if (va) { atomicAdd(&dst->va, va); atomicAdd(&dst->ea, ea); atomicMax(&dst->maxd, mx); atomicMin(&dst->mind, mn); }
        if (ed) atomicAdd(&dst->edges, ed);
        if (ax) atomicAdd(&dst->aux0, ax);
    }
    __syncthreads();
    c = LocalCnt();
}

__device__ __forceinline__ void reset_cnt(IterCnt *c) {
    c->va = 0; c->ea = 0; c->edges = 0; c->maxd = 0; c->mind = 0xffffffffu; c->qlen = 0; c->iqlen = 0;
    c->tf = 0.f; c->te = 0.f; c->Tf = 0.f; c->Te = 0.f;
    c->aux0 = 0u; c->aux1 = 0xffffffffu;
}

// grid-stride helpers
__device__ __forceinline__ long long gtid() { return (long long)blockIdx.x * blockDim.x + threadIdx.x; }
__device__ __forceinline__ long long gthreads() { return (long long)gridDim.x * blockDim.x; }
__device__ __forceinline__ long long gwarp() { return gtid() >> 5; }
__device__ __forceinline__ long long gwarps() { return gthreads() >> 5; }

}  // namespace gsw

namespace gsw {
static_assert(offsetof(IterCnt, va) == 0 && offsetof(IterCnt, edges) == 16 && offsetof(IterCnt, maxd) == 24 &&
                  offsetof(IterCnt, qlen) == 32 && offsetof(IterCnt, tf) == 40 && offsetof(IterCnt, Tf) == 48,
              "cta_read_cnt assumes this layout");
}  // namespace gsw
