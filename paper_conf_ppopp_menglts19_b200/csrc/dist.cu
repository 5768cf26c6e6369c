// dist.cu -- multi-GPU frontier step (the paper itself is single-GPU): 1D vertex
// partition with destination ownership, the per-iteration exchange over NCCL (NVLink 5 /
// NVSwitch), and two more exchange backends that run the SAME partitioned kernels: loopback (p
// virtual ranks on one GPU, exchange = the shared replicated buffers) and host-staged (the caller
// supplies all-gather / all-reduce callbacks, e.g. torch.distributed over gloo, so several
// processes can share one GPU in tests).
//
// Device-resident decisions.  The per-iteration control state (global counts, unvisited counts,
// the next direction, the done flag, per-level records) lives in device memory: every rank's
// `decide` kernel evaluates the same selector rule on the same all-reduced counts, and both
// expand kernels of a level are launched, the one not chosen returning at once.  The host only
// enqueues: it polls the done flag LOOKAHEAD levels behind the stream (pinned copy + event), so
// the stream never drains between levels; the at most LOOKAHEAD no-op levels that follow the last
// one cost a launch and (NCCL) an all-gather each.  Every rank stops after the same number of
// enqueued levels, because the flag it polls is computed from all-reduced values.
//
// BFS level t (every rank / part):
//   push  k_bfs_push: every frontier vertex u of the replicated bitmap FB_t walks its column-slice
//         row "u -> owned targets" (built at create): a lane per short row, the warp for rows up
//         to kHeavy edges, 1024-edge tasks (k_bfs_push_heavy) above; claims by atomicOr on the
//         owned visited map; the rank's slice of FB_{t+1} is marked.
//   pull  k_bfs_pull: the single-GPU list pull (bfs_pull.cuh) over the owned unvisited vertices:
//         first in-neighbour probe, then cursors over the misses; early exit at the first parent.
//   exchange: in-place all-gather of the FB_{t+1} slices (N/8 bytes) + all-reduce of (Va, Ea,
//         edges) -> k_bfs_decide (Via/Eia, direction rule of select.cuh R6, records, done).
// PageRank iteration (every vertex active): owned rows pull the replicated fp32
//   contributions (rows above kHeavy edges as 1024-edge chunk tasks with fp64 partials), each rank
//   writes its slice of the next contributions; all-gather (fp32, N*4 bytes) + all-reduce of the
//   dangling mass.  Fixed iteration count: no host poll at all.
// CC iteration (min-label propagation, DESIGN R8, with the pointer-jumping shortcut
//   label[v] <- label[label[v]] that the replicated labels make local; Soman et al. [53]
//   P:1429-1430): owned rows pull the replicated labels, each rank writes its slice; all-gather
//   (N*4 bytes) + all-reduce of the change count -> k_cc_decide (done when nothing changed).
#include <dlfcn.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <nccl.h>

#include "bfs_pull.cuh"
#include "launch.h"

namespace gsw {

// ------------------------------------------------------------------ NCCL, loaded at run time
struct NcclApi {
    bool tried = false, ok = false;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclGroupStart) groupStart = nullptr;
    decltype(&ncclGroupEnd) groupEnd = nullptr;
    decltype(&ncclGetErrorString) errStr = nullptr;
};
static NcclApi g_nccl;

static bool nccl_load() {
    if (g_nccl.tried) return g_nccl.ok;
    g_nccl.tried = true;
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) {
        const char *p = getenv("GSW_NCCL_PATH");
        if (p) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) { set_error(std::string("NCCL not loadable: ") + dlerror()); return false; }
    g_nccl.getUniqueId = (decltype(g_nccl.getUniqueId))dlsym(h, "ncclGetUniqueId");
    g_nccl.commInitRank = (decltype(g_nccl.commInitRank))dlsym(h, "ncclCommInitRank");
    g_nccl.commDestroy = (decltype(g_nccl.commDestroy))dlsym(h, "ncclCommDestroy");
    g_nccl.allGather = (decltype(g_nccl.allGather))dlsym(h, "ncclAllGather");
    g_nccl.allReduce = (decltype(g_nccl.allReduce))dlsym(h, "ncclAllReduce");
    g_nccl.groupStart = (decltype(g_nccl.groupStart))dlsym(h, "ncclGroupStart");
    g_nccl.groupEnd = (decltype(g_nccl.groupEnd))dlsym(h, "ncclGroupEnd");
    g_nccl.errStr = (decltype(g_nccl.errStr))dlsym(h, "ncclGetErrorString");
    g_nccl.ok = g_nccl.getUniqueId && g_nccl.commInitRank && g_nccl.commDestroy && g_nccl.allGather &&
                g_nccl.allReduce && g_nccl.groupStart && g_nccl.groupEnd && g_nccl.errStr;
    if (!g_nccl.ok) set_error("NCCL symbols missing");
    return g_nccl.ok;
}

#define GSW_NCCL(call)                                                                      \
    do {                                                                                    \
        ncclResult_t _r = (call);                                                           \
        if (_r != ncclSuccess) {                                                            \
            set_error(std::string("NCCL error ") + g_nccl.errStr(_r) + " at " + #call);     \
            return GSW_ENCCL;                                                               \
        }                                                                                   \
    } while (0)

// ------------------------------------------------------------------ partition state
enum DistMode { DM_NCCL = 0, DM_LOOPBACK = 1, DM_HOST = 2 };

constexpr uint32_t kHeavy = 1024;      // rows above this many edges become 1024-edge warp tasks
constexpr int kMaxLevels = 1 << 16;    // per-level records kept on the device
constexpr int kLookaheadMax = 4;       // levels enqueued past the one whose done flag is polled (max)

struct DTask {
    int row;
    uint32_t beg, end;
};

// per-level record on the device (host converts it to gsw_iter_record)
struct DRec {
    long long Va, Ea, Via, Eia, edges;
    int dir, pad;
};

// control block (device): identical on every rank after each decide
struct DCtl {
    unsigned long long tot[4];     // all-reduced {va, ea, edges, changes}
    double dtot;                   // all-reduced f64 (PR dangling mass)
    double pad0;
    long long Via, Eia, nnz_g;     // unvisited vertices / their edges, global nnz
    int dir, done, t, cur;         // cur: the level the next expand runs (graph mode reads it)
    unsigned long long theta, delta;   // SSSP priority threshold and its step (P4)
};

// per-part counters, 64 B apart: {va, ea, edges, changes, f64 bits, -, -, -}
constexpr int kLocStride = 8;

struct DPart {
    int64_t vb = 0;           // first owned vertex (multiple of 64)
    int nloc = 0;             // owned vertices
    uint32_t nnz = 0;         // owned adjacency entries
    uint32_t *roff = nullptr; // nloc+1, rebased to 0
    const int32_t *rcol = nullptr;   // global neighbour ids
    int32_t *rfirst = nullptr;// first in-neighbour of each owned row (-1: empty)
    uint32_t *soff = nullptr; // n_global+1: global source u -> owned targets
    int32_t *scol = nullptr;  // local target ids
    uint32_t *rcol_h = nullptr;   // owned in-edge columns renamed to hub order (PR gathers; nullptr: off)
    unsigned *vis = nullptr;  // visited words of the owned slice (S/32); SSSP: improved in the last push
    unsigned *far = nullptr;  // SSSP far set of the owned slice (S/32)
    const uint32_t *rw = nullptr;   // weights of the owned rows (weighted graphs)
    uint32_t *sw = nullptr;   // weights of the column slice
    DTask *chunks = nullptr;  // heavy owned rows cut into kHeavy-edge chunks (create time)
    unsigned *nchunks = nullptr;
    DTask *ptasks = nullptr;  // push tasks of the current level
    unsigned *nptasks = nullptr;
    uint32_t ptask_cap = 0;
    double *psum = nullptr;   // heavy-row partials (PR sums / CC minima as u32), nloc entries
    unsigned long long *loc = nullptr;   // this part's counters (kLocStride u64)
};

struct DistState {
    int mode = DM_NCCL;
    int nranks = 1, rank = 0;
    int64_t n = 0, S = 0, npad = 0;
    std::vector<DPart> parts;
    unsigned *FB[2] = {nullptr, nullptr};   // replicated frontier bitmaps, npad/32 words
    uint32_t *rep[2] = {nullptr, nullptr};  // replicated per-vertex words: fp32 contributions / labels
    unsigned long long *locs = nullptr;     // parts x kLocStride
    DCtl *ctl = nullptr;
    DRec *recs = nullptr;
    ncclComm_t comm = nullptr;
    unsigned *ntasks = nullptr;             // parts x 32: push-task counters (zeroed by k_bfs_decide)
    int *bdepth = nullptr;                  // BC: replicated depth (npad)
    unsigned long long *bsigma = nullptr;   // BC: replicated path counts (npad)
    double *bomega = nullptr;               // BC: replicated (1 + delta) / sigma (npad)
    bool weighted = false;
    double wbar = 0.0;                      // mean edge weight (SSSP static step c * wbar / dbar)
    gsw_exchange hx{};                      // host-staged backend callbacks
    unsigned char *hsend = nullptr, *hrecv = nullptr;   // pinned staging (host mode)
    size_t hcap = 0;
    int *hdone = nullptr;                   // mapped pinned done flags, one per lookahead slot
    int *hdone_dev = nullptr;               // their device alias (written by k_publish_done)
    int lookahead = 1;                      // GSW_DIST_LOOKAHEAD (1..4); 1 measured best (profiles/r2/part_ab.txt)
    cudaEvent_t evs[kLookaheadMax + 1] = {};
    // graph mode (NCCL / loopback): the whole level loop is one CUDA graph with a device-side WHILE
    // node; instantiated once and re-launched while the output buffer and forced direction match
    cudaGraphExec_t bfs_exec = nullptr;
    const void *bfs_exec_depth = nullptr;
    int bfs_exec_dir = -1;
    cudaStream_t cap = nullptr;             // private stream the graph is captured on (the caller's may be the legacy stream)
    bool graph_failed = false;              // capture / instantiation failed once: host-driven loop
    // hub order for PR: vertices ranked by global degree (descending); the
    // replicated contributions are re-laid out in that order every iteration so the gathers of
    // the hubs share cache lines, as after the single-GPU engine's relabeling
    uint32_t *horder = nullptr;             // npad: vertex of rank i
    uint32_t *hrank = nullptr;              // npad: rank of vertex v
    float *crank = nullptr;                 // npad: contributions in hub order
};

int64_t dist_slice(int64_t n, int32_t p) {
    int64_t per = (n + p - 1) / p;
    return (per + 63) / 64 * 64;
}

// ------------------------------------------------------------------ kernels
namespace {

constexpr int kDB = 256;    // threads per CTA of the partition kernels
constexpr int kDW = kDB / 32;

inline int grid_for(long long work, int sms) {
    long long b = (work + kDB - 1) / kDB;
    return (int)std::max(1LL, std::min(b, (long long)sms * 8));
}

__global__ void k_rebase_offsets(const int64_t *in, int64_t base, uint32_t *out, long long n1) {
    for (long long i = gtid(); i < n1; i += gthreads()) out[i] = (uint32_t)(in[i] - base);
}
__global__ void k_rebase_offsets_u32(const uint32_t *in, uint32_t base, uint32_t *out, long long n1) {
    for (long long i = gtid(); i < n1; i += gthreads()) out[i] = in[i] - base;
}
__global__ void k_first(const uint32_t *roff, const int32_t *rcol, int nloc, int32_t *first) {
    for (long long v = gtid(); v < nloc; v += gthreads()) first[v] = roff[v + 1] > roff[v] ? rcol[roff[v]] : -1;
}
// Hub first (create time): every owned row moves its highest-degree neighbour to the front, so
// the pull's first probe (k_first) meets the likeliest frontier member, as the single-GPU engine's
// degree-ordered relabeling does (C3 p=1: the widest pull level scanned 5.3M edges
// vs 2.8M).  deg: the replicated degree array (all-gathered).  A row's order is irrelevant to
// every other kernel (weights move with their columns).
__global__ void k_degrees(const uint32_t *roff, int nloc, int64_t S, uint32_t *deg_slice) {
    for (long long v = gtid(); v < S; v += gthreads()) deg_slice[v] = v < nloc ? roff[v + 1] - roff[v] : 0u;
}
__global__ void k_hub_first(const uint32_t *roff, int32_t *rcol, uint32_t *rw, int nloc, const uint32_t *deg) {
    for (long long v = gwarp(); v < nloc; v += gwarps()) {
        const uint32_t b = roff[v], e = roff[v + 1];
        unsigned best = 0u;
        uint32_t at = b;
        for (uint32_t k = b + lane_id(); k < e; k += 32) {
            const unsigned dk = deg[rcol[k]];
            if (dk > best || (dk == best && k < at)) { best = dk; at = k; }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned ob = __shfl_xor_sync(0xffffffffu, best, o);
            const uint32_t oa = __shfl_xor_sync(0xffffffffu, at, o);
            if (ob > best || (ob == best && oa < at)) { best = ob; at = oa; }
        }
        if (lane_id() == 0 && e > b && at != b) {
            const int32_t c = rcol[b]; rcol[b] = rcol[at]; rcol[at] = c;
            if (rw) { const uint32_t w = rw[b]; rw[b] = rw[at]; rw[at] = w; }
        }
    }
}
__global__ void k_iota(uint32_t *x, int64_t n) {
    for (long long i = gtid(); i < n; i += gthreads()) x[i] = (uint32_t)i;
}
__global__ void k_invert(const uint32_t *order, int64_t n, uint32_t *rank) {
    for (long long i = gtid(); i < n; i += gthreads()) rank[order[i]] = (uint32_t)i;
}
__global__ void k_rename(const int32_t *col, uint32_t m, const uint32_t *rank, uint32_t *out) {
    for (long long e = gtid(); e < m; e += gthreads()) out[e] = rank[__ldg(col + e)];
}
// contributions re-laid out in hub order: coalesced writes, gathers from the all-gathered array
__global__ void k_hub_layout(const float *c, const uint32_t *order, int64_t n, float *cr) {
    for (long long i = gtid(); i < n; i += gthreads()) cr[i] = c[__ldg(order + i)];
}
// column slice "global source -> owned targets": count, scan, fill
__global__ void k_slice_count(const uint32_t *roff, const int32_t *rcol, int nloc, uint32_t *cnt) {
    for (long long v = gtid(); v < nloc; v += gthreads())
        for (uint32_t e = roff[v]; e < roff[v + 1]; ++e) atomicAdd(cnt + rcol[e], 1u);
}
__global__ void k_slice_fill(const uint32_t *roff, const int32_t *rcol, const uint32_t *rw, int nloc, uint32_t *cursor,
                             int32_t *scol, uint32_t *sw) {
    for (long long v = gtid(); v < nloc; v += gthreads())
        for (uint32_t e = roff[v]; e < roff[v + 1]; ++e) {
            const uint32_t k = atomicAdd(cursor + rcol[e], 1u);
            scol[k] = (int32_t)v;
            if (sw) sw[k] = rw[e];     // symmetric graph: w(u, v) = w(v, u)
        }
}
// sum of the owned rows' weights (for wbar)
__global__ void k_wsum(const uint32_t *w, uint32_t m, unsigned long long *out) {
    unsigned long long s = 0;
    for (long long e = gtid(); e < m; e += gthreads()) s += w[e];
    s = warp_sum(s);
    if (lane_id() == 0 && s) atomicAdd(out, s);
}
// heavy owned rows -> kHeavy-edge chunks (order irrelevant: partials meet in atomics)
__global__ void k_chunks(const uint32_t *roff, int nloc, DTask *tab, unsigned *cnt) {
    for (long long v = gtid(); v < nloc; v += gthreads()) {
        const uint32_t b = roff[v], e = roff[v + 1];
        if (e - b > kHeavy) {
            const unsigned k = (e - b + kHeavy - 1) / kHeavy;
            const unsigned i = atomicAdd(cnt, k);
            for (unsigned j = 0; j < k; ++j) tab[i + j] = DTask{(int)v, b + j * kHeavy, min(e, b + (j + 1) * kHeavy)};
        }
    }
}

// CTA reduction of up to 3 u64 counters + 1 f64 into a part's counter slot (one atomic each)
__device__ __forceinline__ void flush_loc(unsigned long long a, unsigned long long b, unsigned long long c,
                                          double f, unsigned long long *loc) {
    __shared__ unsigned long long s[kDW][3];
    __shared__ double sf[kDW];
    a = warp_sum(a); b = warp_sum(b); c = warp_sum(c); f = warp_sum(f);
    if (lane_id() == 0) { s[threadIdx.x >> 5][0] = a; s[threadIdx.x >> 5][1] = b; s[threadIdx.x >> 5][2] = c; sf[threadIdx.x >> 5] = f; }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long x = 0, y = 0, z = 0;
        double ff = 0.0;
        for (int w = 0; w < kDW; ++w) { x += s[w][0]; y += s[w][1]; z += s[w][2]; ff += sf[w]; }
        if (x) atomicAdd(loc, x);
        if (y) atomicAdd(loc + 1, y);
        if (z) atomicAdd(loc + 2, z);
        if (ff != 0.0) atomicAdd(reinterpret_cast<double *>(loc + 4), ff);
    }
}

__global__ void k_sum_parts(const unsigned long long *locs, int parts, DCtl *ctl) {
    if (threadIdx.x < 4) {
        unsigned long long s = 0;
        for (int p = 0; p < parts; ++p) s += locs[p * kLocStride + threadIdx.x];
        ctl->tot[threadIdx.x] = s;
    } else if (threadIdx.x == 4) {
        double s = 0.0;
        for (int p = 0; p < parts; ++p) s += reinterpret_cast<const double *>(locs + p * kLocStride)[4];
        ctl->dtot = s;
    }
}
__global__ void k_zero_locs(unsigned long long *locs, int parts) {
    for (int i = threadIdx.x; i < parts * kLocStride; i += blockDim.x) locs[i] = 0ull;
}

// ---------------------------------------------------------------- BFS
struct BfsP {
    const uint32_t *roff;
    const int32_t *rcol, *rfirst;
    const uint32_t *soff;
    const int32_t *scol;
    unsigned *vis;
    int *depth;               // owned slice
    int64_t vb, npad;
    int nloc;
    const unsigned *fb;       // FB_t (global)
    unsigned *nfb;            // FB_{t+1} (global; this part writes its slice)
    DTask *tasks;
    unsigned *ntasks;
    uint32_t task_cap;
    unsigned long long *loc;
    const DCtl *ctl;
    int lvl;                  // < 0: graph mode, the level is ctl->cur
};
__device__ __forceinline__ int bfs_lvl(const BfsP &a) { return a.lvl >= 0 ? a.lvl : a.ctl->cur; }

__global__ void k_bfs_init(BfsP a, int64_t src, unsigned *fb0) {
    const int W = (a.nloc + 31) >> 5;
    for (long long v = gtid(); v < a.nloc; v += gthreads()) a.depth[v] = (a.vb + v == src) ? 0 : -1;
    // visited words: a warp per word, a lane per vertex (coalesced offsets, one ballot); the
    // serial 32-vertex loop per thread this replaces cost 56 us at C3
    for (long long w = gwarp(); w < W; w += gwarps()) {
        const long long v = w * 32 + lane_id();
        const bool done = v >= a.nloc || a.roff[v + 1] == a.roff[v] || a.vb + v == src;   // padding, isolated, source
        const unsigned m = __ballot_sync(0xffffffffu, done);
        if (lane_id() == 0) a.vis[w] = m;
    }
    if (gtid() == 0 && src >= a.vb && src < a.vb + a.nloc) {
        const int v = (int)(src - a.vb);
        a.loc[0] = 1ull;
        a.loc[1] = a.roff[v + 1] - a.roff[v];
        atomicOr(fb0 + (src >> 5), 1u << (src & 31));
    }
}

// claim up to 4 local targets (v < 0: none) with their round trips overlapped: visited words,
// then the atomics of the unvisited ones, then the winners' stores and degree loads
__device__ __forceinline__ void push_claim4(const BfsP &a, const int (&v)[4], unsigned long long &va,
                                           unsigned long long &ea, unsigned long long &ed) {
    unsigned w[4], old[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) w[k] = v[k] >= 0 ? a.vis[v[k] >> 5] : ~0u;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const unsigned bit = v[k] >= 0 ? 1u << (v[k] & 31) : 0u;
        old[k] = (v[k] >= 0 && !(w[k] & bit)) ? atomicOr(a.vis + (v[k] >> 5), bit) : ~0u;
        ed += v[k] >= 0 ? 1ull : 0ull;
    }
    const int lvl1 = bfs_lvl(a) + 1;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        if (v[k] < 0 || (old[k] >> (v[k] & 31)) & 1u) continue;
        a.depth[v[k]] = lvl1;
        atomicOr(a.nfb + ((a.vb + v[k]) >> 5), 1u << (v[k] & 31));      // vb is a multiple of 64
        va++;
        ea += a.roff[v[k] + 1] - a.roff[v[k]];
    }
}

// push, light part: a lane per frontier vertex of the warp's bitmap word (rows <= 32 edges, 4
// columns in flight), the whole warp for rows of 33..kHeavy edges (4 edges per lane in flight),
// CTA-wide tasks for longer rows (k_bfs_push_heavy)
__device__ __noinline__ void bfs_push_body(const BfsP &a) {
    const long long FW = a.npad >> 5;
    const unsigned lane = lane_id();
    unsigned long long va = 0, ea = 0, ed = 0;
    for (long long w = gwarp(); w < FW; w += gwarps()) {
        const unsigned word = a.fb[w];
        if (!word) continue;
        const bool mine = (word >> lane) & 1u;
        const long long u = w * 32 + lane;
        uint32_t s0 = 0, s1 = 0;
        if (mine) { s0 = a.soff[u]; s1 = a.soff[u + 1]; }
        const uint32_t L = s1 - s0;
        if (mine && L > kHeavy) {
            const unsigned k = (L + kHeavy - 1) / kHeavy;
            const unsigned i = atomicAdd(a.ntasks, k);
            for (unsigned j = 0; j < k && i + j < a.task_cap; ++j)
                a.tasks[i + j] = DTask{(int)u, s0 + j * kHeavy, min(s1, s0 + (j + 1) * kHeavy)};
        }
        if (mine && L <= 32) {
            for (uint32_t e = s0; e < s1; e += 4) {
                int v[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) v[k] = e + k < s1 ? __ldg(a.scol + e + k) : -1;
                push_claim4(a, v, va, ea, ed);
            }
        }
        unsigned mid = __ballot_sync(0xffffffffu, mine && L > 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t b = __shfl_sync(0xffffffffu, s0, j), e = __shfl_sync(0xffffffffu, s1, j);
            for (uint32_t k = b + lane; k < e; k += 128) {
                int v[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) v[q] = k + 32 * q < e ? __ldg(a.scol + k + 32 * q) : -1;
                push_claim4(a, v, va, ea, ed);
            }
        }
    }
    flush_loc(va, ea, ed, 0.0, a.loc);
}

// heavy rows: a CTA per kHeavy-edge task, 4 edges per thread with their round trips overlapped
// (a warp per task walked 32 dependent claim chains: C3's first push level took 80 us here)
__global__ void __launch_bounds__(kDB) k_bfs_push_heavy(BfsP a) {
    if (a.ctl->done || a.ctl->dir != GSW_PUSH) return;
    a.lvl = bfs_lvl(a);
    const unsigned nt = min(*a.ntasks, a.task_cap);
    unsigned long long va = 0, ea = 0, ed = 0;
    static_assert(kHeavy <= 4 * kDB, "a task fits one pass of the CTA");
    for (unsigned k = blockIdx.x; k < nt; k += gridDim.x) {
        const DTask tk = a.tasks[k];
        int v[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const uint32_t e = tk.beg + threadIdx.x + q * kDB;
            v[q] = e < tk.end ? __ldg(a.scol + e) : -1;
        }
        push_claim4(a, v, va, ea, ed);
    }
    flush_loc(va, ea, ed, 0.0, a.loc);
}

// one launch per level and part: the direction decided on the device (k_bfs_decide) selects the
// push or the pull body; heavy push rows are finished by k_bfs_push_heavy
__global__ void __launch_bounds__(kDB) k_bfs_level(BfsP a) {
    if (a.ctl->done) return;
    a.lvl = bfs_lvl(a);
    if (a.ctl->dir == GSW_PUSH) {
        bfs_push_body(a);
        return;
    }
    __shared__ int lists[(kPullList + kPullWordsPerWarp) * kDW];
    LocalCnt c = bfs_pull_list(a.fb, a.vis, a.depth, a.roff, a.rcol, a.rfirst, a.roff, true, a.lvl,
                               a.nfb + (a.vb >> 5), a.nloc, lists);
    flush_loc(c.va, c.ea, c.edges, 0.0, a.loc);
}

// account level t (its expand and exchange finished, tot = counts of AS_{t+1}) and decide t+1
// (block 0 / thread 0); every thread also clears the bitmap level t+1 will write (FB_t, read by
// level t) and thread 0 the parts' push-task counters, so a level needs no separate memsets
// Graph mode: t = -2 reads the level from ctl->cur, and the WHILE node's condition is set to
// "not done" (cudaGraphSetConditional) so the device decides whether the loop body runs again.
__global__ void k_bfs_decide(DCtl *ctl, DRec *recs, unsigned long long *locs, int parts, int t, long long n,
                             int force_dir, unsigned *clear, long long clear_words, unsigned *ntasks,
                             cudaGraphConditionalHandle cond, int use_cond) {
    for (long long w = gtid(); w < clear_words; w += gthreads()) clear[w] = 0u;
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    if (t == -2) t = ctl->cur;
    ctl->cur = t + 1;
    for (int p = 0; p < parts; ++p) ntasks[p * 32] = 0u;
    const unsigned long long va = ctl->tot[0], ea = ctl->tot[1], ed = ctl->tot[2];
    for (int i = 0; i < parts * kLocStride; ++i) locs[i] = 0ull;
    if (ctl->done) { if (use_cond) cudaGraphSetConditional(cond, 0u); return; }
    if (t >= 0 && t < kMaxLevels) recs[t].edges = (long long)ed;
    if (va == 0) {
        ctl->done = 1;
        if (use_cond) cudaGraphSetConditional(cond, 0u);
        return;
    }
    if (use_cond) cudaGraphSetConditional(cond, 1u);
    ctl->Via -= (long long)va;
    ctl->Eia -= (long long)ea;
    // the single-GPU direction split (select.cuh, R6) on the GLOBAL features
    int dir = ((double)ea * 16.0 > (double)ctl->Eia && (double)va * 2048.0 > (double)n) ? GSW_PULL : GSW_PUSH;
    if (force_dir != GSW_AUTO) dir = force_dir;
    ctl->dir = dir;
    ctl->t = t + 2;                                   // levels with a non-empty active set so far
    if (t + 1 < kMaxLevels) recs[t + 1] = DRec{(long long)va, (long long)ea, ctl->Via, ctl->Eia, 0, dir, 0};
}

// ---------------------------------------------------------------- SSSP (near/far stepping)
// Replicated distances (rep[0], npad u32): rank r relaxes only edges into its owned slice and
// writes only that slice; the slices are all-gathered after every push, so the next round reads
// dist[u] of any frontier vertex locally.
struct SsspP {
    const uint32_t *roff;
    const uint32_t *soff;
    const int32_t *scol;
    const uint32_t *sw;
    unsigned *imp;            // owned: improved by the last push
    unsigned *far;            // owned: improved but above theta (deferred)
    unsigned *dist;           // replicated distances
    int64_t vb, npad;
    int nloc;
    const unsigned *fb;       // the near set N_t (global bitmap)
    unsigned *nfb;            // this part's slice of N_t is written by classify
    DTask *tasks;
    unsigned *ntasks;
    uint32_t task_cap;
    unsigned long long *loc;
    const DCtl *ctl;
};

__global__ void k_sssp_init(SsspP a, int64_t src) {
    const int W = (a.nloc + 31) >> 5;
    for (long long v = gtid(); v < a.nloc; v += gthreads()) a.dist[a.vb + v] = (a.vb + v == src) ? 0u : 0xffffffffu;
    for (long long w = gtid(); w < W; w += gthreads()) {
        unsigned m = 0;
        if (src >= a.vb + w * 32 && src < a.vb + w * 32 + 32 && src < a.vb + a.nloc) m = 1u << ((src - a.vb) & 31);
        a.imp[w] = m;
        a.far[w] = 0u;
    }
}

// Filter of round t: improved or deferred vertices below theta form N_t (this part's slice of the
// replicated bitmap), the rest stays in the far set; counts |N_t|, its edges, |far|
__global__ void __launch_bounds__(kDB) k_sssp_classify(SsspP a) {
    if (a.ctl->done) return;
    const unsigned long long theta = a.ctl->theta;
    const int W = (a.nloc + 31) >> 5;
    unsigned long long va = 0, ea = 0, nf = 0;
    for (long long w = gwarp(); w < W; w += gwarps()) {
        const unsigned cand = a.imp[w] | a.far[w];
        const int v = (int)(w * 32 + lane_id());
        const bool c = (cand >> lane_id()) & 1u;
        bool nr = false;
        if (c) {
            nr = (unsigned long long)a.dist[a.vb + v] < theta;
            if (nr) { va++; ea += a.roff[v + 1] - a.roff[v]; } else nf++;
        }
        const unsigned nm = __ballot_sync(0xffffffffu, nr);
        if (lane_id() == 0) {
            a.nfb[(a.vb >> 5) + w] = nm;
            a.far[w] = cand & ~nm;
            a.imp[w] = 0u;
        }
    }
    flush_loc(va, ea, 0, 0.0, a.loc);
    nf = warp_sum(nf);
    if (lane_id() == 0 && nf) atomicAdd(a.loc + 3, nf);
}

__device__ __forceinline__ void sssp_relax(const SsspP &a, int v, unsigned nd) {
    unsigned *dv = a.dist + a.vb + v;
    if (nd < *dv && nd < atomicMin(dv, nd)) atomicOr(a.imp + (v >> 5), 1u << (v & 31));
}

// Expand of round t: every vertex of N_t relaxes its column-slice row (owned targets)
__global__ void __launch_bounds__(kDB) k_sssp_push(SsspP a) {
    if (a.ctl->done) return;
    const long long FW = a.npad >> 5;
    const unsigned lane = lane_id();
    unsigned long long ed = 0;
    for (long long w = gwarp(); w < FW; w += gwarps()) {
        const unsigned word = a.fb[w];
        if (!word) continue;
        const bool mine = (word >> lane) & 1u;
        const long long u = w * 32 + lane;
        uint32_t s0 = 0, s1 = 0;
        unsigned du = 0;
        if (mine) { s0 = a.soff[u]; s1 = a.soff[u + 1]; du = a.dist[u]; }
        const uint32_t L = s1 - s0;
        if (mine && L > kHeavy) {
            const unsigned k = (L + kHeavy - 1) / kHeavy;
            const unsigned i = atomicAdd(a.ntasks, k);
            for (unsigned j = 0; j < k && i + j < a.task_cap; ++j)
                a.tasks[i + j] = DTask{(int)u, s0 + j * kHeavy, min(s1, s0 + (j + 1) * kHeavy)};
        }
        if (mine && L <= 32)
            for (uint32_t e = s0; e < s1; ++e) { ed++; sssp_relax(a, __ldg(a.scol + e), du + __ldg(a.sw + e)); }
        unsigned mid = __ballot_sync(0xffffffffu, mine && L > 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t b = __shfl_sync(0xffffffffu, s0, j), e = __shfl_sync(0xffffffffu, s1, j);
            const unsigned dj = __shfl_sync(0xffffffffu, du, j);
            for (uint32_t k = b + lane; k < e; k += 32) { ed++; sssp_relax(a, __ldg(a.scol + k), dj + __ldg(a.sw + k)); }
        }
    }
    flush_loc(0, 0, ed, 0.0, a.loc);
}

__global__ void __launch_bounds__(kDB) k_sssp_push_heavy(SsspP a) {
    if (a.ctl->done) return;
    const unsigned nt = min(*a.ntasks, a.task_cap);
    unsigned long long ed = 0;
    for (long long k = gwarp(); k < nt; k += gwarps()) {
        const DTask tk = a.tasks[k];
        const unsigned du = a.dist[tk.row];
        for (uint32_t e = tk.beg + lane_id(); e < tk.end; e += 32) { ed++; sssp_relax(a, __ldg(a.scol + e), du + __ldg(a.sw + e)); }
    }
    flush_loc(0, 0, ed, 0.0, a.loc);
}

// after classify's exchange: empty near set -> advance theta (static delta-stepping, P4) or stop
// when the far set is empty too; records the round; zeroes the counters and push-task counters
__global__ void k_sssp_decide(DCtl *ctl, DRec *recs, unsigned long long *locs, int parts, int t, unsigned *ntasks) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const unsigned long long va = ctl->tot[0], ea = ctl->tot[1], nf = ctl->tot[3];
    for (int i = 0; i < parts * kLocStride; ++i) locs[i] = 0ull;
    for (int p = 0; p < parts; ++p) ntasks[p * 32] = 0u;
    if (ctl->done) return;
    if (va == 0) {
        if (nf == 0) { ctl->done = 1; return; }
        ctl->theta = ctl->theta + ctl->delta;
    }
    if (t < kMaxLevels) recs[t] = DRec{(long long)va, (long long)ea, (long long)nf, 0, 0, GSW_PUSH, (int)min(ctl->theta, 0xffffffffull)};
    ctl->t = t + 1;
}
// edges of round t, read after the push's counters were reduced
__global__ void k_sssp_edges(DCtl *ctl, DRec *recs, unsigned long long *locs, int parts, int t) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    if (t < kMaxLevels && !ctl->done) recs[t].edges = (long long)ctl->tot[2];
    for (int i = 0; i < parts * kLocStride; ++i) locs[i] = 0ull;
}

// ---------------------------------------------------------------- BC (Brandes, per source)
// Replicated depth / sigma / omega: forward level l pulls, for every owned unvisited v, the sum of
// sigma over its in-neighbours at depth l (every parent counts: no early exit); the backward level
// l pulls, for owned v at depth l, delta = sigma(v) * sum over successors w (depth l+1) of
// omega(w) = (1 + delta(w)) / sigma(w).  The owned slices are all-gathered after every level.
struct BcP {
    const uint32_t *roff;
    const int32_t *rcol;
    int64_t vb;
    int nloc;
    int *depth;
    unsigned long long *sigma;
    double *omega;
    double *bc;               // owned slice, accumulated over sources
    const DTask *chunks;
    const unsigned *nchunks;
    double *hacc;             // heavy-row partials (nloc): sigma as u64 bits, or the omega sum
    unsigned long long *loc;
    const DCtl *ctl;
    int src;
};

__global__ void k_bc_init(int *depth, unsigned long long *sigma, int64_t npad, int src) {
    for (long long v = gtid(); v < npad; v += gthreads()) {
        depth[v] = v == src ? 0 : -1;
        sigma[v] = v == src ? 1ull : 0ull;
    }
}

// forward: heavy rows' partial sigma sums over in-neighbours at depth l
__global__ void __launch_bounds__(kDB) k_bc_fwd_heavy(BcP a, int l) {
    if (a.ctl->done) return;
    unsigned long long *acc = reinterpret_cast<unsigned long long *>(a.hacc);
    const unsigned nc = *a.nchunks;
    for (long long k = gwarp(); k < nc; k += gwarps()) {
        const DTask tk = a.chunks[k];
        if (a.depth[a.vb + tk.row] != -1) continue;
        unsigned long long s = 0;
        for (uint32_t e = tk.beg + lane_id(); e < tk.end; e += 32) {
            const int u = __ldg(a.rcol + e);
            if (a.depth[u] == l) s += a.sigma[u];
        }
        s = warp_sum(s);
        if (lane_id() == 0 && s) atomicAdd(acc + tk.row, s);
    }
}

__global__ void __launch_bounds__(kDB) k_bc_fwd(BcP a, int l) {
    if (a.ctl->done) return;
    unsigned long long *acc = reinterpret_cast<unsigned long long *>(a.hacc);
    const unsigned lane = lane_id();
    unsigned long long va = 0, ea = 0, ed = 0;
    for (long long wb = gwarp() * 32; wb < a.nloc; wb += gwarps() * 32) {
        const long long v = wb + lane;
        uint32_t b = 0, e = 0;
        bool open = false;
        if (v < a.nloc) { open = a.depth[a.vb + v] == -1; if (open) { b = a.roff[v]; e = a.roff[v + 1]; } }
        const uint32_t L = e - b;
        unsigned long long sg = 0;
        if (open && L < 32) {
            for (uint32_t k = b; k < e; ++k) {
                const int u = __ldg(a.rcol + k);
                if (a.depth[u] == l) sg += a.sigma[u];
            }
            ed += L;
        } else if (open && L > kHeavy) {
            sg = acc[v];
            acc[v] = 0ull;
            ed += L;
        }
        unsigned mid = __ballot_sync(0xffffffffu, open && L >= 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), ej = __shfl_sync(0xffffffffu, e, j);
            unsigned long long t = 0;
            for (uint32_t k = bj + lane; k < ej; k += 32) {
                const int u = __ldg(a.rcol + k);
                if (a.depth[u] == l) t += a.sigma[u];
            }
            t = warp_sum(t);
            if ((int)lane == j) { sg = t; ed += ej - bj; }
        }
        if (open && sg) {           // v joins level l+1 (plain stores: owned, and read only next level)
            a.depth[a.vb + v] = l + 1;
            a.sigma[a.vb + v] = sg;
            va++;
            ea += L;
        }
    }
    flush_loc(va, ea, ed, 0.0, a.loc);
}

// omega = 1 / sigma for every reached vertex (delta = 0 below the deepest level); local on the
// replicated arrays
__global__ void k_bc_omega0(const int *depth, const unsigned long long *sigma, double *omega, int64_t npad) {
    for (long long v = gtid(); v < npad; v += gthreads())
        omega[v] = depth[v] >= 0 && sigma[v] ? 1.0 / (double)sigma[v] : 0.0;
}

__global__ void __launch_bounds__(kDB) k_bc_bwd_heavy(BcP a, int l) {
    const unsigned nc = *a.nchunks;
    for (long long k = gwarp(); k < nc; k += gwarps()) {
        const DTask tk = a.chunks[k];
        if (a.depth[a.vb + tk.row] != l) continue;
        double s = 0.0;
        for (uint32_t e = tk.beg + lane_id(); e < tk.end; e += 32) {
            const int w = __ldg(a.rcol + e);
            if (a.depth[w] == l + 1) s += a.omega[w];
        }
        s = warp_sum(s);
        if (lane_id() == 0 && s != 0.0) atomicAdd(a.hacc + tk.row, s);
    }
}

__global__ void __launch_bounds__(kDB) k_bc_bwd(BcP a, int l) {
    const unsigned lane = lane_id();
    for (long long wb = gwarp() * 32; wb < a.nloc; wb += gwarps() * 32) {
        const long long v = wb + lane;
        uint32_t b = 0, e = 0;
        bool on = false;
        if (v < a.nloc) { on = a.depth[a.vb + v] == l; if (on) { b = a.roff[v]; e = a.roff[v + 1]; } }
        const uint32_t L = e - b;
        double s = 0.0;
        if (on && L < 32) {
            for (uint32_t k = b; k < e; ++k) {
                const int w = __ldg(a.rcol + k);
                if (a.depth[w] == l + 1) s += a.omega[w];
            }
        } else if (on && L > kHeavy) {
            s = a.hacc[v];
            a.hacc[v] = 0.0;
        }
        unsigned mid = __ballot_sync(0xffffffffu, on && L >= 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), ej = __shfl_sync(0xffffffffu, e, j);
            double t = 0.0;
            for (uint32_t k = bj + lane; k < ej; k += 32) {
                const int w = __ldg(a.rcol + k);
                if (a.depth[w] == l + 1) t += a.omega[w];
            }
            t = warp_sum(t);
            if ((int)lane == j) s = t;
        }
        if (on) {
            const double sg = (double)a.sigma[a.vb + v];
            const double delta = sg * s;
            a.omega[a.vb + v] = (1.0 + delta) / sg;
            if (a.vb + v != a.src) a.bc[v] += delta;
        }
    }
}

__global__ void k_bc_decide(DCtl *ctl, DRec *recs, unsigned long long *locs, int parts, int t) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const unsigned long long va = ctl->tot[0];
    for (int i = 0; i < parts * kLocStride; ++i) locs[i] = 0ull;
    if (ctl->done) return;
    if (va == 0) { ctl->done = 1; return; }
    ctl->t = t + 2;                    // levels with a non-empty set so far (level 0 = the source)
    (void)recs;
}

__global__ void k_zero_f64(double *x, long long n) {
    for (long long i = gtid(); i < n; i += gthreads()) x[i] = 0.0;
}

// ---------------------------------------------------------------- PageRank
struct PrP {
    const uint32_t *roff;
    const int32_t *rcol;
    int64_t vb;
    int nloc;
    const float *cur;         // replicated contributions pr_t(u)/deg(u)
    float *next;              // replicated next contributions (this part writes its slice)
    double *out;              // owned slice output (last iteration) or nullptr
    const DTask *chunks;
    const unsigned *nchunks;
    double *psum;
    unsigned long long *loc;
    const DCtl *ctl;          // dtot = dangling mass of pr_t
    double d, invN;
};

__global__ void k_pr_init(PrP a) {
    double dang = 0.0;
    for (long long v = gtid(); v < a.nloc; v += gthreads()) {
        const uint32_t dg = a.roff[v + 1] - a.roff[v];
        a.next[a.vb + v] = dg ? (float)(a.invN / dg) : 0.f;
        if (!dg) dang += a.invN;
        if (a.out) a.out[v] = a.invN;
        a.psum[v] = 0.0;
    }
    flush_loc(0, 0, 0, dang, a.loc);
}

__global__ void __launch_bounds__(kDB) k_pr_heavy(PrP a) {
    const unsigned nc = *a.nchunks;
    for (long long k = gwarp(); k < nc; k += gwarps()) {
        const DTask tk = a.chunks[k];
        double s = 0.0;
        for (uint32_t e = tk.beg + lane_id(); e < tk.end; e += 32) s += (double)a.cur[__ldg(a.rcol + e)];
        s = warp_sum(s);
        if (lane_id() == 0) atomicAdd(a.psum + tk.row, s);
    }
}

// a lane per row below 32 edges (4 gathers in flight), the warp for rows up to kHeavy, the
// chunk partials for heavier rows
__global__ void __launch_bounds__(kDB) k_pr_rows(PrP a) {
    const double base = (1.0 - a.d) * a.invN + a.d * a.ctl->dtot * a.invN;
    const unsigned lane = lane_id();
    double dang = 0.0;
    for (long long wb = gwarp() * 32; wb < a.nloc; wb += gwarps() * 32) {
        const long long v = wb + lane;
        uint32_t b = 0, e = 0;
        if (v < a.nloc) { b = a.roff[v]; e = a.roff[v + 1]; }
        const uint32_t L = e - b;
        double s = 0.0;
        if (v < a.nloc && L < 32) {
            double s0 = 0.0, s1 = 0.0;
            uint32_t k = b;
            for (; k + 4 <= e; k += 4) {
                const int u0 = __ldg(a.rcol + k), u1 = __ldg(a.rcol + k + 1), u2 = __ldg(a.rcol + k + 2), u3 = __ldg(a.rcol + k + 3);
                s0 += (double)a.cur[u0] + (double)a.cur[u1];
                s1 += (double)a.cur[u2] + (double)a.cur[u3];
            }
            for (; k < e; ++k) s0 += (double)a.cur[__ldg(a.rcol + k)];
            s = s0 + s1;
        } else if (v < a.nloc && L > kHeavy) {
            s = a.psum[v];
            a.psum[v] = 0.0;
        }
        unsigned mid = __ballot_sync(0xffffffffu, v < a.nloc && L >= 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), ej = __shfl_sync(0xffffffffu, e, j);
            double t = 0.0;
            for (uint32_t k = bj + lane; k < ej; k += 32) t += (double)a.cur[__ldg(a.rcol + k)];
            t = warp_sum(t);
            if ((int)lane == j) s = t;
        }
        if (v < a.nloc) {
            const double p = base + a.d * s;
            a.next[a.vb + v] = L ? (float)(p / (double)L) : 0.f;
            if (!L) dang += p;
            if (a.out) a.out[v] = p;
        }
    }
    flush_loc(0, 0, 0, dang, a.loc);
}

// ---------------------------------------------------------------- CC
struct CcP {
    const uint32_t *roff;
    const int32_t *rcol;
    int64_t vb;
    int nloc;
    const uint32_t *cur;      // replicated labels
    uint32_t *next;           // replicated next labels (this part writes its slice)
    int32_t *out;             // owned slice output or nullptr
    const DTask *chunks;
    const unsigned *nchunks;
    uint32_t *hmin;           // heavy-row minima (nloc), ~0 between iterations
    unsigned long long *loc;
    const DCtl *ctl;
};

__global__ void k_cc_init(uint32_t *lab, int64_t npad, uint32_t *hmin, int nloc) {
    for (long long v = gtid(); v < npad; v += gthreads()) lab[v] = (uint32_t)v;
    for (long long v = gtid(); v < nloc; v += gthreads()) hmin[v] = 0xffffffffu;
}

__global__ void __launch_bounds__(kDB) k_cc_heavy(CcP a) {
    if (a.ctl->done) return;
    const unsigned nc = *a.nchunks;
    for (long long k = gwarp(); k < nc; k += gwarps()) {
        const DTask tk = a.chunks[k];
        uint32_t m = 0xffffffffu;
        for (uint32_t e = tk.beg + lane_id(); e < tk.end; e += 32) m = min(m, a.cur[__ldg(a.rcol + e)]);
        m = warp_min(m);
        if (lane_id() == 0) atomicMin(a.hmin + tk.row, m);
    }
}

// label'[v] = min(label[v], min over neighbours), then the shortcut label'[v] = label[label'[v]]
__global__ void __launch_bounds__(kDB) k_cc_rows(CcP a) {
    if (a.ctl->done) return;
    const unsigned lane = lane_id();
    unsigned long long changed = 0;
    for (long long wb = gwarp() * 32; wb < a.nloc; wb += gwarps() * 32) {
        const long long v = wb + lane;
        uint32_t b = 0, e = 0;
        if (v < a.nloc) { b = a.roff[v]; e = a.roff[v + 1]; }
        const uint32_t L = e - b;
        uint32_t m = v < a.nloc ? a.cur[a.vb + v] : 0xffffffffu;
        if (v < a.nloc && L < 32) {
            uint32_t k = b;
            for (; k + 4 <= e; k += 4) {
                const int u0 = __ldg(a.rcol + k), u1 = __ldg(a.rcol + k + 1), u2 = __ldg(a.rcol + k + 2), u3 = __ldg(a.rcol + k + 3);
                m = min(m, min(min(a.cur[u0], a.cur[u1]), min(a.cur[u2], a.cur[u3])));
            }
            for (; k < e; ++k) m = min(m, a.cur[__ldg(a.rcol + k)]);
        } else if (v < a.nloc && L > kHeavy) {
            m = min(m, a.hmin[v]);
            a.hmin[v] = 0xffffffffu;
        }
        unsigned mid = __ballot_sync(0xffffffffu, v < a.nloc && L >= 32 && L <= kHeavy);
        while (mid) {
            const int j = __ffs(mid) - 1;
            mid &= mid - 1;
            const uint32_t bj = __shfl_sync(0xffffffffu, b, j), ej = __shfl_sync(0xffffffffu, e, j);
            uint32_t t = 0xffffffffu;
            for (uint32_t k = bj + lane; k < ej; k += 32) t = min(t, a.cur[__ldg(a.rcol + k)]);
            t = warp_min(t);
            if ((int)lane == j) m = min(m, t);
        }
        if (v < a.nloc) {
            m = min(m, a.cur[m]);                     // pointer jumping on the replicated labels
            a.next[a.vb + v] = m;
            changed += m != a.cur[a.vb + v];
            if (a.out) a.out[v] = (int32_t)m;
        }
    }
    flush_loc(0, 0, 0, 0.0, a.loc);
    changed = warp_sum(changed);
    if (lane == 0 && changed) atomicAdd(a.loc + 3, changed);
}

__global__ void k_cc_decide(DCtl *ctl, unsigned long long *locs, int parts, int t) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const unsigned long long ch = ctl->tot[3];
    for (int i = 0; i < parts * kLocStride; ++i) locs[i] = 0ull;
    if (ctl->done) return;
    ctl->t = t + 1;
    if (ch == 0) ctl->done = 1;
}

}  // namespace

// ------------------------------------------------------------------ workspace + creation
static size_t al(size_t x) { return (x + 255) & ~size_t(255); }
static size_t chunk_cap(uint64_t nnz) { return (size_t)(2 * nnz / kHeavy + 2); }

static size_t dist_bytes(int64_t n, int64_t nnz_total, int32_t nranks, int32_t nparts, int mode, bool weighted) {
    const int64_t S = dist_slice(n, nranks), npad = S * nranks;
    size_t b = 0;
    b += al((size_t)npad / 8) * 2;                           // FB[2]
    b += al((size_t)npad * 4) + 2 * al((size_t)npad * 8);    // BC: depth, sigma, omega (replicated)
    b += al((size_t)npad * 4) * 2;                           // rep[2]
    b += al((size_t)kLocStride * 8 * nparts) + al(sizeof(DCtl)) + al(sizeof(DRec) * kMaxLevels) + al((size_t)128 * nparts);
    for (int p = 0; p < nparts; ++p) {
        b += al((size_t)(S + 1) * 4) + al((size_t)S * 4);    // roff, rfirst
        b += al((size_t)(n + 1) * 4);                        // soff
        b += al((size_t)S / 8 + 8) * 2;                      // vis, far
        b += al((size_t)S * 8);                              // psum
        b += al(256) * 2;                                    // nchunks, nptasks
    }
    // chunk and push-task tables: bounded by the part's nnz, summed over parts <= total nnz
    b += (size_t)nparts * 2 * al(0) + 2 * al(chunk_cap((uint64_t)nnz_total) * sizeof(DTask)) + nparts * 512;
    b += al((size_t)std::max<int64_t>(nnz_total, 1) * 4);   // scol (all parts)
    b += al((size_t)std::max<int64_t>(nnz_total, 1) * 4);   // rcol copy
    if (weighted) b += 2 * al((size_t)std::max<int64_t>(nnz_total, 1) * 4);   // row + slice weights
    b += 3 * al((size_t)npad * 4) + al((size_t)std::max<int64_t>(nnz_total, 1) * 4);   // PR hub order: order, rank, contributions, renamed columns
    if (mode == DM_LOOPBACK) b += al((size_t)(n + 1) * 4);  // full u32 offsets
    size_t cub = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, cub, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)(n + 1));
    b += al(cub) + al((size_t)(n + 1) * 4);                  // scan temp + cursor
    b += al((size_t)(n + 1) * 8);                            // i64 staging of the caller's offsets
    b += al((size_t)npad * 8);                               // output staging (depth / rank / labels)
    return b + (2 << 20);
}

static gsw_status build_slice(gsw_graph g, DPart &p, int64_t n, int32_t *scol, void *cub_tmp, size_t cub_bytes,
                              uint32_t *cursor) {
    cudaStream_t s = g->stream;
    GSW_CUDA(cudaMemsetAsync(p.soff, 0, (size_t)(n + 1) * 4, s));
    k_slice_count<<<grid_for(p.nloc, g->sms), kDB, 0, s>>>(p.roff, p.rcol, p.nloc, p.soff);
    GSW_CUDA(cudaGetLastError());
    size_t cb = cub_bytes;
    GSW_CUDA(cub::DeviceScan::ExclusiveSum(cub_tmp, cb, p.soff, p.soff, (int)(n + 1), s));
    GSW_CUDA(cudaMemcpyAsync(cursor, p.soff, (size_t)(n + 1) * 4, cudaMemcpyDeviceToDevice, s));
    k_slice_fill<<<grid_for(p.nloc, g->sms), kDB, 0, s>>>(p.roff, p.rcol, p.rw, p.nloc, cursor, scol, p.sw);
    GSW_CUDA(cudaGetLastError());
    p.scol = scol;
    return GSW_OK;
}

// ---- exchange (the only place the three backends differ)
static gsw_status host_stage(DistState *d, size_t bytes) {
    if (bytes <= d->hcap) return GSW_OK;
    if (d->hsend) cudaFreeHost(d->hsend);
    if (d->hrecv) cudaFreeHost(d->hrecv);
    d->hsend = d->hrecv = nullptr;
    d->hcap = 0;
    GSW_CUDA(cudaHostAlloc((void **)&d->hsend, bytes, cudaHostAllocDefault));
    GSW_CUDA(cudaHostAlloc((void **)&d->hrecv, bytes * d->nranks, cudaHostAllocDefault));
    d->hcap = bytes;
    return GSW_OK;
}

// in-place all-gather of the rank slices of a replicated buffer: `per` bytes per rank (a frontier
// bitmap: S/8; per-vertex words: 4 S)
static gsw_status ex_allgather(DistState *d, void *buf, size_t per, cudaStream_t s) {
    if (d->mode == DM_LOOPBACK) return GSW_OK;                 // the replica is shared by the parts
    if (d->mode == DM_NCCL) {
        const bool words = per % 4 == 0;
        GSW_NCCL(g_nccl.allGather((char *)buf + (size_t)d->rank * per, buf, words ? per / 4 : per,
                                  words ? ncclUint32 : ncclUint8, d->comm, s));
        return GSW_OK;
    }
    if (gsw_status e = host_stage(d, per)) return e;
    GSW_CUDA(cudaMemcpyAsync(d->hsend, (char *)buf + (size_t)d->rank * per, per, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (d->hx.allgather(d->hx.user, d->hsend, d->hrecv, per) != 0) { set_error("host exchange: allgather callback failed"); return GSW_ENCCL; }
    GSW_CUDA(cudaMemcpyAsync(buf, d->hrecv, per * d->nranks, cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    return GSW_OK;
}

// sum the parts' / ranks' counters into ctl->tot and ctl->dtot
static gsw_status ex_reduce(DistState *d, cudaStream_t s) {
    if (d->mode == DM_LOOPBACK) {
        k_sum_parts<<<1, 32, 0, s>>>(d->locs, (int)d->parts.size(), d->ctl);
        GSW_CUDA(cudaGetLastError());
        return GSW_OK;
    }
    if (d->mode == DM_NCCL) {
        GSW_NCCL(g_nccl.groupStart());
        GSW_NCCL(g_nccl.allReduce(d->locs, d->ctl->tot, 4, ncclUint64, ncclSum, d->comm, s));
        GSW_NCCL(g_nccl.allReduce(d->locs + 4, &d->ctl->dtot, 1, ncclFloat64, ncclSum, d->comm, s));
        GSW_NCCL(g_nccl.groupEnd());
        return GSW_OK;
    }
    unsigned long long h[kLocStride];
    GSW_CUDA(cudaMemcpyAsync(h, d->locs, sizeof(h), cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    double f;
    std::memcpy(&f, h + 4, 8);
    if (d->hx.allreduce_u64(d->hx.user, (uint64_t *)h, 4) != 0 || d->hx.allreduce_f64(d->hx.user, &f, 1) != 0) {
        set_error("host exchange: allreduce callback failed");
        return GSW_ENCCL;
    }
    std::memcpy(h + 4, &f, 8);
    GSW_CUDA(cudaMemcpyAsync(d->ctl->tot, h, 32, cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaMemcpyAsync(&d->ctl->dtot, h + 4, 8, cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    return GSW_OK;
}

gsw_status dist_create(const gsw_csr *rows, int64_t n, const void *nccl_id, const gsw_exchange *hx, int32_t nranks,
                       int32_t rank, int mode, void *workspace, size_t ws_bytes, void *stream, gsw_graph *out) {
    *out = nullptr;
    if (!rows || !rows->row_offsets || (rows->nnz > 0 && !rows->col_indices) || n <= 0 || nranks < 1 ||
        rank < 0 || rank >= nranks) {
        set_error("dist create: bad arguments");
        return GSW_EINVAL;
    }
    if (mode == DM_HOST && (!hx || !hx->allgather || !hx->allreduce_u64 || !hx->allreduce_f64)) {
        set_error("dist create: host exchange needs allgather / allreduce_u64 / allreduce_f64 callbacks");
        return GSW_EINVAL;
    }
    if (n >= (int64_t(1) << 31) - 64 || rows->nnz >= (int64_t(1) << 32)) { set_error("graph too large"); return GSW_EOVERFLOW; }
    const int64_t S = dist_slice(n, nranks);
    const bool loopback = mode == DM_LOOPBACK;
    const int nparts = loopback ? nranks : 1;
    if (!loopback) {
        const int64_t own = std::max<int64_t>(0, std::min<int64_t>(n, (int64_t)(rank + 1) * S) - (int64_t)rank * S);
        if (rows->n != own) { set_error("owned rows must be exactly the rank's slice (gsw_dist_slice)"); return GSW_EINVAL; }
    } else if (rows->n != n) {
        set_error("loopback mode takes the full graph");
        return GSW_EINVAL;
    }
    const size_t need = dist_bytes(n, rows->nnz, nranks, nparts, mode, rows->weights != nullptr);
    if (!workspace || is_device_ptr(workspace) != 1 || ws_bytes < need) {
        set_error("dist workspace must be a device buffer of >= " + std::to_string(need) + " bytes");
        return GSW_ENOMEM;
    }
    gsw_graph g = new gsw_graph_s();
    g->stream = (cudaStream_t)stream;
    g->ws = (char *)workspace;
    g->ws_bytes = ws_bytes;
    cudaError_t e = cudaGetDevice(&g->device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g->sms, cudaDevAttrMultiProcessorCount, g->device);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev0);
    if (e == cudaSuccess) e = cudaEventCreate(&g->ev1);
    if (e != cudaSuccess) { delete g; return cuda_fail(e, "dist create setup"); }
    DistState *d = new DistState();
    g->dist = d;
    d->mode = mode;
    d->nranks = nranks; d->rank = rank;
    d->n = n; d->S = S; d->npad = S * nranks;
    if (hx) d->hx = *hx;
    g->g.n = (int)n;
    g->g.nnz = (uint32_t)rows->nnz;
    auto fail = [&](gsw_status st) { gsw_graph_destroy(g); return st; };
    // the communicator first: every rank arrives here at about the same time (the graph ingest
    // below can take seconds at C5 scale, longer than NCCL's bootstrap waits for its peers)
    if (mode == DM_NCCL) {
        if (!nccl_load()) return fail(GSW_ENCCL);
        if (!nccl_id) { set_error("NCCL mode needs the ncclUniqueId"); return fail(GSW_EINVAL); }
        ncclUniqueId id;
        std::memcpy(&id, nccl_id, sizeof(id));
        ncclResult_t r = g_nccl.commInitRank(&d->comm, nranks, id, rank);
        if (r != ncclSuccess) { set_error(std::string("ncclCommInitRank: ") + g_nccl.errStr(r)); return fail(GSW_ENCCL); }
    }
    for (auto &ev : d->evs)
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "events"));
    if (const char *e = getenv("GSW_DIST_LOOKAHEAD")) d->lookahead = std::max(1, std::min(kLookaheadMax, atoi(e)));
    if (cudaHostAlloc((void **)&d->hdone, sizeof(int) * (kLookaheadMax + 1), cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer((void **)&d->hdone_dev, d->hdone, 0) != cudaSuccess)
        return fail(cuda_fail(cudaGetLastError(), "pinned flags"));
    Workspace ws{g->ws, ws_bytes, 0};
    d->FB[0] = (unsigned *)ws.take(d->npad / 8);
    d->FB[1] = (unsigned *)ws.take(d->npad / 8);
    d->rep[0] = (uint32_t *)ws.take(d->npad * 4);
    d->rep[1] = (uint32_t *)ws.take(d->npad * 4);
    d->locs = (unsigned long long *)ws.take((size_t)kLocStride * 8 * nparts);
    d->ctl = (DCtl *)ws.take(sizeof(DCtl));
    d->recs = (DRec *)ws.take(sizeof(DRec) * kMaxLevels);
    d->ntasks = (unsigned *)ws.take((size_t)128 * nparts);
    d->bdepth = (int *)ws.take((size_t)d->npad * 4);
    d->bsigma = (unsigned long long *)ws.take((size_t)d->npad * 8);
    d->bomega = (double *)ws.take((size_t)d->npad * 8);
    int64_t *staging = (int64_t *)ws.take((size_t)(n + 1) * 8);
    size_t cub_bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, cub_bytes, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)(n + 1));
    void *cub_tmp = ws.take(cub_bytes);
    uint32_t *cursor = (uint32_t *)ws.take((size_t)(n + 1) * 4);
    int32_t *scol_all = (int32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4);
    int32_t *col = (int32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4);
    uint32_t *full_off = loopback ? (uint32_t *)ws.take((size_t)(n + 1) * 4) : nullptr;
    d->weighted = rows->weights != nullptr;
    uint32_t *wrow = d->weighted ? (uint32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4) : nullptr;
    uint32_t *wslice = d->weighted ? (uint32_t *)ws.take((size_t)std::max<int64_t>(rows->nnz, 1) * 4) : nullptr;
    if (d->weighted && (!wrow || !wslice)) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
    DTask *chunk_all = (DTask *)ws.take(chunk_cap((uint64_t)rows->nnz) * sizeof(DTask));
    DTask *task_all = (DTask *)ws.take(chunk_cap((uint64_t)rows->nnz) * sizeof(DTask));
    if (!d->FB[1] || !d->rep[1] || !d->locs || !d->ctl || !d->recs || !d->ntasks || !d->bomega || !staging || !cub_tmp || !cursor || !scol_all ||
        !col || (loopback && !full_off) || !chunk_all || !task_all) {
        set_error("dist workspace too small");
        return fail(GSW_ENOMEM);
    }
    cudaStream_t s = g->stream;
    // adjacency on the device
    const int64_t *off64 = rows->row_offsets;
    if (!is_device_ptr(off64)) {
        if (cudaMemcpyAsync(staging, off64, (size_t)(rows->n + 1) * 8, cudaMemcpyHostToDevice, s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "copy offsets"));
        off64 = staging;
    }
    if (rows->nnz > 0 && cudaMemcpyAsync(col, rows->col_indices, (size_t)rows->nnz * 4,
                                         is_device_ptr(rows->col_indices) ? cudaMemcpyDeviceToDevice
                                                                          : cudaMemcpyHostToDevice, s) != cudaSuccess)
        return fail(cuda_fail(cudaGetLastError(), "copy columns"));
    if (d->weighted && rows->nnz > 0 &&
        cudaMemcpyAsync(wrow, rows->weights, (size_t)rows->nnz * 4,
                        is_device_ptr(rows->weights) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, s) != cudaSuccess)
        return fail(cuda_fail(cudaGetLastError(), "copy weights"));
    if (loopback) k_rebase_offsets<<<grid_for(n + 1, g->sms), kDB, 0, s>>>(off64, 0, full_off, n + 1);
    std::vector<int64_t> hoff;
    if (loopback) {
        hoff.resize(n + 1);
        if (cudaMemcpyAsync(hoff.data(), off64, (size_t)(n + 1) * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "read offsets"));
    }
    int32_t *scol_cur = scol_all;
    DTask *chunk_cur = chunk_all, *task_cur = task_all;
    for (int p = 0; p < nparts; ++p) {
        DPart P;
        const int r = loopback ? p : rank;
        P.vb = (int64_t)r * S;
        P.nloc = (int)std::max<int64_t>(0, std::min<int64_t>(n, P.vb + S) - P.vb);
        P.roff = (uint32_t *)ws.take((size_t)(S + 1) * 4);
        P.rfirst = (int32_t *)ws.take((size_t)S * 4 + 4);
        P.soff = (uint32_t *)ws.take((size_t)(n + 1) * 4);
        P.vis = (unsigned *)ws.take((size_t)S / 8 + 8);
        P.far = (unsigned *)ws.take((size_t)S / 8 + 8);
        P.psum = (double *)ws.take((size_t)S * 8 + 8);
        P.nchunks = (unsigned *)ws.take(256);
        P.nptasks = d->ntasks ? d->ntasks + 32 * p : nullptr;
        P.loc = d->locs + (size_t)p * kLocStride;
        if (!P.roff || !P.rfirst || !P.soff || !P.vis || !P.far || !P.psum || !P.nchunks || !P.nptasks) {
            set_error("dist workspace too small");
            return fail(GSW_ENOMEM);
        }
        if (loopback) {
            const int64_t e0 = P.nloc ? hoff[P.vb] : 0, e1 = P.nloc ? hoff[P.vb + P.nloc] : 0;
            P.nnz = (uint32_t)(e1 - e0);
            P.rcol = col + e0;
            if (wrow) { P.rw = wrow + e0; P.sw = wslice + e0; }
            if (P.nloc)
                k_rebase_offsets_u32<<<grid_for(P.nloc + 1, g->sms), kDB, 0, s>>>(full_off + P.vb, (uint32_t)e0, P.roff, P.nloc + 1);
        } else {
            P.nnz = (uint32_t)rows->nnz;
            P.rcol = col;
            if (wrow) { P.rw = wrow; P.sw = wslice; }
            k_rebase_offsets<<<grid_for(P.nloc + 1, g->sms), kDB, 0, s>>>(off64, 0, P.roff, P.nloc + 1);
        }
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "rebase"));
        if (gsw_status st = build_slice(g, P, n, scol_cur, cub_tmp, cub_bytes, cursor)) return fail(st);
        k_first<<<grid_for(P.nloc, g->sms), kDB, 0, s>>>(P.roff, P.rcol, P.nloc, P.rfirst);
        P.chunks = chunk_cur;
        P.ptasks = task_cur;
        P.ptask_cap = (uint32_t)chunk_cap(P.nnz);
        if (cudaMemsetAsync(P.nchunks, 0, 4, s) != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "memset"));
        k_chunks<<<grid_for(P.nloc, g->sms), kDB, 0, s>>>(P.roff, P.nloc, P.chunks, P.nchunks);
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "chunks"));
        scol_cur += P.nnz;
        chunk_cur += chunk_cap(P.nnz);
        task_cur += chunk_cap(P.nnz);
        d->parts.push_back(P);
    }
    // hub first: all-gather the degrees into rep[0], reorder every owned row, redo the first-neighbour table
    if (!(std::getenv("GSW_DIST_HUBFIRST") && *std::getenv("GSW_DIST_HUBFIRST") == '0')) {
        for (auto &P : d->parts)
            k_degrees<<<grid_for(S, g->sms), kDB, 0, s>>>(P.roff, P.nloc, S, d->rep[0] + P.vb);
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "degrees"));
        if (gsw_status st = ex_allgather(d, d->rep[0], (size_t)S * 4, s)) return fail(st);
        for (auto &P : d->parts) {
            if (!P.nloc) continue;
            k_hub_first<<<grid_for((long long)P.nloc * 32, g->sms), kDB, 0, s>>>(P.roff, const_cast<int32_t *>(P.rcol),
                                                                               const_cast<uint32_t *>(P.rw), P.nloc, d->rep[0]);
            k_first<<<grid_for(P.nloc, g->sms), kDB, 0, s>>>(P.roff, P.rcol, P.nloc, P.rfirst);
        }
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "hub first"));
    }
    // PR hub order: rank every vertex by its global degree (the degrees are in rep[0] after the hub
    // step; they are gathered here otherwise), rename the owned columns once
    const char *ho = std::getenv("GSW_DIST_PR_HUBORDER");
    if (!(ho && *ho == '0')) {
        d->horder = (uint32_t *)ws.take((size_t)d->npad * 4);
        d->hrank = (uint32_t *)ws.take((size_t)d->npad * 4);
        d->crank = (float *)ws.take((size_t)d->npad * 4);
        if (!d->horder || !d->hrank || !d->crank) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
        const char *hf = std::getenv("GSW_DIST_HUBFIRST");
        if (hf && *hf == '0') {                        // degrees not gathered by the hub-first step
            for (auto &P : d->parts)
                k_degrees<<<grid_for(S, g->sms), kDB, 0, s>>>(P.roff, P.nloc, S, d->rep[0] + P.vb);
            if (gsw_status st = ex_allgather(d, d->rep[0], (size_t)S * 4, s)) return fail(st);
        }
        // descending radix sort of (degree, vertex) with double buffers: rep[0]/rep[1] for the keys,
        // the BC scratch (bdepth) and horder for the values, bsigma as the sort's temp storage
        k_iota<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(reinterpret_cast<uint32_t *>(d->bdepth), d->npad);
        cub::DoubleBuffer<uint32_t> keys(d->rep[0], d->rep[1]);
        cub::DoubleBuffer<uint32_t> vals(reinterpret_cast<uint32_t *>(d->bdepth), d->horder);
        size_t tb = 0;
        cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, keys, vals, (int)d->npad, 0, 32, s);
        if (tb > (size_t)d->npad * 8) { set_error("dist workspace too small (hub-order sort)"); return fail(GSW_ENOMEM); }
        if (cub::DeviceRadixSort::SortPairsDescending(d->bsigma, tb, keys, vals, (int)d->npad, 0, 32, s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "hub-order sort"));
        if (vals.Current() != d->horder &&
            cudaMemcpyAsync(d->horder, vals.Current(), (size_t)d->npad * 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "hub order"));
        k_invert<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(d->horder, d->npad, d->hrank);
        for (auto &P : d->parts) {
            P.rcol_h = (uint32_t *)ws.take((size_t)std::max<uint32_t>(P.nnz, 1) * 4);
            if (!P.rcol_h) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
            if (P.nnz) k_rename<<<grid_for(P.nnz, g->sms), kDB, 0, s>>>(P.rcol, P.nnz, d->hrank, P.rcol_h);
        }
        if (cudaGetLastError() != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "hub order"));
    }
    g->scratch = (char *)ws.take((size_t)d->npad * 8);      // output staging (host outputs)
    g->scratch_bytes = (size_t)d->npad * 8;
    if (!g->scratch) { set_error("dist workspace too small"); return fail(GSW_ENOMEM); }
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail(cuda_fail(cudaGetLastError(), "dist create"));
    // global nnz (once): every rank's owned entries, summed by the exchange
    {
        unsigned long long h[kLocStride] = {};
        for (auto &P : d->parts) h[0] += P.nnz;            // loopback: part 0's slot carries the total
        if (cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * nparts, s) != cudaSuccess ||
            cudaMemcpyAsync(d->locs, h, sizeof(h), cudaMemcpyHostToDevice, s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "nnz"));
        if (wrow && rows->nnz > 0) k_wsum<<<grid_for(rows->nnz, g->sms), kDB, 0, s>>>(wrow, (uint32_t)rows->nnz, d->locs + 1);
        if (gsw_status st = ex_reduce(d, s)) return fail(st);
        unsigned long long tot[4];
        if (cudaMemcpyAsync(tot, d->ctl->tot, 32, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "nnz"));
        DCtl c{};
        c.nnz_g = (long long)tot[0];
        d->wbar = tot[0] ? (double)tot[1] / (double)tot[0] : 1.0;
        if (cudaMemcpyAsync(d->ctl, &c, sizeof(c), cudaMemcpyHostToDevice, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return fail(cuda_fail(cudaGetLastError(), "ctl"));
    }
    *out = g;
    return GSW_OK;
}

void dist_destroy(DistState *d) {
    if (!d) return;
    if (d->bfs_exec) cudaGraphExecDestroy(d->bfs_exec);
    if (d->cap) cudaStreamDestroy(d->cap);
    if (d->comm && g_nccl.ok) g_nccl.commDestroy(d->comm);
    for (auto &ev : d->evs) if (ev) cudaEventDestroy(ev);
    if (d->hdone) cudaFreeHost(d->hdone);
    if (d->hsend) cudaFreeHost(d->hsend);
    if (d->hrecv) cudaFreeHost(d->hrecv);
    delete d;
}

// Pipelined termination: after enqueueing iteration t, poll the done flag of iteration
// t - LOOKAHEAD (host mode: of t itself, its exchange has synchronised already).  Returns through
// *stop whether the host should stop enqueueing.
__global__ void k_publish_done(const DCtl *ctl, volatile int *flag) {
    if (threadIdx.x == 0) { *flag = ctl->done; __threadfence_system(); }
}

static gsw_status poll_done(DistState *d, int t, cudaStream_t s, bool *stop) {
    const int R = d->lookahead + 1;
    // the flag goes to mapped host memory from a one-thread kernel: no copy-engine round trip in
    // the stream between two levels
    k_publish_done<<<1, 32, 0, s>>>(d->ctl, d->hdone_dev + (t % R));
    GSW_CUDA(cudaGetLastError());
    GSW_CUDA(cudaEventRecord(d->evs[t % R], s));
    const int lag = d->mode == DM_HOST ? 0 : d->lookahead;
    *stop = false;
    if (t >= lag) {
        GSW_CUDA(cudaEventSynchronize(d->evs[(t - lag) % R]));
        *stop = d->hdone[(t - lag) % R] != 0;
    }
    return GSW_OK;
}

static void reset_ctl_host(DCtl &c, long long nnz_g, long long n) {
    c = DCtl{};
    c.nnz_g = nnz_g;
    c.Via = n;
    c.Eia = nnz_g;
    c.dir = GSW_PUSH;
}

static gsw_status read_nnz_g(DistState *d, cudaStream_t s, long long *nnz_g) {
    GSW_CUDA(cudaMemcpyAsync(nnz_g, &d->ctl->nnz_g, 8, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed BFS
gsw_status dist_bfs(gsw_graph g, int32_t source, int32_t *depth_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (source < 0 || source >= d->n) { set_error("gsw_bfs: source out of range"); return GSW_EINVAL; }
    if (!depth_out) { set_error("gsw_bfs: depth is NULL"); return GSW_EINVAL; }
    const int fdir = g->forced.direction;
    if (fdir != GSW_AUTO && fdir != GSW_PUSH && fdir != GSW_PULL) { set_error("gsw_bfs: bad forced direction"); return GSW_EUNSUPPORTED; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->mode == DM_LOOPBACK ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(depth_out) == 1;
    int *depth = dev_out ? depth_out : (int *)g->scratch;
    const size_t FBB = (size_t)d->npad / 8;
    long long nnz_g = 0;
    if (gsw_status e = read_nnz_g(d, s, &nnz_g)) return e;
    DCtl c0;
    reset_ctl_host(c0, nnz_g, d->n);
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemcpyAsync(d->ctl, &c0, sizeof(c0), cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaMemsetAsync(d->FB[0], 0, FBB, s));
    GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
    std::vector<BfsP> pa(parts);
    for (int p = 0; p < parts; ++p) {
        const DPart &P = d->parts[p];
        pa[p] = BfsP{P.roff, P.rcol, P.rfirst, P.soff, P.scol, P.vis, depth + (d->mode == DM_LOOPBACK ? P.vb : 0),
                     P.vb, d->npad, P.nloc, nullptr, nullptr, P.ptasks, P.nptasks, P.ptask_cap, P.loc, d->ctl, 0};
        k_bfs_init<<<grid_for(std::max(P.nloc, 1), g->sms), kDB, 0, s>>>(pa[p], source, d->FB[0]);
    }
    GSW_CUDA(cudaGetLastError());
    if (gsw_status e = ex_allgather(d, d->FB[0], (size_t)d->S / 8, s)) return e;      // the owner's source bit
    // level-0 features (Va = 1, Ea = deg(source)) through the same exchange, then the decision
    if (gsw_status e = ex_reduce(d, s)) return e;
    const int grid = g->sms * 8;
    const long long FBW = d->npad / 32;
    k_bfs_decide<<<g->sms, kDB, 0, s>>>(d->ctl, d->recs, d->locs, parts, -1, d->n, fdir, d->FB[1], FBW, d->ntasks,
                                        cudaGraphConditionalHandle{}, 0);
    GSW_CUDA(cudaGetLastError());
    // graph mode: the level loop as one CUDA graph whose WHILE node the decide kernel drives, so
    // the host neither polls nor enqueues per level (NCCL / loopback; GSW_DIST_GRAPH=0 disables)
    // Default: loopback and single-rank NCCL.  With several NCCL ranks the graph holds NCCL's
    // collectives inside a conditional body, which only this one-GPU build could not exercise, so
    // it is opt-in there (GSW_DIST_GRAPH=1); a capture or instantiation failure falls back to the
    // host-driven loop either way.
    const char *gm = std::getenv("GSW_DIST_GRAPH");
    bool graph_mode = d->mode != DM_HOST && !d->graph_failed &&
                      (gm ? *gm != '0' : (d->mode == DM_LOOPBACK || d->nranks == 1));
    if (graph_mode) {
        if (!d->bfs_exec || d->bfs_exec_depth != (const void *)depth || d->bfs_exec_dir != fdir) {
            if (d->bfs_exec) { cudaGraphExecDestroy(d->bfs_exec); d->bfs_exec = nullptr; }
            cudaGraph_t gr = nullptr;
            GSW_CUDA(cudaGraphCreate(&gr, 0));
            cudaGraphConditionalHandle cond;
            GSW_CUDA(cudaGraphConditionalHandleCreate(&cond, gr, 1u, cudaGraphCondAssignDefault));
            cudaGraphNodeParams cp = {};
            cp.type = cudaGraphNodeTypeConditional;
            cp.conditional.handle = cond;
            cp.conditional.type = cudaGraphCondTypeWhile;
            cp.conditional.size = 1;
            cudaGraphNode_t node;
            GSW_CUDA(cudaGraphAddNode(&node, gr, nullptr, 0, &cp));
            cudaGraph_t body = cp.conditional.phGraph_out[0];
            if (!d->cap) GSW_CUDA(cudaStreamCreateWithFlags(&d->cap, cudaStreamNonBlocking));
            const cudaStream_t run = s;
            s = d->cap;                                   // the enqueues below are captured, not run
            GSW_CUDA(cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
            gsw_status cs = GSW_OK;
            for (int par = 0; par < 2 && cs == GSW_OK; ++par) {      // two levels per body: fixed FB parity
                unsigned *fb = d->FB[par], *nfb = d->FB[par ^ 1];
                for (int p = 0; p < parts; ++p) {
                    BfsP a = pa[p];
                    a.fb = fb; a.nfb = nfb; a.lvl = -1;
                    if (!a.nloc) continue;
                    k_bfs_level<<<grid, kDB, 0, s>>>(a);
                    k_bfs_push_heavy<<<g->sms * 2, kDB, 0, s>>>(a);
                }
                if (cudaGetLastError() != cudaSuccess) { cs = GSW_ECUDA; break; }
                if ((cs = ex_allgather(d, nfb, (size_t)d->S / 8, s)) != GSW_OK) break;
                if ((cs = ex_reduce(d, s)) != GSW_OK) break;
                k_bfs_decide<<<g->sms, kDB, 0, s>>>(d->ctl, d->recs, d->locs, parts, -2, d->n, fdir, fb, FBW, d->ntasks,
                                                    cond, 1);
            }
            cudaGraph_t cap = nullptr;
            const cudaError_t ce = cudaStreamEndCapture(s, &cap);
            s = run;
            cudaError_t ie = cudaErrorUnknown;
            if (cs == GSW_OK && ce == cudaSuccess) ie = cudaGraphInstantiate(&d->bfs_exec, gr, 0);
            cudaGraphDestroy(gr);
            if (ie != cudaSuccess) {
                // fall back to the host-driven loop for this handle (nothing of the capture ran)
                cudaGetLastError();
                d->bfs_exec = nullptr;
                d->graph_failed = true;
                graph_mode = false;
                if (std::getenv("GSW_VERBOSE"))
                    std::fprintf(stderr, "gsw: dist BFS graph capture failed (%s), host-driven loop\n",
                                 cudaGetErrorString(ce != cudaSuccess ? ce : ie));
            } else {
                d->bfs_exec_depth = depth;
                d->bfs_exec_dir = fdir;
            }
        }
        if (graph_mode) GSW_CUDA(cudaGraphLaunch(d->bfs_exec, s));
    }
    int t = 0;
    for (; !graph_mode; ++t) {
        unsigned *fb = d->FB[t & 1], *nfb = d->FB[(t + 1) & 1];
        for (int p = 0; p < parts; ++p) {
            BfsP a = pa[p];
            a.fb = fb; a.nfb = nfb; a.lvl = t;
            if (!a.nloc) continue;
            k_bfs_level<<<grid, kDB, 0, s>>>(a);
            k_bfs_push_heavy<<<g->sms * 2, kDB, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        if (gsw_status e = ex_allgather(d, nfb, (size_t)d->S / 8, s)) return e;
        if (gsw_status e = ex_reduce(d, s)) return e;
        k_bfs_decide<<<g->sms, kDB, 0, s>>>(d->ctl, d->recs, d->locs, parts, t, d->n, fdir, fb, FBW, d->ntasks,
                                            cudaGraphConditionalHandle{}, 0);
        GSW_CUDA(cudaGetLastError());
        bool stop = false;
        if (gsw_status e = poll_done(d, t, s, &stop)) return e;
        if (stop || t + 1 >= kMaxLevels) break;
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(depth_out, depth, (size_t)out_len * 4, cudaMemcpyDeviceToHost, s));
    DCtl cend;
    GSW_CUDA(cudaMemcpyAsync(&cend, d->ctl, sizeof(cend), cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    const int levels = std::min(cend.t, kMaxLevels);     // levels with a non-empty active set
    std::vector<DRec> h(levels);
    if (levels) GSW_CUDA(cudaMemcpy(h.data(), d->recs, sizeof(DRec) * levels, cudaMemcpyDeviceToHost));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        unsigned long long edges = 0, bytes = 0;
        for (int i = 0; i < levels; ++i) {
            const unsigned long long Va = h[i].Va, next = i + 1 < levels ? (unsigned long long)h[i + 1].Va : 0ull;
            edges += h[i].edges;
            // SURVEY 8(d) D0, summed over the ranks: push 12|F| + 4E + 8|F'|, pull N/4 + 8|U| + 4S + 4|F'|
            bytes += h[i].dir == GSW_PUSH ? 12ull * Va + 4ull * h[i].edges + 8ull * next
                                          : (unsigned long long)d->n / 4 + 8ull * (unsigned long long)std::max(0LL, h[i].Via) +
                                                4ull * h[i].edges + 4ull * next;
            if (st->records && i < st->max_records) {
                gsw_iter_record &r = st->records[i];
                r = gsw_iter_record{};
                r.iteration = i; r.direction = h[i].dir; r.format = GSW_BITMAP;
                r.load_balance = h[i].dir == GSW_PULL ? GSW_LB_THREAD : GSW_LB_TWC; r.fusion = GSW_FUSED;
                r.Va = h[i].Va; r.Ea = h[i].Ea; r.Via = h[i].Via; r.Eia = h[i].Eia; r.edges = h[i].edges;
                r.ctas = grid;
            }
        }
        st->iterations = levels;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)edges;
        st->bytes_alg = (int64_t)bytes;
    }
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed SSSP
// Near/far rounds with a static step (P4 "static" candidate; forced UNORDERED = Bellman-Ford,
// theta = infinity): classify -> all-gather of the near-set slices + counts -> decide (theta,
// done) -> push over the column slices (atomicMin on owned distances) -> all-gather of the
// distance slices.  The dynamic law of the single-GPU kernel is not used here.
gsw_status dist_sssp(gsw_graph g, int32_t source, uint32_t *dist_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (source < 0 || source >= d->n) { set_error("gsw_sssp: source out of range"); return GSW_EINVAL; }
    if (!dist_out) { set_error("gsw_sssp: dist is NULL"); return GSW_EINVAL; }
    if (!d->weighted) { set_error("gsw_sssp: the partitioned graph has no weights"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->mode == DM_LOOPBACK ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(dist_out) == 1;
    unsigned *distv = d->rep[0];
    long long nnz_g = 0;
    if (gsw_status e = read_nnz_g(d, s, &nnz_g)) return e;
    DCtl c0;
    reset_ctl_host(c0, nnz_g, d->n);
    const gsw_config &fc = g->forced;
    const double dbar = (double)nnz_g / (double)d->n;
    const double d0 = fc.delta0 ? (double)fc.delta0 : 32.0 * d->wbar / std::max(dbar, 1e-9);   // P:660-661, R6b
    c0.delta = (unsigned long long)std::max(1.0, std::min(d0, 2147483647.0));
    c0.theta = fc.stepping == GSW_STEP_UNORDERED ? 0xffffffffull : c0.delta;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemcpyAsync(d->ctl, &c0, sizeof(c0), cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
    GSW_CUDA(cudaMemsetAsync(d->ntasks, 0, (size_t)128 * parts, s));
    GSW_CUDA(cudaMemsetAsync(d->FB[0], 0, (size_t)d->npad / 8, s));   // padding words stay 0 (never classified)
    std::vector<SsspP> pa(parts);
    for (int p = 0; p < parts; ++p) {
        const DPart &P = d->parts[p];
        pa[p] = SsspP{P.roff, P.soff, P.scol, P.sw, P.vis, P.far, distv, P.vb, d->npad, P.nloc, nullptr, nullptr,
                      P.ptasks, P.nptasks, P.ptask_cap, P.loc, d->ctl};
        k_sssp_init<<<grid_for(std::max(P.nloc, 1), g->sms), kDB, 0, s>>>(pa[p], source);
    }
    GSW_CUDA(cudaGetLastError());
    if (gsw_status e = ex_allgather(d, distv, (size_t)d->S * 4, s)) return e;
    const int grid = g->sms * 8;
    unsigned *nb = d->FB[0];
    int t = 0;
    for (;; ++t) {
        for (int p = 0; p < parts; ++p) {
            SsspP a = pa[p];
            a.fb = nb; a.nfb = nb;
            if (a.nloc) k_sssp_classify<<<grid, kDB, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        if (gsw_status e = ex_allgather(d, nb, (size_t)d->S / 8, s)) return e;
        if (gsw_status e = ex_reduce(d, s)) return e;
        k_sssp_decide<<<1, 32, 0, s>>>(d->ctl, d->recs, d->locs, parts, t, d->ntasks);
        for (int p = 0; p < parts; ++p) {
            SsspP a = pa[p];
            a.fb = nb; a.nfb = nb;
            if (!a.nloc) continue;
            k_sssp_push<<<grid, kDB, 0, s>>>(a);
            k_sssp_push_heavy<<<g->sms * 2, kDB, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        if (gsw_status e = ex_allgather(d, distv, (size_t)d->S * 4, s)) return e;
        if (gsw_status e = ex_reduce(d, s)) return e;
        k_sssp_edges<<<1, 32, 0, s>>>(d->ctl, d->recs, d->locs, parts, t);
        GSW_CUDA(cudaGetLastError());
        bool stop = false;
        if (gsw_status e = poll_done(d, t, s, &stop)) return e;
        if (stop || t + 1 >= (1 << 24)) break;
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    const unsigned *own = distv + (d->mode == DM_LOOPBACK ? 0 : d->parts[0].vb);
    GSW_CUDA(cudaMemcpyAsync(dist_out, own, (size_t)out_len * 4, dev_out ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s));
    DCtl cend;
    GSW_CUDA(cudaMemcpyAsync(&cend, d->ctl, sizeof(cend), cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    const int rounds = cend.t;
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        const int nrec = std::min(rounds, kMaxLevels);
        std::vector<DRec> h(nrec);
        if (nrec) GSW_CUDA(cudaMemcpy(h.data(), d->recs, sizeof(DRec) * nrec, cudaMemcpyDeviceToHost));
        unsigned long long edges = 0, bytes = 0;
        for (int i = 0; i < nrec; ++i) {
            edges += h[i].edges;
            bytes += 12ull * h[i].Va + 8ull * h[i].edges + 8ull * (i + 1 < nrec ? h[i + 1].Va : 0);
            if (st->records && i < st->max_records) {
                gsw_iter_record &r = st->records[i];
                r = gsw_iter_record{};
                r.iteration = i; r.direction = GSW_PUSH; r.format = GSW_BITMAP; r.load_balance = GSW_LB_TWC;
                r.stepping = fc.stepping == GSW_STEP_UNORDERED ? GSW_STEP_UNORDERED : GSW_STEP_STATIC;
                r.fusion = GSW_STANDALONE;
                r.Va = h[i].Va; r.Ea = h[i].Ea; r.edges = h[i].edges; r.theta = (uint32_t)h[i].pad;
                r.ctas = grid;
            }
        }
        st->iterations = rounds;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)edges;
        st->bytes_alg = (int64_t)bytes;
    }
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed BC
gsw_status dist_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (!bc_out) { set_error("gsw_bc: bc is NULL"); return GSW_EINVAL; }
    if (nsrc < 0 || (nsrc > 0 && !sources)) { set_error("gsw_bc: bad sources"); return GSW_EINVAL; }
    if (is_device_ptr(sources) == 1) { set_error("gsw_bc: sources must be a host array"); return GSW_EINVAL; }
    for (int i = 0; i < nsrc; ++i)
        if (sources[i] < 0 || sources[i] >= d->n) { set_error("gsw_bc: source out of range"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->mode == DM_LOOPBACK ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(bc_out) == 1;
    double *bc = dev_out ? bc_out : (double *)g->scratch;
    long long nnz_g = 0;
    if (gsw_status e = read_nnz_g(d, s, &nnz_g)) return e;
    const int grid = g->sms * 8;
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    k_zero_f64<<<grid_for(out_len, g->sms), kDB, 0, s>>>(bc, out_len);
    for (auto &P : d->parts) k_zero_f64<<<grid_for(std::max(P.nloc, 1), g->sms), kDB, 0, s>>>(P.psum, P.nloc);
    GSW_CUDA(cudaGetLastError());
    auto args = [&](int p, int src) {
        const DPart &P = d->parts[p];
        return BcP{P.roff, P.rcol, P.vb, P.nloc, d->bdepth, d->bsigma, d->bomega,
                   bc + (d->mode == DM_LOOPBACK ? P.vb : 0), P.chunks, P.nchunks, P.psum, P.loc, d->ctl, src};
    };
    long long levels_total = 0, edges_total = 0;
    for (int si = 0; si < nsrc; ++si) {
        const int src = sources[si];
        DCtl c0;
        reset_ctl_host(c0, nnz_g, d->n);
        GSW_CUDA(cudaMemcpyAsync(d->ctl, &c0, sizeof(c0), cudaMemcpyHostToDevice, s));
        GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
        k_bc_init<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(d->bdepth, d->bsigma, d->npad, src);
        GSW_CUDA(cudaGetLastError());
        // forward levels (device-side stop, polled two levels behind)
        int t = 0;
        for (;; ++t) {
            for (int p = 0; p < parts; ++p) {
                if (!d->parts[p].nloc) continue;
                const BcP a = args(p, src);
                k_bc_fwd_heavy<<<g->sms * 2, kDB, 0, s>>>(a, t);
                k_bc_fwd<<<grid, kDB, 0, s>>>(a, t);
            }
            GSW_CUDA(cudaGetLastError());
            if (gsw_status e = ex_allgather(d, d->bdepth, (size_t)d->S * 4, s)) return e;
            if (gsw_status e = ex_allgather(d, d->bsigma, (size_t)d->S * 8, s)) return e;
            if (gsw_status e = ex_reduce(d, s)) return e;
            k_bc_decide<<<1, 32, 0, s>>>(d->ctl, d->recs, d->locs, parts, t);
            GSW_CUDA(cudaGetLastError());
            bool stop = false;
            if (gsw_status e = poll_done(d, t, s, &stop)) return e;
            if (stop || t + 1 >= kMaxLevels) break;
        }
        DCtl cf;
        GSW_CUDA(cudaMemcpyAsync(&cf, d->ctl, sizeof(cf), cudaMemcpyDeviceToHost, s));
        GSW_CUDA(cudaStreamSynchronize(s));
        const int L = std::max(1, cf.t);          // levels 0 .. L-1 are non-empty
        levels_total += L;
        edges_total += (long long)L * nnz_g;
        // backward levels L-2 .. 1 (the deepest level has delta = 0; the source gets no credit)
        k_bc_omega0<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(d->bdepth, d->bsigma, d->bomega, d->npad);
        for (int l = L - 2; l >= 1; --l) {
            for (int p = 0; p < parts; ++p) {
                if (!d->parts[p].nloc) continue;
                const BcP a = args(p, src);
                k_bc_bwd_heavy<<<g->sms * 2, kDB, 0, s>>>(a, l);
                k_bc_bwd<<<grid, kDB, 0, s>>>(a, l);
            }
            GSW_CUDA(cudaGetLastError());
            if (gsw_status e = ex_allgather(d, d->bomega, (size_t)d->S * 8, s)) return e;
        }
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(bc_out, bc, (size_t)out_len * 8, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = (int32_t)levels_total;
        st->gpu_ms = ms;
        st->edges_touched = edges_total;
        st->bytes_alg = (int64_t)(4ull * (unsigned long long)edges_total * 2);   // forward + backward column reads
    }
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed PageRank
gsw_status dist_pr(gsw_graph g, double damping, int32_t iters, double *rank_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (!rank_out || iters < 0 || !(damping >= 0.0 && damping <= 1.0)) { set_error("gsw_pr: bad arguments"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->mode == DM_LOOPBACK ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(rank_out) == 1;
    double *out = dev_out ? rank_out : (double *)g->scratch;
    const double invN = 1.0 / (double)d->n;
    float *C[2] = {reinterpret_cast<float *>(d->rep[0]), reinterpret_cast<float *>(d->rep[1])};
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
    GSW_CUDA(cudaMemsetAsync(C[0], 0, (size_t)d->npad * 4, s));
    const bool hub = d->crank != nullptr;          // gathers in hub order (create time)
    auto args = [&](int p, const float *cur, float *next, bool last) {
        const DPart &P = d->parts[p];
        return PrP{P.roff, hub ? reinterpret_cast<const int32_t *>(P.rcol_h) : P.rcol, P.vb, P.nloc,
                   hub ? d->crank : cur, next, last ? out + (d->mode == DM_LOOPBACK ? P.vb : 0) : nullptr,
                   P.chunks, P.nchunks, P.psum, P.loc, d->ctl, damping, invN};
    };
    auto relayout = [&](const float *c) {
        if (hub) k_hub_layout<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(c, d->horder, d->npad, d->crank);
    };
    for (int p = 0; p < parts; ++p)
        k_pr_init<<<grid_for(std::max(d->parts[p].nloc, 1), g->sms), kDB, 0, s>>>(args(p, nullptr, C[0], iters == 0));
    GSW_CUDA(cudaGetLastError());
    if (gsw_status e = ex_allgather(d, C[0], (size_t)d->S * 4, s)) return e;
    if (gsw_status e = ex_reduce(d, s)) return e;
    relayout(C[0]);
    const int grid = g->sms * 8;
    unsigned long long nnz_loc = 0;
    for (auto &P : d->parts) nnz_loc += P.nnz;
    for (int t = 0; t < iters; ++t) {
        GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
        for (int p = 0; p < parts; ++p) {
            if (!d->parts[p].nloc) continue;
            const PrP a = args(p, C[t & 1], C[(t + 1) & 1], t == iters - 1);
            k_pr_heavy<<<grid, kDB, 0, s>>>(a);
            k_pr_rows<<<grid, kDB, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        if (gsw_status e = ex_allgather(d, C[(t + 1) & 1], (size_t)d->S * 4, s)) return e;
        if (gsw_status e = ex_reduce(d, s)) return e;
        if (t + 1 < iters) relayout(C[(t + 1) & 1]);
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank_out, out, (size_t)out_len * 8, cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = iters;
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)nnz_loc * iters;
        // per iteration: 4 B per owned in-edge column + owned rows (offsets 4 B, contribution
        // write 4 B) + the fp32 all-gather (N * 4 B received); gathers of the replicated
        // contributions are L2 probes (D0) at C3 sizes
        st->bytes_alg = (int64_t)((4ull * nnz_loc + 8ull * (unsigned long long)out_len + 4ull * d->npad) * iters);
    }
    return GSW_OK;
}

// ------------------------------------------------------------------ distributed CC
gsw_status dist_cc(gsw_graph g, int32_t *label_out, gsw_run_stats *st) {
    DistState *d = g->dist;
    cudaStream_t s = g->stream;
    if (!label_out) { set_error("gsw_cc: label is NULL"); return GSW_EINVAL; }
    const int parts = (int)d->parts.size();
    const int64_t out_len = d->mode == DM_LOOPBACK ? d->n : d->parts[0].nloc;
    const bool dev_out = is_device_ptr(label_out) == 1;
    int32_t *out = dev_out ? label_out : (int32_t *)g->scratch;
    long long nnz_g = 0;
    if (gsw_status e = read_nnz_g(d, s, &nnz_g)) return e;
    DCtl c0;
    reset_ctl_host(c0, nnz_g, d->n);
    GSW_CUDA(cudaEventRecord(g->ev0, s));
    GSW_CUDA(cudaMemcpyAsync(d->ctl, &c0, sizeof(c0), cudaMemcpyHostToDevice, s));
    GSW_CUDA(cudaMemsetAsync(d->locs, 0, (size_t)kLocStride * 8 * parts, s));
    for (int p = 0; p < parts; ++p) {
        const DPart &P = d->parts[p];
        k_cc_init<<<grid_for(d->npad, g->sms), kDB, 0, s>>>(d->rep[0], p == 0 ? d->npad : 0,
                                                            reinterpret_cast<uint32_t *>(P.psum), P.nloc);
    }
    GSW_CUDA(cudaGetLastError());
    const int grid = g->sms * 8;
    unsigned long long nnz_loc = 0;
    for (auto &P : d->parts) nnz_loc += P.nnz;
    int t = 0;
    for (;; ++t) {
        const uint32_t *cur = d->rep[t & 1];
        uint32_t *next = d->rep[(t + 1) & 1];
        for (int p = 0; p < parts; ++p) {
            const DPart &P = d->parts[p];
            if (!P.nloc) continue;
            const CcP a{P.roff, P.rcol, P.vb, P.nloc, cur, next, out + (d->mode == DM_LOOPBACK ? P.vb : 0), P.chunks,
                        P.nchunks, reinterpret_cast<uint32_t *>(P.psum), P.loc, d->ctl};
            k_cc_heavy<<<grid, kDB, 0, s>>>(a);
            k_cc_rows<<<grid, kDB, 0, s>>>(a);
        }
        GSW_CUDA(cudaGetLastError());
        if (gsw_status e = ex_allgather(d, next, (size_t)d->S * 4, s)) return e;
        if (gsw_status e = ex_reduce(d, s)) return e;
        k_cc_decide<<<1, 32, 0, s>>>(d->ctl, d->locs, parts, t);
        GSW_CUDA(cudaGetLastError());
        bool stop = false;
        if (gsw_status e = poll_done(d, t, s, &stop)) return e;
        if (stop || t + 1 >= kMaxLevels) break;
    }
    GSW_CUDA(cudaEventRecord(g->ev1, s));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(label_out, out, (size_t)out_len * 4, cudaMemcpyDeviceToHost, s));
    DCtl cend;
    GSW_CUDA(cudaMemcpyAsync(&cend, d->ctl, sizeof(cend), cudaMemcpyDeviceToHost, s));
    GSW_CUDA(cudaStreamSynchronize(s));
    if (st) {
        float ms = 0.f;
        GSW_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = cend.t;                       // iterations until nothing changed
        st->gpu_ms = ms;
        st->edges_touched = (int64_t)nnz_loc * cend.t;
        st->bytes_alg = (int64_t)((4ull * nnz_loc + 12ull * (unsigned long long)out_len + 4ull * d->npad) * cend.t);
    }
    return GSW_OK;
}

size_t dist_workspace(int64_t n, int64_t nnz, int32_t nranks, int32_t nparts, int mode, bool weighted) {
    return dist_bytes(n, nnz, nranks, nparts, mode, weighted);
}

gsw_status dist_unique_id(void *id128) {
    if (!id128) { set_error("null id"); return GSW_EINVAL; }
    if (!nccl_load()) return GSW_ENCCL;
    ncclUniqueId id;
    GSW_NCCL(g_nccl.getUniqueId(&id));
    std::memcpy(id128, &id, sizeof(id));
    return GSW_OK;
}

}  // namespace gsw
