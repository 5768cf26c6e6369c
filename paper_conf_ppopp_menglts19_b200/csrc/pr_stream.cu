// pr_stream.cu -- PageRank pull as an edge-tiled stream: the STRICT (equal-edges-per-tile, merge-
// path lineage) load-balance candidate of PR's Expand, designed for B200.
//
// Same iteration as pr.cu (reading R7 / SURVEY Q9):
//   pr_{t+1}(v) = (1-d)/N + d * ( sum_{u in N_in(v)} pr_t(u)/deg_out(u) + D_t/N ),  D_t = dangling mass
// with every vertex and edge active.  Differences from pr.cu, all aimed at the HBM/L2
// roofline of a whole-graph gather:
//   * one 1024-thread CTA per SM; the in-edge array is cut into tiles of kTile edges (8 per
//     thread); tiles are dealt round-robin to CTAs, so work is equal by construction (hub rows
//     span many tiles, short rows share a tile);
//   * the column indices of the next warp-tile are prefetched into registers (streaming 16-byte
//     loads, ld.global.cs) while the current one is reduced, together with the first 32 row
//     offsets and the tile geometry; the remaining row offsets of a tile are staged in a per-warp
//     shared-memory buffer (plain loads -- an earlier plan for a TMA bulk copy was not kept);
//   * contributions pr_t(u)/deg_out(u) are stored as fp32 (accumulation stays fp64); the first K
//     of them -- the highest-degree vertices after graph.cu's degree-ordered relabeling, ~55% of
//     all gathers on R-MAT -- are cached in shared memory for the whole iteration, the rest are
//     gathered through L1/L2;
//   * each thread walks its 8 consecutive edges serially; rows that end inside a thread are
//     finished in place, rows crossing thread boundaries are combined by a CTA-wide segmented
//     scan of the per-thread carries, rows crossing tile boundaries by fp64 atomics that the tile
//     holding the row's last edge finishes after a grid barrier (phase B);
//   * rows without in-edges (the isolated tail after relabeling) are finished from a list.
#include "engine.cuh"
#include "internal.h"
#include "launch.h"

#include <cstdlib>

namespace gsw {

constexpr int kSBlock = 1024;
constexpr int kSWarps = kSBlock / 32;
#ifndef GSW_PR_EPT
#define GSW_PR_EPT 12      // 8: C3 2,648 it/s, 12: 2,812, 16: 2,783 (profiles/r2/pr_ept_cc_jump_ab.txt)
#endif
constexpr int kEpt = GSW_PR_EPT;              // edges per lane per warp-tile (A/B knob: GSW_PR_EPT)
constexpr int kWt = 32 * kEpt;                // edges per warp-tile
constexpr int kWBuf = 320;                    // row offsets a warp keeps in shared memory per tile

struct PrsArgs {
    DevGraph g;
    bool sym;                 // CSC == CSR: in-degree == out-degree
    double damping;
    int iters;
    int K;                    // contributions cached in shared memory
    double *out;              // final ranks, caller order
    float *contrib[2];        // pr/deg_out (0 for dangling), double buffered
    double *sum;              // fp64 accumulator of tile-crossing rows (zero between iterations)
    double *dsum;             // dangling mass D_t, iters+1 entries
    uint32_t *wt_row;         // nwt+1: row holding the first edge of each warp-tile (+ row of the last edge)
    int *empty;               // rows without in-edges
    unsigned *nempty;
    unsigned nwt;
    RunCommon rc;
};

// predicated global load (0 when !pred): no branch, so the compiler keeps all gathers in flight
__device__ __forceinline__ float ld_pred_f32(const float *p, bool pred) {
    float v = 0.f;
    asm("{\n .reg .pred q;\n setp.ne.u32 q, %2, 0;\n @q ld.global.f32 %0, [%1];\n}" : "+f"(v) : "l"(p), "r"((unsigned)pred));
    return v;
}

__device__ __forceinline__ int4 ld_stream4(const int4 *p) {
    int4 v;
    asm volatile("ld.global.cs.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

struct PrsEpi {
    const uint32_t *off;      // out-CSR offsets (out-degree)
    const uint32_t *perm;
    double *out;
    float *cnext;
    double base, d;
    bool last;
    __device__ __forceinline__ void finish(int v, double s, uint32_t dg, double &dang) const {
        const double p = base + d * s;
        if (last) out[perm ? perm[v] : v] = p;
        cnext[v] = dg ? (float)p * __frcp_rn((float)dg) : 0.f;   // fp32 store; no fp64 divide slow-path call
        if (!dg) dang += p;
    }
    __device__ __forceinline__ uint32_t deg_out(int v) const { return __ldg(off + v + 1) - __ldg(off + v); }
};

__device__ __forceinline__ double block_sum_1024(double v, double *sh) {
    v = warp_sum(v);
    __syncthreads();
    if (lane_id() == 0) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    double s = lane_id() < (unsigned)kSWarps ? sh[lane_id()] : 0.0;
    return warp_sum(s);
}

__device__ __forceinline__ void load_cols(const int32_t *in_col, uint32_t e0, uint32_t nnz, int (&c)[kEpt]) {
    if (e0 + kEpt <= nnz) {
#pragma unroll
        for (int h = 0; h < kEpt / 4; ++h) {
            const int4 x = ld_stream4(reinterpret_cast<const int4 *>(in_col + e0 + 4 * h));
            c[4 * h] = x.x; c[4 * h + 1] = x.y; c[4 * h + 2] = x.z; c[4 * h + 3] = x.w;
        }
    } else {
#pragma unroll
        for (int j = 0; j < kEpt; ++j) c[j] = e0 + j < nnz ? __ldg(in_col + e0 + j) : 0;
    }
}

__global__ void __launch_bounds__(kSBlock, 1) pr_stream_kernel(PrsArgs a) {
    extern __shared__ __align__(16) unsigned char dyn[];
    float *cache = reinterpret_cast<float *>(dyn);
    __shared__ uint32_t wbuf[kSWarps][kWBuf];
    __shared__ double shsum[kSWarps];

    const RunCommon &rc = a.rc;
    const GridBarrier bar = make_bar(rc);
    unsigned epoch = 0;
    const int n = a.g.n;
    const uint32_t nnz = a.g.nnz;
    const double N = (double)n, d = a.damping;
    const uint32_t *in_off = a.g.in_off;
    const int32_t *in_col = a.g.in_col;
    const unsigned tid = threadIdx.x, lane = lane_id(), wid = tid >> 5;
    uint32_t *const sb = wbuf[wid];

    // ---- init: pr_0 = 1/N -> contrib_0 (fp32), D_0; warp-tile table; rows without in-edges
    double dang = 0.0;
    for (long long v = gtid(); v < n; v += gthreads()) {
        const uint32_t dg = __ldg(a.g.off + v + 1) - __ldg(a.g.off + v);
        a.contrib[0][v] = dg ? (float)(1.0 / N) * __frcp_rn((float)dg) : 0.f;
        a.sum[v] = 0.0;
        if (!dg) dang += 1.0 / N;
        if (a.iters == 0) a.out[v] = 1.0 / N;
    }
    // rows without in-edges: one atomic per 1024-vertex chunk
    for (long long c0 = (long long)blockIdx.x * kSBlock; c0 < n; c0 += (long long)gridDim.x * kSBlock) {
        const long long v = c0 + tid;
        const bool e = v < n && __ldg(in_off + v + 1) == __ldg(in_off + v);
        const unsigned m = __ballot_sync(0xffffffffu, e);
        __shared__ unsigned wcnt[kSWarps], cbase;
        if (lane == 0) wcnt[wid] = __popc(m);
        __syncthreads();
        if (tid == 0) {
            unsigned s = 0;
            for (int i = 0; i < kSWarps; ++i) { const unsigned c = wcnt[i]; wcnt[i] = s; s += c; }
            cbase = s ? atomicAdd(a.nempty, s) : 0u;
        }
        __syncthreads();
        if (e) a.empty[cbase + wcnt[wid] + __popc(m & lanemask_lt())] = (int)v;
        __syncthreads();
    }
    for (long long i = gtid(); i <= a.iters; i += gthreads()) a.dsum[i] = 0.0;
    // wt_row[q] = last row r with in_off[r] <= q*kWt (a non-empty row); wt_row[nwt] = row of edge nnz-1
    for (long long q = gtid(); q <= (long long)a.nwt; q += gthreads()) {
        const uint32_t x = q < a.nwt ? (uint32_t)q * kWt : nnz - 1;
        int lo = 0, hi = n - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (__ldg(in_off + mid) <= x) lo = mid; else hi = mid - 1;
        }
        a.wt_row[q] = (uint32_t)lo;
    }
    grid_sync(bar, epoch);
    {
        const double s = block_sum_1024(dang, shsum);
        if (tid == 0 && s != 0.0) atomicAdd(a.dsum, s);
    }
    grid_sync(bar, epoch);
    const unsigned nempty = *(volatile const unsigned *)a.nempty;
    const int K = a.K;
    const unsigned NW = gridDim.x * kSWarps;
    const unsigned w0 = blockIdx.x * kSWarps + wid;          // this warp's first warp-tile

    Book book;
    Features f = rc.base;
    f.Va = n; f.Ea = (long long)nnz; f.Via = 0; f.Eia = 0;
    f.maxd = 0; f.mind = 0;
    const DevCfg cfg{GSW_PULL, GSW_BITMAP, GSW_LB_STRICT, GSW_STEP_REMAIN, GSW_FUSED};
    int t = 0;
    for (; t < a.iters; ++t) {
        if (is_book()) {
            book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
            if (t > 0) {
                book.bytes += 4ull * nnz + 12ull * n;
                book.edges += nnz;
                if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)nnz;
            }
        }
        f.iter = t;
        write_record(rc, t, cfg, f, 0u);
        __shared__ double sD;
        if (tid == 0) sD = *(volatile const double *)(a.dsum + t);
        if (is_book()) book_expand(book);
        double dloc = 0.0;
        const float *cur = a.contrib[t & 1];
        // hub cache: contributions of vertices [0, K)
        for (int k = tid * 4; k < K; k += kSBlock * 4) {
            if (k + 4 <= K) *reinterpret_cast<float4 *>(cache + k) = *reinterpret_cast<const float4 *>(cur + k);
            else for (int j = k; j < K; ++j) cache[j] = cur[j];
        }
        __syncthreads();
        // epilogue parameters live in shared memory / the parameter bank, not in registers
        __shared__ double sbase;
        if (tid == 0) sbase = (1.0 - d) / N + d * sD / N;
        __syncthreads();
        const bool last = t == a.iters - 1;
        float *const cnext = a.contrib[(t + 1) & 1];
        auto finish = [&](int v, double s, uint32_t dg) {
            const double p = sbase + a.damping * s;
            if (last) a.out[a.g.perm ? a.g.perm[v] : v] = p;
            cnext[v] = dg ? (float)p * __frcp_rn((float)dg) : 0.f;   // fp32 store; no fp64 divide slow-path call
            if (!dg) dloc += p;
        };
        auto deg_out = [&](int v) -> uint32_t { return __ldg(a.g.off + v + 1) - __ldg(a.g.off + v); };

        // ---- phase A: every warp runs its own warp-tiles w0, w0+NW, ... (no CTA barriers); the
        // next tile's columns, first 32 row offsets and geometry are prefetched one tile ahead
        unsigned q = w0;
        int cols[kEpt];
        uint32_t lo = 0, hi = 0, pre_off = 0;
        if (q < a.nwt) {
            load_cols(in_col, q * kWt + lane * kEpt, nnz, cols);
            lo = a.wt_row[q]; hi = a.wt_row[q + 1];
            pre_off = lo + lane <= hi + 1 ? __ldg(in_off + lo + lane) : 0u;
        }
        for (; q < a.nwt; q += NW) {
            // gathers of this tile: all global loads back to back (predicated), then the cache hits
            float val[kEpt];
#pragma unroll
            for (int j = 0; j < kEpt; ++j) val[j] = ld_pred_f32(cur + cols[j], cols[j] >= K);
#pragma unroll
            for (int j = 0; j < kEpt; ++j) {
                const float c = cache[cols[j] < K ? cols[j] : 0];
                if (cols[j] < K) val[j] = c;
            }
            // prefetch the next tile
            const unsigned qn = q + NW;
            uint32_t nlo = 0, nhi = 0;
            if (qn < a.nwt) {
                load_cols(in_col, qn * kWt + lane * kEpt, nnz, cols);
                nlo = a.wt_row[qn]; nhi = a.wt_row[qn + 1];
            }
            const uint32_t ts = q * (uint32_t)kWt, te = min(ts + (uint32_t)kWt, nnz);
            if (lo == hi) {
                // the whole tile lies in row lo (hub rows): a warp sum, no row walk
                const uint32_t e0 = ts + lane * kEpt;
                double acc = 0.0;
#pragma unroll
                for (int j = 0; j < kEpt; ++j) acc += e0 + j < te ? (double)val[j] : 0.0;
                acc = warp_sum(acc);
                const uint32_t rb = __shfl_sync(0xffffffffu, pre_off, 0), re = __shfl_sync(0xffffffffu, pre_off, 1);
                if (lane == 0) {
                    if (rb < ts || re > te) atomicAdd(a.sum + lo, acc);      // finished in phase B
                    else finish((int)lo, acc, a.sym ? re - rb : deg_out((int)lo));
                }
                lo = nlo; hi = nhi;
                if (qn < a.nwt) pre_off = lo + lane <= hi + 1 ? __ldg(in_off + lo + lane) : 0u;
                continue;
            }
            // row offsets of this tile (rows lo .. hi+1) into the warp's buffer
            const unsigned cnt = hi - lo + 2;
            const uint32_t *so;
            __syncwarp();
            if (cnt <= (unsigned)kWBuf) {
                sb[lane] = pre_off;
                for (unsigned i = 32 + lane; i < cnt; i += 32) sb[i] = __ldg(in_off + lo + i);
                so = sb;
            } else {
                so = in_off + lo;
            }
            __syncwarp();
            const uint32_t e0 = ts + lane * kEpt;
            const int m = e0 < te ? (int)min((uint32_t)kEpt, te - e0) : 0;
            int ckey = -2 - (int)lane;           // carry key (global row) or a unique breaker
            double cval = 0.0;
            int fin_row = -1;
            double fin_val = 0.0;
            if (m > 0) {
                int blo = 0, bhi = (int)cnt - 2;
                while (blo < bhi) {
                    const int mid = (blo + bhi + 1) >> 1;
                    if (so[mid] <= e0) blo = mid; else bhi = mid - 1;
                }
                int ri = blo;
                uint32_t rb = so[ri], re = so[ri + 1];
                bool first = true, have = false;
                double acc = 0.0;
#pragma unroll
                for (int j = 0; j < kEpt; ++j) {
                    if (j < m) {
                        const uint32_t e = e0 + j;
                        while (e >= re) {
                            if (have) {
                                const int r = (int)lo + ri;
                                if (first && rb < e0) { fin_row = r; fin_val = acc; }
                                else finish(r, acc, a.sym ? re - rb : deg_out(r));
                            }
                            first = false; have = false; acc = 0.0;
                            ++ri; rb = re; re = so[ri + 1];
                        }
                        acc += (double)val[j];
                        have = true;
                    }
                }
                const int r = (int)lo + ri;
                if (re > e0 + (uint32_t)m) { ckey = r; cval = acc; }      // continues past this lane
                else if (first && rb < e0) { fin_row = r; fin_val = acc; }
                else finish(r, acc, a.sym ? re - rb : deg_out(r));
            }
            // warp segmented inclusive scan of the carries (keys form contiguous runs)
            double sv = cval;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double ov = __shfl_up_sync(0xffffffffu, sv, o);
                const int ok = __shfl_up_sync(0xffffffffu, ckey, o);
                if (lane >= (unsigned)o && ok == ckey) sv += ov;
            }
            const double prev_v = __shfl_up_sync(0xffffffffu, sv, 1);
            int prev_k = __shfl_up_sync(0xffffffffu, ckey, 1);     // every lane must take part
            if (lane == 0) prev_k = -1;
            if (fin_row >= 0) {
                const double tot = fin_val + (prev_k == fin_row ? prev_v : 0.0);
                if (fin_row == (int)lo && so[0] < ts) atomicAdd(a.sum + fin_row, tot);   // started in an earlier tile
                else finish(fin_row, tot, a.sym ? so[fin_row - lo + 1] - so[fin_row - lo] : deg_out(fin_row));
            }
            if (lane == 31 && ckey >= 0) atomicAdd(a.sum + ckey, sv);     // continues into a later tile
            // next tile's first 32 row offsets
            lo = nlo; hi = nhi;
            if (qn < a.nwt) pre_off = lo + lane <= hi + 1 ? __ldg(in_off + lo + lane) : 0u;
        }
        // rows without in-edges
        for (long long i = gtid(); i < nempty; i += gthreads()) {
            const int v = a.empty[i];
            finish(v, 0.0, deg_out(v));
        }
        grid_sync(bar, epoch);
        // ---- phase B: the warp-tile holding the last edge of a tile-crossing row finishes it
        for (long long qq = gtid(); qq < a.nwt; qq += gthreads()) {
            const uint32_t r = a.wt_row[qq];
            const uint32_t qs = (uint32_t)qq * kWt;
            const uint32_t rb = __ldg(in_off + r), re = __ldg(in_off + r + 1);
            if (rb < qs && re <= qs + (uint32_t)kWt) {
                const double s = a.sum[r];
                a.sum[r] = 0.0;
                finish((int)r, s, a.sym ? re - rb : deg_out((int)r));
            }
        }
        {
            const double s = block_sum_1024(dloc, shsum);
            if (tid == 0 && s != 0.0) atomicAdd(a.dsum + t + 1, s);
        }
        grid_sync(bar, epoch);
    }
    if (is_book()) {
        if (t > 0) {
            book.bytes += 4ull * nnz + 12ull * n + 12ull * n;     // last iteration + caller-order output
            book.edges += nnz;
            if (t - 1 < kMaxHist) rc.rec[t - 1].edges = (long long)nnz;
        }
        book_start(book, rc, t, rc.cnt + ((t + 1) % 3));
        book_finish(book, rc, t);
    }
}

// K: contributions cached per CTA, from the opt-in shared memory per block
static int stream_cache_entries(gsw_graph g, size_t *smem_bytes) {
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, g->device);
    const size_t static_bytes = sizeof(uint32_t) * kSWarps * kWBuf + 2048;   // warp buffers, scratch
    long long avail = (long long)optin - (long long)static_bytes - 16;
    // Cache size (profiles/r2/pr_cache_sweep.txt, tools/pr_ab.py): every shared-memory byte the hub
    // cache takes is an L1 byte the gathers lose (one CTA per SM; the carveout steps 132 / 164 /
    // 196 / 228 KB), and the whole opt-in size (~46K entries, L1 ~28 KB) was the worst choice:
    // C3 11.5 ms vs 7.6 ms at 28,672 entries (2,629 it/s), C4 19.3 vs 12.4 ms, C1 0.43 vs 0.37 ms.
    // Graphs whose contributions overflow L2 (C5) want a smaller cache still: 12,288 entries
    // 166 ms vs 179 ms at 28,672 (and 402 ms at the maximum).
    int l2 = 0;
    if (cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g->device) != cudaSuccess) { cudaGetLastError(); l2 = 0; }
    const long long want = (l2 > 0 && (double)g->g.n * 4.0 > 0.5 * (double)l2) ? 12288 : 28672;
    long long K = std::min<long long>(want, avail > 0 ? (avail / 16) * 4 : 0);
    K = std::min<long long>(K, ((long long)g->g.n / 4) * 4);
    if (const char *e = getenv("GSW_PR_CACHE")) K = std::min<long long>(K, (atoll(e) / 4) * 4);   // tests
    if (K < 0) K = 0;
    *smem_bytes = (size_t)(K + 4) * 4;
    return (int)K;
}

gsw_status run_pr_stream(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *st) {
    const int n = g->g.n;
    Workspace ws{g->scratch, g->scratch_bytes, 0};
    const bool dev_out = is_device_ptr(rank) == 1;
    PrsArgs a{};
    a.g = g->g;
    a.sym = g->symmetric;
    a.damping = damping;
    a.iters = iters;
    a.nwt = (unsigned)(((uint64_t)g->g.nnz + kWt - 1) / kWt);
    a.out = dev_out ? rank : (double *)ws.take((size_t)n * 8);
    a.contrib[0] = (float *)ws.take((size_t)n * 4 + 16);
    a.contrib[1] = (float *)ws.take((size_t)n * 4 + 16);
    a.sum = (double *)ws.take((size_t)n * 8);
    a.dsum = (double *)ws.take((size_t)(iters + 1) * 8);
    a.wt_row = (uint32_t *)ws.take(((size_t)a.nwt + 2) * 4);
    a.empty = (int *)ws.take((size_t)n * 4 + 4);
    a.nempty = (unsigned *)ws.take(256);
    size_t smem = 0;
    a.K = stream_cache_entries(g, &smem);
    // control blocks (grid = one CTA per SM)
    RunCommon &rc = a.rc;
    rc.ctl = (Ctl *)ws.take(sizeof(Ctl));
    rc.cnt = (IterCnt *)ws.take(3 * sizeof(IterCnt));
    rc.hist = (Hist *)ws.take(sizeof(Hist) * kMaxHist);
    rc.rec = (gsw_iter_record *)ws.take(sizeof(gsw_iter_record) * kMaxHist);
    rc.partial = (uint32_t *)ws.take(sizeof(uint32_t) * (g->sms + 1));
    if (!a.out || !a.contrib[1] || !a.sum || !a.dsum || !a.wt_row || !a.empty || !a.nempty || !rc.ctl ||
        !rc.cnt || !rc.hist || !rc.rec || !rc.partial) {
        set_error("workspace too small");
        return GSW_ENOMEM;
    }
    rc.force = g->forced;
    const Attrs &A = g->attrs;
    Features f{};
    f.N = (float)A.N; f.M = (float)A.M; f.dbar = (float)A.dbar; f.sd = (float)A.sd; f.rd = (float)A.rd;
    f.gini = (float)A.gini; f.her = (float)A.her;
    rc.base = f;
    GSW_CUDA(cudaEventRecord(g->ev0, g->stream));   // device time of the call starts with its resets
    GSW_CUDA(cudaMemsetAsync(rc.ctl, 0, sizeof(Ctl), g->stream));
    GSW_CUDA(cudaMemsetAsync(a.nempty, 0, 4, g->stream));
    GSW_CUDA(cudaFuncSetAttribute((const void *)pr_stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)smem));
    int nb = 0;
    GSW_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void *)pr_stream_kernel, kSBlock, smem));
    if (nb < 1) { set_error("pr_stream_kernel does not fit on an SM"); return GSW_ECUDA; }
    void *args[] = {&a};
    GSW_CUDA(cudaLaunchCooperativeKernel((const void *)pr_stream_kernel, dim3(g->sms), dim3(kSBlock), args, smem,
                                         g->stream));
    GSW_CUDA(cudaEventRecord(g->ev1, g->stream));
    if (!dev_out) GSW_CUDA(cudaMemcpyAsync(rank, a.out, (size_t)n * 8, cudaMemcpyDeviceToHost, g->stream));
    LaunchInfo li;
    li.grid = g->sms;
    return finish_run(g, a.rc, li, st);
}

}  // namespace gsw
