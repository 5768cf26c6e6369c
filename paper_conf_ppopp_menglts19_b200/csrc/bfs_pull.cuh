// bfs_pull.cuh -- the B200 list pull of BFS (the THREAD candidate on the bitmap format, P:374-393
// "edge skipping" Fig. 2), shared by the single-GPU persistent kernel (bfs.cu) and the
// partitioned per-level kernels (dist.cu, where V / depth / nfb are the rank's owned slice and
// the in-neighbour ids are global).
#pragma once
#include "common.cuh"

namespace gsw {

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
#ifndef GSW_PULL_CUR
#define GSW_PULL_CUR 4
#endif
#ifndef GSW_PULL_BATCH
#define GSW_PULL_BATCH 8
#endif
constexpr int kPullCur = GSW_PULL_CUR;       // pass-2 cursors per lane
// Chunk hand-out: each CTA owns the chunks blockIdx.x, blockIdx.x + gridDim.x, ... (so every CTA
// sees every region of the degree-ordered id range) and its warps take them one at a time from a
// shared-memory counter.  Measured per warp (GSW_PULL_PROF, profiles/r2/pull_warp_profile_c3.txt):
// with the static warp-strided hand-out C3's widest pull level took 51-56 us while the median warp
// finished in 23 us -- the level's time was its slowest warps.  GSW_PULL_DYN=0: static hand-out.
#ifndef GSW_PULL_DYN
#define GSW_PULL_DYN 1
#endif
constexpr int kPullBatch = GSW_PULL_BATCH;   // pass-1 words probed per batch (loads in flight per lane)
constexpr int kPullWordsPerWarp = 16;
constexpr int kPullList = kPullWordsPerWarp * 32;
// GSW_PULL_BOUNDS=1: pass 1 also loads the row bounds of every probed vertex (coalesced, in the
// same batch as in_first), so a hit's degree needs no later round trip (A/B build knob)
#ifndef GSW_PULL_BOUNDS
#define GSW_PULL_BOUNDS 0
#endif
static __device__ __noinline__ LocalCnt bfs_pull_list(const unsigned *__restrict__ fb, unsigned *__restrict__ V,
                                               int *__restrict__ depth, const uint32_t *__restrict__ in_off,
                                               const int32_t *__restrict__ in_col, const int32_t *__restrict__ in_first,
                                               const uint32_t *__restrict__ out_off, bool symmetric, int lvl,
                                               unsigned *__restrict__ nfb, int n, int *lists) {
    LocalCnt cnt;
    const int W = (n + 31) >> 5;
    const unsigned lane = lane_id();
    int *list = lists + (threadIdx.x >> 5) * (kPullList + kPullWordsPerWarp);
    unsigned *found_bits = reinterpret_cast<unsigned *>(list + kPullList);
#if GSW_PULL_DYN
    __shared__ unsigned s_next;
    __syncthreads();
    if (threadIdx.x == 0) s_next = 0u;
    __syncthreads();
    for (;;) {
        unsigned k = 0;
        if (lane == 0) k = atomicAdd(&s_next, 1u);
        k = __shfl_sync(0xffffffffu, k, 0);
        const long long chunk = blockIdx.x + (long long)k * gridDim.x;
        if (chunk * kPullWordsPerWarp >= W) break;
#else
    for (long long chunk = gwarp(); chunk * kPullWordsPerWarp < W; chunk += gwarps()) {
#endif
        const long long w0 = chunk * kPullWordsPerWarp;
        unsigned word = 0, orig = ~0u;
        if (lane < (unsigned)kPullWordsPerWarp && w0 + lane < W) {
            orig = V[w0 + lane];
            word = ~orig;                                   // padding bits are set in V
            found_bits[lane] = 0u;
        }
        __syncwarp();                                       // found_bits reset before lane 0's stores
        // pass 1: probe the first in-neighbour (the highest-degree one) of every unvisited vertex,
        // coalesced through in_first, 8 words in flight (one load + one probe per vertex: the row
        // bounds are not needed yet).  Hits go to the top of the list (their degrees are loaded
        // in one batch afterwards), misses to the bottom (pass 2 scans them from their 2nd edge).
        unsigned total = 0, nhit = 0;                        // warp-uniform list lengths
        unsigned nz = __ballot_sync(0xffffffffu, word != 0u);  // words with unvisited vertices
#pragma unroll 1
        while (nz) {
            int y[kPullBatch], kk[kPullBatch];
#if GSW_PULL_BOUNDS
            uint32_t hb[kPullBatch], he[kPullBatch];
            const uint32_t *o = symmetric ? in_off : out_off;
#endif
#pragma unroll
            for (int j = 0; j < kPullBatch; ++j) {
                kk[j] = nz ? __ffs(nz) - 1 : -1;              // warp-uniform
                nz &= nz - 1u;
            }
#pragma unroll
            for (int j = 0; j < kPullBatch; ++j) {
                const unsigned wm = __shfl_sync(0xffffffffu, word, kk[j] < 0 ? 0 : kk[j]);
                const bool act = kk[j] >= 0 && ((wm >> lane) & 1u);   // padding bits are set in V: v < n
                y[j] = act ? __ldg(in_first + (int)((w0 + kk[j]) * 32 + lane)) : -2;
#if GSW_PULL_BOUNDS
                const int vv = (int)((w0 + kk[j]) * 32 + lane);
                hb[j] = act ? __ldg(o + vv) : 0u;
                he[j] = act ? __ldg(o + vv + 1) : 0u;
#endif
            }
            unsigned p[kPullBatch];
#pragma unroll
            for (int j = 0; j < kPullBatch; ++j) p[j] = y[j] >= 0 ? fb[y[j] >> 5] : 0u;
#pragma unroll
            for (int j = 0; j < kPullBatch; ++j) {
                const int v = (int)((w0 + kk[j]) * 32 + lane);
                const bool hit = y[j] >= 0 && ((p[j] >> (y[j] & 31)) & 1u);
                if (y[j] >= 0) cnt.edges++;
                if (hit) depth[v] = lvl + 1;
                const unsigned hm = __ballot_sync(0xffffffffu, hit);
                if (lane == 0 && kk[j] >= 0) found_bits[kk[j]] = hm;
#if GSW_PULL_BOUNDS
                if (hit) cnt.add_vertex(he[j] - hb[j]);
#else
                if (hit) list[kPullList - 1 - (nhit + __popc(hm & lanemask_lt()))] = v;
                nhit += __popc(hm);
#endif
                const bool miss = y[j] >= 0 && !hit;
                const unsigned mm = __ballot_sync(0xffffffffu, miss);
                if (miss) list[total + __popc(mm & lanemask_lt())] = v;
                total += __popc(mm);
            }
        }
        __syncwarp();
        // degrees of the hits (Table 1 Ea of the next active set), 8 rows in flight per lane
        for (unsigned i0 = lane; i0 < nhit; i0 += 32 * 8) {
            int hv[8];
            uint32_t hb[8], he[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) hv[j] = i0 + 32 * j < nhit ? list[kPullList - 1 - (i0 + 32 * j)] : -1;
            const uint32_t *o = symmetric ? in_off : out_off;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                hb[j] = hv[j] >= 0 ? __ldg(o + hv[j]) : 0u;
                he[j] = hv[j] >= 0 ? __ldg(o + hv[j] + 1) : 0u;
            }
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (hv[j] >= 0) cnt.add_vertex(he[j] - hb[j]);
        }
        // pass 2: cursors over the misses, from their second edge, two edges per step (both
        // columns of a step usually share a sector; the probes are independent)
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
            int y0[kPullCur], y1[kPullCur];
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) {
                const bool a0 = v[j] >= 0 && e[j] < end[j], a1 = v[j] >= 0 && e[j] + 1 < end[j];
                y0[j] = a0 ? __ldg(in_col + e[j]) : -1;
                y1[j] = a1 ? __ldg(in_col + e[j] + 1) : -1;
            }
            unsigned p0[kPullCur], p1[kPullCur];
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) {
                p0[j] = y0[j] >= 0 ? fb[y0[j] >> 5] : 0u;
                p1[j] = y1[j] >= 0 ? fb[y1[j] >> 5] : 0u;
            }
            int nv[kPullCur];
#pragma unroll
            for (int j = 0; j < kPullCur; ++j) {
                nv[j] = v[j];
                if (v[j] < 0) continue;
                bool done = false;
                if (y0[j] >= 0) {
                    cnt.edges += y1[j] >= 0 ? 2 : 1;
                    if (((p0[j] >> (y0[j] & 31)) & 1u) || (y1[j] >= 0 && ((p1[j] >> (y1[j] & 31)) & 1u))) {
                        const int x = v[j];
                        depth[x] = lvl + 1;
                        atomicOr(found_bits + ((x >> 5) - w0), 1u << (x & 31));   // shared memory
                        cnt.add_vertex(symmetric ? end[j] - beg[j] : __ldg(out_off + x + 1) - __ldg(out_off + x));
                        done = true;
                    } else if ((e[j] += 2) >= end[j]) {
                        done = true;
                    }
                } else {
                    done = true;                     // single-edge row (its only edge missed in pass 1)
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

}  // namespace gsw
