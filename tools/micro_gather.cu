// micro_gather.cu -- ceiling of the PageRank pull's dominant access on B200: random 4-byte
// gathers from an L2-resident array (C3: contributions of 4.19M vertices = 16.8 MB) driven by a
// streamed index array read from HBM (C3: 128M column indices = 513 MB), as in pr_stream.cu.
//   mode 0: stream the indices only (sum them)            -> HBM stream ceiling
//   mode 1: stream + gather x[idx] for every index        -> L2 random-gather ceiling
//   mode 2: as 1, but indices below H hit a shared-memory copy of x[0..H) (hub cache)
// Indices: uniform over [0, n) (worst case for L2 sectors) or a power law (R-MAT-like skew).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_gather tools/micro_gather.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

//   mode 3: cluster of K CTAs shares one hub cache of K*H entries: CTA r holds x[r H, (r+1) H),
//           gathers below K*H read the owner's shared memory through DSMEM
template <int EPT>
__global__ void __launch_bounds__(1024, 1) k_gather_dsmem(const int4 *__restrict__ idx4, long long m4,
                                                          const float *__restrict__ x, int H, float *out) {
    extern __shared__ float cache[];
    cg::cluster_group cl = cg::this_cluster();
    const unsigned K = cl.num_blocks(), r = cl.block_rank();
    for (int i = threadIdx.x; i < H; i += blockDim.x) cache[i] = x[r * H + i];
    cl.sync();
    float *rc[16];
    for (unsigned c = 0; c < K; ++c) rc[c] = cl.map_shared_rank(cache, c);
    const int KH = (int)K * H;
    float acc = 0.f;
    const long long T = (long long)gridDim.x * blockDim.x;
    for (long long b = blockIdx.x * (long long)blockDim.x + threadIdx.x; b < m4 / (EPT / 4); b += T) {
        int id[EPT];
#pragma unroll
        for (int h = 0; h < EPT / 4; ++h) {
            const int4 v = __ldcs(idx4 + b * (EPT / 4) + h);
            id[4 * h] = v.x; id[4 * h + 1] = v.y; id[4 * h + 2] = v.z; id[4 * h + 3] = v.w;
        }
        float g[EPT];
#pragma unroll
        for (int j = 0; j < EPT; ++j) {
            const int i = id[j];
            if (i < KH) { const unsigned o = (unsigned)i / (unsigned)H; g[j] = rc[o][i - (int)o * H]; }
            else g[j] = __ldg(x + i);
        }
#pragma unroll
        for (int j = 0; j < EPT; ++j) acc += g[j];
    }
    cl.sync();
    if (acc == 1234.5f) *out = acc;
}

template <int MODE, int EPT>
__global__ void __launch_bounds__(1024, 1) k_gather(const int4 *__restrict__ idx4, long long m4, const float *__restrict__ x,
                                                    int H, float *out) {
    extern __shared__ float cache[];
    if (MODE == 2) {
        for (int i = threadIdx.x; i < H; i += blockDim.x) cache[i] = x[i];
        __syncthreads();
    }
    float acc = 0.f;
    const long long T = (long long)gridDim.x * blockDim.x;
    for (long long b = blockIdx.x * (long long)blockDim.x + threadIdx.x; b < m4 / (EPT / 4); b += T) {
        int id[EPT];
#pragma unroll
        for (int h = 0; h < EPT / 4; ++h) {
            const int4 v = __ldcs(idx4 + b * (EPT / 4) + h);
            id[4 * h] = v.x; id[4 * h + 1] = v.y; id[4 * h + 2] = v.z; id[4 * h + 3] = v.w;
        }
        float g[EPT];
#pragma unroll
        for (int j = 0; j < EPT; ++j) {
            if (MODE == 0) g[j] = (float)id[j];
            else if (MODE == 1) g[j] = __ldg(x + id[j]);
            else g[j] = id[j] < H ? cache[id[j]] : __ldg(x + id[j]);
        }
#pragma unroll
        for (int j = 0; j < EPT; ++j) acc += g[j];
    }
    if (acc == 1234.5f) *out = acc;
}

int main() {
    const int n = 1 << 22;
    const long long m = 128ll << 20;
    std::vector<int> hu(m), hp(m);
    unsigned long long s = 88172645463325252ull;
    auto rnd = [&]() { s ^= s << 13; s ^= s >> 7; s ^= s << 17; return s; };
    for (long long i = 0; i < m; ++i) hu[i] = (int)(rnd() % n);
    // power law over degree-ordered ids: P(id < k) ~ (k/n)^0.25 (about half the mass in the top 1%)
    for (long long i = 0; i < m; ++i) {
        const double u = (double)(rnd() >> 11) / 9007199254740992.0;
        long long k = (long long)(n * u * u * u * u);
        hp[i] = (int)(k < n ? k : n - 1);
    }
    int *du, *dp;
    float *x, *out;
    cudaMalloc(&du, m * 4);
    cudaMalloc(&dp, m * 4);
    cudaMalloc(&x, n * 4);
    cudaMalloc(&out, 64);
    cudaMemcpy(du, hu.data(), m * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dp, hp.data(), m * 4, cudaMemcpyHostToDevice);
    cudaMemset(x, 0, n * 4);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int H = 28672;
    cudaFuncSetAttribute(k_gather<2, 12>, cudaFuncAttributeMaxDynamicSharedMemorySize, H * 4);
    cudaFuncSetAttribute(k_gather<2, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, H * 4);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int dist = 0; dist < 2; ++dist) {
        const int4 *idx = reinterpret_cast<const int4 *>(dist ? dp : du);
        for (int mode = 0; mode < 3; ++mode) {
            for (int ept : {12, 16}) {
                float best = 1e9f;
                for (int rep = 0; rep < 5; ++rep) {
                    cudaEventRecord(e0);
                    const long long m4 = m / 4;
                    if (ept == 12) {
                        if (mode == 0) k_gather<0, 12><<<sms, 1024>>>(idx, m4 - m4 % 3, x, H, out);
                        if (mode == 1) k_gather<1, 12><<<sms, 1024>>>(idx, m4 - m4 % 3, x, H, out);
                        if (mode == 2) k_gather<2, 12><<<sms, 1024, H * 4>>>(idx, m4 - m4 % 3, x, H, out);
                    } else {
                        if (mode == 0) k_gather<0, 16><<<sms, 1024>>>(idx, m4, x, H, out);
                        if (mode == 1) k_gather<1, 16><<<sms, 1024>>>(idx, m4, x, H, out);
                        if (mode == 2) k_gather<2, 16><<<sms, 1024, H * 4>>>(idx, m4, x, H, out);
                    }
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms;
                    cudaEventElapsedTime(&ms, e0, e1);
                    best = ms < best ? ms : best;
                }
                printf("%s mode=%d (%s) ept=%d: %.1f us  %.1f G idx/s  stream %.0f GB/s  err=%s\n",
                       dist ? "powerlaw" : "uniform ", mode,
                       mode == 0 ? "stream only" : mode == 1 ? "stream+gather" : "stream+gather, smem hub cache", ept,
                       best * 1e3, m / (best * 1e6), m * 4.0 / (best * 1e6), cudaGetErrorString(cudaGetLastError()));
            }
        }
    }
    // mode 3: DSMEM-shared hub cache over clusters of 2 and 4 (power-law indices)
    cudaFuncSetAttribute(k_gather_dsmem<12>, cudaFuncAttributeMaxDynamicSharedMemorySize, H * 4);
    for (int K : {1, 2, 4}) {
        const int4 *idx = reinterpret_cast<const int4 *>(dp);
        const long long m4 = m / 4 - (m / 4) % 3;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(sms - sms % K);
        cfg.blockDim = dim3(1024);
        cfg.dynamicSmemBytes = H * 4;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = K; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        int ncl = 0;
        cudaOccupancyMaxActiveClusters(&ncl, k_gather_dsmem<12>, &cfg);
        if (ncl * K < (int)cfg.gridDim.x) cfg.gridDim = dim3(ncl * K);
        float best = 1e9f;
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(e0);
            cudaLaunchKernelEx(&cfg, k_gather_dsmem<12>, idx, m4, (const float *)x, H, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = ms < best ? ms : best;
        }
        printf("powerlaw mode=3 (DSMEM hub cache, cluster %d = %d entries, grid %u) ept=12: %.1f us  %.1f G idx/s  err=%s\n",
               K, K * H, cfg.gridDim.x, best * 1e3, m / (best * 1e6), cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
