// micro_cluster_coop.cu -- can a cooperative (co-resident, grid-barrier) persistent kernel also be
// a thread-block-cluster launch on B200, and what do a cluster barrier and a software grid
// barrier cost inside it?  Standalone probe for the cluster tier idea.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_cluster_coop tools/micro_cluster_coop.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__global__ void k_probe(unsigned *ctr, int iters, int mode, unsigned long long *out) {
    cg::cluster_group cl = cg::this_cluster();
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        if (mode == 0) {
            cl.sync();                                   // barrier.cluster
        } else {
            __syncthreads();                             // flip-bit software grid barrier
            if (threadIdx.x == 0) {
                const unsigned add = blockIdx.x == 0 ? 0x80000000u - (gridDim.x - 1u) : 1u;
                __threadfence();
                const unsigned old = atomicAdd(ctr, add);
                volatile unsigned *p = ctr;
                while (((old ^ *p) & 0x80000000u) == 0u) {}
                __threadfence();
            }
            __syncthreads();
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[mode] = clock64() - t0;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned *ctr;
    unsigned long long *out;
    cudaMalloc(&ctr, 256);
    cudaMalloc(&out, 64);
    for (int per_sm : {1, 2}) {
        for (int csize : {2, 4, 8}) {
            const int grid = sms * per_sm;
            if (grid % csize) { printf("grid %d not divisible by cluster %d\n", grid, csize); continue; }
            for (int mode = 0; mode < 2; ++mode) {
                cudaMemset(ctr, 0, 256);
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(grid);
                cfg.blockDim = dim3(256);
                cudaLaunchAttribute at[2];
                at[0].id = cudaLaunchAttributeCooperative;
                at[0].val.cooperative = 1;
                at[1].id = cudaLaunchAttributeClusterDimension;
                at[1].val.clusterDim.x = csize; at[1].val.clusterDim.y = 1; at[1].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 2;
                int iters = 20000;
                cudaEvent_t e0, e1;
                cudaEventCreate(&e0); cudaEventCreate(&e1);
                cudaEventRecord(e0);
                cudaError_t err = cudaLaunchKernelEx(&cfg, k_probe, ctr, iters, mode, out);
                cudaEventRecord(e1);
                cudaError_t e2 = cudaDeviceSynchronize();
                float ms = 0;
                cudaEventElapsedTime(&ms, e0, e1);
                printf("per_sm=%d cluster=%d %s: launch=%s sync=%s  %.3f us/barrier\n", per_sm, csize,
                       mode == 0 ? "cluster.sync" : "grid barrier", cudaGetErrorString(err), cudaGetErrorString(e2),
                       ms * 1e3 / iters);
            }
        }
    }
    return 0;
}
