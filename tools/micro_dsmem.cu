// micro_dsmem.cu -- cost of one "exchange a small record with every CTA of the cluster" step on
// B200, the per-level synchronisation of the BFS team tier (bfs.cu bfs_team):
//   mode 0: cluster barrier only
//   mode 1: barrier, then warp 0 lane c reads CTA c's record through DSMEM (pull)
//   mode 2: warp 0 lane c stores my record into CTA c's slot array (push), barrier, local reads
//   mode 3: as 1, but the record is written by thread 0 right before the barrier (as bfs_team)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_dsmem tools/micro_dsmem.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

struct Rec { unsigned qn, mx, mn, pad; unsigned long long ea; };

__global__ void k_ex(int iters, int mode, unsigned long long *out, unsigned *sink) {
    __shared__ Rec mine[2];
    __shared__ Rec slots[2][16];
    __shared__ unsigned tot;
    cg::cluster_group cl = cg::this_cluster();
    const unsigned k = cl.num_blocks(), r = cl.block_rank(), tid = threadIdx.x;
    unsigned acc = 0;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        const int p = i & 1;
        if (mode == 0) {
            cl.sync();
            acc += tid;
        } else if (mode == 1 || mode == 3) {
            if (tid == 0) mine[p] = Rec{r + i, r, r, 0, (unsigned long long)i};
            cl.sync();
            if (tid < 32) {
                unsigned q = 0;
                if (tid < k) {
                    const Rec *rm = cl.map_shared_rank(&mine[p], tid);
                    q = rm->qn + rm->mx + rm->mn + (unsigned)rm->ea;
                }
                for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
                if (tid == 0) tot = q;
            }
            __syncthreads();
            acc += tot;
        } else {
            if (tid < k) {
                Rec *rs = cl.map_shared_rank(&slots[p][r], tid);
                *rs = Rec{r + i, r, r, 0, (unsigned long long)i};
            }
            cl.sync();
            if (tid < 32) {
                unsigned q = 0;
                if (tid < k) { const Rec &m = slots[p][tid]; q = m.qn + m.mx + m.mn + (unsigned)m.ea; }
                for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
                if (tid == 0) tot = q;
            }
            __syncthreads();
            acc += tot;
        }
    }
    cl.sync();
    if (blockIdx.x == 0 && tid == 0) out[mode] = clock64() - t0;
    if (acc == 0x12345678u) *sink = acc;
}

int main() {
    unsigned long long *out;
    unsigned *sink;
    cudaMalloc(&out, 64);
    cudaMalloc(&sink, 64);
    cudaFuncSetAttribute(k_ex, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    for (int csize : {2, 4, 8, 16}) {
        for (int mode = 0; mode < 3; ++mode) {
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(csize);
            cfg.blockDim = dim3(256);
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = csize; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            const int iters = 20000;
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            cudaEventRecord(e0);
            cudaError_t err = cudaLaunchKernelEx(&cfg, k_ex, iters, mode, out, sink);
            cudaEventRecord(e1);
            cudaError_t e2 = cudaDeviceSynchronize();
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("cluster=%2d mode=%d (%s): %s/%s  %.3f us/step\n", csize, mode,
                   mode == 0 ? "barrier only" : mode == 1 ? "barrier + DSMEM pull" : "DSMEM push + barrier",
                   cudaGetErrorString(err), cudaGetErrorString(e2), ms * 1e3 / iters);
        }
    }
    return 0;
}
