// micro_barrier.cu -- cost of one grid-wide barrier inside a persistent cooperative kernel on
// B200, for several implementations and grid sizes.  Standalone tool (not part of libgsw).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_barrier tools/micro_barrier.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_release_add(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// A: counter + generation word (libgsw v0)
__global__ void bar_a(unsigned *ctr, unsigned *gen, int iters) {
    unsigned epoch = 0;
    for (int i = 0; i < iters; ++i) {
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned target = epoch + 1;
            __threadfence();
            unsigned prev = atomicAdd(ctr, 1u);
            if (prev == target * gridDim.x - 1) { __threadfence(); st_release(gen, target); }
            else while (ld_acquire(gen) < target) {}
            __threadfence();
        }
        epoch++;
        __syncthreads();
    }
}
// B: release-reduction arrival, everybody polls the counter (no generation word, no fences)
__global__ void bar_b(unsigned *ctr, unsigned *gen, int iters) {
    for (int i = 0; i < iters; ++i) {
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned target = (unsigned)(i + 1) * gridDim.x;
            red_release_add(ctr, 1u);
            while (ld_acquire(ctr) < target) {}
        }
        __syncthreads();
    }
}
// C: acq_rel atomic arrival + generation word with the last arriver publishing, no extra fences
__global__ void bar_c(unsigned *ctr, unsigned *gen, int iters) {
    for (int i = 0; i < iters; ++i) {
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned target = i + 1;
            unsigned prev;
            asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(ctr) : "memory");
            if (prev == target * gridDim.x - 1) st_release(gen, target);
            else while (ld_acquire(gen) < target) {}
        }
        __syncthreads();
    }
}
// D: cooperative groups grid sync
__global__ void bar_d(unsigned *, unsigned *, int iters) {
    cg::grid_group g = cg::this_grid();
    for (int i = 0; i < iters; ++i) g.sync();
}
// E: hierarchical: CTAs arrive at one of 8 sub-counters, sub-leaders arrive at the top counter
__global__ void bar_e(unsigned *ctr, unsigned *gen, int iters) {
    const unsigned G = gridDim.x, NS = 16;
    unsigned grp = blockIdx.x % NS;
    unsigned gsize = G / NS + (grp < G % NS ? 1 : 0);
    for (int i = 0; i < iters; ++i) {
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned target = i + 1;
            unsigned prev;
            asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(ctr + 32 * (1 + grp)) : "memory");
            if (prev == target * gsize - 1) {
                unsigned p2;
                asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(p2) : "l"(ctr) : "memory");
                if (p2 == target * NS - 1) st_release(gen, target);
            }
            while (ld_acquire(gen) < target) {}
        }
        __syncthreads();
    }
}

typedef void (*kfn)(unsigned *, unsigned *, int);

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned *buf;
    cudaMalloc(&buf, 1 << 16);
    kfn ks[] = {bar_a, bar_b, bar_c, bar_d, bar_e};
    const char *names[] = {"A ctr+gen+fences", "B red.release+poll ctr", "C atom.acq_rel+gen", "D cg::grid.sync", "E hier16+gen"};
    int per_sm[] = {1, 2, 4, 8};
    int iters = 20000;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int k = 0; k < 5; ++k) {
        for (int p : per_sm) {
            int grid = sms * p;
            for (int rep = 0; rep < 2; ++rep) {
                cudaMemset(buf, 0, 1 << 16);
                unsigned *ctr = buf, *gen = buf + 1024;
                void *args[] = {&ctr, &gen, &iters};
                cudaEventRecord(e0);
                cudaError_t err = cudaLaunchCooperativeKernel((void *)ks[k], dim3(grid), dim3(256), args, 0, 0);
                cudaEventRecord(e1);
                cudaError_t e2 = cudaDeviceSynchronize();
                float ms = 0;
                cudaEventElapsedTime(&ms, e0, e1);
                if (rep == 1)
                    printf("%-24s grid=%5d (%d/SM): %7.3f us/barrier %s %s\n", names[k], grid, p, ms * 1e3 / iters,
                           err ? cudaGetErrorString(err) : "", e2 ? cudaGetErrorString(e2) : "");
            }
        }
    }
    return 0;
}
