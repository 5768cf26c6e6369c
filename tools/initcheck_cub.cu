// initcheck_cub.cu -- is compute-sanitizer initcheck blind to CUB radix-sort output on sm_100a?
// Sorts (key, value) pairs with cub::DeviceRadixSort::SortPairsDescending exactly as graph.cu's
// relabeling does, then reads the sorted values in a plain kernel and checks them on the host.
// If initcheck reports "uninitialized" reads of a buffer whose contents are verifiably correct,
// its reports on graph.cu's perm (round 2) are the same false positive.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o build/initcheck_cub tools/initcheck_cub.cu
#include <cstdio>
#include <vector>
#include <cub/device/device_radix_sort.cuh>

__global__ void k_read(const unsigned *v, int n, unsigned long long *sum) {
    unsigned long long s = 0;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) s += v[i];
    atomicAdd(sum, s);
}

int main() {
    const int n = 2048;
    std::vector<unsigned> hk(n), hv(n);
    for (int i = 0; i < n; ++i) { hk[i] = (unsigned)((i * 2654435761u) % 97u); hv[i] = (unsigned)i; }
    unsigned *k0, *k1, *v0, *v1;
    unsigned long long *sum;
    cudaMalloc(&k0, n * 4); cudaMalloc(&k1, n * 4); cudaMalloc(&v0, n * 4); cudaMalloc(&v1, n * 4);
    cudaMalloc(&sum, 8);
    cudaMemcpy(k0, hk.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(v0, hv.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMemset(sum, 0, 8);
    size_t tb = 0;
    cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, k0, k1, v0, v1, n, 0, 32);
    void *tmp;
    cudaMalloc(&tmp, tb);
    cub::DeviceRadixSort::SortPairsDescending(tmp, tb, k0, k1, v0, v1, n, 0, 32);
    k_read<<<8, 256>>>(v1, n, sum);
    unsigned long long s = 0;
    cudaMemcpy(&s, sum, 8, cudaMemcpyDeviceToHost);
    std::vector<unsigned> out(n);
    cudaMemcpy(out.data(), v1, n * 4, cudaMemcpyDeviceToHost);
    std::vector<int> seen(n, 0);
    bool perm = true;
    for (unsigned x : out) { if (x >= (unsigned)n || seen[x]++) perm = false; }
    printf("sum of sorted values %llu (expected %llu), output is a permutation: %s\n", s,
           (unsigned long long)n * (n - 1) / 2, perm ? "yes" : "NO");
    return 0;
}
