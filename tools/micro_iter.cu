// micro_iter.cu -- cost of the persistent engine's per-iteration skeleton, adding one piece at a
// time (standalone diagnostic tool, not part of libgsw).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude -Ipaper_conf_ppopp_menglts19_b200/csrc \
//        -o build/micro_iter tools/micro_iter.cu
#include <cstdio>

#include "engine.cuh"
#include "lb.cuh"

using namespace gsw;

struct NopOp {
    using Probe = unsigned;
    using Tok = unsigned;
    using Aux = unsigned;
    static constexpr bool kEarlyExit = false;
    __device__ bool skip(int) const { return false; }
    __device__ Probe probe(int, uint32_t, int) const { return 0; }
    __device__ Tok act(int, uint32_t, int, Probe) const { return 0; }
    __device__ Aux aux(int, uint32_t, int, Tok) const { return 0; }
    __device__ bool commit(int, uint32_t, int, Tok, Aux, LocalCnt &) const { return false; }
};

__global__ void __launch_bounds__(kBlock, 4) k_iter(int variant, int iters, unsigned *bar_mem, IterCnt *cnt,
                                                    gsw_iter_record *rec, const uint32_t *off, const int *col,
                                                    int *q) {
    __shared__ LbSmem sm;
    __shared__ uint32_t red[kWarps + 1];
    GridBarrier bar{bar_mem, bar_mem + 32, bar_mem + 64};
    unsigned epoch = 0;
    Book book;
    Features f{};
    gsw_config force{};
    RunCommon rc{};
    rc.rec = rec;
    for (int t = 0; t < iters; ++t) {
        IterCnt *cur = cnt + (t % 3), *nxt = cnt + ((t + 1) % 3);
        if (variant >= 1) {
            CntView cv = cta_read_cnt(cur);
            f.Va = cv.va + 1; f.Ea = cv.ea;
        }
        if (variant >= 2) {
            if (is_book()) book_start(book, rc, t, nxt);
            DevCfg c = select_traversal(f, force);
            write_record(rc, t & 1023, c, f, 0u);
            if (is_book()) reset_cnt(cnt + ((t + 2) % 3));
            if (is_book()) book_expand(book);
        }
        LocalCnt lc;
        if (variant >= 3) {
            NopOp op;
            lc = run_lb(GSW_LB_WM, QueueSrc{q, 1u}, Adj{off, col}, op, sm, red, bar, epoch, nullptr, nullptr);
        }
        if (variant >= 4) flush_counts(lc, nxt);
        grid_sync(bar, epoch);
    }
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned *bar;
    IterCnt *cnt;
    gsw_iter_record *rec;
    uint32_t *off;
    int *col, *q;
    cudaMalloc(&bar, 4096);
    cudaMalloc(&cnt, 3 * sizeof(IterCnt));
    cudaMalloc(&rec, 1024 * sizeof(gsw_iter_record));
    cudaMalloc(&off, 16);
    cudaMalloc(&col, 16);
    cudaMalloc(&q, 16);
    cudaMemset(cnt, 0, 3 * sizeof(IterCnt));
    uint32_t hoff[2] = {0, 2};
    cudaMemcpy(off, hoff, 8, cudaMemcpyHostToDevice);
    cudaMemset(col, 0, 16);
    cudaMemset(q, 0, 16);
    const char *names[] = {"barrier only", "+cta_read_cnt", "+select/record/book", "+noinline LB call (WM, 1 item)",
                           "+flush_counts"};
    int iters = 5000;
    for (int per : {1, 2, 4}) {
        for (int v = 0; v <= 4; ++v) {
            cudaMemset(bar, 0, 4096);
            void *args[] = {&v, &iters, &bar, &cnt, &rec, &off, &col, &q};
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            cudaEventRecord(e0);
            cudaError_t err = cudaLaunchCooperativeKernel((void *)k_iter, dim3(sms * per), dim3(kBlock), args, 0, 0);
            cudaEventRecord(e1);
            cudaError_t e2 = cudaDeviceSynchronize();
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("grid %4d  %-34s %7.3f us/iter %s %s\n", sms * per, names[v], ms * 1e3 / iters,
                   err ? cudaGetErrorString(err) : "", e2 ? cudaGetErrorString(e2) : "");
        }
    }
    return 0;
}
