// Micro-benchmark: cost of a grid-wide barrier on B200 (cooperative groups
// grid.sync vs a hand-written sense-reversal barrier), per barrier.
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;

__global__ void k_cg(int iters, double *sink) {
    cg::grid_group g = cg::this_grid();
    double acc = 0;
    for (int i = 0; i < iters; i++) { acc += i; g.sync(); }
    if (acc < 0) sink[0] = acc;
}

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
// counter[0] = arrivals, counter[1] = generation
__device__ __forceinline__ void my_sync(unsigned *bar, unsigned nblocks, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned g = gen;
        unsigned prev;
        asm volatile("atom.add.release.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(bar) : "memory");
        if (prev == nblocks - 1) {
            bar[0] = 0;
            asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(bar + 1), "r"(g + 1) : "memory");
        } else {
            while (ld_acquire(bar + 1) == g) { }
        }
    }
    gen++;
    __syncthreads();
}

__global__ void k_my(int iters, unsigned *bar, double *sink) {
    unsigned gen = 0;
    double acc = 0;
    for (int i = 0; i < iters; i++) { acc += i; my_sync(bar, gridDim.x, gen); }
    if (acc < 0) sink[0] = acc;
}

int main() {
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    double *sink; cudaMalloc(&sink, 8);
    unsigned *bar; cudaMalloc(&bar, 8);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    int iters = 2000;
    for (int bps : {1, 2, 4}) for (int thr : {256, 512}) {
        int grid = nsm * bps;
        void *args[] = {&iters, &sink};
        cudaLaunchCooperativeKernel((void *)k_cg, grid, thr, args, 0, 0);
        cudaEventRecord(a);
        cudaLaunchCooperativeKernel((void *)k_cg, grid, thr, args, 0, 0);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        cudaMemset(bar, 0, 8);
        void *args2[] = {&iters, &bar, &sink};
        cudaLaunchCooperativeKernel((void *)k_my, grid, thr, args2, 0, 0);
        cudaMemset(bar, 0, 8);
        cudaEventRecord(a);
        cudaLaunchCooperativeKernel((void *)k_my, grid, thr, args2, 0, 0);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms2; cudaEventElapsedTime(&ms2, a, b);
        printf("grid %d x %d: cg.sync %.3f us, own barrier %.3f us  (%s)\n", grid, thr, 1e3 * ms / iters,
               1e3 * ms2 / iters, cudaGetErrorString(cudaGetLastError()));
    }
}
