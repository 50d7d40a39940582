// Micro-benchmark: L1 data-pipe wavefronts of one warp-wide load, by width and
// by the number of distinct addresses in the warp (read with ncu:
// l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum / _mem_shared.sum per launch).
#include <cstdio>
#include <cstdint>

template <int MODE>
__global__ void k(const double *__restrict__ src, double *out, int iters, int distinct) {
    __shared__ __align__(16) double sm[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) sm[i] = i;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int grp = lane % distinct;                     // lanes sharing an address
    const double *p = src + 4 * (grp + 64 * (blockIdx.x % 64));
    double acc = 0;
    for (int it = 0; it < iters; it++) {
        double a, b, c, d;
        if (MODE == 0) {        // 256-bit
            asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
        } else if (MODE == 1) { // 128-bit
            asm volatile("ld.global.nc.v2.f64 {%0,%1}, [%2];" : "=d"(a), "=d"(b) : "l"(p)); c = d = 0;
        } else if (MODE == 2) { // 64-bit
            asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(a) : "l"(p)); b = c = d = 0;
        } else {                // shared 128-bit
            const double2 v = reinterpret_cast<const double2 *>(sm)[grp * 2];
            a = v.x; b = v.y; c = d = 0;
        }
        acc += a + b + c + d;
        p += 4 * 64 * 64;       // new lines each iteration (stays in L1/L2: small footprint wraps)
        if (p > src + (1 << 20)) p -= (1 << 20);
    }
    if (acc == -1.0) out[0] = acc;
}

int main() {
    double *src, *out;
    cudaMalloc(&src, (2 << 20) * sizeof(double));
    cudaMemset(src, 0, (2 << 20) * sizeof(double));
    cudaMalloc(&out, 64);
    const int iters = 64;
    for (int d : {1, 2, 4, 8, 32}) {
        k<0><<<148, 256>>>(src, out, iters, d);
        k<1><<<148, 256>>>(src, out, iters, d);
        k<2><<<148, 256>>>(src, out, iters, d);
        k<3><<<148, 256>>>(src, out, iters, d);
    }
    cudaDeviceSynchronize();
    printf("done %s (warp-loads per launch: %d)\n", cudaGetErrorString(cudaGetLastError()), 148 * 8 * iters);
}
