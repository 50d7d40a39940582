// Micro-benchmark: throughput cost (SM cycles per warp instruction) of the
// L1 data-pipe operations the fused particle kernel is built from, by width
// and by how many distinct addresses / lines the 32 lanes touch.  Every
// operation is timed with CUDA events over many back-to-back independent
// instructions (8 warps x 4 blocks per SM, all SMs, 8 in flight per warp), so the number printed is
// the issue-limited cost per warp instruction on one SM.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o wf_cost wf_cost.cu
#include <cstdint>
#include <cstdio>

enum {
    G256, G128, G64, G32, G16,   // global ld.nc of that width (bits)
    S256, S128, S64,             // shared loads
    SHFL32, SHFL64,              // shuffles (idx)
    RED64,                       // red.global.add.f64
    NMODES
};
static const char *names[] = {"ldg.256", "ldg.128", "ldg.64", "ldg.32", "ldg.16",
                              "lds.256(2x128)", "lds.128", "lds.64", "shfl.32", "shfl.64",
                              "red.f64"};

// distinct: number of distinct addresses in the warp; spread: bytes between them
template <int MODE>
__global__ void __launch_bounds__(256) k(const char *__restrict__ src, double *out, int iters,
                                         int distinct, int spread, int active = 32, int contig = 0) {
    __shared__ __align__(32) double sm[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) sm[i] = i;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int grp = contig ? lane / (32 / distinct) : lane % distinct;
    const long long woff = (long long)(threadIdx.x >> 5) * 4096;   // 32 KB per window, shared by all SMs: L1-resident
    const char *p = src + woff + (long long)grp * spread;
    double acc = 0;
    unsigned acci = 0;
    double *dst = out + 1024 + grp * (spread / 8) + (long long)(blockIdx.x * 8 + (threadIdx.x >> 5)) * 4096;   // per-warp region: no inter-warp contention
#pragma unroll 1
    for (int it = 0; it < iters; it++) {
        // 8 independent instructions per iteration, consumed after all issued
        double r[8];
        unsigned ri[8];
#pragma unroll
        for (int k = 0; k < 8; k++) {
            const char *q = p + k * 4096 + ((it & 1) << 15);   // depends on it: not hoisted
            r[k] = 0;
            ri[k] = 0;
            if (lane >= active) {
            } else if (MODE == G256) {
                double a, b, c, d;
                asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
                             : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(q));
                r[k] = a + b + c + d;
            } else if (MODE == G128) {
                double a, b;
                asm volatile("ld.global.nc.v2.f64 {%0,%1}, [%2];" : "=d"(a), "=d"(b) : "l"(q));
                r[k] = a + b;
            } else if (MODE == G64) {
                asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(r[k]) : "l"(q));
            } else if (MODE == G32) {
                asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(ri[k]) : "l"(q));
            } else if (MODE == G16) {
                unsigned short a;
                asm volatile("ld.global.nc.u16 %0, [%1];" : "=h"(a) : "l"(q));
                ri[k] = a;
            } else if (MODE == S256 || MODE == S128 || MODE == S64) {
                const int idx = ((grp * (spread / 8)) + k * 64 + (it & 1) * 32) & 1023 & ~3;
                const unsigned sa = (unsigned)__cvta_generic_to_shared(sm + idx);
                if (MODE == S64) {
                    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(r[k]) : "r"(sa));
                } else {
                    double a, b;
                    asm volatile("ld.shared.v2.f64 {%0,%1}, [%2];" : "=d"(a), "=d"(b) : "r"(sa));
                    r[k] = a + b;
                    if (MODE == S256) {
                        asm volatile("ld.shared.v2.f64 {%0,%1}, [%2];" : "=d"(a), "=d"(b) : "r"(sa + 16));
                        r[k] += a + b;
                    }
                }
            } else if (MODE == SHFL32) {
                unsigned v = acci + it + k;
                asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, 0xffffffff;" : "=r"(ri[k]) : "r"(v), "r"(grp));
            } else if (MODE == SHFL64) {
                r[k] = __shfl_sync(0xffffffffu, acc + (double)k, grp);
            } else if (MODE == RED64) {
                asm volatile("red.global.add.f64 [%0], %1;" :: "l"(dst + k * 512), "d"(1.0) : "memory");
            }
        }
#pragma unroll
        for (int k = 0; k < 8; k++) {
            acc += r[k];
            acci += ri[k];
        }
    }
    if (acc == -1.0 || acci == 12345u) out[0] = acc + acci;
}

template <int MODE>
static float run(const char *src, double *out, int iters, int d, int spread, int active = 32, int contig = 0) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k<MODE><<<148 * 4, 256>>>(src, out, 8, d, spread);   // warm
    cudaEventRecord(e0);
    k<MODE><<<148 * 4, 256>>>(src, out, iters, d, spread, active, contig);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main() {
    char *src;
    double *out;
    cudaMalloc(&src, 64 << 20);
    cudaMemset(src, 0, 64 << 20);
    const size_t ob = 8ull * (1024 + 148 * 4 * 8 * 4096ull + 64 * 1024);
    cudaMalloc(&out, ob);
    cudaMemset(out, 0, ob);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const int iters = 1024;
    const double winstr_per_sm = 4.0 * 8 * iters * 8;
    printf("mode distinct spread_B cycles_per_warp_instr (SM clock %d MHz)\n", clk_khz / 1000);


    printf("contiguous lane groups (lanes 0..32/d-1 share line 0, ...), spread 128\n");
    for (int d : {1, 2, 4, 8}) {
        auto cyc = [&](float t) { return (double)t * 1e-3 * clk_khz * 1e3 / winstr_per_sm; };
        printf("d=%d contig: ldg.256 %6.2f ldg.64 %6.2f lds.128 %6.2f | interleaved: ldg.256 %6.2f\n", d,
               cyc(run<G256>(src, out, iters, d, 128, 32, 1)), cyc(run<G64>(src, out, iters, d, 128, 32, 1)),
               cyc(run<S128>(src, out, iters, d, 128, 32, 1)), cyc(run<G256>(src, out, iters, d, 128, 32, 0)));
    }
    printf("red.f64, per-warp region (no contention): active lanes x distinct lines\n");
    for (int act : {1, 4, 8, 16, 32}) {
        auto cyc = [&](float t) { return (double)t * 1e-3 * clk_khz * 1e3 / winstr_per_sm; };
        printf("active=%2d d=1 %7.2f  d=32(sp128) %7.2f  d=32(sp8) %7.2f\n", act, cyc(run<RED64>(src, out, 256, 1, 128, act)) * 4,
               cyc(run<RED64>(src, out, 256, 32, 128, act)) * 4, cyc(run<RED64>(src, out, 256, 32, 8, act)) * 4);
    }
    printf("partial warps: active lanes, each on its own line (spread 128) or all on one line\n");
    for (int act : {1, 2, 4, 8, 16}) {
        for (int d : {1, 32}) {
            const float a256 = run<G256>(src, out, iters, d, 128, act);
            const float a64 = run<G64>(src, out, iters, d, 128, act);
            const float a32 = run<G32>(src, out, iters, d, 128, act);
            const float s128 = run<S128>(src, out, iters, d, 32, act);
            auto cyc = [&](float t) { return (double)t * 1e-3 * clk_khz * 1e3 / winstr_per_sm; };
            printf("active=%2d d=%2d  ldg.256 %6.2f  ldg.64 %6.2f  ldg.32 %6.2f  lds.128(sp32) %6.2f\n", act,
                   d, cyc(a256), cyc(a64), cyc(a32), cyc(s128));
        }
    }
    for (int spread : {32, 128}) {
        for (int d : {1, 2, 4, 8, 16, 32}) {
            float t[NMODES];
            t[G256] = run<G256>(src, out, iters, d, spread);
            t[G128] = run<G128>(src, out, iters, d, spread);
            t[G64] = run<G64>(src, out, iters, d, spread);
            t[G32] = run<G32>(src, out, iters, d, spread);
            t[G16] = run<G16>(src, out, iters, d, spread);
            t[S256] = run<S256>(src, out, iters, d, spread);
            t[S128] = run<S128>(src, out, iters, d, spread);
            t[S64] = run<S64>(src, out, iters, d, spread);
            t[SHFL32] = run<SHFL32>(src, out, iters, d, spread);
            t[SHFL64] = run<SHFL64>(src, out, iters, d, spread);
            t[RED64] = run<RED64>(src, out, iters, d, spread);
            for (int m = 0; m < NMODES; m++) {
                const double cyc = (double)t[m] * 1e-3 * clk_khz * 1e3 / winstr_per_sm;
                printf("%-15s d=%2d spread=%3d  %7.2f\n", names[m], d, spread, cyc);
            }
        }
    }
    cudaDeviceSynchronize();
    printf("status %s\n", cudaGetErrorString(cudaGetLastError()));
}
