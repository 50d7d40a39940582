// opp_em.h -- kernels of the CabanaPIC-style electromagnetic particle loop
// (config C3): Interpolate and the fused
// Move_Deposit (Boris push + face-crossing move + Eq. 11 current deposit).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace opp {

constexpr int kEmNI = 18;   // interpolator doubles per cell
constexpr int kEmNA = 12;   // accumulator doubles per cell (jx[4], jy[4], jz[4])

struct EmCounters {
    unsigned long long n_crossings, n_capped;
    unsigned max_crossings, pad;
    unsigned long long n_work;   // particles deferred to the continuation pass
};

struct EmArgs {
    long long n, cap;          // particles, SoA column stride (elements)
    double *off, *u;           // [3][cap] offsets in [-1, 1], momenta u = gamma v / c
    const double *w;           // [cap] weights
    int32_t *cell;             // [cap]
    const double *interp;      // [nc][18]
    const int32_t *c2c;        // [nc][6] faces -x,+x,-y,+y,-z,+z
    long long nc;
    double *acc;               // [nc][12]
    double qdt_2mc, cdt[3], qsp;
    int kcap;
    int dep;                   // 0: 12 reductions per segment and lane; 1: warp-aggregated
    EmCounters *cnt;
    uint32_t *work;            // deferred particles (face crossers), capacity >= n; null: no deferral
};

cudaError_t launch_em_interpolate(int nx, int ny, int nz, const double *e, const double *b,
                                  double *interp, cudaStream_t s);
cudaError_t launch_em_move_deposit(const EmArgs &a, int nsm, cudaStream_t s);
cudaError_t launch_em_accumulate_current(const double *acc, const int32_t *c2c, long long nc,
                                         const double h[3], double dt, double *J, cudaStream_t s);
cudaError_t launch_em_advance_b(const double *e, double *b, const int32_t *c2c, long long nc,
                                const double h[3], double fdt, cudaStream_t s);
cudaError_t launch_em_advance_e(double *e, const double *b, const double *J, const int32_t *c2c,
                                long long nc, const double h[3], double dt, cudaStream_t s);

}  // namespace opp
