// opp_boltz.cu -- sm_100a kernels of the Boltzmann-electron (nonlinear) field
// solve (internal).
//
// Mini-FEM-PIC's field solve is a Newton loop of ComputeF1Vector (the
// nonlinear residual), ComputeJMatrix (its Jacobian) and a linear solve
// (PETSc KSP in the paper; §4.1.1).
// readings B1-B4 fix the formulas the paper only names:
//   F_n = (K phi)_n - rhs_scale Q_n + ne m_n exp((phi_n - phi0) / te)  (free n)
//   J   = K + diag(ne m_n / te exp((phi_n - phi0) / te))
// with m_n the lumped P1 mass.  Kernels:
//   k_lumped_mass   m_n = sum over the node's cells of |V_e| / 4 (fixed order)
//   k_newton_eval   ONE pass over K (sliced ELLPACK, warp = slice, lane = row)
//                   computes K phi, F (written as the CG load -F), the
//                   Jacobian values (K's values, the diagonal entry raised by
//                   the electron term), its Jacobi inverse diagonal and the
//                   block partials of ||F||^2 -- ComputeF1Vector and
//                   ComputeJMatrix fused, K read once per Newton step
//   k_sum_final     fixed-order sum of the partials (deterministic norm)
//   k_newton_start / k_newton_update   phi_D = dval_D, phi_F = phi0 or warm;
//                   phi_F += delta_F
// The linear step J_FF delta_F = -F_F runs through the persistent cooperative
// CG kernel of opp_field.cu (launch_cg) on a FieldMat that shares K's
// sparsity and has J's values, J's Jacobi diagonal and zero Dirichlet data.
// Roofline: k_newton_eval streams the padded matrix once (12 B per entry:
// col + K value read, J value written = 20 B with the write) -- L2-resident
// at C2 (31 MB of K); the CG iterations dominate the solve (opp_field.cu).
#include <algorithm>

#include "opp_field.h"

namespace opp {
namespace {

constexpr int kBzThreads = 256;

__global__ void k_lumped_mass(const double *__restrict__ xyz, const int32_t *__restrict__ c2n,
                              const int32_t *__restrict__ n2c_ptr, const int32_t *__restrict__ n2c,
                              long long nn, double *__restrict__ m) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= nn) return;
    double acc = 0.0;
    for (int e = n2c_ptr[i]; e < n2c_ptr[i + 1]; e++) {
        int4 n = reinterpret_cast<const int4 *>(c2n)[n2c[e]];
        double a[3], b[3], c[3];
        for (int k = 0; k < 3; k++) {
            double p0 = xyz[3ll * n.x + k];
            a[k] = xyz[3ll * n.y + k] - p0;
            b[k] = xyz[3ll * n.z + k] - p0;
            c[k] = xyz[3ll * n.w + k] - p0;
        }
        double det = a[0] * (b[1] * c[2] - b[2] * c[1]) + a[1] * (b[2] * c[0] - b[0] * c[2]) +
                     a[2] * (b[0] * c[1] - b[1] * c[0]);
        acc += fabs(det) / 24.0;     // |V_e| / 4, V_e = det / 6
    }
    m[i] = acc;
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__global__ void __launch_bounds__(kBzThreads)
    k_newton_eval(FieldMat K, double *__restrict__ jval, double *__restrict__ jdinv,
                  const double *__restrict__ Q, const double *__restrict__ phi,
                  const double *__restrict__ m, NewtonCoef co, double *__restrict__ rhsv,
                  double *__restrict__ part) {
    __shared__ double sm[kBzThreads / 32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long TW = ((long long)gridDim.x * blockDim.x) >> 5;
    double acc = 0.0;
    for (long long sl = gw; sl < K.nslices; sl += TW) {
        const long long i = sl * kSell + lane;
        const long long off = K.slice_off[sl];
        const int W = (int)((K.slice_off[sl + 1] - off) / kSell);
        const bool row = i < K.nn;
        const bool freerow = row && !K.dmask[i];
        double kphi = 0.0, kii = 0.0;
        int kd = -1;
        for (int k = 0; k < W; k++) {
            const long long q = off + (long long)kSell * k + lane;
            const int c = K.col[q];
            const double v = K.val[q];
            if (row) kphi += v * phi[c];
            if (kd < 0 && c == (int)i) { kd = k; kii = v; }
            jval[q] = v;
        }
        if (!row) continue;
        double F = 0.0;
        if (freerow) {
            const double e = exp((phi[i] - co.phi0) * co.inv_te);
            const double d = co.ne * m[i] * e * co.inv_te;
            F = kphi - co.rhs_scale * Q[i] + co.ne * m[i] * e;
            if (kd >= 0) jval[off + (long long)kSell * kd + lane] = kii + d;
            jdinv[i] = 1.0 / (kii + d);
        } else {
            jdinv[i] = 1.0;
        }
        rhsv[i] = -F;
        acc += F * F;
    }
    acc = warp_sum(acc);
    if (lane == 0) sm[wid] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < kBzThreads / 32; w++) t += sm[w];
        part[blockIdx.x] = t;
    }
}

// Multi-rank form (slab partition): y = K phi with the interface rows already
// summed over ranks (halo), K.dinv = 1 / the summed diagonal.  The electron
// diagonal is added to the Jacobian values on the owning rank only (own[i] =
// 1), so the halo-summed SpMV of the CG applies K + diag(d) exactly once.
__global__ void __launch_bounds__(kBzThreads)
    k_newton_eval_y(FieldMat K, const double *__restrict__ y, const double *__restrict__ own,
                    double *__restrict__ jval, double *__restrict__ jdinv,
                    const double *__restrict__ Q, const double *__restrict__ phi,
                    const double *__restrict__ m, NewtonCoef co, double *__restrict__ rhsv) {
    const int lane = threadIdx.x & 31;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long TW = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long sl = gw; sl < K.nslices; sl += TW) {
        const long long i = sl * kSell + lane;
        const long long off = K.slice_off[sl];
        const int W = (int)((K.slice_off[sl + 1] - off) / kSell);
        const bool row = i < K.nn;
        int kd = -1;
        for (int k = 0; k < W; k++) {
            const long long q = off + (long long)kSell * k + lane;
            const int c = K.col[q];
            if (kd < 0 && c == (int)i) kd = k;
            jval[q] = K.val[q];
        }
        if (!row) continue;
        double F = 0.0;
        if (!K.dmask[i]) {
            const double e = exp((phi[i] - co.phi0) * co.inv_te);
            const double d = co.ne * m[i] * e * co.inv_te;
            F = y[i] - co.rhs_scale * Q[i] + co.ne * m[i] * e;
            if (kd >= 0 && own[i] > 0.0) jval[off + (long long)kSell * kd + lane] += d;
            jdinv[i] = 1.0 / (1.0 / K.dinv[i] + d);
        } else {
            jdinv[i] = 1.0;
        }
        rhsv[i] = -F;
    }
}

__global__ void k_sum_final(const double *__restrict__ part, int nblk, double *out) {
    const int lane = threadIdx.x;
    double t = 0.0;
    for (int b = lane; b < nblk; b += 32) t += part[b];
    t = warp_sum(t);
    if (lane == 0) *out = t;
}

__global__ void k_newton_start(FieldMat K, double *phi, double phi0, int warm) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= K.nn) return;
    phi[i] = K.dmask[i] ? K.dval[i] : (warm ? phi[i] : phi0);
}

__global__ void k_newton_update(FieldMat K, double *phi, const double *__restrict__ delta) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= K.nn) return;
    if (!K.dmask[i]) phi[i] += delta[i];
}

// warm_start 2 of opp_field_solve: x0 = 2 x_{n-1} - x_{n-2} on free rows,
// then xprev = x_{n-1} (linear extrapolation of the last two solutions)
__global__ void k_extrapolate(FieldMat K, double *x, double *xprev) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= K.nn || K.dmask[i]) return;
    const double xc = x[i];
    x[i] = 2.0 * xc - xprev[i];
    xprev[i] = xc;
}

inline unsigned blocks_of(long long n) { return (unsigned)((n + kBzThreads - 1) / kBzThreads); }

}  // namespace

int newton_eval_blocks(const FieldMat &K, int nsm) {
    long long need = (K.nslices + kBzThreads / 32 - 1) / (kBzThreads / 32);
    long long cap = (long long)nsm * 8;
    return (int)std::max<long long>(1, std::min(need, cap));
}

cudaError_t launch_lumped_mass(const double *xyz, const int32_t *c2n, const int32_t *n2c_ptr,
                               const int32_t *n2c, long long nn, double *m, cudaStream_t s) {
    if (nn <= 0) return cudaSuccess;
    k_lumped_mass<<<blocks_of(nn), kBzThreads, 0, s>>>(xyz, c2n, n2c_ptr, n2c, nn, m);
    return cudaGetLastError();
}

cudaError_t launch_newton_eval(const FieldMat &K, double *jval, double *jdinv, const double *Q,
                               const double *phi, const double *m, const NewtonCoef &co,
                               double *rhsv, double *part, int nblk, double *norm2,
                               cudaStream_t s) {
    k_newton_eval<<<nblk, kBzThreads, 0, s>>>(K, jval, jdinv, Q, phi, m, co, rhsv, part);
    k_sum_final<<<1, 32, 0, s>>>(part, nblk, norm2);
    return cudaGetLastError();
}

cudaError_t launch_newton_eval_y(const FieldMat &K, const double *y, const double *own,
                                 double *jval, double *jdinv, const double *Q, const double *phi,
                                 const double *m, const NewtonCoef &co, double *rhsv, int nblk,
                                 cudaStream_t s) {
    k_newton_eval_y<<<nblk, kBzThreads, 0, s>>>(K, y, own, jval, jdinv, Q, phi, m, co, rhsv);
    return cudaGetLastError();
}

cudaError_t launch_newton_start(const FieldMat &K, double *phi, double phi0, int warm,
                                cudaStream_t s) {
    if (K.nn <= 0) return cudaSuccess;
    k_newton_start<<<blocks_of(K.nn), kBzThreads, 0, s>>>(K, phi, phi0, warm);
    return cudaGetLastError();
}

cudaError_t launch_newton_update(const FieldMat &K, double *phi, const double *delta,
                                 cudaStream_t s) {
    if (K.nn <= 0) return cudaSuccess;
    k_newton_update<<<blocks_of(K.nn), kBzThreads, 0, s>>>(K, phi, delta);
    return cudaGetLastError();
}

cudaError_t launch_extrapolate(const FieldMat &K, double *x, double *xprev, cudaStream_t s) {
    if (K.nn <= 0) return cudaSuccess;
    k_extrapolate<<<blocks_of(K.nn), kBzThreads, 0, s>>>(K, x, xprev);
    return cudaGetLastError();
}

}  // namespace opp
