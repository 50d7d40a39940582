// opp_field.h -- the electrostatic field solve of libopp (internal): P1 FEM
// Poisson matrix in sliced-ELLPACK form, a persistent cooperative CG kernel and
// the cell-field kernel (Fig. 1
// step 1, 469-479, 1044-1068, 1604-1612).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace opp {

constexpr int kSell = 32;   // rows per slice (one warp, lane = row)

// K stored as SELL-32: slice s holds rows [32 s, 32 s + 32); its width
// W_s = max nnz of those rows; entry k of row 32 s + l is at
// slice_off[s] + 32 k + l (column-major inside the slice: a warp's 32 lanes
// read 32 consecutive values).  Padding: col = the row itself, val = 0.
// Dirichlet rows are identity rows; free rows keep their Dirichlet columns
// (needed once, for the lifted initial residual).
struct FieldMat {
    long long nn = 0, nslices = 0, nnz_pad = 0;
    int64_t *slice_off = nullptr;   // [nslices + 1]
    int32_t *col = nullptr;         // [nnz_pad]
    double *val = nullptr;          // [nnz_pad]
    double *dinv = nullptr;         // [nn] Jacobi: 1 / K_ii (1 on Dirichlet rows)
    int32_t *dmask = nullptr;       // [nn] 1 = Dirichlet node
    double *dval = nullptr;         // [nn] Dirichlet values (0 on free nodes)
};

// Device-side solver state (read back by opp_get_field_stats).
struct CgState {
    int iterations;
    int converged;
    double rr0;          // ||b_F - K_FD phi_D||^2 (the stopping reference)
    double rr;           // ||r||^2 at exit (recursive residual)
    double pad[5];
};

struct CgArgs {
    FieldMat K;
    const double *Q;     // node charge
    double *x;           // node potential (in: warm start, out: solution)
    double *r, *u, *w, *p, *s;   // work vectors [nn]
    double *m0, *m1, *z, *q;     // pipelined CG (k_pcg): M^-1 w (two buffers), z, q
    double *part;        // [3 * grid] block partial sums
    CgState *st;
    double rhs_scale, tol;
    int max_iter, warm, precond;
    int pipelined;       // 1: k_pcg (one grid barrier per iteration), 0: k_cg
};

// Per-row assembly from the node->cell CSR (deterministic order, no atomics).
cudaError_t launch_field_assemble(const double *xyz, const int32_t *c2n, const int32_t *n2c_ptr,
                                  const int32_t *n2c, const FieldMat &K, cudaStream_t s);
// One cooperative launch runs the whole CG solve (grid = nsm x min(occupancy,
// max_bps) blocks, fewer if the matrix has fewer slices); returns the grid used.
cudaError_t launch_cg(const CgArgs &a, int nsm, int max_bps, cudaStream_t s, int *grid_out);
// E_c = -sum_i phi[c2n[c][i]] grad(lambda_i) -> ef (AoS [nc][3]) and, if
// non-NULL, the padded copy the particle kernels read.
cudaError_t launch_efield(const double *xyz, const int32_t *c2n, const double *phi, long long nc,
                          double *ef, double4 *efp, cudaStream_t s);

}  // namespace opp

// ---- slab CG (nranks > 1, or opp_field_params.slab_cg): one kernel per
// phase, the partial SpMV rows of interface nodes completed by the charge
// halo exchange, dot products over owned nodes reduced across ranks.
namespace opp {
cudaError_t launch_cg_x0(const FieldMat &K, double *x, int warm, cudaStream_t s);
// y = K v over all local rows; yd (may be NULL) = the Dirichlet-column part.
cudaError_t launch_spmv(const FieldMat &K, const double *v, double *y, double *yd, int nsm,
                        cudaStream_t s);
// r = b - y, beff = b - yd on free rows (0 on Dirichlet rows), u = M^-1 r, p = s = 0.
cudaError_t launch_cg_r0(const FieldMat &K, const double *Q, double rhs_scale, const double *y,
                         const double *yd, double *r, double *u, double *p, double *sv,
                         double *beff, int precond, cudaStream_t s);
// out[k] = sum_i own[i] * a_k[i] * b_k[i], k < nv (deterministic two-pass sum).
cudaError_t launch_dots(long long n, const double *own, int nv, const double *const *va,
                        const double *const *vb, double *part, int nblk, double *out,
                        cudaStream_t s);
// Slab CG (nranks > 1) driven from the device: the per-rank dot products
// of an iteration are all-gathered on the stream and summed in rank order by
// one thread, which also forms alpha, beta and the stop test, so the host
// enqueues iterations in batches and reads one flag per batch.
struct CgCoef {
    double alpha, beta, gamma_old, stop, rr0, rho;
    int it, done, first, pad;
};
// init: rr0 = the gathered ||b_eff||^2, stop = tol^2 rr0; else one iteration's
// (gamma, delta, rho) -> it, done, alpha, beta (Chronopoulos-Gear, as k_cg)
cudaError_t launch_cg_coef(const double *gathered, int nranks, int nv, CgCoef *c, double tol,
                           int max_iter, int init, cudaStream_t s);
cudaError_t launch_cg_update_dev(const FieldMat &K, const CgCoef *c, double *x, double *r, double *u,
                                 const double *w, double *p, double *sv, int precond, cudaStream_t s);
cudaError_t launch_cg_update(const FieldMat &K, double alpha, double beta, double *x, double *r,
                             double *u, const double *w, double *p, double *sv, int precond,
                             cudaStream_t s);
// diag[i] = K_ii (local partial on interface rows); then dinv from the summed diag.
cudaError_t launch_diag(const FieldMat &K, double *diag, cudaStream_t s);
cudaError_t launch_dinv(const FieldMat &K, const double *diag, cudaStream_t s);
}  // namespace opp

// ---- Boltzmann-electron Newton solve (opp_boltz.cu; SURVEY.md §8(f) NEXT-4,
// DESIGN.md §11 readings B1-B4)
namespace opp {
struct NewtonCoef {
    double rhs_scale, ne, phi0, inv_te;
};
// m_n = sum over the node's cells of |V_e| / 4 (lumped P1 mass)
cudaError_t launch_lumped_mass(const double *xyz, const int32_t *c2n, const int32_t *n2c_ptr,
                               const int32_t *n2c, long long nn, double *m, cudaStream_t s);
// blocks of k_newton_eval (= the partial count launch_newton_eval reduces)
int newton_eval_blocks(const FieldMat &K, int nsm);
// One pass over K: rhsv = -F(phi) (0 on Dirichlet rows), jval / jdinv = the
// Jacobian's values and Jacobi inverse diagonal, *norm2 = ||F||^2 (fixed order).
cudaError_t launch_newton_eval(const FieldMat &K, double *jval, double *jdinv, const double *Q,
                               const double *phi, const double *m, const NewtonCoef &co,
                               double *rhsv, double *part, int nblk, double *norm2,
                               cudaStream_t s);
// Multi-rank form: y = the halo-summed K phi; the electron diagonal goes into
// the Jacobian values where own[i] > 0 only; no norm (own-weighted dots follow).
cudaError_t launch_newton_eval_y(const FieldMat &K, const double *y, const double *own,
                                 double *jval, double *jdinv, const double *Q, const double *phi,
                                 const double *m, const NewtonCoef &co, double *rhsv, int nblk,
                                 cudaStream_t s);
cudaError_t launch_newton_start(const FieldMat &K, double *phi, double phi0, int warm,
                                cudaStream_t s);
// free rows: x <- 2 x - xprev, xprev <- old x (warm_start 2 of opp_field_solve)
cudaError_t launch_extrapolate(const FieldMat &K, double *x, double *xprev, cudaStream_t s);
cudaError_t launch_newton_update(const FieldMat &K, double *phi, const double *delta,
                                 cudaStream_t s);
}  // namespace opp
