// gen_cuda.cu -- device twin of gen/__init__.py's seeded input generators.
//
// INPUT GENERATION ONLY (no method arithmetic).  Reproduces gen.u01,
// gen.seed_particles and gen.inject_batch bit for bit (explicit
// round-to-nearest ops in the numpy evaluation order), so the bench can
// create 50M+ particle workloads in milliseconds; tests/test_gen_cuda.py
// checks the bit-identity.  Outputs are AoS ([n][3] pos/vel), device memory.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ unsigned long long mix(unsigned long long z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

__device__ __forceinline__ double u01(unsigned long long key, unsigned long long idx) {
    unsigned long long z = key + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    return (double)(mix(z) >> 11) * (1.0 / 9007199254740992.0);
}

unsigned long long host_mix(unsigned long long z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

unsigned long long key_of(unsigned long long seed, int stream) {
    return host_mix(seed ^ ((unsigned long long)stream << 48));
}

__device__ __forceinline__ double dm(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double da(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double ds(double a, double b) { return __dsub_rn(a, b); }

struct Keys {
    unsigned long long cell, point, vel, face, injpt;
};

__global__ void k_seed(const double *__restrict__ xyz, const int *__restrict__ c2n, long long nc,
                       long long first, long long n, Keys k, double drift, double spread, long long id_base,
                       const long long *__restrict__ hot, long long nhot, double frac,
                       double *pos, double *vel, int *cell, long long *id) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        // particle first + i of the seeded population (chunked generation)
        const unsigned long long ui = (unsigned long long)(first + i);
        double u = u01(k.cell, ui * 2ull);
        long long c = (long long)dm(u, (double)nc);
        if (c > nc - 1) c = nc - 1;
        if (nhot > 0) {
            double pick = u01(k.cell, ui * 2ull + 1ull);
            long long h = (long long)dm(u, (double)nhot);
            if (h > nhot - 1) h = nhot - 1;
            if (pick < frac) c = hot[h];
        }
        double s0 = u01(k.point, ui * 3ull), s1 = u01(k.point, ui * 3ull + 1ull),
               s2 = u01(k.point, ui * 3ull + 2ull);
        // sort ascending (exact)
        double t;
        if (s0 > s1) { t = s0; s0 = s1; s1 = t; }
        if (s1 > s2) { t = s1; s1 = s2; s2 = t; }
        if (s0 > s1) { t = s0; s0 = s1; s1 = t; }
        const double b0 = s0, b1 = ds(s1, s0), b2 = ds(s2, s1), b3 = ds(1.0, s2);
        const int n0 = c2n[4 * c], n1 = c2n[4 * c + 1], n2 = c2n[4 * c + 2], n3 = c2n[4 * c + 3];
        for (int d = 0; d < 3; d++) {
            double p = dm(b0, xyz[3 * (long long)n0 + d]);
            p = da(p, dm(b1, xyz[3 * (long long)n1 + d]));
            p = da(p, dm(b2, xyz[3 * (long long)n2 + d]));
            p = da(p, dm(b3, xyz[3 * (long long)n3 + d]));
            pos[3 * i + d] = p;
            double v = dm(ds(dm(2.0, u01(k.vel, ui * 3ull + (unsigned long long)d)), 1.0), spread);
            if (d == 2) v = da(v, drift);
            vel[3 * i + d] = v;
        }
        cell[i] = (int)c;
        id[i] = id_base + first + i;
    }
}

__global__ void k_inject(const double *__restrict__ xyz, const long long *__restrict__ inlet,
                         long long nf, long long step, long long n_inj, Keys k, double v_inj,
                         long long id_base, double *pos, double *vel, int *cell, long long *id) {
    for (long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x; j < n_inj;
         j += (long long)gridDim.x * blockDim.x) {
        const unsigned long long g = (unsigned long long)step * (unsigned long long)n_inj + (unsigned long long)j;
        long long f = (long long)dm(u01(k.face, g), (double)nf);
        if (f > nf - 1) f = nf - 1;
        double a = u01(k.injpt, g * 2ull), b = u01(k.injpt, g * 2ull + 1ull);
        if (da(a, b) > 1.0) {
            a = ds(1.0, a);
            b = ds(1.0, b);
        }
        const long long na = inlet[4 * f + 1], nb = inlet[4 * f + 2], ncn = inlet[4 * f + 3];
        for (int d = 0; d < 3; d++) {
            const double pa = xyz[3 * na + d], pb = xyz[3 * nb + d], pc = xyz[3 * ncn + d];
            pos[3 * j + d] = da(da(pa, dm(a, ds(pb, pa))), dm(b, ds(pc, pa)));
            vel[3 * j + d] = d == 2 ? v_inj : 0.0;
        }
        cell[j] = (int)inlet[4 * f];
        id[j] = id_base + step * n_inj + j;
    }
}

Keys keys(unsigned long long seed) {
    return Keys{key_of(seed, 0), key_of(seed, 1), key_of(seed, 2), key_of(seed, 3), key_of(seed, 4)};
}

// Two-stream population of gen.em.two_stream (config C3): particle p in cell
// p / ppc, offsets 2 u - 1, beams +-v0 along z (even / odd p) plus the
// per-plane perturbation table, thermal spread vth (2 u - 1).  SoA outputs.
__global__ void k_em_two_stream(long long n, int ppc, long long nxy, unsigned long long ko0,
                                unsigned long long ko1, unsigned long long ko2,
                                unsigned long long ku0, unsigned long long ku1,
                                unsigned long long ku2, double v0, double vth, double w,
                                const double *__restrict__ tab, double *off, double *u,
                                double *wout, int *cell) {
    for (long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x; p < n;
         p += (long long)gridDim.x * blockDim.x) {
        const long long c = p / ppc;
        const unsigned long long i = (unsigned long long)p;
        off[p] = ds(dm(2.0, u01(ko0, i)), 1.0);
        off[n + p] = ds(dm(2.0, u01(ko1, i)), 1.0);
        off[2 * n + p] = ds(dm(2.0, u01(ko2, i)), 1.0);
        const double sgn = (p % 2 == 0) ? 1.0 : -1.0;
        u[p] = dm(vth, ds(dm(2.0, u01(ku0, i)), 1.0));
        u[n + p] = dm(vth, ds(dm(2.0, u01(ku1, i)), 1.0));
        u[2 * n + p] = da(da(dm(sgn, v0), tab[c / nxy]), dm(vth, ds(dm(2.0, u01(ku2, i)), 1.0)));
        wout[p] = w;
        cell[p] = (int)c;
    }
}

}  // namespace

extern "C" int gen_seed_particles(const double *xyz, const int *c2n, long long nc, long long first,
                                  long long n,
                                  unsigned long long seed, double drift, double spread,
                                  long long id_base, const long long *hot, long long nhot,
                                  double frac, double *pos, double *vel, int *cell, long long *id,
                                  void *stream) {
    if (n <= 0) return 0;
    long long g = (n + 255) / 256;
    if (g > 148 * 16) g = 148 * 16;
    k_seed<<<(int)g, 256, 0, (cudaStream_t)stream>>>(xyz, c2n, nc, first, n, keys(seed), drift, spread,
                                                     id_base, hot, nhot, frac, pos, vel, cell, id);
    return (int)cudaGetLastError();
}

extern "C" int gen_inject_batch(const double *xyz, const long long *inlet, long long nf,
                                long long step, long long n_inj, unsigned long long seed,
                                double v_inj, long long id_base, double *pos, double *vel,
                                int *cell, long long *id, void *stream) {
    if (n_inj <= 0) return 0;
    long long g = (n_inj + 255) / 256;
    if (g > 148 * 16) g = 148 * 16;
    k_inject<<<(int)g, 256, 0, (cudaStream_t)stream>>>(xyz, inlet, nf, step, n_inj, keys(seed),
                                                       v_inj, id_base, pos, vel, cell, id);
    return (int)cudaGetLastError();
}

extern "C" int gen_em_two_stream(int nx, int ny, int nz, int ppc, unsigned long long seed,
                                 double v0, double vth, double w, const double *tab, double *off,
                                 double *u, double *wout, int *cell, void *stream) {
    const long long n = (long long)nx * ny * nz * ppc;
    if (n <= 0) return 0;
    long long g = (n + 255) / 256;
    if (g > 148 * 16) g = 148 * 16;
    k_em_two_stream<<<(int)g, 256, 0, (cudaStream_t)stream>>>(
        n, ppc, (long long)nx * ny, key_of(seed, 10), key_of(seed, 11), key_of(seed, 12),
        key_of(seed, 13), key_of(seed, 14), key_of(seed, 15), v0, vth, w, tab, off, u, wout, cell);
    return (int)cudaGetLastError();
}
