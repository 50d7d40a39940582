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
    // slab partition (opp_em_set_partition): cells [c0, c1) are this rank's
    // (single domain: [0, nc)); a particle whose path enters another rank's
    // cell stops on the face and is recorded as a migrant: its index, the face
    // point in the new cell's offsets, the rest of its streak, the crossings
    // so far and the new cell (mig_n == null: single domain, never happens)
    long long c0, c1;
    unsigned long long *mig_n;
    uint32_t *mig_i;
    double *mig_p, *mig_d;     // [3][mig_cap]
    int32_t *mig_c, *mig_k;
    long long mig_cap;
};

// One migrating particle on the wire (opp_em_move_deposit_slab): face point,
// rest of the streak, momentum, weight, id, new cell, crossings so far.
struct EmRecord {
    double p[3], d[3], u[3], w;
    long long id;
    int32_t cell, k;
};
static_assert(sizeof(EmRecord) == 96, "EmRecord is 96 bytes");

// Slab ranges: rank r owns cells [lo[r], lo[r + 1]).
constexpr int kEmMaxRanks = 64;
struct EmRanges {
    long long lo[kEmMaxRanks + 1];
    int n;
};

cudaError_t launch_em_interpolate(int nx, int ny, int nz, const double *e, const double *b,
                                  double *interp, cudaStream_t s, long long c0 = 0, long long c1 = -1);
cudaError_t launch_em_move_deposit(const EmArgs &a, int nsm, cudaStream_t s);
// Slabs: the received particles [first, first + m) resume their walk from
// (off, cell) with the rest of their streak d[3][m] and crossings k[m].
cudaError_t launch_em_continue(const EmArgs &a, long long first, long long m, const double *d,
                               const int32_t *k, int nsm, cudaStream_t s);
// migrants -> records, grouped by destination rank (cursor[r] = first slot);
// dest rank of a cell: the rank whose cell range [lo, hi) holds it
cudaError_t launch_em_mig_count(const EmArgs &a, const EmRanges &rr, unsigned long long *counts,
                                cudaStream_t s);
cudaError_t launch_em_mig_pack(const EmArgs &a, const EmRanges &rr, unsigned long long *cursor,
                               const long long *id, EmRecord *out, uint32_t *holes, cudaStream_t s);
// records -> particles [first, first + m) (d, k of each into dbuf / kbuf)
cudaError_t launch_em_mig_unpack(const EmArgs &a, long long *id, const EmRecord *in, long long first,
                                 long long m, double *dbuf, int32_t *kbuf, cudaStream_t s);
// (field kernels: cells [c0, c1) of the nc; c1 < 0: all)
cudaError_t launch_em_accumulate_current(const double *acc, const int32_t *c2c, long long nc,
                                         const double h[3], double dt, double *J, cudaStream_t s,
                                         long long c0 = 0, long long c1 = -1);
cudaError_t launch_em_advance_b(const double *e, double *b, const int32_t *c2c, long long nc,
                                const double h[3], double fdt, cudaStream_t s, long long c0 = 0,
                                long long c1 = -1);
cudaError_t launch_em_advance_e(double *e, const double *b, const double *J, const int32_t *c2c,
                                long long nc, const double h[3], double dt, cudaStream_t s,
                                long long c0 = 0, long long c1 = -1);

}  // namespace opp
