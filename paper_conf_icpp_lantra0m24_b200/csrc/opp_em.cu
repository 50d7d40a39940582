// opp_em.cu -- sm_100a kernels of the CabanaPIC-style electromagnetic loop
// (config C3).
//
// k_em_move_deposit is the paper's Move_Deposit routine ("calculating new
// positions and velocities, moving to the correct final cell, and depositing
// current into an accumulator in a single routine"), one
// particle per lane:
//   1. gather the cell's 18-double interpolator (nine 128-bit loads) and
//      evaluate E (bilinear) and B (linear) at the particle's offsets;
//   2. relativistic Boris push of u = gamma v / c (Eqs. 7-9 with B);
//   3. streak d = (2 c dt / h) u / gamma in offset units;
//   4. walk the straight path through the faces it crosses, in order, the next
//      cell read from the c2c map, depositing for every
//      segment the Eq. 11 current of the cell's 12 edges
//      in closed form: Q da/4 [(1 + sb mb)(1 + sc mc) + sb sc db dc / 12];
//   5. warp-aggregated accumulation: the lanes depositing into one cell are
//      summed by a 16-value reduce-scatter over the warp (16 shuffles of
//      doubles) and leave as one 12-lane reduction instruction -- in
//      cell-sorted storage (~750 particles per cell) nearly every warp's
//      first segments share one cell.
// Arithmetic that decides a result (push, streak, face times, positions) uses
// explicit round-to-nearest intrinsics, in the oracle's evaluation order
// (oracle/em.c), so cells and offsets match it bit for bit.
#include "opp_em.h"

#include <algorithm>

namespace opp {
namespace {

__device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double sub(double a, double b) { return __dsub_rn(a, b); }
__device__ __forceinline__ double dvd(double a, double b) { return __ddiv_rn(a, b); }

// ---------------------------------------------------------------------------
// Interpolate: edge E / face B on the periodic grid ->
// per-cell interpolator (bilinear E_a in the two transverse offsets, linear
// B_a).  Same layouts and evaluation order as the oracle's em_interpolate.
// ---------------------------------------------------------------------------
__global__ void k_em_interpolate(int nx, int ny, int nz, const double *__restrict__ e,
                                 const double *__restrict__ b, double *__restrict__ interp, long long c0,
                                 long long c1) {
    const long long nc = (long long)nx * ny * nz;
    for (long long c = c0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; c < c1;
         c += (long long)gridDim.x * blockDim.x) {
        const int i = (int)(c % nx), j = (int)((c / nx) % ny), k = (int)(c / ((long long)nx * ny));
        const int ip = (i + 1) % nx, jp = (j + 1) % ny, kp = (k + 1) % nz;
        auto id = [&](int I, int J, int K) { return I + (long long)nx * (J + (long long)ny * K); };
        double v[3][4];
        v[0][0] = e[id(i, j, k)];           v[0][1] = e[id(i, jp, k)];
        v[0][2] = e[id(i, j, kp)];          v[0][3] = e[id(i, jp, kp)];
        v[1][0] = e[nc + id(i, j, k)];      v[1][1] = e[nc + id(i, j, kp)];
        v[1][2] = e[nc + id(ip, j, k)];     v[1][3] = e[nc + id(ip, j, kp)];
        v[2][0] = e[2 * nc + id(i, j, k)];  v[2][1] = e[2 * nc + id(ip, j, k)];
        v[2][2] = e[2 * nc + id(i, jp, k)]; v[2][3] = e[2 * nc + id(ip, jp, k)];
        double *f = interp + kEmNI * c;
#pragma unroll
        for (int a = 0; a < 3; a++) {
            const double *q = v[a];
            f[4 * a + 0] = dvd(add(add(q[0], q[1]), add(q[2], q[3])), 4.0);
            f[4 * a + 1] = dvd(add(sub(q[1], q[0]), sub(q[3], q[2])), 4.0);
            f[4 * a + 2] = dvd(add(sub(q[2], q[0]), sub(q[3], q[1])), 4.0);
            f[4 * a + 3] = dvd(sub(sub(q[3], q[2]), sub(q[1], q[0])), 4.0);
        }
        const double b0x = b[id(i, j, k)], b1x = b[id(ip, j, k)];
        const double b0y = b[nc + id(i, j, k)], b1y = b[nc + id(i, jp, k)];
        const double b0z = b[2 * nc + id(i, j, k)], b1z = b[2 * nc + id(i, j, kp)];
        f[12] = dvd(add(b0x, b1x), 2.0); f[13] = dvd(sub(b1x, b0x), 2.0);
        f[14] = dvd(add(b0y, b1y), 2.0); f[15] = dvd(sub(b1y, b0y), 2.0);
        f[16] = dvd(add(b0z, b1z), 2.0); f[17] = dvd(sub(b1z, b0z), 2.0);
    }
}

// ---------------------------------------------------------------------------
// Move_Deposit
// ---------------------------------------------------------------------------
__device__ __forceinline__ double2 ldnc2(const double *p) {
    double2 v;
    asm("ld.global.nc.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
}

// Eq. 11 of one straight segment p -> q in offset units, charge Q, closed
// form: edge k = (sb, sc) along axis a, transverse offsets (b, c) =
// ((a+1)%3, (a+2)%3), order (-,-), (+,-), (-,+), (+,+).
__device__ __forceinline__ void seg_current(const double p[3], const double q[3], double Q,
                                            double v[kEmNA]) {
    double d[3], m[3];
#pragma unroll
    for (int a = 0; a < 3; a++) {
        d[a] = sub(q[a], p[a]);
        m[a] = mul(0.5, add(p[a], q[a]));
    }
#pragma unroll
    for (int a = 0; a < 3; a++) {
        const int b = (a + 1) % 3, c = (a + 2) % 3;
        const double A = mul(mul(Q, d[a]), 0.25);
        const double cr = mul(mul(d[b], d[c]), 1.0 / 12.0);
        const double bm = sub(1.0, m[b]), bp = add(1.0, m[b]);
        const double cm = sub(1.0, m[c]), cp = add(1.0, m[c]);
        v[4 * a + 0] = mul(A, add(mul(bm, cm), cr));
        v[4 * a + 1] = mul(A, sub(mul(bp, cm), cr));
        v[4 * a + 2] = mul(A, sub(mul(bm, cp), cr));
        v[4 * a + 3] = mul(A, add(mul(bp, cp), cr));
    }
}

// Sum the 12 values of every lane in `grp` (lanes outside contribute 0) by a
// reduce-scatter over 16 slots (xor 16, 8, 4, 2 halve the slots, xor 1
// completes): even lanes 2s (s < 12) then hold slot s and issue one
// reduction each -- one 12-lane instruction on 96 contiguous bytes.
__device__ __forceinline__ void rs_deposit(double *__restrict__ acc_cell, bool in,
                                           const double v[kEmNA]) {
    const unsigned FULL = 0xffffffffu, lane = threadIdx.x & 31u;
    double s8[8];
    const bool h16 = lane & 16u;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const double lo = in ? v[i] : 0.0;
        const double hi = (in && i + 8 < kEmNA) ? v[i + 8] : 0.0;
        const double keep = h16 ? hi : lo, send = h16 ? lo : hi;
        s8[i] = add(keep, __shfl_xor_sync(FULL, send, 16));
    }
    double s4[4];
    const bool h8 = lane & 8u;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const double keep = h8 ? s8[i + 4] : s8[i], send = h8 ? s8[i] : s8[i + 4];
        s4[i] = add(keep, __shfl_xor_sync(FULL, send, 8));
    }
    double s2[2];
    const bool h4 = lane & 4u;
#pragma unroll
    for (int i = 0; i < 2; i++) {
        const double keep = h4 ? s4[i + 2] : s4[i], send = h4 ? s4[i] : s4[i + 2];
        s2[i] = add(keep, __shfl_xor_sync(FULL, send, 4));
    }
    const bool h2 = lane & 2u;
    double t = add(h2 ? s2[1] : s2[0], __shfl_xor_sync(FULL, h2 ? s2[0] : s2[1], 2));
    t = add(t, __shfl_xor_sync(FULL, t, 1));
    const int slot = (h16 ? 8 : 0) + (h8 ? 4 : 0) + (h4 ? 2 : 0) + (h2 ? 1 : 0);
    if (!(lane & 1u) && slot < kEmNA) atomicAdd(acc_cell + slot, t);
}

// Deposit one segment per lane (lanes with has = false contribute nothing).
// DEP 1: at most OPP_EM_DIRECT active lanes (the later move rounds: only the
// particles still crossing faces) reduce directly -- an fp64 reduction costs
// the L1 ~2 cycles per lane, cheaper than any warp-wide shuffle reduction of
// 12 values.  Otherwise lanes are grouped by cell (match_any).  Up to
// OPP_EM_RS_MAX groups: one reduce-scatter (above) per group.  More groups (the two beams of a
// two-stream population drift apart, so a warp's lanes spread over a few
// cells): a log-step tree sums each group's 12 values into its lowest lane,
// then the (group, slot) pairs are dealt out 32 per pass -- lane j takes pair
// 32 r + j: its group's leader and slot -- so each reduction instruction
// covers up to 32 pairs (consecutive slots of a cell are adjacent doubles).
// DEP 0: 12 reductions per lane.
#ifndef OPP_EM_DIRECT
#define OPP_EM_DIRECT 8   // active lanes at or below which segments reduce directly
                          // (C3: 0 -> 8 lanes: 5.38 -> 4.80 ms; 12, 16: same)
#endif
#ifndef OPP_EM_RS_MAX
#define OPP_EM_RS_MAX 3   // cells per warp at or below which each gets a reduce-scatter
                          // (C3: 1, 2, 3 within 1%; 6: 8% slower)
#endif
#ifndef OPP_EM_SMEM_SUM
#define OPP_EM_SMEM_SUM 1   // > OPP_EM_RS_MAX cells per warp: transpose through shared memory
                            // (C3: 4.50 -> 4.16 ms vs the shuffle tree + deal)
#endif
constexpr int kEmBufLd = 33;   // row stride (doubles) of the per-warp transpose buffer

template <int DEP>
__device__ __forceinline__ void em_deposit(double *__restrict__ acc, bool has, int key,
                                           const double vin[kEmNA], double *__restrict__ buf) {
    const unsigned FULL = 0xffffffffu, lane = threadIdx.x & 31u;
    if (DEP == 0) {
        if (has) {
            double *a = acc + (long long)kEmNA * key;
#pragma unroll
            for (int s = 0; s < kEmNA; s++) atomicAdd(a + s, vin[s]);
        }
        return;
    }
    const unsigned act = __ballot_sync(FULL, has);
    if (!act) return;
    if (__popc(act) <= OPP_EM_DIRECT) {   // a few lanes (later move rounds): direct reductions
        if (has) {
            double *a = acc + (long long)kEmNA * key;
#pragma unroll
            for (int s = 0; s < kEmNA; s++) atomicAdd(a + s, vin[s]);
        }
        return;
    }
    const unsigned peers = __match_any_sync(FULL, has ? key : -1 - (int)lane);
    const unsigned lead = __ballot_sync(FULL, has && (int)lane == __ffs(peers) - 1);
    const int G = __popc(lead);
    if (G <= OPP_EM_RS_MAX) {   // one reduce-scatter per cell
        unsigned l = lead;
        do {
            const int L = __ffs(l) - 1;
            l &= l - 1u;
            const int kL = __shfl_sync(FULL, key, L);
            rs_deposit(acc + (long long)kEmNA * kL, has && key == kL, vin);
        } while (l);
        return;
    }
    if (OPP_EM_SMEM_SUM) {
        // transpose: buf[slot][lane]; then lane j sums (cell g, slot s) pair
        // 32 r + j over the members of cell g -- about 12 G x (32 / G) / 32 =
        // 12 iterations for any number of cells, where shuffle reductions cost
        // a full warp pass per cell
        if (has) {
#pragma unroll
            for (int s = 0; s < kEmNA; s++) buf[s * kEmBufLd + lane] = vin[s];
        }
        __syncwarp();
        const int P = G * kEmNA;
        for (int base = 0; base < P; base += 32) {
            const int pr = base + (int)lane;
            const bool act = pr < P;
            const int g = act ? pr / kEmNA : 0, sl = act ? pr - g * kEmNA : 0;
            const int L = (int)__fns(lead, 0, g + 1);
            unsigned m = __shfl_sync(FULL, peers, L);
            const int kL = __shfl_sync(FULL, key, L);
            if (act) {
                const double *row = buf + sl * kEmBufLd;
                double sum = 0.0;
                while (m) {
                    const int k = __ffs(m) - 1;
                    m &= m - 1u;
                    sum = add(sum, row[k]);
                }
                atomicAdd(acc + (long long)kEmNA * kL + sl, sum);
            }
        }
        __syncwarp();
        return;
    }
    double v[kEmNA];
#pragma unroll
    for (int s = 0; s < kEmNA; s++) v[s] = has ? vin[s] : 0.0;
    // tree: each round a lane absorbs the next still-present lane of its group
    int rel = __popc(peers & ((1u << lane) - 1u));
    unsigned up = has ? (peers & ~((2u << lane) - 1u)) : 0u;
    if (lane == 31) up = 0;
    while (__any_sync(FULL, up != 0)) {
        const int nx = up ? __ffs(up) - 1 : (int)lane;
#pragma unroll
        for (int s = 0; s < kEmNA; s++) {
            const double t = __shfl_sync(FULL, v[s], nx);
            if (up) v[s] = add(v[s], t);
        }
        const unsigned gone = __ballot_sync(FULL, (rel & 1) != 0);
        up &= ~gone;
        rel >>= 1;
    }
    // deal the G x 12 (leader, slot) pairs over the lanes, 32 per pass
    const int P = G * kEmNA;
    for (int base = 0; base < P; base += 32) {
        const int pr = base + (int)lane;
        const bool act = pr < P;
        const int g = act ? pr / kEmNA : 0, sl = act ? pr - g * kEmNA : 0;
        const int L = (int)__fns(lead, 0, g + 1);
        double val = 0.0;
#pragma unroll
        for (int s = 0; s < kEmNA; s++) {
            const double t = __shfl_sync(FULL, v[s], L);
            if (s == sl) val = t;
        }
        const int kL = __shfl_sync(FULL, key, L);
        if (act) atomicAdd(acc + (long long)kEmNA * kL + sl, val);
    }
}

// Face hit by the streak d from p (first along the path; t = 1 ends inside)
// and the segment's end point q (exactly on the face when one is hit).
__device__ __forceinline__ int em_face(const double p[3], const double d[3], double q[3]) {
    double t = 1.0;
    int face = -1;
    // one division site per axis (the oracle's two branches differ only in
    // the numerator): divergent lanes would otherwise run both
#pragma unroll
    for (int ax = 0; ax < 3; ax++) {
        const bool pos = d[ax] > 0.0;
        if (d[ax] != 0.0) {
            const double ta = dvd(sub(pos ? 1.0 : -1.0, p[ax]), d[ax]);
            if (ta < t) { t = ta; face = 2 * ax + (pos ? 1 : 0); }
        }
    }
#pragma unroll
    for (int ax = 0; ax < 3; ax++) q[ax] = add(p[ax], mul(t, d[ax]));
    if (face >= 0) {
        const double fv = (face & 1) ? 1.0 : -1.0;
        const int fa = face >> 1;
        q[0] = fa == 0 ? fv : q[0];
        q[1] = fa == 1 ? fv : q[1];
        q[2] = fa == 2 ? fv : q[2];
    }
    return face;
}

// Cross `face`: the rest of the streak continues from the face point in the
// neighbour, with the offset along the face axis flipped.
__device__ __forceinline__ void em_cross(double p[3], double d[3], const double q[3], int face,
                                         int &c, const int32_t *__restrict__ c2c) {
#pragma unroll
    for (int ax = 0; ax < 3; ax++) {
        d[ax] = sub(d[ax], sub(q[ax], p[ax]));
        p[ax] = q[ax];
    }
    const int fa = face >> 1;
    p[0] = fa == 0 ? -p[0] : p[0];
    p[1] = fa == 1 ? -p[1] : p[1];
    p[2] = fa == 2 ? -p[2] : p[2];
    c = __ldg(c2c + 6 * (long long)c + face);
}

// Streak of the (already pushed) momentum u, offset units.
__device__ __forceinline__ void em_streak(const EmArgs &a, const double uu[3], double d[3]) {
    const double rg = dvd(1.0, __dsqrt_rn(add(1.0, add(add(mul(uu[0], uu[0]), mul(uu[1], uu[1])),
                                                         mul(uu[2], uu[2])))));
    d[0] = mul(a.cdt[0], mul(uu[0], rg));
    d[1] = mul(a.cdt[1], mul(uu[1], rg));
    d[2] = mul(a.cdt[2], mul(uu[2], rg));
}

// Slabs: a cell of another rank (cells outside [c0, c1))
__device__ __forceinline__ bool em_foreign(const EmArgs &a, int c) {
    return (long long)c < a.c0 || (long long)c >= a.c1;
}
// Record migrants (warp-aggregated append): index, face point, rest of the
// streak, new cell, crossings so far; the particle's slot becomes a hole.
__device__ __forceinline__ void em_mig_push(const EmArgs &a, bool pred, long long i, const double p[3],
                                            const double d[3], int c, int k) {
    const unsigned FULL = 0xffffffffu, lane = threadIdx.x & 31u;
    const unsigned m = __ballot_sync(FULL, pred);
    if (!m) return;
    unsigned long long base = 0;
    const int leader = __ffs(m) - 1;
    if ((int)lane == leader) base = atomicAdd(a.mig_n, (unsigned long long)__popc(m));
    base = __shfl_sync(FULL, base, leader);
    if (pred) {
        const unsigned long long sl = base + __popc(m & ((1u << lane) - 1u));
        a.mig_i[sl] = (uint32_t)i;
        for (int ax = 0; ax < 3; ax++) {
            a.mig_p[ax * a.mig_cap + sl] = p[ax];
            a.mig_d[ax * a.mig_cap + sl] = d[ax];
        }
        a.mig_c[sl] = c;
        a.mig_k[sl] = k;
        a.cell[i] = -1;
    }
}

// Per-warp queue of particles still crossing faces (OPP_EM_QUEUE): their later
// move rounds run in batches of 32, so a round never runs for a handful of
// lanes (a round costs the warp the same ~250 instructions for 2 lanes as
// for 32).  Ring of kEmQ slots in shared memory: position, remaining streak,
// cell, crossings so far, particle index.
constexpr int kEmQ = 64;
struct EmQueue {
    double *p[3], *d[3];
    int *c, *k, *i;
    unsigned head, tail;   // warp-uniform
    __device__ __forceinline__ unsigned count() const { return tail - head; }
    __device__ __forceinline__ void push(bool pred, const double pp[3], const double dd[3], int cc,
                                         int kk, int ii) {
        const unsigned m = __ballot_sync(0xffffffffu, pred);
        if (!m) return;
        const unsigned lane = threadIdx.x & 31u;
        if (pred) {
            const unsigned sl = (tail + __popc(m & ((1u << lane) - 1u))) & (kEmQ - 1);
            p[0][sl] = pp[0]; p[1][sl] = pp[1]; p[2][sl] = pp[2];
            d[0][sl] = dd[0]; d[1][sl] = dd[1]; d[2][sl] = dd[2];
            c[sl] = cc; k[sl] = kk; i[sl] = ii;
        }
        tail += __popc(m);
        __syncwarp();
    }
};
constexpr int kEmQBytes = kEmQ * (6 * 8 + 3 * 4);                  // per warp
constexpr int kEmBufBytes = kEmNA * kEmBufLd * 8;                   // per warp
#ifndef OPP_EM_QUEUE
#define OPP_EM_QUEUE 1   // C3: 4.16 -> 3.77 ms with direct reductions for the queued rounds
#endif
#ifndef OPP_EM_QDEP
#define OPP_EM_QDEP 0    // 1: warp-aggregated deposits for queued rounds (scattered cells: 4.56 ms)
#endif

#ifndef OPP_EM_MINB
#define OPP_EM_MINB 3   // resident blocks per SM (80 registers); 4 spills and measured slower
#endif
// One move round for up to 32 queued particles (lane j takes entry head + j).
template <int DEP, bool SLAB>
__device__ __forceinline__ void em_queue_round(const EmArgs &a, EmQueue &qs, double *wbuf,
                                               unsigned long long &ncross, unsigned long long &ncap,
                                               unsigned &maxk) {
    const unsigned lane = threadIdx.x & 31u;
    const unsigned take = min(32u, qs.count());
    const bool has = lane < take;
    double p[3] = {0, 0, 0}, d[3] = {0, 0, 0};
    int c = 0, k = 0, i = 0;
    if (has) {
        const unsigned sl = (qs.head + lane) & (kEmQ - 1);
        p[0] = qs.p[0][sl]; p[1] = qs.p[1][sl]; p[2] = qs.p[2][sl];
        d[0] = qs.d[0][sl]; d[1] = qs.d[1][sl]; d[2] = qs.d[2][sl];
        c = qs.c[sl]; k = qs.k[sl]; i = qs.i[sl];
    }
    __syncwarp();
    qs.head += take;
    double v[kEmNA], q[3] = {p[0], p[1], p[2]};
    int face = -1;
    if (has) {
        face = em_face(p, d, q);
        seg_current(p, q, mul(a.qsp, __ldg(a.w + i)), v);
    } else {
#pragma unroll
        for (int s = 0; s < kEmNA; s++) v[s] = 0.0;
    }
    // queued particles sit in scattered cells: direct reductions (OPP_EM_QDEP=1: warp-aggregated)
    em_deposit<OPP_EM_QDEP ? DEP : 0>(a.acc, has, c, v, wbuf);
    bool again = false, capped = false, migr = false;
    if (has) {
        if (face >= 0 && k < a.kcap) {
            em_cross(p, d, q, face, c, a.c2c);
            k++;
            if (SLAB && em_foreign(a, c)) migr = true;
            else again = true;
        } else {
            capped = face >= 0;
            a.off[i] = q[0]; a.off[a.cap + i] = q[1]; a.off[2 * a.cap + i] = q[2];
            a.cell[i] = c;
            ncross += (unsigned)k;
            ncap += capped;
            maxk = max(maxk, (unsigned)k);
        }
    }
    if (SLAB) em_mig_push(a, migr, i, p, d, c, k);
    qs.push(again, p, d, c, k, i);
}

// SLAB: this rank owns cells [c0, c1); a walk entering another rank's cell
// stops there and migrates (the single-domain instance has none of it).
template <int DEP, bool QUEUE, bool SLAB>
__global__ void __launch_bounds__(256, OPP_EM_MINB) k_em_move_deposit(EmArgs a) {
    const unsigned FULL = 0xffffffffu, lane = threadIdx.x & 31u;
    extern __shared__ __align__(16) char em_dyn[];   // per warp: transpose buffer, then the queue
    char *wbase = em_dyn + (size_t)(threadIdx.x >> 5) * (kEmBufBytes + (QUEUE ? kEmQBytes : 0));
    double *wbuf = reinterpret_cast<double *>(wbase);
    EmQueue qs{};
    if (QUEUE) {
        char *qb = wbase + kEmBufBytes;
        for (int a_ = 0; a_ < 3; a_++) qs.p[a_] = reinterpret_cast<double *>(qb + a_ * kEmQ * 8);
        for (int a_ = 0; a_ < 3; a_++) qs.d[a_] = reinterpret_cast<double *>(qb + (3 + a_) * kEmQ * 8);
        qs.c = reinterpret_cast<int *>(qb + 6 * kEmQ * 8);
        qs.k = qs.c + kEmQ;
        qs.i = qs.k + kEmQ;
        qs.head = qs.tail = 0;
    }
    const long long nwarps = (long long)gridDim.x * (blockDim.x >> 5);
    const long long gw = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    unsigned long long ncross = 0, ncap = 0;
    unsigned maxk = 0;
    for (long long base = gw * 32; base < a.n; base += nwarps * 32) {
        const long long i = base + lane;
        const bool valid = i < a.n;
        int c = 0;
        double p[3] = {0, 0, 0}, uu[3] = {0, 0, 0}, w = 0;
        if (valid) {
            c = a.cell[i];
            p[0] = a.off[i]; p[1] = a.off[a.cap + i]; p[2] = a.off[2 * a.cap + i];
            uu[0] = a.u[i]; uu[1] = a.u[a.cap + i]; uu[2] = a.u[2 * a.cap + i];
            w = a.w[i];
        }
        double d[3] = {0, 0, 0};
        double Q = 0;
        if (valid) {
            // 1. interpolate E, B at the offsets (oracle em_fields order)
            const double *f = a.interp + (long long)kEmNI * c;
            double F[kEmNI];
#pragma unroll
            for (int k = 0; k < kEmNI / 2; k++) {
                const double2 t = ldnc2(f + 2 * k);
                F[2 * k] = t.x;
                F[2 * k + 1] = t.y;
            }
            const double x = p[0], y = p[1], z = p[2];
            const double Ex = add(add(F[0], mul(y, F[1])), mul(z, add(F[2], mul(y, F[3]))));
            const double Ey = add(add(F[4], mul(z, F[5])), mul(x, add(F[6], mul(z, F[7]))));
            const double Ez = add(add(F[8], mul(x, F[9])), mul(y, add(F[10], mul(x, F[11]))));
            const double Bx = add(F[12], mul(x, F[13]));
            const double By = add(F[14], mul(y, F[15]));
            const double Bz = add(F[16], mul(z, F[17]));
            // 2. Boris (oracle em_boris order)
            const double q2 = a.qdt_2mc;
            const double h0 = mul(q2, Ex), h1 = mul(q2, Ey), h2 = mul(q2, Ez);
            double m0 = add(uu[0], h0), m1 = add(uu[1], h1), m2 = add(uu[2], h2);
            const double gam = __dsqrt_rn(add(1.0, add(add(mul(m0, m0), mul(m1, m1)), mul(m2, m2))));
            const double r = dvd(q2, gam);
            const double t0 = mul(r, Bx), t1 = mul(r, By), t2 = mul(r, Bz);
            const double tt = add(add(mul(t0, t0), mul(t1, t1)), mul(t2, t2));
            const double p0 = add(m0, sub(mul(m1, t2), mul(m2, t1)));
            const double p1 = add(m1, sub(mul(m2, t0), mul(m0, t2)));
            const double p2 = add(m2, sub(mul(m0, t1), mul(m1, t0)));
            const double sc = dvd(2.0, add(1.0, tt));
            const double s0 = mul(sc, t0), s1 = mul(sc, t1), s2 = mul(sc, t2);
            m0 = add(m0, sub(mul(p1, s2), mul(p2, s1)));
            m1 = add(m1, sub(mul(p2, s0), mul(p0, s2)));
            m2 = add(m2, sub(mul(p0, s1), mul(p1, s0)));
            uu[0] = add(m0, h0); uu[1] = add(m1, h1); uu[2] = add(m2, h2);
            // 3. streak in offset units
            em_streak(a, uu, d);
            Q = mul(a.qsp, w);
            a.u[i] = uu[0]; a.u[a.cap + i] = uu[1]; a.u[2 * a.cap + i] = uu[2];
        }
        // 4. move through the faces crossed; one segment per lane per round,
        //    deposited warp-aggregated (rounds continue while any lane moves);
        //    QUEUE: a particle that crosses a face continues in the warp's queue
        bool moving = valid;
        int k = 0;
        bool capped = false, queued = false, migr = false;
        while (__any_sync(FULL, moving)) {
            double v[kEmNA];
            int face = -1;
            double q[3] = {p[0], p[1], p[2]};
            if (moving) {
                face = em_face(p, d, q);
                seg_current(p, q, Q, v);
            } else {
#pragma unroll
                for (int s = 0; s < kEmNA; s++) v[s] = 0.0;
            }
            em_deposit<DEP>(a.acc, moving, c, v, wbuf);
            if (moving) {
                if (face < 0) {
                    p[0] = q[0]; p[1] = q[1]; p[2] = q[2];
                    moving = false;
                } else if (k >= a.kcap) {
                    p[0] = q[0]; p[1] = q[1]; p[2] = q[2];
                    capped = true;
                    moving = false;
                } else {
                    em_cross(p, d, q, face, c, a.c2c);
                    k++;
                    if (SLAB && em_foreign(a, c)) {   // slab: the rest of the walk is another rank's
                        migr = true;
                        moving = false;
                    } else if (QUEUE) {
                        queued = true;
                        moving = false;
                    }
                }
            }
        }
        if (SLAB) em_mig_push(a, migr, i, p, d, c, k);
        if (valid && !queued && !migr) {
            a.off[i] = p[0]; a.off[a.cap + i] = p[1]; a.off[2 * a.cap + i] = p[2];
            a.cell[i] = c;
            ncross += (unsigned)k;
            ncap += capped;
            maxk = max(maxk, (unsigned)k);
        }
        if (QUEUE) {
            qs.push(queued, p, d, c, k, (int)i);
            while (qs.count() >= 32) em_queue_round<DEP, SLAB>(a, qs, wbuf, ncross, ncap, maxk);
        }
    }
    if (QUEUE)
        while (qs.count() > 0) em_queue_round<DEP, SLAB>(a, qs, wbuf, ncross, ncap, maxk);
    const unsigned sc = __reduce_add_sync(FULL, (unsigned)ncross);
    const unsigned scap = __reduce_add_sync(FULL, (unsigned)ncap);
    const unsigned mk = __reduce_max_sync(FULL, maxk);
    if (lane == 0) {
        if (sc) atomicAdd(&a.cnt->n_crossings, (unsigned long long)sc);
        if (scap) atomicAdd(&a.cnt->n_capped, (unsigned long long)scap);
        if (mk) atomicMax(&a.cnt->max_crossings, mk);
    }
}

// Slabs: particles received from another rank resume their walk -- from the
// face point (off) in their new cell with the rest of the streak d and the
// crossings k -- one per lane, depositing every segment directly (they are
// few and in scattered cells); one that enters yet another rank's cell
// migrates again.  The segment sequence is the one the single-domain kernel
// walks, so deposits and final states are those of one domain.
__global__ void __launch_bounds__(256) k_em_continue(EmArgs a, long long first, long long m,
                                                     const double *__restrict__ dbuf,
                                                     const int32_t *__restrict__ kbuf) {
    const unsigned FULL = 0xffffffffu, lane = threadIdx.x & 31u;
    unsigned long long ncross = 0, ncap = 0;
    unsigned maxk = 0;
    const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
    for (long long base = ((long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < m;
         base += nw * 32) {
        const long long t = base + lane;
        const bool valid = t < m;
        const long long i = first + t;
        int c = 0, k = 0;
        double p[3] = {0, 0, 0}, d[3] = {0, 0, 0}, Q = 0;
        if (valid) {
            c = a.cell[i];
            p[0] = a.off[i]; p[1] = a.off[a.cap + i]; p[2] = a.off[2 * a.cap + i];
            d[0] = dbuf[t]; d[1] = dbuf[m + t]; d[2] = dbuf[2 * m + t];
            k = kbuf[t];
            Q = mul(a.qsp, a.w[i]);
        }
        bool moving = valid, capped = false, migr = false;
        while (moving) {
            double v[kEmNA], q[3];
            const int face = em_face(p, d, q);
            seg_current(p, q, Q, v);
            double *acc = a.acc + (long long)kEmNA * c;
#pragma unroll
            for (int s_ = 0; s_ < kEmNA; s_++) atomicAdd(acc + s_, v[s_]);
            if (face < 0 || k >= a.kcap) {
                p[0] = q[0]; p[1] = q[1]; p[2] = q[2];
                capped = face >= 0;
                moving = false;
            } else {
                em_cross(p, d, q, face, c, a.c2c);
                k++;
                if (em_foreign(a, c)) {
                    migr = true;
                    moving = false;
                }
            }
        }
        em_mig_push(a, migr, i, p, d, c, k);
        if (valid && !migr) {
            a.off[i] = p[0]; a.off[a.cap + i] = p[1]; a.off[2 * a.cap + i] = p[2];
            a.cell[i] = c;
            ncross += (unsigned)k;
            ncap += capped;
            maxk = max(maxk, (unsigned)k);
        }
    }
    const unsigned sc = __reduce_add_sync(FULL, (unsigned)ncross);
    const unsigned scap = __reduce_add_sync(FULL, (unsigned)ncap);
    const unsigned mk = __reduce_max_sync(FULL, maxk);
    if (lane == 0) {
        if (sc) atomicAdd(&a.cnt->n_crossings, (unsigned long long)sc);
        if (scap) atomicAdd(&a.cnt->n_capped, (unsigned long long)scap);
        if (mk) atomicMax(&a.cnt->max_crossings, mk);
    }
}

__device__ __forceinline__ int em_owner(const EmRanges &rr, long long c) {
    for (int r = 0; r < rr.n; r++)
        if (c >= rr.lo[r] && c < rr.lo[r + 1]) return r;
    return -1;
}

__global__ void k_em_mig_count(EmArgs a, EmRanges rr, unsigned long long *counts) {
    __shared__ unsigned long long sc[kEmMaxRanks];
    for (int r = threadIdx.x; r < rr.n; r += blockDim.x) sc[r] = 0;
    __syncthreads();
    const unsigned long long m = *a.mig_n;
    for (unsigned long long j = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; j < m;
         j += (unsigned long long)gridDim.x * blockDim.x) {
        const int o = em_owner(rr, a.mig_c[j]);
        if (o >= 0) atomicAdd(&sc[o], 1ull);
    }
    __syncthreads();
    for (int r = threadIdx.x; r < rr.n; r += blockDim.x)
        if (sc[r]) atomicAdd(&counts[r], sc[r]);
}

__global__ void k_em_mig_pack(EmArgs a, EmRanges rr, unsigned long long *cursor,
                              const long long *__restrict__ id, EmRecord *out, uint32_t *holes) {
    const unsigned long long m = *a.mig_n;
    for (unsigned long long j = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; j < m;
         j += (unsigned long long)gridDim.x * blockDim.x) {
        const int o = em_owner(rr, a.mig_c[j]);
        const long long i = a.mig_i[j];
        holes[j] = (uint32_t)i;
        if (o < 0) continue;
        EmRecord r;
        for (int ax = 0; ax < 3; ax++) {
            r.p[ax] = a.mig_p[ax * a.mig_cap + j];
            r.d[ax] = a.mig_d[ax * a.mig_cap + j];
            r.u[ax] = a.u[ax * a.cap + i];
        }
        r.w = a.w[i];
        r.id = id ? id[i] : i;
        r.cell = a.mig_c[j];
        r.k = a.mig_k[j];
        out[atomicAdd(&cursor[o], 1ull)] = r;
    }
}

__global__ void k_em_mig_unpack(EmArgs a, long long *id, const EmRecord *__restrict__ in, long long first,
                                long long m, double *dbuf, int32_t *kbuf) {
    for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < m;
         t += (long long)gridDim.x * blockDim.x) {
        const EmRecord r = in[t];
        const long long i = first + t;
        for (int ax = 0; ax < 3; ax++) {
            a.off[ax * a.cap + i] = r.p[ax];
            a.u[ax * a.cap + i] = r.u[ax];
            dbuf[ax * m + t] = r.d[ax];
        }
        const_cast<double *>(a.w)[i] = r.w;
        if (id) id[i] = r.id;
        a.cell[i] = r.cell;
        kbuf[t] = r.k;
    }
}

// ---------------------------------------------------------------------------
// Field side: AccumulateCurrent, AdvanceB, AdvanceE on the
// Yee-staggered periodic grid, neighbours read through c2c (f = -x,+x,-y,+y,
// -z,+z).  One thread per cell; the oracle's operation order (oracle/em_field.py)
// so results are bit-identical.  E_a / J_a live on the cell's edge along a at
// the (-,-) corner of its transverse offsets, B_a on its face at offset -1.
// ---------------------------------------------------------------------------
__global__ void k_em_accumulate_current(const double *__restrict__ acc,
                                        const int32_t *__restrict__ c2c, long long nc, double sx,
                                        double sy, double sz, double *__restrict__ J, long long c0,
                                        long long c1) {
    for (long long c = c0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; c < c1;
         c += (long long)gridDim.x * blockDim.x) {
        const int *nb = c2c + 6 * c;
        const int xm = nb[0], ym = nb[2], zm = nb[4];
        const int ymzm = __ldg(c2c + 6 * (long long)ym + 4);   // (j-1, k-1)
        const int xmzm = __ldg(c2c + 6 * (long long)xm + 4);   // (i-1, k-1)
        const int xmym = __ldg(c2c + 6 * (long long)xm + 2);   // (i-1, j-1)
        const double *A = acc;
        // x edge: cells (i,j,k) (-,-), (i,j-1,k) (+,-), (i,j,k-1) (-,+), (i,j-1,k-1) (+,+)
        double jx = add(add(add(A[kEmNA * c + 0], A[kEmNA * (long long)ym + 1]),
                            A[kEmNA * (long long)zm + 2]), A[kEmNA * (long long)ymzm + 3]);
        // y edge (transverse z, x): (i,j,k), (i,j,k-1), (i-1,j,k), (i-1,j,k-1)
        double jy = add(add(add(A[kEmNA * c + 4], A[kEmNA * (long long)zm + 5]),
                            A[kEmNA * (long long)xm + 6]), A[kEmNA * (long long)xmzm + 7]);
        // z edge (transverse x, y): (i,j,k), (i-1,j,k), (i,j-1,k), (i-1,j-1,k)
        double jz = add(add(add(A[kEmNA * c + 8], A[kEmNA * (long long)xm + 9]),
                            A[kEmNA * (long long)ym + 10]), A[kEmNA * (long long)xmym + 11]);
        J[c] = dvd(jx, sx);
        J[nc + c] = dvd(jy, sy);
        J[2 * nc + c] = dvd(jz, sz);
    }
}

__global__ void k_em_advance_b(const double *__restrict__ e, double *__restrict__ b,
                               const int32_t *__restrict__ c2c, long long nc, double hx, double hy,
                               double hz, double fdt, long long c0, long long c1) {
    for (long long c = c0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; c < c1;
         c += (long long)gridDim.x * blockDim.x) {
        const int *nb = c2c + 6 * c;
        const long long xp = nb[1], yp = nb[3], zp = nb[5];
        const double ex = e[c], ey = e[nc + c], ez = e[2 * nc + c];
        const double cx = sub(dvd(sub(e[2 * nc + yp], ez), hy), dvd(sub(e[nc + zp], ey), hz));
        const double cy = sub(dvd(sub(e[zp], ex), hz), dvd(sub(e[2 * nc + xp], ez), hx));
        const double cz = sub(dvd(sub(e[nc + xp], ey), hx), dvd(sub(e[yp], ex), hy));
        b[c] = sub(b[c], mul(fdt, cx));
        b[nc + c] = sub(b[nc + c], mul(fdt, cy));
        b[2 * nc + c] = sub(b[2 * nc + c], mul(fdt, cz));
    }
}

__global__ void k_em_advance_e(double *__restrict__ e, const double *__restrict__ b,
                               const double *__restrict__ J, const int32_t *__restrict__ c2c,
                               long long nc, double hx, double hy, double hz, double dt, long long c0,
                               long long c1) {
    for (long long c = c0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; c < c1;
         c += (long long)gridDim.x * blockDim.x) {
        const int *nb = c2c + 6 * c;
        const long long xm = nb[0], ym = nb[2], zm = nb[4];
        const double bx = b[c], by = b[nc + c], bz = b[2 * nc + c];
        const double cx = sub(dvd(sub(bz, b[2 * nc + ym]), hy), dvd(sub(by, b[nc + zm]), hz));
        const double cy = sub(dvd(sub(bx, b[zm]), hz), dvd(sub(bz, b[2 * nc + xm]), hx));
        const double cz = sub(dvd(sub(by, b[nc + xm]), hx), dvd(sub(bx, b[ym]), hy));
        e[c] = add(e[c], mul(dt, sub(cx, J[c])));
        e[nc + c] = add(e[nc + c], mul(dt, sub(cy, J[nc + c])));
        e[2 * nc + c] = add(e[2 * nc + c], mul(dt, sub(cz, J[2 * nc + c])));
    }
}

}  // namespace

static int em_grid(long long n) { return (int)std::max(1LL, std::min<long long>((n + 255) / 256, 4096)); }

cudaError_t launch_em_accumulate_current(const double *acc, const int32_t *c2c, long long nc,
                                         const double h[3], double dt, double *J, cudaStream_t s,
                                         long long c0, long long c1) {
    if (c1 < 0) c1 = nc;
    // scale 2 dt h_b h_c, formed as the oracle forms it: (2.0 * dt) * h_b * h_c
    const double sx = 2.0 * dt * h[1] * h[2], sy = 2.0 * dt * h[2] * h[0], sz = 2.0 * dt * h[0] * h[1];
    k_em_accumulate_current<<<em_grid(c1 - c0), 256, 0, s>>>(acc, c2c, nc, sx, sy, sz, J, c0, c1);
    return cudaGetLastError();
}

cudaError_t launch_em_advance_b(const double *e, double *b, const int32_t *c2c, long long nc,
                                const double h[3], double fdt, cudaStream_t s, long long c0, long long c1) {
    if (c1 < 0) c1 = nc;
    k_em_advance_b<<<em_grid(c1 - c0), 256, 0, s>>>(e, b, c2c, nc, h[0], h[1], h[2], fdt, c0, c1);
    return cudaGetLastError();
}

cudaError_t launch_em_advance_e(double *e, const double *b, const double *J, const int32_t *c2c,
                                long long nc, const double h[3], double dt, cudaStream_t s, long long c0,
                                long long c1) {
    if (c1 < 0) c1 = nc;
    k_em_advance_e<<<em_grid(c1 - c0), 256, 0, s>>>(e, b, J, c2c, nc, h[0], h[1], h[2], dt, c0, c1);
    return cudaGetLastError();
}

cudaError_t launch_em_interpolate(int nx, int ny, int nz, const double *e, const double *b,
                                  double *interp, cudaStream_t s, long long c0, long long c1) {
    const long long nc = (long long)nx * ny * nz;
    if (c1 < 0) c1 = nc;
    k_em_interpolate<<<em_grid(c1 - c0), 256, 0, s>>>(nx, ny, nz, e, b, interp, c0, c1);
    return cudaGetLastError();
}

template <int DEP, bool QUEUE, bool SLAB>
static cudaError_t em_launch(const EmArgs &a, int nsm, cudaStream_t s) {
    const int smem = 8 * (kEmBufBytes + (QUEUE ? kEmQBytes : 0));
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_em_move_deposit<DEP, QUEUE, SLAB>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int per = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_em_move_deposit<DEP, QUEUE, SLAB>, 256, smem);
    const long long need = (a.n + 255) / 256;
    const long long grid = std::max(1LL, std::min<long long>(need, (long long)nsm * std::max(per, 1)));
    k_em_move_deposit<DEP, QUEUE, SLAB><<<(int)grid, 256, smem, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_em_move_deposit(const EmArgs &a, int nsm, cudaStream_t s) {
    const bool queue = OPP_EM_QUEUE && a.kcap > 0 && a.n < (1LL << 31);
    if (a.mig_n) {   // slabs
        if (a.dep == 1) return queue ? em_launch<1, true, true>(a, nsm, s) : em_launch<1, false, true>(a, nsm, s);
        return queue ? em_launch<0, true, true>(a, nsm, s) : em_launch<0, false, true>(a, nsm, s);
    }
    if (a.dep == 1) return queue ? em_launch<1, true, false>(a, nsm, s) : em_launch<1, false, false>(a, nsm, s);
    return queue ? em_launch<0, true, false>(a, nsm, s) : em_launch<0, false, false>(a, nsm, s);
}

cudaError_t launch_em_continue(const EmArgs &a, long long first, long long m, const double *d,
                               const int32_t *k, int nsm, cudaStream_t s) {
    if (m <= 0) return cudaSuccess;
    const long long g = std::max(1LL, std::min<long long>((m + 255) / 256, (long long)nsm * 8));
    k_em_continue<<<(int)g, 256, 0, s>>>(a, first, m, d, k);
    return cudaGetLastError();
}

cudaError_t launch_em_mig_count(const EmArgs &a, const EmRanges &rr, unsigned long long *counts,
                                cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(counts, 0, sizeof(unsigned long long) * rr.n, s);
    if (e != cudaSuccess) return e;
    k_em_mig_count<<<em_grid(a.mig_cap), 256, 0, s>>>(a, rr, counts);
    return cudaGetLastError();
}

cudaError_t launch_em_mig_pack(const EmArgs &a, const EmRanges &rr, unsigned long long *cursor,
                               const long long *id, EmRecord *out, uint32_t *holes, cudaStream_t s) {
    k_em_mig_pack<<<em_grid(a.mig_cap), 256, 0, s>>>(a, rr, cursor, id, out, holes);
    return cudaGetLastError();
}

cudaError_t launch_em_mig_unpack(const EmArgs &a, long long *id, const EmRecord *in, long long first,
                                 long long m, double *dbuf, int32_t *kbuf, cudaStream_t s) {
    if (m <= 0) return cudaSuccess;
    k_em_mig_unpack<<<em_grid(m), 256, 0, s>>>(a, id, in, first, m, dbuf, kbuf);
    return cudaGetLastError();
}

}  // namespace opp
