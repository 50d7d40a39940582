// opp_kernels.cu -- sm_100a kernels of the OP-PIC electrostatic particle loop.
//
// The hot kernel is k_push_move_deposit: one thread per particle, a
// warp-uniform grid-stride loop over the SoA particle columns, the cell
// field and the 128-B walk line gathered through the read-only path, the
// walk bounded by H_pass hops (leftovers go to a compacted worklist that
// k_move_continue finishes), and the Eq. 10 deposit as fp64 reductions
// (optionally warp-aggregated over runs of equal cells).
//
// All arithmetic that decides a result (push, barycentric coordinates, the
// overlay centre) is written with explicit round-to-nearest intrinsics
// (__dmul_rn/__dadd_rn/__dsub_rn/__ddiv_rn), so no FMA contraction happens
// regardless of compiler flags.
#include "opp_internal.h"
#include "opp_kernels.h"

#include <climits>

namespace opp {

namespace {

constexpr int ST_DONE = 0, ST_MOVE = 1, ST_REMOVE = 2, ST_MIGRATE = 3;

__device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double sub(double a, double b) { return __dsub_rn(a, b); }

struct Line {
    double g0, g1, g2, g3, g4, g5, g6, g7, g8, px, py, pz;
    int4 cc, cn;
};

__device__ __forceinline__ Line load_line(const WalkLine *__restrict__ lines, int c) {
    const double2 *L = reinterpret_cast<const double2 *>(lines + c);
    double2 a0 = __ldg(L + 0), a1 = __ldg(L + 1), a2 = __ldg(L + 2);
    double2 a3 = __ldg(L + 3), a4 = __ldg(L + 4), a5 = __ldg(L + 5);
    const int4 *I = reinterpret_cast<const int4 *>(L + 6);
    Line l;
    l.g0 = a0.x; l.g1 = a0.y; l.g2 = a1.x; l.g3 = a1.y; l.g4 = a2.x; l.g5 = a2.y;
    l.g6 = a3.x; l.g7 = a3.y; l.g8 = a4.x; l.px = a4.y; l.py = a5.x; l.pz = a5.y;
    l.cc = __ldg(I);
    l.cn = __ldg(I + 1);
    return l;
}

// Barycentric coordinates, node-relative form, fixed evaluation order.
__device__ __forceinline__ void bary(const Line &l, double x, double y, double z, double &l0,
                                     double &l1, double &l2, double &l3) {
    double d0 = sub(x, l.px), d1 = sub(y, l.py), d2 = sub(z, l.pz);
    l1 = add(add(mul(l.g0, d0), mul(l.g1, d1)), mul(l.g2, d2));
    l2 = add(add(mul(l.g3, d0), mul(l.g4, d1)), mul(l.g5, d2));
    l3 = add(add(mul(l.g6, d0), mul(l.g7, d1)), mul(l.g8, d2));
    l0 = sub(1.0, add(add(l1, l2), l3));
}

__device__ __forceinline__ bool in01(double v) { return v >= 0.0 && v <= 1.0; }

// Multi-hop walk (Fig. 6 template 1098-1124).  `cell` is a
// global id in/out; stops when inside (DONE), at H_cap (DONE, capped), when
// hops reaches stop_at (NEED_MOVE: deferred), across a boundary face
// (NEED_REMOVE) or into a cell another rank owns (NEED_MIGRATE).
template <bool MULTI>
__device__ __forceinline__ int walk(const StepArgs &a, int &cell, double x, double y, double z,
                                    int &hops, int stop_at, double &l0, double &l1, double &l2,
                                    double &l3, int &capped, int4 &cn) {
    for (;;) {
        Line L = load_line(a.lines, cell - a.cell_base);
        bary(L, x, y, z, l0, l1, l2, l3);
        cn = L.cn;
        if (in01(l0) && in01(l1) && in01(l2) && in01(l3)) return ST_DONE;
        if (hops >= a.hcap) {
            capped = 1;
            return ST_DONE;
        }
        if (hops >= stop_at) return ST_MOVE;
        int nb = L.cc.x;
        double m = l0;
        if (l1 < m) { m = l1; nb = L.cc.y; }
        if (l2 < m) { m = l2; nb = L.cc.z; }
        if (l3 < m) { nb = L.cc.w; }
        if (nb < 0) return ST_REMOVE;
        if (MULTI && (unsigned)(nb - a.cell_base) >= (unsigned)a.n_cells) {
            cell = nb;
            return ST_MIGRATE;
        }
        cell = nb;
        hops++;
    }
}

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

// Warp-aggregated append: one atomic per warp, returns this lane's slot.
__device__ __forceinline__ unsigned long long warp_append(bool pred, unsigned long long *counter) {
    unsigned m = __ballot_sync(0xffffffffu, pred);
    if (!m) return 0;
    int leader = __ffs(m) - 1;
    unsigned long long base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(counter, (unsigned long long)__popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
    return base + __popc(m & ((1u << lane_id()) - 1u));
}

// Deposit of Eq. 10: Q[c2n[cell][i]] += w * lambda_i.
// DEP 0: one fp64 reduction per (particle, node).
// DEP 1: runs of lanes with the same cell (same 4 nodes) are summed with a
//        segmented suffix scan (5 shuffle steps) and the run head issues the
//        4 reductions -- "warp-level aggregation of same-cell deposits".
template <int DEP>
__device__ __forceinline__ void deposit(double *__restrict__ Q, bool done, int cell, int4 cn,
                                        double w, double l0, double l1, double l2, double l3) {
    double v0 = mul(w, l0), v1 = mul(w, l1), v2 = mul(w, l2), v3 = mul(w, l3);
    if (DEP == 0) {
        if (done) {
            atomicAdd(Q + cn.x, v0);
            atomicAdd(Q + cn.y, v1);
            atomicAdd(Q + cn.z, v2);
            atomicAdd(Q + cn.w, v3);
        }
        return;
    }
    const unsigned lane = lane_id();
    int key = done ? cell : -2 - (int)lane;
    if (!done) { v0 = v1 = v2 = v3 = 0.0; }
    int prev = __shfl_up_sync(0xffffffffu, key, 1);
    bool head = (lane == 0) || (prev != key);
    unsigned heads = __ballot_sync(0xffffffffu, head);
    unsigned above = heads & ~((2u << lane) - 1u);   // heads strictly above this lane
    if (lane == 31) above = 0;
    int run_end = above ? (__ffs(above) - 2) : 31;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        double t0 = __shfl_down_sync(0xffffffffu, v0, off);
        double t1 = __shfl_down_sync(0xffffffffu, v1, off);
        double t2 = __shfl_down_sync(0xffffffffu, v2, off);
        double t3 = __shfl_down_sync(0xffffffffu, v3, off);
        if ((int)lane + off <= run_end) {
            v0 = add(v0, t0); v1 = add(v1, t1); v2 = add(v2, t2); v3 = add(v3, t3);
        }
    }
    if (head && done) {
        atomicAdd(Q + cn.x, v0);
        atomicAdd(Q + cn.y, v1);
        atomicAdd(Q + cn.z, v2);
        atomicAdd(Q + cn.w, v3);
    }
}

// SR deposit, phase 1: store (cell, w*lambda[4]) records.
__device__ __forceinline__ void sr_store(const StepArgs &a, bool done, int cell, double w,
                                         double l0, double l1, double l2, double l3) {
    unsigned long long slot = warp_append(done, &a.cnt->n_sr);
    if (done) {
        a.sr_cell[slot] = cell - a.cell_base;
        a.sr_val[slot] = mul(w, l0);
        a.sr_val[a.cap + slot] = mul(w, l1);
        a.sr_val[2 * a.cap + slot] = mul(w, l2);
        a.sr_val[3 * a.cap + slot] = mul(w, l3);
    }
}

// Per-warp flush of walk statistics.
__device__ __forceinline__ void flush_stats(DevCounters *c, unsigned hops, unsigned maxh,
                                            unsigned capped, unsigned removed) {
    unsigned sh = __reduce_add_sync(0xffffffffu, hops);
    unsigned mh = __reduce_max_sync(0xffffffffu, maxh);
    unsigned sc = __reduce_add_sync(0xffffffffu, capped);
    unsigned sr = __reduce_add_sync(0xffffffffu, removed);
    if (lane_id() == 0) {
        if (sh) atomicAdd(&c->total_hops, (unsigned long long)sh);
        if (mh) atomicMax(&c->max_hops, mh);
        if (sc) atomicAdd(&c->n_capped, (unsigned long long)sc);
        if (sr) atomicAdd(&c->n_removed, (unsigned long long)sr);
    }
}

// DH seed (S19): the overlay cell's tet, else unchanged.
__device__ __forceinline__ int dh_seed(const Overlay &ov, double x, double y, double z, int cell) {
    double t0 = __ddiv_rn(sub(x, ov.x0[0]), ov.dx);
    double t1 = __ddiv_rn(sub(y, ov.x0[1]), ov.dx);
    double t2 = __ddiv_rn(sub(z, ov.x0[2]), ov.dx);
    if (!(t0 >= 0.0) || !(t1 >= 0.0) || !(t2 >= 0.0)) return cell;
    double f0 = floor(t0), f1 = floor(t1), f2 = floor(t2);
    if (f0 >= (double)ov.n[0] || f1 >= (double)ov.n[1] || f2 >= (double)ov.n[2]) return cell;
    long long g = (long long)f0 + (long long)ov.n[0] * ((long long)f1 + (long long)ov.n[1] * (long long)f2);
    int s = __ldg(ov.map + g);
    return s >= 0 ? s : cell;
}

}  // namespace

// ---------------------------------------------------------------------------
// The fused push / move / deposit kernel (CalcPosVel + Move + DepositCharge,
// PAPER.md:1586-1604, fused).  CONT = continuation pass over the worklist.
// ---------------------------------------------------------------------------
template <int DEP, bool DH, bool CONT, bool MULTI>
__global__ void __launch_bounds__(256) k_push_move_deposit(StepArgs a) {
    const unsigned long long n = CONT ? *(volatile unsigned long long *)&a.cnt->n_work
                                      : *(volatile unsigned long long *)&a.cnt->n;
    const unsigned lane = lane_id();
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned my_hops = 0, my_max = 0, my_capped = 0, my_removed = 0;
    const int stop_at = CONT ? INT_MAX : a.hpass;
    for (unsigned long long i0 = (unsigned long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
         i0 < n; i0 += stride) {
        const unsigned long long k = i0 + lane;
        const bool valid = k < n;
        int status = ST_REMOVE + 100;   // "no particle"
        int cell = 0, hops = 0, capped = 0;
        double l0 = 0, l1 = 0, l2 = 0, l3 = 0;
        int4 cn = make_int4(0, 0, 0, 0);
        unsigned long long i = k;
        if (valid) {
            double x, y, z;
            if (CONT) {
                i = a.work[k];
                hops = a.work_hops[k];
                x = a.pos[i]; y = a.pos[a.cap + i]; z = a.pos[2 * a.cap + i];
                cell = a.p2c[i];
            } else {
                x = a.pos[i]; y = a.pos[a.cap + i]; z = a.pos[2 * a.cap + i];
                double vx = a.vel[i], vy = a.vel[a.cap + i], vz = a.vel[2 * a.cap + i];
                cell = a.p2c[i];
                // gather the cell-constant field, leap-frog push (569-583, 1576-1590)
                const double *Ep = reinterpret_cast<const double *>(a.ef + (cell - a.cell_base));
                const double2 Exy = __ldg(reinterpret_cast<const double2 *>(Ep));
                const double Ez = __ldg(Ep + 2);
                vx = add(vx, mul(a.c1, Exy.x));
                vy = add(vy, mul(a.c1, Exy.y));
                vz = add(vz, mul(a.c1, Ez));
                x = add(x, mul(vx, a.dt));
                y = add(y, mul(vy, a.dt));
                z = add(z, mul(vz, a.dt));
                a.pos[i] = x; a.pos[a.cap + i] = y; a.pos[2 * a.cap + i] = z;
                a.vel[i] = vx; a.vel[a.cap + i] = vy; a.vel[2 * a.cap + i] = vz;
                if (DH) cell = dh_seed(a.ov, x, y, z, cell);
            }
            status = walk<MULTI>(a, cell, x, y, z, hops, stop_at, l0, l1, l2, l3, capped, cn);
            if (status != ST_MOVE) {
                my_hops += (unsigned)hops;
                my_max = max(my_max, (unsigned)hops);
                my_capped += (unsigned)capped;
            }
            a.p2c[i] = (status == ST_REMOVE) ? -1 : cell;
            my_removed += (status == ST_REMOVE);
        }
        const bool done = valid && status == ST_DONE;
        if (DEP == 2) {
            sr_store(a, done, cell, a.w, l0, l1, l2, l3);
        } else {
            deposit<DEP>(a.Q, done, cell, cn, a.w, l0, l1, l2, l3);
        }
        // holes and the deferred-walk worklist
        const bool rem = valid && status == ST_REMOVE;
        unsigned long long hs = warp_append(rem, &a.cnt->n_holes);
        if (rem) a.holes[hs] = (uint32_t)i;
        if (!CONT) {
            const bool mv = valid && status == ST_MOVE;
            unsigned long long ws = warp_append(mv, &a.cnt->n_work);
            if (mv) {
                a.work[ws] = (uint32_t)i;
                a.work_hops[ws] = hops;
            }
        }
    }
    flush_stats(a.cnt, my_hops, my_max, my_capped, my_removed);
}

// ---------------------------------------------------------------------------
// Step prologue: zero node charge, reset the per-step counters.
// ---------------------------------------------------------------------------
__global__ void k_step_begin(double *Q, long long nn, DevCounters *c, int zero) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        c->n_before = c->n;
        c->cum_pushed += c->n;
        c->cum_steps += 1;
        c->n_inj_last = c->n_injected;
        c->n_injected = 0;
        c->n_holes = 0;
        c->n_work = 0;
        c->total_hops = 0;
        c->n_capped = 0;
        c->max_hops = 0;
        c->n_removed = 0;
        c->n_sr = 0;
        c->n_head = 0;
        c->n_tail = 0;
    }
    if (zero)
        for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nn;
             i += (long long)gridDim.x * blockDim.x)
            Q[i] = 0.0;
}

// ---------------------------------------------------------------------------
// Hole fill: N' = N - R.  Plan: holes below N' form the
// head list; tail slots [N', N) still holding a particle (p2c >= 0) form the
// tail list; both have the same length.  Move: tail[k] -> head[k].
// ---------------------------------------------------------------------------
__global__ void k_fill_plan(const uint32_t *__restrict__ holes, const int32_t *__restrict__ p2c,
                            DevCounters *c, uint32_t *head, uint32_t *tail) {
    const unsigned long long R = c->n_holes, N = c->n, Np = N - R;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long k0 = (unsigned long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
         k0 < R; k0 += stride) {
        unsigned long long k = k0 + lane_id();
        bool v = k < R;
        uint32_t h = v ? holes[k] : 0;
        bool is_head = v && h < Np;
        unsigned long long s = warp_append(is_head, &c->n_head);
        if (is_head) head[s] = h;
        bool is_tail = v && p2c[Np + k] >= 0;
        unsigned long long t = warp_append(is_tail, &c->n_tail);
        if (is_tail) tail[t] = (uint32_t)(Np + k);
    }
}

__global__ void k_fill_move(ColSet cols, DevCounters *c, const uint32_t *__restrict__ head,
                            const uint32_t *__restrict__ tail) {
    const unsigned long long m = c->n_head;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        c->n_removed_last = c->n_holes;
        c->n = c->n - c->n_holes;
        c->n_holes = 0;
    }
    for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (unsigned long long)gridDim.x * blockDim.x) {
        const unsigned long long d = head[k], s = tail[k];
        for (int j = 0; j < cols.n; j++) {
            const ColDesc cd = cols.c[j];
            for (int e = 0; e < cd.dim; e++) {
                const long long off = (long long)e * cd.cap;
                if (cd.elem_bytes == 8) {
                    long long *p = reinterpret_cast<long long *>(cd.ptr);
                    p[off + d] = p[off + s];
                } else {
                    int *p = reinterpret_cast<int *>(cd.ptr);
                    p[off + d] = p[off + s];
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------
// Injection (OPP_ITERATE_INJECTED range): AoS sources ->
// SoA columns at [N, N+n); the last block to finish commits N += n.
// ---------------------------------------------------------------------------
__global__ void k_inject(ColSet cols, long long n_inj, DevCounters *c) {
    __shared__ unsigned long long base_s;
    if (threadIdx.x == 0) base_s = *(volatile unsigned long long *)&c->n;
    __syncthreads();
    const unsigned long long base = base_s;
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < n_inj;
         k += (long long)gridDim.x * blockDim.x) {
        for (int j = 0; j < cols.n; j++) {
            const ColDesc cd = cols.c[j];
            for (int e = 0; e < cd.dim; e++) {
                const long long src = k * cd.dim + e;
                const long long dst = (long long)e * cd.cap + (long long)base + k;
                if (cd.elem_bytes == 8)
                    reinterpret_cast<long long *>(cd.ptr)[dst] =
                        reinterpret_cast<const long long *>(cols.src[j])[src];
                else
                    reinterpret_cast<int *>(cd.ptr)[dst] = reinterpret_cast<const int *>(cols.src[j])[src];
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        unsigned long long t = atomicAdd(&c->inj_done_blocks, 1ull);
        if (t == gridDim.x - 1) {
            c->n = base + (unsigned long long)n_inj;
            c->n_injected += (unsigned long long)n_inj;
            c->inj_done_blocks = 0;
            __threadfence();
        }
    }
}

// ---------------------------------------------------------------------------
// Mesh preparation (once per mesh / per field update; not on the step path).
// ---------------------------------------------------------------------------
// Walk lines: g rows = (b x c, c x a, a x b) / det with a,b,c the edges
// p1-p0, p2-p0, p3-p0 and det = a . (b x c) (Cramer's rule).
__global__ void k_build_lines(const double *__restrict__ xyz, const int32_t *__restrict__ c2n,
                              const int32_t *__restrict__ c2c, long long nc, WalkLine *out,
                              DevCounters *cnt) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < nc;
         c += (long long)gridDim.x * blockDim.x) {
        int n0 = c2n[4 * c], n1 = c2n[4 * c + 1], n2 = c2n[4 * c + 2], n3 = c2n[4 * c + 3];
        double p[3], a[3], b[3], e[3];
        for (int k = 0; k < 3; k++) {
            p[k] = xyz[3 * (long long)n0 + k];
            a[k] = sub(xyz[3 * (long long)n1 + k], p[k]);
            b[k] = sub(xyz[3 * (long long)n2 + k], p[k]);
            e[k] = sub(xyz[3 * (long long)n3 + k], p[k]);
        }
        double bxc[3] = {sub(mul(b[1], e[2]), mul(b[2], e[1])), sub(mul(b[2], e[0]), mul(b[0], e[2])),
                         sub(mul(b[0], e[1]), mul(b[1], e[0]))};
        double cxa[3] = {sub(mul(e[1], a[2]), mul(e[2], a[1])), sub(mul(e[2], a[0]), mul(e[0], a[2])),
                         sub(mul(e[0], a[1]), mul(e[1], a[0]))};
        double axb[3] = {sub(mul(a[1], b[2]), mul(a[2], b[1])), sub(mul(a[2], b[0]), mul(a[0], b[2])),
                         sub(mul(a[0], b[1]), mul(a[1], b[0]))};
        double det = add(add(mul(a[0], bxc[0]), mul(a[1], bxc[1])), mul(a[2], bxc[2]));
        if (!(det > 0.0)) atomicOr(&cnt->err_flags, 1u);
        WalkLine L;
        for (int k = 0; k < 3; k++) {
            L.g[k] = __ddiv_rn(bxc[k], det);
            L.g[3 + k] = __ddiv_rn(cxa[k], det);
            L.g[6 + k] = __ddiv_rn(axb[k], det);
            L.p0[k] = p[k];
        }
        for (int k = 0; k < 4; k++) {
            L.c2c[k] = c2c[4 * c + k];
            L.c2n[k] = c2n[4 * c + k];
        }
        out[c] = L;
    }
}

__global__ void k_pack_field(const double *__restrict__ ef, long long nc, double4 *out) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < nc;
         c += (long long)gridDim.x * blockDim.x)
        out[c] = make_double4(ef[3 * c], ef[3 * c + 1], ef[3 * c + 2], 0.0);
}

// Overlay cell-map (S19): every overlay cell whose centre lies in tet c
// (all lambda >= 0) takes min(global id); INT_MAX -> -1 afterwards.
__global__ void k_overlay_init(int32_t *map, long long n) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        map[i] = INT_MAX;
}

__global__ void k_overlay_build(const WalkLine *__restrict__ lines, const double *__restrict__ xyz,
                                long long nc, int cell_base, Overlay ov, int32_t *map) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < nc;
         c += (long long)gridDim.x * blockDim.x) {
        Line L = load_line(lines, (int)c);
        int nodes[4] = {L.cn.x, L.cn.y, L.cn.z, L.cn.w};
        double lo[3], hi[3];
        for (int k = 0; k < 3; k++) {
            lo[k] = hi[k] = xyz[3 * (long long)nodes[0] + k];
            for (int q = 1; q < 4; q++) {
                double v = xyz[3 * (long long)nodes[q] + k];
                lo[k] = fmin(lo[k], v);
                hi[k] = fmax(hi[k], v);
            }
        }
        int g0[3], g1[3];
        for (int k = 0; k < 3; k++) {
            g0[k] = max(0, (int)floor((lo[k] - ov.x0[k]) / ov.dx - 0.5) - 1);
            g1[k] = min(ov.n[k] - 1, (int)ceil((hi[k] - ov.x0[k]) / ov.dx - 0.5) + 1);
        }
        for (int gz = g0[2]; gz <= g1[2]; gz++)
            for (int gy = g0[1]; gy <= g1[1]; gy++)
                for (int gx = g0[0]; gx <= g1[0]; gx++) {
                    double x = add(ov.x0[0], mul(add((double)gx, 0.5), ov.dx));
                    double y = add(ov.x0[1], mul(add((double)gy, 0.5), ov.dx));
                    double z = add(ov.x0[2], mul(add((double)gz, 0.5), ov.dx));
                    double l0, l1, l2, l3;
                    bary(L, x, y, z, l0, l1, l2, l3);
                    if (l0 >= 0.0 && l1 >= 0.0 && l2 >= 0.0 && l3 >= 0.0)
                        atomicMin(map + gx + (long long)ov.n[0] * (gy + (long long)ov.n[1] * gz),
                                  (int)c + cell_base);
                }
    }
}

__global__ void k_overlay_finish(int32_t *map, long long n) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        if (map[i] == INT_MAX) map[i] = -1;
}

// ---------------------------------------------------------------------------
// SR deposit (Fig. 3: store values and keys -> sort by
// key -> reduce by key), with the key = local cell (dense in [0, nc)), so the
// sort is a counting sort: histogram -> exclusive scan -> scatter; the
// per-cell reduction then sums each cell's contiguous segment and the
// per-node pass gathers the 4 sums of every incident cell through a
// node->(cell,slot) CSR -- no floating-point atomics at all.
// ---------------------------------------------------------------------------
__global__ void k_sr_hist(const int32_t *__restrict__ sr_cell, const DevCounters *c,
                          unsigned *hist) {
    const unsigned long long m = c->n_sr;
    for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (unsigned long long)gridDim.x * blockDim.x)
        atomicAdd(hist + sr_cell[k], 1u);
}

// Single-block exclusive scan of nc+1 counters (nc ~ 1e6: a few microseconds).
__global__ void k_scan_1block(const unsigned *in, unsigned *out, long long n) {
    __shared__ unsigned long long warp_sums[32];
    __shared__ unsigned long long carry_s;
    if (threadIdx.x == 0) carry_s = 0;
    __syncthreads();
    for (long long base = 0; base < n; base += blockDim.x) {
        long long i = base + threadIdx.x;
        unsigned long long v = i < n ? in[i] : 0;
        unsigned long long x = v;
        for (int off = 1; off < 32; off <<= 1) {
            unsigned long long t = __shfl_up_sync(0xffffffffu, x, off);
            if ((int)lane_id() >= off) x += t;
        }
        if (lane_id() == 31) warp_sums[threadIdx.x >> 5] = x;
        __syncthreads();
        if (threadIdx.x < 32) {
            unsigned long long s = (threadIdx.x < (blockDim.x >> 5)) ? warp_sums[threadIdx.x] : 0;
            for (int off = 1; off < 32; off <<= 1) {
                unsigned long long t = __shfl_up_sync(0xffffffffu, s, off);
                if ((int)threadIdx.x >= off) s += t;
            }
            warp_sums[threadIdx.x] = s;
        }
        __syncthreads();
        unsigned long long wpre = (threadIdx.x >> 5) ? warp_sums[(threadIdx.x >> 5) - 1] : 0;
        unsigned long long carry = carry_s;
        if (i < n) out[i] = (unsigned)(carry + wpre + x - v);
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry_s = carry + wpre + x;
        __syncthreads();
    }
}

__global__ void k_sr_scatter(const int32_t *__restrict__ sr_cell, const double *__restrict__ sr_val,
                             long long cap, const DevCounters *c, unsigned *cursor,
                             double *sorted) {
    const unsigned long long m = c->n_sr;
    for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (unsigned long long)gridDim.x * blockDim.x) {
        unsigned pos = atomicAdd(cursor + sr_cell[k], 1u);
        sorted[4ull * pos + 0] = sr_val[k];
        sorted[4ull * pos + 1] = sr_val[cap + k];
        sorted[4ull * pos + 2] = sr_val[2 * cap + k];
        sorted[4ull * pos + 3] = sr_val[3 * cap + k];
    }
}

// per-cell reduce: cellsum[c][i] = sum over the cell's segment
__global__ void k_sr_cell_reduce(const unsigned *__restrict__ start, const double *__restrict__ sorted,
                                 long long nc, double *cellsum) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < nc;
         c += (long long)gridDim.x * blockDim.x) {
        unsigned b = start[c], e = start[c + 1];
        double s0 = 0, s1 = 0, s2 = 0, s3 = 0;
        for (unsigned k = b; k < e; k++) {
            const double4 v = *reinterpret_cast<const double4 *>(sorted + 4ull * k);
            s0 = add(s0, v.x); s1 = add(s1, v.y); s2 = add(s2, v.z); s3 = add(s3, v.w);
        }
        *reinterpret_cast<double4 *>(cellsum + 4 * c) = make_double4(s0, s1, s2, s3);
    }
}

// per-node gather over the node -> (4*cell + slot) CSR; Q[n] (+)= sum
__global__ void k_sr_node_gather(const int32_t *__restrict__ n2cs_ptr, const int32_t *__restrict__ n2cs,
                                 const double *__restrict__ cellsum, long long nn, double *Q) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < nn;
         v += (long long)gridDim.x * blockDim.x) {
        double s = 0.0;
        for (int k = n2cs_ptr[v]; k < n2cs_ptr[v + 1]; k++) s = add(s, cellsum[n2cs[k]]);
        Q[v] = add(Q[v], s);
    }
}

// ---------------------------------------------------------------------------
// Launchers (host side of this translation unit)
// ---------------------------------------------------------------------------
template <int DEP, bool DH, bool CONT, bool MULTI>
static cudaError_t launch_pmd_t(const StepArgs &a, int grid, cudaStream_t s) {
    k_push_move_deposit<DEP, DH, CONT, MULTI><<<grid, 256, 0, s>>>(a);
    return cudaGetLastError();
}

template <bool CONT>
static cudaError_t launch_pmd_c(int dep, bool dh, bool multi, const StepArgs &a, int grid,
                                cudaStream_t s) {
#define OPP_CASE(D, H, M) \
    if (dep == D && dh == H && multi == M) return launch_pmd_t<D, H, CONT, M>(a, grid, s);
    OPP_CASE(0, false, false) OPP_CASE(0, true, false) OPP_CASE(1, false, false)
    OPP_CASE(1, true, false) OPP_CASE(2, false, false) OPP_CASE(2, true, false)
    OPP_CASE(0, false, true) OPP_CASE(0, true, true) OPP_CASE(1, false, true)
    OPP_CASE(1, true, true) OPP_CASE(2, false, true) OPP_CASE(2, true, true)
#undef OPP_CASE
    return cudaErrorInvalidValue;
}

cudaError_t launch_push_move_deposit(int dep, bool dh, bool multi, bool cont, const StepArgs &a,
                                     int grid, cudaStream_t s) {
    return cont ? launch_pmd_c<true>(dep, dh, multi, a, grid, s)
                : launch_pmd_c<false>(dep, dh, multi, a, grid, s);
}

int pmd_blocks_per_sm(int dep, bool dh) {
    int nb = 0;
    cudaError_t e;
    if (dep == 1)
        e = dh ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_push_move_deposit<1, true, false, false>, 256, 0)
               : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_push_move_deposit<1, false, false, false>, 256, 0);
    else
        e = dh ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_push_move_deposit<0, true, false, false>, 256, 0)
               : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_push_move_deposit<0, false, false, false>, 256, 0);
    return (e == cudaSuccess && nb > 0) ? nb : 1;
}

cudaError_t launch_step_begin(double *Q, long long nn, DevCounters *c, int zero, int grid,
                              cudaStream_t s) {
    k_step_begin<<<grid, 256, 0, s>>>(Q, nn, c, zero);
    return cudaGetLastError();
}

cudaError_t launch_fill(const ColSet &cols, DevCounters *c, const uint32_t *holes,
                        const int32_t *p2c, uint32_t *head, uint32_t *tail, int grid,
                        cudaStream_t s) {
    k_fill_plan<<<grid, 256, 0, s>>>(holes, p2c, c, head, tail);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    k_fill_move<<<grid, 256, 0, s>>>(cols, c, head, tail);
    return cudaGetLastError();
}

cudaError_t launch_inject(const ColSet &cols, long long n, DevCounters *c, int grid, cudaStream_t s) {
    k_inject<<<grid, 256, 0, s>>>(cols, n, c);
    return cudaGetLastError();
}

cudaError_t launch_build_lines(const double *xyz, const int32_t *c2n, const int32_t *c2c,
                               long long nc, WalkLine *out, DevCounters *cnt, cudaStream_t s) {
    int grid = (int)((nc + 255) / 256);
    if (grid < 1) grid = 1;
    k_build_lines<<<grid, 256, 0, s>>>(xyz, c2n, c2c, nc, out, cnt);
    return cudaGetLastError();
}

cudaError_t launch_pack_field(const double *ef, long long nc, double4 *out, cudaStream_t s) {
    int grid = (int)((nc + 255) / 256);
    if (grid < 1) grid = 1;
    k_pack_field<<<grid, 256, 0, s>>>(ef, nc, out);
    return cudaGetLastError();
}

cudaError_t launch_overlay(const WalkLine *lines, const double *xyz, long long nc, int cell_base,
                           const Overlay &ov, int32_t *map, cudaStream_t s) {
    long long tot = (long long)ov.n[0] * ov.n[1] * ov.n[2];
    int g1 = (int)((tot + 255) / 256), g2 = (int)((nc + 255) / 256);
    k_overlay_init<<<g1 > 0 ? g1 : 1, 256, 0, s>>>(map, tot);
    k_overlay_build<<<g2 > 0 ? g2 : 1, 256, 0, s>>>(lines, xyz, nc, cell_base, ov, map);
    k_overlay_finish<<<g1 > 0 ? g1 : 1, 256, 0, s>>>(map, tot);
    return cudaGetLastError();
}

cudaError_t launch_sr(const StepArgs &a, long long nc, long long nn, unsigned *hist,
                      unsigned *start, double *sorted, double *cellsum, const int32_t *n2cs_ptr,
                      const int32_t *n2cs, int grid, cudaStream_t s) {
    cudaMemsetAsync(hist, 0, sizeof(unsigned) * (nc + 1), s);
    k_sr_hist<<<grid, 256, 0, s>>>(a.sr_cell, a.cnt, hist);
    k_scan_1block<<<1, 1024, 0, s>>>(hist, start, nc + 1);
    cudaMemcpyAsync(hist, start, sizeof(unsigned) * (nc + 1), cudaMemcpyDeviceToDevice, s);
    k_sr_scatter<<<grid, 256, 0, s>>>(a.sr_cell, a.sr_val, a.cap, a.cnt, hist, sorted);
    int gc = (int)((nc + 255) / 256), gn = (int)((nn + 255) / 256);
    k_sr_cell_reduce<<<gc > 0 ? gc : 1, 256, 0, s>>>(start, sorted, nc, cellsum);
    k_sr_node_gather<<<gn > 0 ? gn : 1, 256, 0, s>>>(n2cs_ptr, n2cs, cellsum, nn, a.Q);
    return cudaGetLastError();
}

}  // namespace opp
