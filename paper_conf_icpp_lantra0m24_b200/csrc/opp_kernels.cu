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

#include <algorithm>
#include <climits>

namespace opp {

namespace {

constexpr int ST_DONE = 0, ST_MOVE = 1, ST_REMOVE = 2, ST_MIGRATE = 3, ST_NONE = 100;

__device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double sub(double a, double b) { return __dsub_rn(a, b); }

struct Line {
    double g0, g1, g2, g3, g4, g5, g6, g7, g8, px, py, pz;
    int4 cc, cn;
};

#ifndef OPP_LAZY_LINE
// 1: a visit loads only the 96 B lambda needs (gradients, p0: three 256-bit
// loads); the neighbour ids (c2c) are loaded by the lanes that hop and the
// node ids (c2n) by the lanes that issue the deposit reductions.  An L1 load
// costs ~8 SM cycles per 256-bit warp instruction and distinct line even for
// one active lane (scripts/micro/wf_cost.cu), so the fourth sector of every
// visit was a quarter of the walk's L1 data-pipe time.
#define OPP_LAZY_LINE 1
#endif
constexpr bool kLazyLine = OPP_LAZY_LINE != 0;

// One 128-B walk line: four 256-bit read-only loads (LDG.E.256), or the first
// three (lazy: the c2c / c2n sector is read on demand, below).
__device__ __forceinline__ Line load_line(const WalkLine *__restrict__ lines, int c) {
    const double *L = reinterpret_cast<const double *>(lines + c);
    Line l;
    asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(l.g0), "=d"(l.g1), "=d"(l.g2), "=d"(l.g3) : "l"(L));
    asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(l.g4), "=d"(l.g5), "=d"(l.g6), "=d"(l.g7) : "l"(L + 4));
    asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(l.g8), "=d"(l.px), "=d"(l.py), "=d"(l.pz) : "l"(L + 8));
    if (!kLazyLine) {
        asm("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
            : "=r"(l.cc.x), "=r"(l.cc.y), "=r"(l.cc.z), "=r"(l.cc.w),
              "=r"(l.cn.x), "=r"(l.cn.y), "=r"(l.cn.z), "=r"(l.cn.w) : "l"(L + 12));
    }
    return l;
}

// c2c of local cell c (walk line bytes 96..111) and c2n (112..127).
__device__ __forceinline__ int4 line_c2c(const WalkLine *__restrict__ lines, int c) {
    return __ldg(reinterpret_cast<const int4 *>(reinterpret_cast<const double *>(lines + c) + 12));
}
__device__ __forceinline__ int4 line_c2n(const WalkLine *__restrict__ lines, int c) {
    return __ldg(reinterpret_cast<const int4 *>(reinterpret_cast<const double *>(lines + c) + 14));
}
__device__ __forceinline__ int line_node(const WalkLine *__restrict__ lines, int c, int q) {
    return __ldg(reinterpret_cast<const int *>(reinterpret_cast<const double *>(lines + c) + 14) + q);
}
// the neighbours of the cell whose line L is (lc: its local index)
__device__ __forceinline__ int4 cc_of(const WalkLine *__restrict__ lines, const Line &L, int lc) {
    return kLazyLine ? line_c2c(lines, lc) : L.cc;
}

// Cell field E (double4, 32-B aligned): one 256-bit read-only load, or
// (OPP_E_NARROW) a 128-bit + a 64-bit load of just the 24 B used.
#ifndef OPP_E_NARROW
#define OPP_E_NARROW 0
#endif
__device__ __forceinline__ void load_E(const double4 *__restrict__ ef, int lc, double2 &exy,
                                       double &ez) {
    if (OPP_E_NARROW) {
        const double *p = reinterpret_cast<const double *>(ef + lc);
        exy = __ldg(reinterpret_cast<const double2 *>(p));
        ez = __ldg(p + 2);
        return;
    }
    double pad;
    asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(exy.x), "=d"(exy.y), "=d"(ez), "=d"(pad) : "l"(ef + lc));
}

// Overlay slot of overlay cell (ix, iy, iz): 4x4x2 bricks of 32 ints (one
// 128-B line), so the particles of one tet -- a few overlay cells in every
// direction -- touch a few lines instead of one line per (iy, iz) row.
__device__ __forceinline__ long long ov_slot32(const Overlay &ov, int ix, int iy, int iz) {
    const long long b = (long long)(ix >> 2) +
                        (long long)ov.nb[0] * ((long long)(iy >> 2) + (long long)ov.nb[1] * (iz >> 1));
    return b * 32 + (ix & 3) + 4 * (iy & 3) + 16 * (iz & 1);
}

__device__ __forceinline__ long long ov_slot16(const Overlay &ov, int ix, int iy, int iz) {
    const unsigned b = (unsigned)(ix >> 2) +
                       (unsigned)ov.nbc[0] * ((unsigned)(iy >> 2) + (unsigned)ov.nbc[1] * (unsigned)(iz >> 2));
    return (long long)b * 64 + (ix & 3) + 4 * (iy & 3) + 16 * (iz & 3);
}

// Slot of overlay cell (ix, iy, iz) in the active layout, and its tet.
__device__ __forceinline__ long long ov_slot(const Overlay &ov, int ix, int iy, int iz) {
    return ov.compact ? ov_slot16(ov, ix, iy, iz) : ov_slot32(ov, ix, iy, iz);
}
__device__ __forceinline__ int ov_value(const Overlay &ov, long long slot) {
    if (ov.compact) {   // the two loads are independent: one round trip
        const int o = __ldg(ov.off + slot);
        const int b = __ldg(ov.base + (slot >> 6));
        return o == -32768 ? -1 : b + o;
    }
    return __ldg(ov.map + slot);
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
// global id in/out and L its already-loaded walk line; stops when inside
// (DONE), at H_cap (DONE, capped), when hops reaches stop_at (NEED_MOVE:
// deferred), across a boundary face (NEED_REMOVE) or into a cell another
// rank owns (NEED_MIGRATE).
// Position source for the walk: registers, or (TMA-pipelined kernel) the
// warp's shared output buffer, re-read at every visit so the three doubles do
// not occupy registers across the line-load latency.
struct PosRegs {
    double x, y, z;
    __device__ __forceinline__ void get(double &a, double &b, double &c) const { a = x; b = y; c = z; }
};
struct PosSmem {
    const double *p;   // p[0], p[32], p[64]
    __device__ __forceinline__ void get(double &a, double &b, double &c) const {
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(a) : "r"((unsigned)__cvta_generic_to_shared(p)));
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(b) : "r"((unsigned)__cvta_generic_to_shared(p + 32)));
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(c) : "r"((unsigned)__cvta_generic_to_shared(p + 64)));
    }
};

template <bool MULTI, typename PS>
__device__ __forceinline__ int walk_from(const StepArgs &a, int &cell, Line L, const PS &ps,
                                         int &hops, int stop_at, double &l0, double &l1,
                                         double &l2, double &l3, int &capped, int4 &cn) {
    for (;;) {
        double x, y, z;
        ps.get(x, y, z);
        bary(L, x, y, z, l0, l1, l2, l3);
        cn = L.cn;
        if (in01(l0) && in01(l1) && in01(l2) && in01(l3)) return ST_DONE;
        if (hops >= a.hcap) {
            capped = 1;
            return ST_DONE;
        }
        if (hops >= stop_at) return ST_MOVE;
        const int4 cc = cc_of(a.lines, L, cell - a.cell_base);
        int nb = cc.x;
        double m = l0;
        if (l1 < m) { m = l1; nb = cc.y; }
        if (l2 < m) { m = l2; nb = cc.z; }
        if (l3 < m) { nb = cc.w; }
        if (nb < 0) return ST_REMOVE;
        if (MULTI && (unsigned)(nb - a.cell_base) >= (unsigned)a.n_cells) {
            cell = nb;       // the hop into the other rank's cell counts here
            hops++;
            return ST_MIGRATE;
        }
        cell = nb;
        hops++;
        L = load_line(a.lines, cell - a.cell_base);
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
// DEP 1: lanes with the same cell (same 4 nodes) are aggregated inside the
//        warp before one set of 4 reductions per cell -- "warp-level
//        aggregation of same-cell deposits before global atomics".
//
// Lanes with the same key are found with __match_any_sync wherever they sit
// in the warp.  A lane alone with its cell reduces straight to Q.  Each
// group of >= 2 lanes (in cell-sorted storage: the one or two cells a warp's
// slice covers, while the few particles that hopped are mostly alone) is
// summed by a full-warp reduce-scatter -- xor 16 halves the 4 values, xor 8
// halves them again, xor 4/2/1 finish -- 12 shuffles and 6 adds per group;
// lanes 0, 8, 16, 24 then hold the group's 4 sums and issue one reduction
// each.  With more than kMaxRsGroups groups a log-step tree over each group
// (lowest lane issues the 4 reductions) is cheaper.
#ifndef OPP_RS_GROUPS
#define OPP_RS_GROUPS 0   // C2: 0 (always the tree) 1.894 ms, 3: 1.912, 8: 2.35
#endif
constexpr int kMaxRsGroups = OPP_RS_GROUPS;
#ifndef OPP_DEP_MERGE
#define OPP_DEP_MERGE 1   // singles through the tree too: C2 pass 1 1.901 -> 1.849 ms, C5 2.80 -> 2.71
#endif

// Node ids of the depositing cell: from the walk line already in registers,
// or (lazy line) loaded by the lanes that issue the reductions only.
struct CnSrc {
    const WalkLine *lines;
    int base;   // cell_base: key - base is the local cell
    __device__ __forceinline__ int4 get(int key, int4 cn) const {
        return kLazyLine ? line_c2n(lines, key - base) : cn;
    }
    __device__ __forceinline__ int node(int key, int4 cn, int q) const {
        if (kLazyLine) return line_node(lines, key - base, q);
        return q == 0 ? cn.x : q == 1 ? cn.y : q == 2 ? cn.z : cn.w;
    }
};

__device__ __forceinline__ void red4(double *__restrict__ Q, int4 cn, double v0, double v1,
                                     double v2, double v3) {
    atomicAdd(Q + cn.x, v0);
    atomicAdd(Q + cn.y, v1);
    atomicAdd(Q + cn.z, v2);
    atomicAdd(Q + cn.w, v3);
}

// Log-step tree over every peer group of the lanes with `act` set.
__device__ __forceinline__ void deposit_tree(double *__restrict__ Q, bool act, unsigned peers,
                                             const CnSrc &cs, int key, int4 cn, double v0,
                                             double v1, double v2, double v3) {
    const unsigned lane = lane_id();
    const int first = __ffs(peers) - 1;
    int rel = __popc(peers & ((1u << lane) - 1u));       // my rank inside the group
    unsigned up = peers & ~((2u << lane) - 1u);           // group lanes above me
    if (lane == 31) up = 0;
    // the lowest lane of each group fetches the node ids while the tree runs
    if (act && (int)lane == first) cn = cs.get(key, cn);
    while (__any_sync(0xffffffffu, up != 0)) {
        const int next = up ? __ffs(up) - 1 : (int)lane;
        const double t0 = __shfl_sync(0xffffffffu, v0, next);
        const double t1 = __shfl_sync(0xffffffffu, v1, next);
        const double t2 = __shfl_sync(0xffffffffu, v2, next);
        const double t3 = __shfl_sync(0xffffffffu, v3, next);
        if (up) {
            v0 = add(v0, t0); v1 = add(v1, t1); v2 = add(v2, t2); v3 = add(v3, t3);
        }
        // lanes at odd group rank have been absorbed by their lower neighbour
        const unsigned gone = __ballot_sync(0xffffffffu, (rel & 1) != 0);
        up &= ~gone;
        rel >>= 1;
    }
    if (act && (int)lane == first) red4(Q, cn, v0, v1, v2, v3);
}

// Warp-aggregated deposit of (key, cn, v0..v3) for the lanes with `done`
// (key: the cell; lanes with equal keys have equal cn).
__device__ __forceinline__ void deposit_agg(double *__restrict__ Q, const CnSrc &cs, bool done,
                                            int key, int4 cn, double v0, double v1, double v2,
                                            double v3) {
    const unsigned FULL = 0xffffffffu;
    const unsigned lane = lane_id();
    const unsigned peers = __match_any_sync(FULL, done ? key : -2 - (int)lane);
    const bool single = peers == (1u << lane);
    if (OPP_DEP_MERGE && kMaxRsGroups == 0) {
        // singles ride through the tree as groups of one, so every cell's
        // four reductions leave in the same four instructions (the fixed
        // cost of a reduction instruction is paid once, not twice)
        if (__any_sync(FULL, done)) deposit_tree(Q, done, peers, cs, key, cn, v0, v1, v2, v3);
        return;
    }
    if (done && single) red4(Q, cs.get(key, cn), v0, v1, v2, v3);
    unsigned lead = __ballot_sync(FULL, done && !single && (int)lane == __ffs(peers) - 1);
    if (!lead) return;
    if (__popc(lead) > kMaxRsGroups) {
        deposit_tree(Q, done && !single, peers, cs, key, cn, v0, v1, v2, v3);
        return;
    }
    const bool h16 = (lane & 16u) != 0, h8 = (lane & 8u) != 0;
    do {
        const int L = __ffs(lead) - 1;
        lead &= lead - 1u;
        const unsigned gm = __shfl_sync(FULL, peers, L);
        const bool in = done && ((gm >> lane) & 1u);
        const double a0 = in ? v0 : 0.0, a1 = in ? v1 : 0.0, a2 = in ? v2 : 0.0, a3 = in ? v3 : 0.0;
        double k0 = h16 ? a2 : a0, k1 = h16 ? a3 : a1;    // the pair this lane keeps
        const double s0 = h16 ? a0 : a2, s1 = h16 ? a1 : a3;
        k0 = add(k0, __shfl_xor_sync(FULL, s0, 16));
        k1 = add(k1, __shfl_xor_sync(FULL, s1, 16));
        double t = h8 ? k1 : k0;
        t = add(t, __shfl_xor_sync(FULL, h8 ? k0 : k1, 8));
        t = add(t, __shfl_xor_sync(FULL, t, 4));
        t = add(t, __shfl_xor_sync(FULL, t, 2));
        t = add(t, __shfl_xor_sync(FULL, t, 1));
        // lane 8q holds the sum of value q = 2*h16 + h8
        const int q = 2 * (int)h16 + (int)h8;
        if (kLazyLine) {
            const int kL = __shfl_sync(FULL, key, L);
            if ((lane & 7u) == 0) atomicAdd(Q + cs.node(kL, cn, q), t);
        } else {
            const int n0 = __shfl_sync(FULL, cn.x, L), n1 = __shfl_sync(FULL, cn.y, L);
            const int n2 = __shfl_sync(FULL, cn.z, L), n3 = __shfl_sync(FULL, cn.w, L);
            if ((lane & 7u) == 0) {
                const int node = h16 ? (h8 ? n3 : n2) : (h8 ? n1 : n0);
                atomicAdd(Q + node, t);
            }
        }
    } while (lead);
}

template <int DEP>
__device__ __forceinline__ void deposit(double *__restrict__ Q, const CnSrc &cs, bool done,
                                        int cell, int4 cn, double w, double l0, double l1,
                                        double l2, double l3) {
    double v0 = mul(w, l0), v1 = mul(w, l1), v2 = mul(w, l2), v3 = mul(w, l3);
    if (DEP == 0) {
        if (done) red4(Q, cs.get(cell, cn), v0, v1, v2, v3);
        return;
    }
    deposit_agg(Q, cs, done, cell, cn, v0, v1, v2, v3);
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
// dh_slot: the overlay slot of a position, -1 outside the overlay box.
__device__ __forceinline__ long long dh_slot(const Overlay &ov, double x, double y, double z) {
    const double inv = ov.inv_dx;
    double t0 = mul(sub(x, ov.x0[0]), inv);
    double t1 = mul(sub(y, ov.x0[1]), inv);
    double t2 = mul(sub(z, ov.x0[2]), inv);
    if (!(t0 >= 0.0) || !(t1 >= 0.0) || !(t2 >= 0.0)) return -1;
    // floor(t) for t >= 0 as one saturating fp64 -> int conversion each (the
    // conversion unit is the slow part of this lookup; no FRND + I2F pair);
    // t >= 2^31 saturates to INT_MAX and fails the range test like floor(t).
    const int f0 = __double2int_rd(t0), f1 = __double2int_rd(t1), f2 = __double2int_rd(t2);
    if (f0 >= ov.n[0] || f1 >= ov.n[1] || f2 >= ov.n[2]) return -1;
    return ov_slot(ov, f0, f1, f2);
}

__device__ __forceinline__ int dh_seed(const Overlay &ov, double x, double y, double z, int cell) {
    const long long g = dh_slot(ov, x, y, z);
    if (g < 0) return cell;
    int s = ov_value(ov, g);
    return s >= 0 ? s : cell;
}

// DH mode 2 (reading S19''): a particle no longer inside its cell (L = its
// line) takes the overlay seed; one still inside keeps cell and line.
__device__ __forceinline__ void dh_if_left(const StepArgs &a, double x, double y, double z,
                                           int &cell, Line &L) {
    double l0, l1, l2, l3;
    bary(L, x, y, z, l0, l1, l2, l3);
    if (in01(l0) && in01(l1) && in01(l2) && in01(l3)) return;
    const int sc = dh_seed(a.ov, x, y, z, cell);
    if (sc != cell) {
        cell = sc;
        L = load_line(a.lines, sc - a.cell_base);
    }
}

}  // namespace

// ---------------------------------------------------------------------------
// Per-particle body shared by the fused kernel (both its TMA-tiled and its
// direct paths) and the continuation pass.  Must be called by full warps
// (the deposit / append collectives use all 32 lanes); `valid` masks lanes
// without a particle.  On return x..vz and cell hold what is written back
// (cell = -1 for a hole).
// ---------------------------------------------------------------------------
struct Tally {
    unsigned hops = 0, maxh = 0, capped = 0, removed = 0;
};

// Block b visits groups of K consecutive tiles round-robin: group g goes to
// block g % G.  K = 1 sweeps the array as one moving window (small L2 working
// set when storage is cell-sorted); larger K gives each SM runs of adjacent
// cells (L1 reuse) while the window stays G*K tiles.
struct TileMap {
    unsigned long long ntiles, G, K, b;
    __device__ __forceinline__ unsigned long long count() const {
        const unsigned long long ng = (ntiles + K - 1) / K;
        if (b >= ng) return 0;
        const unsigned long long nb = (ng - 1 - b) / G + 1;
        unsigned long long c = nb * K;
        if (b + (nb - 1) * G == ng - 1) c -= ng * K - ntiles;
        return c;
    }
    __device__ __forceinline__ unsigned long long tile(unsigned long long it) const {
        return ((it / K) * G + b) * K + it % K;
    }
};

// Sequential walk over a block's tiles without 64-bit divisions.
struct TileIter {
    unsigned group_first, sub, K, step;   // step = G * K; tile ids < 2^32 / kTile
    __device__ __forceinline__ TileIter(const TileMap &m)
        : group_first((unsigned)(m.b * m.K)), sub(0), K((unsigned)m.K), step((unsigned)(m.G * m.K)) {}
    __device__ __forceinline__ unsigned long long tile() const { return group_first + sub; }
    __device__ __forceinline__ void next() {
        if (++sub == K) {
            sub = 0;
            group_first += step;
        }
    }
};

// TMA-pipelined kernel geometry: tiles of kTile particles, kStages stages.
constexpr int kTile = 256;
constexpr int kConsumerWarps = kTile / 32;
constexpr int kTiledThreads = kTile + 32;
#ifndef OPP_STAGES
#define OPP_STAGES 2   // measured on C2: 2 stages leave more of the L1/shared array to
                       // L1 for the walk lines (pmd 1.91 -> 1.87 ms vs 4 stages)
#endif
#ifndef OPP_MINB_HI
#define OPP_MINB_HI 3   // resident blocks per SM the register budget is cut for
#endif
constexpr int kStages = OPP_STAGES;
constexpr int kStageBytes = kTile * (6 * 8 + 4);
constexpr int kRingBytesPerWarp = 64 * 12 + 128;   // holes ring (4 B) + work ring (4 B + 4 B hops) + lane permutation (32 x 4 B)
#ifndef OPP_SEED_PERM
#define OPP_SEED_PERM 0   // 1: regroup a warp's lanes by seed cell before the first walk-line load
                          // (C2: parity green, pass 1 1.844 -> 1.884 ms: the shuffles cost more than
                          // the cheaper line loads save -- off)
#endif
#ifndef OPP_TMA_OUT
// 0: results leave as coalesced per-lane stores (C2: pmd 1.99 vs 2.06 ms --
// staging the stores in shared memory cost L1 data-pipe wavefronts twice,
// the shared stores and the bulk copy's reads); 1: per-warp shared buffer +
// cp.async.bulk shared -> global
#define OPP_TMA_OUT 0
#endif
constexpr int kRingBase = kStages * kStageBytes + 2 * kStages * 8 +
                          (OPP_TMA_OUT ? (kTile / 32) * 32 * (6 * 8 + 4) : 0);
constexpr int kTiledSmem = kRingBase + (kTile / 32) * kRingBytesPerWarp;

struct StageView {
    double *c[6];   // x, y, z, vx, vy, vz
    int *cell;
};
__device__ __forceinline__ StageView stage_view(char *smem, int s) {
    StageView v;
    char *b = smem + (size_t)s * kStageBytes;
    for (int k = 0; k < 6; k++) v.c[k] = reinterpret_cast<double *>(b + k * kTile * 8);
    v.cell = reinterpret_cast<int *>(b + 6 * kTile * 8);
    return v;
}


// Per-warp output buffers (TMA-out): 2 x [6 x 32 doubles | 32 ints] after the
// stages and the barriers.
constexpr int kOutBytes = 32 * (6 * 8 + 4);
constexpr int kOutBase = kStages * kStageBytes + 2 * kStages * 8;

// Per-warp staging ring for appends to a global list (holes, deferred
// walks): items are buffered in shared memory and leave 32 at a time with one
// global atomic, instead of one single-address atomic per warp-iteration
// (those serialise in L2 when every warp appends).
constexpr int kRing = 64;
struct WarpRing {
    uint32_t *va;          // shared ring of values
    int32_t *vb;           // optional second value (hop counts), may be null
    unsigned head, tail;   // warp-uniform
};
struct Appends {
    WarpRing holes, work;
};

__device__ __forceinline__ void ring_push(WarpRing &r, bool pred, uint32_t va, int32_t vb) {
    const unsigned m = __ballot_sync(0xffffffffu, pred);
    if (!m) return;
    const unsigned lane = threadIdx.x & 31u;
    const unsigned slot = r.tail + __popc(m & ((1u << lane) - 1u));
    if (pred) {
        r.va[slot & (kRing - 1)] = va;
        if (r.vb) r.vb[slot & (kRing - 1)] = vb;
    }
    r.tail += __popc(m);
}

__device__ __forceinline__ void ring_flush(WarpRing &r, unsigned long long *counter, uint32_t *ga,
                                           int32_t *gb, bool all) {
    const unsigned lane = threadIdx.x & 31u;
    while (r.tail - r.head >= 32u || (all && r.tail != r.head)) {
        const unsigned k = min(32u, r.tail - r.head);
        __syncwarp();
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(counter, (unsigned long long)k);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (lane < k) {
            const unsigned sl = (r.head + lane) & (kRing - 1);
            ga[base + lane] = r.va[sl];
            if (gb) gb[base + lane] = r.vb[sl];
        }
        __syncwarp();
        r.head += k;
    }
}

__device__ __forceinline__ void mbar_arrive_fwd(uint64_t *b);
__device__ __forceinline__ void fence_proxy_async_fwd();

// Gathers of the NEXT slice issued one slice ahead by the TMA-pipelined
// consumer (OPP_PREFETCH_NEXT): the cell field and the speculative overlay
// entry only depend on the streamed state, so they leave the per-slice
// dependent chain (their latency hides behind the current slice's walk).
struct Pre {
    long long slot;
    int val;
    double2 Exy;
    double Ez;
};

// `release`: the stage mbarrier to arrive on once this warp no longer needs
// the shared-memory copy of its particles (TMA-pipelined kernel; every lane
// valid) -- after the push has consumed all seven loaded values, so no shared
// load is still pending when the producer's next bulk copy overwrites it.
template <int DEP, int DH, bool CONT, bool MULTI, bool SOUT = false>
__device__ __forceinline__ void pmd_body(const StepArgs &a, bool valid, unsigned long long i,
                                         int hops, double &x, double &y, double &z, double &vx,
                                         double &vy, double &vz, int &cell, Tally &t,
                                         uint64_t *release = nullptr, double *sout = nullptr,
                                         int sj = 0, Appends *ap = nullptr,
                                         const Pre *pre = nullptr, int *perm = nullptr) {
    int status = ST_NONE;
    int capped = 0;
    double l0 = 0, l1 = 0, l2 = 0, l3 = 0;
    int4 cn = make_int4(0, 0, 0, 0);
    // output position: i (in place), or dest[i] on a sort-fused step
    unsigned long long o = (!CONT && a.dest && valid) ? (unsigned long long)__ldg(a.dest + i) : i;
    if (valid && a.dbg == 1) {   // diagnostic: stream only
        vx = add(vx, a.c1); x = add(x, mul(vx, a.dt));
        a.pos[i] = x; a.pos[a.cap + i] = y; a.pos[2 * a.cap + i] = z;
        a.vel[i] = vx; a.vel[a.cap + i] = vy; a.vel[2 * a.cap + i] = vz;
        valid = false;
    }
    if (valid && a.dbg == 2) {   // diagnostic: stream + E gather
        const double *Ep = reinterpret_cast<const double *>(a.ef + (cell - a.cell_base));
        vx = add(vx, mul(a.c1, __ldg(Ep))); x = add(x, mul(vx, a.dt));
        a.pos[i] = x; a.pos[a.cap + i] = y; a.pos[2 * a.cap + i] = z;
        a.vel[i] = vx; a.vel[a.cap + i] = vy; a.vel[2 * a.cap + i] = vz;
        valid = false;
    }
    if (valid) {
        const int lc = cell - a.cell_base;
        // First visit.  Direct paths issue the walk line together with E (one
        // round trip).  The TMA-out path issues it after the push (through an
        // opaque dependency on the pushed x) so the 32 line registers and the
        // particle state are never live at once: fewer registers, more warps.
        Line L;
        if (!(SOUT && !CONT)) L = load_line(a.lines, lc);
        if (!CONT) {
            // gather the cell-constant field, leap-frog push (569-583, 1576-1590)
            // DH: the overlay entry of the drift-only position x + v dt is
            // fetched together with E; it is used only when the pushed
            // position lies in the same overlay cell (all but ~|c1 E dt| / dx
            // of the particles), so the seed is exactly that of the pushed
            // position and the lookup leaves the dependent chain.
            long long spec_slot = -1;
            int spec_val = -1;
            double2 Exy;
            double Ez;
            if (pre) {
                spec_slot = pre->slot;
                spec_val = pre->val;
                Exy = pre->Exy;
                Ez = pre->Ez;
            } else {
                if (DH == 1) {
                    spec_slot = dh_slot(a.ov, add(x, mul(vx, a.dt)), add(y, mul(vy, a.dt)),
                                        add(z, mul(vz, a.dt)));
                    spec_val = ov_value(a.ov, spec_slot >= 0 ? spec_slot : 0);
                }
                load_E(a.ef, lc, Exy, Ez);
            }
            vx = add(vx, mul(a.c1, Exy.x));
            vy = add(vy, mul(a.c1, Exy.y));
            vz = add(vz, mul(a.c1, Ez));
            x = add(x, mul(vx, a.dt));
            y = add(y, mul(vy, a.dt));
            z = add(z, mul(vz, a.dt));
            // position and velocity are final now: store them before the walk
            // (TMA-out path: into the shared stage, bulk-stored by the warp)
            if (SOUT && sout) {   // per-warp output buffer: 6 columns of 32 doubles
                sout[sj] = x; sout[32 + sj] = y; sout[64 + sj] = z;
                sout[96 + sj] = vx; sout[128 + sj] = vy; sout[160 + sj] = vz;
            } else {
                a.pos_out[o] = x; a.pos_out[a.cap + o] = y; a.pos_out[2 * a.cap + o] = z;
                a.vel_out[o] = vx; a.vel_out[a.cap + o] = vy; a.vel_out[2 * a.cap + o] = vz;
            }
            if (release) {
                fence_proxy_async_fwd();   // generic reads before the async-proxy refill
                __syncwarp();
                if ((threadIdx.x & 31u) == 0) mbar_arrive_fwd(release);
            }
            if (DH == 1) {   // seed every particle from the overlay
                const long long g = dh_slot(a.ov, x, y, z);
                int v = g == spec_slot ? spec_val : (g >= 0 ? ov_value(a.ov, g) : -1);
                if (g < 0) v = -1;
                int sc = v >= 0 ? v : cell;
                if (sc != cell) {
                    cell = sc;
                    if (!SOUT) L = load_line(a.lines, sc - a.cell_base);
                }
            }
            if (SOUT && DH == 1 && perm) {
                // regroup the warp's particles by seed cell (contiguous lanes share
                // a cell): a 256-bit load costs the L1 ~2 cycles per distinct line
                // per 8-lane quarter, so interleaved seeds (~6 per warp) cost ~27
                // cycles per walk-line load and grouped ones ~17.  Position, cell
                // and output slot move; v is already stored.
                const unsigned FULL = 0xffffffffu, ln = threadIdx.x & 31u;
                const unsigned peers = __match_any_sync(FULL, cell);
                const int leader = __ffs(peers) - 1;
                const int sz = (int)ln == leader ? __popc(peers) : 0;
                int incl = sz;
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const int tq = __shfl_up_sync(FULL, incl, d);
                    if ((int)ln >= d) incl += tq;
                }
                const int dest = __shfl_sync(FULL, incl - sz, leader) + __popc(peers & ((1u << ln) - 1u));
                perm[dest] = (int)ln;
                __syncwarp();
                const int src = perm[ln];
                __syncwarp();
                x = __shfl_sync(FULL, x, src);
                y = __shfl_sync(FULL, y, src);
                z = __shfl_sync(FULL, z, src);
                cell = __shfl_sync(FULL, cell, src);
                o = __shfl_sync(FULL, o, src);
            }
            if (SOUT) {
                int zero;
                asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, %1;\n\tmov.b32 %0, 0;\n\t}"
                             : "=r"(zero) : "d"(z));
                L = load_line(a.lines, cell - a.cell_base + zero);
            }
            if (DH == 2) dh_if_left(a, x, y, z, cell, L);
        }
        const int stop_at = a.dbg == 3 ? 0 : (CONT ? INT_MAX : a.hpass);
        status = walk_from<MULTI>(a, cell, L, PosRegs{x, y, z}, hops, stop_at, l0, l1, l2, l3,
                                  capped, cn);
        if (a.dbg == 3 && status == ST_MOVE) status = ST_DONE;
        if (status != ST_MOVE && status != ST_MIGRATE) {   // counted where the walk ends
            t.hops += (unsigned)hops;
            t.maxh = max(t.maxh, (unsigned)hops);
            t.capped += (unsigned)capped;
        }
        t.removed += (status == ST_REMOVE);
    }
    const bool done = status == ST_DONE && a.dbg == 0;
    if (DEP == 2) {
        sr_store(a, done, cell, a.w, l0, l1, l2, l3);
    } else {
        deposit<DEP>(a.Q, CnSrc{a.lines, a.cell_base}, done, cell, cn, a.w, l0, l1, l2, l3);
    }
    // holes, the deferred-walk worklist, migrants
    const bool rem = status == ST_REMOVE || status == ST_MIGRATE;
    if (ap) {
        ring_push(ap->holes, rem, (uint32_t)o, 0);
        ring_flush(ap->holes, &a.cnt->n_holes, a.holes, nullptr, false);
        if (!CONT) {
            ring_push(ap->work, status == ST_MOVE, (uint32_t)o, hops);
            ring_flush(ap->work, &a.cnt->n_work, a.work, a.work_hops, false);
        }
    } else {
        unsigned long long hs = warp_append(rem, &a.cnt->n_holes);
        if (rem) a.holes[hs] = (uint32_t)o;
        if (!CONT) {
            const bool mv = status == ST_MOVE;
            unsigned long long ws = warp_append(mv, &a.cnt->n_work);
            if (mv) {
                a.work[ws] = (uint32_t)o;
                a.work_hops[ws] = hops;
            }
        }
    }
    if (MULTI) {
        const bool mg = status == ST_MIGRATE;
        unsigned long long ms = warp_append(mg, &a.cnt->n_mig);
        if (mg) {
            a.mig[ms] = (uint32_t)o;
            a.mig_cell[ms] = cell;
            a.mig_hops[ms] = hops;
        }
    }
    if (rem) cell = -1;
    if (perm) a.p2c_out[o] = cell;   // regrouped lanes store their own particle's cell
}

// ---------------------------------------------------------------------------
// Direct-load variant: warps stride over [lo, hi) one particle per lane; the
// next particle's state is loaded before the current one walks (a register
// double buffer), so the HBM stream stays in flight during the latency-bound
// walk.  Used for the continuation pass, the ragged tail of the tiled
// kernel, and as the non-TMA variant of pass 1.
// ---------------------------------------------------------------------------
struct PState {
    double x, y, z, vx, vy, vz;
    int cell, hops;
    unsigned long long i;
    bool valid;
};

template <bool CONT>
__device__ __forceinline__ void load_pstate(const StepArgs &a, unsigned long long k,
                                            unsigned long long hi, PState &p) {
    p.valid = k < hi;
    p.i = k;
    p.hops = 0;
    p.cell = 0;
    p.x = p.y = p.z = p.vx = p.vy = p.vz = 0.0;
    if (p.valid) {
        if (CONT) {
            p.i = a.work[k];
            p.hops = a.work_hops[k];
        }
        p.x = a.pos[p.i]; p.y = a.pos[a.cap + p.i]; p.z = a.pos[2 * a.cap + p.i];
        if (!CONT) { p.vx = a.vel[p.i]; p.vy = a.vel[a.cap + p.i]; p.vz = a.vel[2 * a.cap + p.i]; }
        p.cell = a.p2c[p.i];
    }
}

template <int DEP, int DH, bool CONT, bool MULTI>
__device__ __forceinline__ void pmd_direct_range(const StepArgs &a, unsigned long long lo,
                                                 unsigned long long hi, unsigned long long first,
                                                 unsigned long long stride, Tally &t) {
    unsigned long long i0 = lo + first;
    if (i0 >= hi) return;
    PState cur;
    load_pstate<CONT>(a, i0 + lane_id(), hi, cur);
    for (; i0 < hi; i0 += stride) {
        PState nxt;
        const bool more = i0 + stride < hi;
        if (more) load_pstate<CONT>(a, i0 + stride + lane_id(), hi, nxt);
        pmd_body<DEP, DH, CONT, MULTI>(a, cur.valid, cur.i, cur.hops, cur.x, cur.y, cur.z, cur.vx,
                                       cur.vy, cur.vz, cur.cell, t);
        if (cur.valid) a.p2c_out[(!CONT && a.dest) ? (unsigned long long)__ldg(a.dest + cur.i) : cur.i] = cur.cell;
        if (more) cur = nxt;
    }
}

// Pass 1 (direct variant): every block owns one contiguous chunk of the
// particle array, so in cell-sorted storage the walk lines a block touches
// stay hot in its SM's L1.  Continuation: grid-stride over the worklist.
template <int DEP, int DH, bool CONT, bool MULTI>
__global__ void __launch_bounds__(256) k_push_move_deposit(StepArgs a) {
    Tally t;
    if (CONT) {
        const unsigned long long n = *(volatile unsigned long long *)&a.cnt->n_work;
        pmd_direct_range<DEP, DH, true, MULTI>(
            a, 0, n, (unsigned long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31u),
            (unsigned long long)gridDim.x * blockDim.x, t);
    } else {
        const unsigned long long n = *(volatile unsigned long long *)&a.cnt->n;
        const TileMap tm{(n + 255) / 256, gridDim.x, (unsigned long long)a.tile_group, blockIdx.x};
        const unsigned long long my = tm.count();
        TileIter ti(tm);
        for (unsigned long long it = 0; it < my; it++, ti.next()) {
            const unsigned long long lo = ti.tile() * 256;
            pmd_direct_range<DEP, DH, false, MULTI>(a, lo, lo + 256 < n ? lo + 256 : n,
                                                    threadIdx.x & ~31u, 256, t);
        }
    }
    flush_stats(a.cnt, t.hops, t.maxh, t.capped, t.removed);
}

// ---------------------------------------------------------------------------
// The fused push / move / deposit kernel, TMA-pipelined (CalcPosVel + Move +
// DepositCharge of PAPER.md:1586-1604 in one pass).  Each block owns a
// contiguous range of kTile-particle tiles (L1 locality of the walk lines in
// cell-sorted storage).  A producer warp streams each tile's 7 SoA column
// segments global -> shared with cp.async.bulk (complete_tx on the stage's
// `full` mbarrier) up to kStages tiles ahead; each of the 8 consumer warps
// copies its 32 particles out of the stage, releases it (`empty` mbarrier,
// one arrival per warp) and then pushes / walks / deposits, storing results
// with coalesced stores.  No block-wide barrier inside the loop: a warp whose
// lanes walk far never stalls the others.  The ragged tail (< kTile) takes
// the direct path.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)),
                 "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// Blocking wait on an mbarrier phase.  try_wait with a suspend-time hint
// parks the thread in hardware until the phase completes (or the hint
// expires), instead of spinning through the L1 data pipe.
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done) : "r"(smem_u32(b)), "r"(parity), "r"(1000000u) : "memory");
    } while (!done);
}
__device__ __forceinline__ void mbar_wait_sleep(uint64_t *b, uint32_t parity) { mbar_wait(b, parity); }
__device__ __forceinline__ void mbar_arrive_fwd(uint64_t *b) { mbar_arrive(b); }
__device__ __forceinline__ bool mbar_test(uint64_t *b, uint32_t parity) {
    uint32_t done;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done) : "r"(smem_u32(b)), "r"(parity) : "memory");
    return done != 0;
}
__device__ __forceinline__ void prefetch_l1(const void *p) {
    asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}
__device__ __forceinline__ void fence_proxy_async_fwd() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read1() {
    asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }


// producer: load tile `tile` into stage s
__device__ __forceinline__ void issue_tile_load(const StepArgs &a, char *smem, uint64_t *full,
                                                int s, unsigned long long tile) {
    StageView v = stage_view(smem, s);
    const unsigned long long base = tile * kTile;
    mbar_expect_tx(&full[s], kStageBytes);
    for (int k = 0; k < 3; k++) {
        bulk_g2s(v.c[k], a.pos + k * a.cap + base, kTile * 8, &full[s]);
        bulk_g2s(v.c[3 + k], a.vel + k * a.cap + base, kTile * 8, &full[s]);
    }
    bulk_g2s(v.cell, a.p2c + base, kTile * 4, &full[s]);
}

// Producer-warp L1 warming for tile p (already issued; waits until landed).
__device__ __forceinline__ void warm_tile(const StepArgs &a, char *smem, uint64_t *full,
                                          unsigned long long p, unsigned lane) {
    const int sp = (int)(p % kStages);
    mbar_wait(&full[sp], (uint32_t)((p / kStages) & 1ull));
    const int *cells = stage_view(smem, sp).cell + lane * (kTile / 32);
    int prev = INT_MIN;
    int4 cc[kTile / 32];
    int lcs[kTile / 32];
    int nd = 0;
#pragma unroll
    for (int k = 0; k < kTile / 32; k++) {
        const int lc = cells[k] - a.cell_base;
        if (lc == prev || (unsigned)lc >= (unsigned)a.n_cells) continue;
        prev = lc;
        lcs[nd] = lc;
        cc[nd] = __ldg(reinterpret_cast<const int4 *>(reinterpret_cast<const double *>(a.lines + lc) + 12));
        prefetch_l1(a.ef + lc);
        nd++;
    }
    for (int k = 0; k < nd; k++) {
        const int nb[4] = {cc[k].x, cc[k].y, cc[k].z, cc[k].w};
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const int ln = nb[q] - a.cell_base;
            if (nb[q] >= 0 && (unsigned)ln < (unsigned)a.n_cells) prefetch_l1(a.lines + ln);
        }
        (void)lcs;
    }
}

#ifndef OPP_PRE
#define OPP_PRE 0   // 1: issue the next slice's E / overlay gathers one slice ahead
                    // (C2: pmd 1.98 vs 1.94 ms -- the extra stage reads cost more L1
                    // data-pipe wavefronts than the hidden latency saves)
#endif
template <int DEP, int DH, bool MULTI, bool REFILL, int MINB>
__global__ void __launch_bounds__(kTiledThreads, MINB) k_push_move_deposit_tiled(StepArgs a) {
    constexpr bool PRE = OPP_PRE != 0;
    constexpr bool TMA_OUT = OPP_TMA_OUT != 0;
    extern __shared__ __align__(128) char smem[];
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + kStages * kStageBytes);
    uint64_t *empty = full + kStages;
    const unsigned long long n = *(volatile unsigned long long *)&a.cnt->n;
    const unsigned long long ntiles = n / kTile;
    const unsigned long long G = gridDim.x;
    const TileMap tm{ntiles, G, (unsigned long long)a.tile_group, blockIdx.x};
    const unsigned long long my = tm.count();
    const int warp = threadIdx.x >> 5;
    const unsigned lane = lane_id();
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumerWarps);
        }
        fence_proxy_async();
    }
    __syncthreads();
    if (warp == kConsumerWarps) {
        // producer warp: lane 0 streams tiles kStages ahead of the slowest
        // consumer; then the whole warp warms the SM's L1 for the tile that
        // landed before: the walk lines and fields of its (few, cell-sorted)
        // start cells and the lines of their four face neighbours -- the
        // cells the consumers' first visit and first hop will touch.
        TileIter ti(tm);
        for (unsigned long long it = 0; it < my; it++, ti.next()) {
            const int s = (int)(it % kStages);
            if (lane == 0) {
                if (it >= kStages) mbar_wait_sleep(&empty[s], (uint32_t)(((it / kStages) - 1) & 1ull));
                issue_tile_load(a, smem, full, s, ti.tile());
            }
            __syncwarp();
            if (a.prefetch && it >= 1) warm_tile(a, smem, full, it - 1, lane);
        }
        if (a.prefetch && my >= 1) warm_tile(a, smem, full, my - 1, lane);
        return;
    }
    Tally t;
    if (!REFILL) {
        // Consumer warp, warp-synchronous: one 32-particle slice per tile;
        // the slice is copied to registers and the stage released at once.
        // Input: the warp copies its slice to registers, forces the shared
        // loads to complete, fences the generic proxy against the producer's
        // next bulk copy and releases the stage at once.  Output: results go
        // to a per-warp double buffer in shared memory and leave with
        // cp.async.bulk shared -> global (256-B / 128-B segments per column),
        // so the LSU pipe carries no particle stores.
        Appends ap;
        {
            char *rb = smem + kRingBase + (size_t)warp * kRingBytesPerWarp;
            ap.holes = WarpRing{reinterpret_cast<uint32_t *>(rb), nullptr, 0u, 0u};
            ap.work = WarpRing{reinterpret_cast<uint32_t *>(rb + 4 * kRing),
                               reinterpret_cast<int32_t *>(rb + 8 * kRing), 0u, 0u};
        }
        TileIter ti(tm);
        Pre cur{-1, -1, make_double2(0.0, 0.0), 0.0};
        bool have_cur = false;
        for (unsigned long long it = 0; it < my; it++, ti.next()) {
            const int s = (int)(it % kStages);
            const int ob_i = 0;   // one output buffer per warp (keeps 3 blocks / SM in smem)
            mbar_wait(&full[s], (uint32_t)((it / kStages) & 1ull));
            StageView v = stage_view(smem, s);
            const int j = threadIdx.x;
            double x = v.c[0][j], y = v.c[1][j], z = v.c[2][j];
            double vx = v.c[3][j], vy = v.c[4][j], vz = v.c[5][j];
            int cell = v.cell[j];
            Pre nxt;
            bool have_nxt = false;
            if (PRE && it + 1 < my) {
                const int s1 = (int)((it + 1) % kStages);
                const bool landed = __all_sync(0xffffffffu,
                                               mbar_test(&full[s1], (uint32_t)(((it + 1) / kStages) & 1ull)));
                if (landed) {
                    StageView v1 = stage_view(smem, s1);
                    const double x1 = v1.c[0][j], y1 = v1.c[1][j], z1 = v1.c[2][j];
                    const double vx1 = v1.c[3][j], vy1 = v1.c[4][j], vz1 = v1.c[5][j];
                    const int c1 = v1.cell[j];
                    nxt.slot = -1;
                    nxt.val = -1;
                    if (DH == 1) {
                        nxt.slot = dh_slot(a.ov, add(x1, mul(vx1, a.dt)), add(y1, mul(vy1, a.dt)),
                                           add(z1, mul(vz1, a.dt)));
                        nxt.val = ov_value(a.ov, nxt.slot >= 0 ? nxt.slot : 0);
                    }
                    load_E(a.ef, c1 - a.cell_base, nxt.Exy, nxt.Ez);
                    have_nxt = true;
                }
            }
            const unsigned long long h = (unsigned long long)__double_as_longlong(x) ^
                                         (unsigned long long)__double_as_longlong(y) ^
                                         (unsigned long long)__double_as_longlong(z) ^
                                         (unsigned long long)__double_as_longlong(vx) ^
                                         (unsigned long long)__double_as_longlong(vy) ^
                                         (unsigned long long)__double_as_longlong(vz) ^
                                         (unsigned long long)(unsigned)cell;
            asm volatile("" ::"l"(h));   // the shared loads have landed
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&empty[s]);
                if (it >= 1) bulk_wait_read0();   // the previous stores have read the buffer
            }
            __syncwarp();
            const unsigned long long tile = ti.tile();
            const unsigned long long i = tile * kTile + j;
            double *o = reinterpret_cast<double *>(smem + kOutBase +
                                                   (size_t)(warp + ob_i) * kOutBytes);
            // results leave through the shared buffer + bulk stores (TMA_OUT),
            // or (sort-fused step / OPP_TMA_OUT=0) as coalesced per-lane stores
            double *obuf = (TMA_OUT && !a.dest) ? o : nullptr;
            int *perm = (OPP_SEED_PERM && DH == 1 && !obuf)
                             ? reinterpret_cast<int *>(smem + kRingBase + (size_t)warp * kRingBytesPerWarp + 64 * 12)
                             : nullptr;
            pmd_body<DEP, DH, false, MULTI, true>(a, true, i, 0, x, y, z, vx, vy, vz, cell, t,
                                                  nullptr, obuf, (int)lane, &ap,
                                                  (PRE && have_cur) ? &cur : nullptr, perm);
            if (PRE) {
                cur = nxt;
                have_cur = have_nxt;
            }
            if (!obuf) {
                if (!perm) a.p2c_out[a.dest ? (unsigned long long)__ldg(a.dest + i) : i] = cell;
                continue;
            }
            reinterpret_cast<int *>(o + 192)[lane] = cell;
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
                const unsigned long long g0 = tile * kTile + warp * 32;
                for (int k = 0; k < 3; k++) {
                    bulk_s2g(a.pos + k * a.cap + g0, o + 32 * k, 256);
                    bulk_s2g(a.vel + k * a.cap + g0, o + 32 * (3 + k), 256);
                }
                bulk_s2g(a.p2c + g0, o + 192, 128);
                bulk_commit();
            }
        }
        ring_flush(ap.holes, &a.cnt->n_holes, a.holes, nullptr, true);
        ring_flush(ap.work, &a.cnt->n_work, a.work, a.work_hops, true);
        if (lane == 0) bulk_wait_all();
        // the ragged tail (< kTile particles) is done by k_push_move_deposit_tail
        flush_stats(a.cnt, t.hops, t.maxh, t.capped, t.removed);
        return;
    }
    // Consumer warp with per-lane refill: its particle stream is its 32-slot slice of every tile.
    // Lanes are refilled independently: whenever a lane's particle finishes
    // (DONE / REMOVE / deferred / migrating) it takes the next stream entry,
    // so every iteration advances 32 walks by one cell visit instead of
    // waiting for the warp's longest walk.
    const unsigned long long total = 32ull * my;
    unsigned long long pos = 0;
    long long waited = -1;
    bool active = false;
    double x = 0, y = 0, z = 0;
    int cell = 0, hops = 0;
    unsigned long long i = 0;
    Line L;
    const unsigned lt_mask = (1u << lane) - 1u;
    for (;;) {
        // ---- refill idle lanes from the stream
        const unsigned need = __ballot_sync(0xffffffffu, !active);
        if (need && pos < total) {
            const unsigned long long avail = total - pos;
            const int k = (int)min((unsigned long long)__popc(need), avail);
            const int r = __popc(need & lt_mask);
            const bool take = !active && r < k;
            const long long last_tile = (long long)((pos + k - 1) / 32);
            if (last_tile > waited) {
                mbar_wait(&full[last_tile % kStages], (uint32_t)((last_tile / kStages) & 1));
                waited = last_tile;
            }
            double vx = 0, vy = 0, vz = 0;
            if (take) {
                const unsigned long long p = pos + r, it = p / 32;
                const int j = warp * 32 + (int)(p % 32);
                StageView v = stage_view(smem, (int)(it % kStages));
                x = v.c[0][j]; y = v.c[1][j]; z = v.c[2][j];
                vx = v.c[3][j]; vy = v.c[4][j]; vz = v.c[5][j];
                cell = v.cell[j];
                i = tm.tile(it) * kTile + j;
                hops = 0;
            }
            const unsigned long long pos0 = pos, npos = pos + k;
            pos = npos;
            if (take) {
                const int lc = cell - a.cell_base;
                L = load_line(a.lines, lc);
                double2 Exy;
                double Ez;
                load_E(a.ef, lc, Exy, Ez);
                vx = add(vx, mul(a.c1, Exy.x));
                vy = add(vy, mul(a.c1, Exy.y));
                vz = add(vz, mul(a.c1, Ez));
                x = add(x, mul(vx, a.dt));
                y = add(y, mul(vy, a.dt));
                z = add(z, mul(vz, a.dt));
                a.pos[i] = x; a.pos[a.cap + i] = y; a.pos[2 * a.cap + i] = z;
                a.vel[i] = vx; a.vel[a.cap + i] = vy; a.vel[2 * a.cap + i] = vz;
                if (DH == 1) {
                    const int sc = dh_seed(a.ov, x, y, z, cell);
                    if (sc != cell) {
                        cell = sc;
                        L = load_line(a.lines, sc - a.cell_base);
                    }
                }
                if (DH == 2) dh_if_left(a, x, y, z, cell, L);
                active = true;
            }
            // the push has consumed the shared copies: release fully read slices
            fence_proxy_async();
            __syncwarp();
            if (lane == 0)
                for (unsigned long long tt = pos0 / 32; tt < npos / 32; tt++)
                    mbar_arrive(&empty[tt % kStages]);
        }
        if (!__any_sync(0xffffffffu, active)) break;
        // ---- one cell visit per active lane
        int status = ST_NONE;
        int capped = 0;
        double l0 = 0, l1 = 0, l2 = 0, l3 = 0;
        int4 cn = make_int4(0, 0, 0, 0);
        if (active) {
            bary(L, x, y, z, l0, l1, l2, l3);
            cn = L.cn;
            if (in01(l0) && in01(l1) && in01(l2) && in01(l3)) {
                status = ST_DONE;
            } else if (hops >= a.hcap) {
                status = ST_DONE;
                capped = 1;
            } else if (hops >= a.hpass) {
                status = ST_MOVE;
            } else {
                const int4 cc = cc_of(a.lines, L, cell - a.cell_base);
                int nb = cc.x;
                double m = l0;
                if (l1 < m) { m = l1; nb = cc.y; }
                if (l2 < m) { m = l2; nb = cc.z; }
                if (l3 < m) { nb = cc.w; }
                if (nb < 0) {
                    status = ST_REMOVE;
                } else if (MULTI && (unsigned)(nb - a.cell_base) >= (unsigned)a.n_cells) {
                    cell = nb;
                    hops++;
                    status = ST_MIGRATE;
                } else {
                    cell = nb;
                    hops++;
                    L = load_line(a.lines, nb - a.cell_base);
                }
            }
        }
        const bool fin = status != ST_NONE;
        if (fin && status != ST_MOVE && status != ST_MIGRATE) {
            t.hops += (unsigned)hops;
            t.maxh = max(t.maxh, (unsigned)hops);
            t.capped += (unsigned)capped;
        }
        t.removed += (status == ST_REMOVE);
        const bool done = status == ST_DONE;
        if (DEP == 2) sr_store(a, done, cell, a.w, l0, l1, l2, l3);
        else deposit<DEP>(a.Q, CnSrc{a.lines, a.cell_base}, done, cell, cn, a.w, l0, l1, l2, l3);
        const bool rem = status == ST_REMOVE || status == ST_MIGRATE;
        unsigned long long hs = warp_append(rem, &a.cnt->n_holes);
        if (rem) a.holes[hs] = (uint32_t)i;
        const bool mv = status == ST_MOVE;
        unsigned long long ws = warp_append(mv, &a.cnt->n_work);
        if (mv) {
            a.work[ws] = (uint32_t)i;
            a.work_hops[ws] = hops;
        }
        if (MULTI) {
            const bool mg = status == ST_MIGRATE;
            unsigned long long ms = warp_append(mg, &a.cnt->n_mig);
            if (mg) {
                a.mig[ms] = (uint32_t)i;
                a.mig_cell[ms] = cell;
                a.mig_hops[ms] = hops;
            }
        }
        if (fin) {
            a.p2c[i] = rem ? -1 : cell;
            active = false;
        }
    }
    flush_stats(a.cnt, t.hops, t.maxh, t.capped, t.removed);
}

// Ragged tail of the TMA-pipelined pass: particles [floor(n / kTile) * kTile, n)
// (fewer than kTile), one block, direct loads.  A separate launch so the
// register-heavy direct path does not set the pipelined kernel's allocation.
template <int DEP, int DH, bool MULTI>
__global__ void __launch_bounds__(256) k_push_move_deposit_tail(StepArgs a) {
    const unsigned long long n = *(volatile unsigned long long *)&a.cnt->n;
    const unsigned long long lo = n / kTile * kTile;
    Tally t;
    pmd_direct_range<DEP, DH, false, MULTI>(a, lo, n, threadIdx.x & ~31u, 256, t);
    flush_stats(a.cnt, t.hops, t.maxh, t.capped, t.removed);
}

// ---------------------------------------------------------------------------
// Continuation walk with per-lane refill: finishes the deferred walks (and
// received migrants).  Each lane carries one particle and advances it by one
// cell visit per iteration; a lane whose particle finished claims the next
// worklist entry (the warp leader claims a batch with one atomic), so every
// iteration keeps ~32 walks in flight instead of waiting for the longest walk
// of the warp.  Small register footprint -> many resident warps to hide the
// L2 latency of the line gathers.
// ---------------------------------------------------------------------------
template <int DEP, bool MULTI>
__global__ void __launch_bounds__(256, 4) k_walk_refill(StepArgs a) {
    const unsigned long long nw = *(volatile unsigned long long *)&a.cnt->n_work;
    const unsigned lane = lane_id();
    const unsigned lt = (1u << lane) - 1u;
    // Warps walk the worklist in 32-entry groups, group g = gw + k * nwarps
    // (no shared claim counter: a single-address atomic per refill serialises
    // in L2), so the entries in flight form one moving window of the worklist
    // -- and of the mesh, since the list follows the cell-sorted storage.
    const unsigned long long nwarps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
    const unsigned long long gw = (unsigned long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const unsigned long long gstep = nwarps * 32;
    unsigned long long gstart = gw * 32;                          // current group
    unsigned long long cur = gstart;                              // next unclaimed entry
    unsigned long long gend = gstart + 32 < nw ? gstart + 32 : nw;
    __shared__ uint32_t hring[8][kRing];
    WarpRing hr{hring[threadIdx.x >> 5], nullptr, 0u, 0u};
    Tally t;
    bool active = false, more = gstart < nw;
    unsigned long long i = 0;
    int cell = 0, hops = 0;
    double x = 0, y = 0, z = 0;
    Line L;
    for (;;) {
        const unsigned need = __ballot_sync(0xffffffffu, !active);
        if (need && more) {
            // the r-th needing lane takes the r-th unclaimed entry: first from
            // the current group, then from the warp's next group
            const unsigned r = __popc(need & lt), k = __popc(need);
            const unsigned long long left = gend - cur;
            const unsigned long long nstart = gstart + gstep;
            const unsigned long long nend = nstart + 32 < nw ? nstart + 32 : nw;
            unsigned long long q = ~0ull;
            if (r < left) q = cur + r;
            else if (nstart + (r - left) < nend) q = nstart + (r - left);
            if (k < left) {
                cur += k;
            } else {
                gstart = nstart;
                gend = nend;
                cur = nstart + (k - left);
                if (gstart >= nw) {
                    more = false;
                } else if (cur >= gend) {
                    gstart += gstep;
                    cur = gstart;
                    gend = gstart + 32 < nw ? gstart + 32 : nw;
                    more = gstart < nw;
                }
            }
            if (!active && q != ~0ull) {
                i = a.work[q];
                hops = a.work_hops[q];
                x = a.pos[i]; y = a.pos[a.cap + i]; z = a.pos[2 * a.cap + i];
                cell = a.p2c[i];
                L = load_line(a.lines, cell - a.cell_base);
                active = true;
            }
        }
        if (!__any_sync(0xffffffffu, active)) break;
        int status = ST_NONE, capped = 0;
        double l0 = 0, l1 = 0, l2 = 0, l3 = 0;
        int4 cn = make_int4(0, 0, 0, 0);
        if (active) {
            bary(L, x, y, z, l0, l1, l2, l3);
            cn = L.cn;
            if (in01(l0) && in01(l1) && in01(l2) && in01(l3)) {
                status = ST_DONE;
            } else if (hops >= a.hcap) {
                status = ST_DONE;
                capped = 1;
            } else {
                const int4 cc = cc_of(a.lines, L, cell - a.cell_base);
                int nb = cc.x;
                double m = l0;
                if (l1 < m) { m = l1; nb = cc.y; }
                if (l2 < m) { m = l2; nb = cc.z; }
                if (l3 < m) { nb = cc.w; }
                if (nb < 0) {
                    status = ST_REMOVE;
                } else if (MULTI && (unsigned)(nb - a.cell_base) >= (unsigned)a.n_cells) {
                    cell = nb;
                    hops++;
                    status = ST_MIGRATE;
                } else {
                    cell = nb;
                    hops++;
                    L = load_line(a.lines, nb - a.cell_base);
                }
            }
        }
        const bool fin = status != ST_NONE;
        if (fin && status != ST_MIGRATE) {
            t.hops += (unsigned)hops;
            t.maxh = max(t.maxh, (unsigned)hops);
            t.capped += (unsigned)capped;
        }
        t.removed += (status == ST_REMOVE);
        const bool done = status == ST_DONE;
        if (DEP == 2) sr_store(a, done, cell, a.w, l0, l1, l2, l3);
        else deposit<DEP>(a.Q, CnSrc{a.lines, a.cell_base}, done, cell, cn, a.w, l0, l1, l2, l3);
        const bool rem = status == ST_REMOVE || status == ST_MIGRATE;
        ring_push(hr, rem, (uint32_t)i, 0);
        ring_flush(hr, &a.cnt->n_holes, a.holes, nullptr, false);
        if (MULTI) {
            const bool mg = status == ST_MIGRATE;
            unsigned long long ms = warp_append(mg, &a.cnt->n_mig);
            if (mg) {
                a.mig[ms] = (uint32_t)i;
                a.mig_cell[ms] = cell;
                a.mig_hops[ms] = hops;
            }
        }
        if (fin) {
            a.p2c[i] = rem ? -1 : cell;
            active = false;
        }
    }
    ring_flush(hr, &a.cnt->n_holes, a.holes, nullptr, true);
    flush_stats(a.cnt, t.hops, t.maxh, t.capped, t.removed);
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
        c->n_mig = 0;
        c->n_mig_out = 0;
        c->n_mig_in = 0;
        c->work_cursor = 0;
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
        const Line L = load_line(lines, (int)c);
        const int4 cn = line_c2n(lines, (int)c);
        int nodes[4] = {cn.x, cn.y, cn.z, cn.w};
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
                        atomicMin(map + ov_slot32(ov, gx, gy, gz), (int)c + cell_base);
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
// Multi-block exclusive scan of unsigned counts (3 phases: tile sums, scan of
// the tile sums in one block, tile scans plus offsets).  Tile = 4096.
// ---------------------------------------------------------------------------
constexpr int kScanTile = 4096;   // 1024 threads x 4 elements

__device__ __forceinline__ unsigned long long block_exclusive_scan(unsigned long long v,
                                                                   unsigned long long *warp_buf,
                                                                   unsigned long long *total) {
    unsigned long long x = v;
    for (int off = 1; off < 32; off <<= 1) {
        unsigned long long t = __shfl_up_sync(0xffffffffu, x, off);
        if ((int)lane_id() >= off) x += t;
    }
    const int wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (lane_id() == 31) warp_buf[wid] = x;
    __syncthreads();
    if (wid == 0) {
        unsigned long long s = (int)lane_id() < nw ? warp_buf[lane_id()] : 0;
        for (int off = 1; off < 32; off <<= 1) {
            unsigned long long t = __shfl_up_sync(0xffffffffu, s, off);
            if ((int)lane_id() >= off) s += t;
        }
        warp_buf[lane_id()] = s;
    }
    __syncthreads();
    unsigned long long pre = wid ? warp_buf[wid - 1] : 0;
    if (total) *total = warp_buf[nw - 1];
    return pre + x - v;
}

__global__ void __launch_bounds__(1024) k_scan_tiles(const unsigned *__restrict__ in, long long n,
                                                     unsigned long long *tile_sum) {
    __shared__ unsigned long long wb[32];
    const long long base = (long long)blockIdx.x * kScanTile + 4 * threadIdx.x;
    unsigned long long v = 0;
    for (int k = 0; k < 4; k++)
        if (base + k < n) v += in[base + k];
    unsigned long long tot;
    block_exclusive_scan(v, wb, &tot);
    if (threadIdx.x == 0) tile_sum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(1024) k_scan_top(unsigned long long *tile_sum, long long ntiles) {
    __shared__ unsigned long long wb[32];
    __shared__ unsigned long long carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (long long b = 0; b < ntiles; b += blockDim.x) {
        long long i = b + threadIdx.x;
        unsigned long long v = i < ntiles ? tile_sum[i] : 0;
        unsigned long long tot;
        unsigned long long ex = block_exclusive_scan(v, wb, &tot);
        unsigned long long c = carry;
        __syncthreads();
        if (i < ntiles) tile_sum[i] = c + ex;
        if (threadIdx.x == 0) carry = c + tot;
        __syncthreads();
    }
}

__global__ void __launch_bounds__(1024) k_scan_apply(const unsigned *__restrict__ in, long long n,
                                                     const unsigned long long *__restrict__ tile_off,
                                                     unsigned *out) {
    __shared__ unsigned long long wb[32];
    const long long base = (long long)blockIdx.x * kScanTile + 4 * threadIdx.x;
    unsigned e[4];
    unsigned long long v = 0;
    for (int k = 0; k < 4; k++) {
        e[k] = base + k < n ? in[base + k] : 0u;
        v += e[k];
    }
    unsigned long long ex = block_exclusive_scan(v, wb, nullptr) + tile_off[blockIdx.x];
    for (int k = 0; k < 4; k++) {
        if (base + k < n) out[base + k] = (unsigned)ex;
        ex += e[k];
    }
}

// ---------------------------------------------------------------------------
// Sort by cell (particle sorting as an auxiliary call;
// here also the step's compaction): counting sort keyed by the local cell.
// Holes (p2c = -1) are dropped, so the sorted set is also hole-free.  Runs of
// equal cells inside a warp are aggregated into one atomic.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void run_info(int key, unsigned &heads, int &run_start, int &run_len,
                                         bool &head) {
    const unsigned lane = lane_id();
    int prev = __shfl_up_sync(0xffffffffu, key, 1);
    head = (lane == 0) || (prev != key);
    heads = __ballot_sync(0xffffffffu, head);
    unsigned below = heads & ((2u << lane) - 1u);      // heads at or below this lane
    if (lane == 31) below = heads;
    run_start = 31 - __clz(below);
    unsigned above = heads & ~((2u << lane) - 1u);
    if (lane == 31) above = 0;
    int run_end = above ? (__ffs(above) - 2) : 31;
    run_len = run_end - run_start + 1;
}

// Sort bucket of a cell: its locality key (see opp_init_params.sort_axis) or
// the local cell index.
__device__ __forceinline__ unsigned bucket_of(const uint32_t *__restrict__ skey, int lc) {
    return skey ? __ldg(skey + lc) : (unsigned)lc;
}

__global__ void k_cell_hist(const int32_t *__restrict__ p2c, const DevCounters *c, int cell_base,
                            const uint32_t *__restrict__ skey, unsigned *hist) {
    const unsigned long long n = c->n;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i0 = (unsigned long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
         i0 < n; i0 += stride) {
        const unsigned long long i = i0 + lane_id();
        int cell = i < n ? p2c[i] : -1;
        int key = cell >= 0 ? cell : -2 - (int)lane_id();
        unsigned heads;
        int rs, rl;
        bool head;
        run_info(key, heads, rs, rl, head);
        if (head && cell >= 0) atomicAdd(hist + bucket_of(skey, cell - cell_base), (unsigned)rl);
    }
}

// Phase 1: destination slot of every particle (run heads take one atomic
// per run of equal cells); holes get 0xffffffff.
__global__ void k_sort_rank(const int32_t *__restrict__ p2c, const DevCounters *c, int cell_base,
                            const uint32_t *__restrict__ skey, unsigned *cursor, uint32_t *dest,
                            uint32_t *src_of) {
    const unsigned long long n = c->n;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i0 = (unsigned long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
         i0 < n; i0 += stride) {
        const unsigned long long i = i0 + lane_id();
        int cell = i < n ? p2c[i] : -1;
        int key = cell >= 0 ? cell : -2 - (int)lane_id();
        unsigned heads;
        int rs, rl;
        bool head;
        run_info(key, heads, rs, rl, head);
        unsigned base = 0;
        if (head && cell >= 0)
            base = atomicAdd(cursor + bucket_of(skey, cell - cell_base), (unsigned)rl);
        base = __shfl_sync(0xffffffffu, base, rs);
        if (cell >= 0) {
            src_of[base + (lane_id() - rs)] = (uint32_t)i;   // inverse permutation
            if (dest) dest[i] = base + (lane_id() - rs);      // forward (sort fused into the move)
        }
    }
}

// Phase 2: gather move dst[d] = src[src_of[d]] for d in [0, total): the
// writes stream in order (full sectors, no read-modify-write of partially
// written sectors), the reads of nearly sorted data hit sectors that their
// neighbours in d fetched a moment ago.
constexpr int kSortUnroll = 4;
__global__ void __launch_bounds__(256) k_sort_gather(ColSet src, ColSet dst,
                                                     const uint32_t *__restrict__ src_of,
                                                     const unsigned *__restrict__ total_p,
                                                     int u0, int u1) {
    const unsigned long long n = *total_p;
    const unsigned long long span = (unsigned long long)blockDim.x * kSortUnroll;
    for (unsigned long long b = (unsigned long long)blockIdx.x * span; b < n;
         b += (unsigned long long)gridDim.x * span) {
        unsigned long long dd[kSortUnroll];
        uint32_t ss[kSortUnroll];
#pragma unroll
        for (int u = 0; u < kSortUnroll; u++) {
            dd[u] = b + (unsigned long long)u * blockDim.x + threadIdx.x;
            ss[u] = dd[u] < n ? __ldg(src_of + dd[u]) : 0u;
        }
        int u = 0;   // flattened (column, component) index; this launch moves [u0, u1)
        for (int j = 0; j < src.n; j++) {
            const ColDesc cs = src.c[j], cd = dst.c[j];
            for (int e = 0; e < cs.dim; e++, u++) {
                if (u < u0 || u >= u1) continue;
                if (cs.elem_bytes == 8) {
                    const long long *sp = reinterpret_cast<const long long *>(cs.ptr) + e * cs.cap;
                    long long *dp = reinterpret_cast<long long *>(cd.ptr) + e * cd.cap;
                    long long v[kSortUnroll];
#pragma unroll
                    for (int u = 0; u < kSortUnroll; u++) v[u] = dd[u] < n ? __ldg(sp + ss[u]) : 0;
#pragma unroll
                    for (int u = 0; u < kSortUnroll; u++) if (dd[u] < n) dp[dd[u]] = v[u];
                } else {
                    const int *sp = reinterpret_cast<const int *>(cs.ptr) + e * cs.cap;
                    int *dp = reinterpret_cast<int *>(cd.ptr) + e * cd.cap;
                    int v[kSortUnroll];
#pragma unroll
                    for (int u = 0; u < kSortUnroll; u++) v[u] = dd[u] < n ? __ldg(sp + ss[u]) : 0;
#pragma unroll
                    for (int u = 0; u < kSortUnroll; u++) if (dd[u] < n) dp[dd[u]] = v[u];
                }
            }
        }
    }
}

// Sort-fused step: the columns the move does not write (ids, user dats)
// follow their particles, dst[dest[i]] = src[i] for i < n.
__global__ void __launch_bounds__(256) k_scatter_cols(ColSet src, ColSet dst,
                                                      const uint32_t *__restrict__ dest,
                                                      const DevCounters *c) {
    const unsigned long long n = c->n;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        const unsigned long long d = __ldg(dest + i);
        for (int j = 0; j < src.n; j++) {
            const ColDesc cs = src.c[j], cd = dst.c[j];
            for (int e = 0; e < cs.dim; e++) {
                if (cs.elem_bytes == 8)
                    reinterpret_cast<long long *>(cd.ptr)[e * cd.cap + d] =
                        __ldg(reinterpret_cast<const long long *>(cs.ptr) + e * cs.cap + i);
                else
                    reinterpret_cast<int *>(cd.ptr)[e * cd.cap + d] =
                        __ldg(reinterpret_cast<const int *>(cs.ptr) + e * cs.cap + i);
            }
        }
    }
}

// n := number of sorted (hole-free) particles; holes consumed.
__global__ void k_sort_commit(DevCounters *c, const unsigned *start_total) {
    c->n_removed_last = c->n_holes;
    c->n = *start_total;
    c->n_holes = 0;
}

// ---------------------------------------------------------------------------
// Particle migration between slabs (mark -> pack into one
// buffer -> send/recv -> unpack to the end of the dats -> continue the walk).
// A record holds every particle column (AoS bytes, the p2c slot carrying the
// target global cell) followed by the hop count (S4: hops travel with the
// particle).
// ---------------------------------------------------------------------------
__device__ __forceinline__ int owner_of(const RankRanges &rr, int cell) {
    for (int r = 0; r < rr.n; r++)
        if (cell >= rr.lo[r] && cell < rr.hi[r]) return r;
    return -1;
}

__global__ void k_mig_count(const int32_t *__restrict__ mig_cell, const DevCounters *c, RankRanges rr,
                            unsigned long long *counts) {
    __shared__ unsigned long long sc[kMaxRanks];
    for (int r = threadIdx.x; r < rr.n; r += blockDim.x) sc[r] = 0;
    __syncthreads();
    const unsigned long long m = c->n_mig;
    for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (unsigned long long)gridDim.x * blockDim.x) {
        int o = owner_of(rr, mig_cell[k]);
        if (o >= 0) atomicAdd(&sc[o], 1ull);
    }
    __syncthreads();
    for (int r = threadIdx.x; r < rr.n; r += blockDim.x)
        if (sc[r]) atomicAdd(&counts[r], sc[r]);
}

__device__ __forceinline__ void copy_elem(char *dst, const char *src, int eb) {
    if (eb == 8) *reinterpret_cast<long long *>(dst) = *reinterpret_cast<const long long *>(src);
    else *reinterpret_cast<int *>(dst) = *reinterpret_cast<const int *>(src);
}

__global__ void k_mig_pack(ColSet cols, int p2c_col, const uint32_t *__restrict__ mig,
                           const int32_t *__restrict__ mig_cell, const int32_t *__restrict__ mig_hops,
                           const DevCounters *c, RankRanges rr, unsigned long long *cursor,
                           char *sendbuf, int rec_bytes) {
    const unsigned long long m = c->n_mig;
    for (unsigned long long k = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (unsigned long long)gridDim.x * blockDim.x) {
        const int o = owner_of(rr, mig_cell[k]);
        if (o < 0) continue;
        const unsigned long long slot = atomicAdd(&cursor[o], 1ull);
        char *rec = sendbuf + slot * (unsigned long long)rec_bytes;
        const unsigned long long i = mig[k];
        int off = 0;
        for (int j = 0; j < cols.n; j++) {
            const ColDesc cd = cols.c[j];
            off = (off + cd.elem_bytes - 1) & ~(cd.elem_bytes - 1);   // natural alignment
            for (int e = 0; e < cd.dim; e++) {
                if (j == p2c_col) *reinterpret_cast<int *>(rec + off) = mig_cell[k];
                else copy_elem(rec + off, cd.ptr + ((long long)e * cd.cap + (long long)i) * cd.elem_bytes,
                               cd.elem_bytes);
                off += cd.elem_bytes;
            }
        }
        *reinterpret_cast<int *>(rec + off) = mig_hops[k];
    }
}

// Append R received records at [N, N+R); they become the continuation
// worklist; the last block commits N += R and resets the migrant list.
__global__ void k_mig_unpack(ColSet cols, const char *__restrict__ recvbuf, long long R, int rec_bytes,
                             DevCounters *c, uint32_t *work, int32_t *work_hops) {
    __shared__ unsigned long long base_s;
    if (threadIdx.x == 0) base_s = *(volatile unsigned long long *)&c->n;
    __syncthreads();
    const unsigned long long base = base_s;
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < R;
         k += (long long)gridDim.x * blockDim.x) {
        const char *rec = recvbuf + k * (long long)rec_bytes;
        const unsigned long long i = base + k;
        int off = 0;
        for (int j = 0; j < cols.n; j++) {
            const ColDesc cd = cols.c[j];
            off = (off + cd.elem_bytes - 1) & ~(cd.elem_bytes - 1);
            for (int e = 0; e < cd.dim; e++) {
                copy_elem(cd.ptr + ((long long)e * cd.cap + (long long)i) * cd.elem_bytes, rec + off,
                          cd.elem_bytes);
                off += cd.elem_bytes;
            }
        }
        work[k] = (uint32_t)i;
        work_hops[k] = *reinterpret_cast<const int *>(rec + off);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        unsigned long long t = atomicAdd(&c->unpack_done_blocks, 1ull);
        if (t == gridDim.x - 1) {
            c->n = base + (unsigned long long)R;
            c->n_work = (unsigned long long)R;
            c->work_cursor = 0;
            c->n_mig_out += c->n_mig;
            c->n_mig = 0;
            c->n_mig_in += (unsigned long long)R;
            c->unpack_done_blocks = 0;
            __threadfence();
        }
    }
}

// Node-charge halo: interface nodes' partial sums.
__global__ void k_halo_pack(const double *__restrict__ Q, const int32_t *__restrict__ idx, long long m,
                            double *out) {
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (long long)gridDim.x * blockDim.x)
        out[k] = Q[idx[k]];
}

__global__ void k_halo_add(double *Q, const int32_t *__restrict__ idx, long long m,
                           const double *__restrict__ in) {
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (long long)gridDim.x * blockDim.x)
        atomicAdd(Q + idx[k], in[k]);
}

// ---------------------------------------------------------------------------
// Launchers (host side of this translation unit)
// ---------------------------------------------------------------------------

long long scan_tiles(long long n) { return n > 0 ? (n + kScanTile - 1) / kScanTile : 1; }

cudaError_t scan_exclusive(const unsigned *in, unsigned *out, long long n,
                           unsigned long long *tile_sums, cudaStream_t s) {
    long long tiles = scan_tiles(n);
    k_scan_tiles<<<(int)tiles, 1024, 0, s>>>(in, n, tile_sums);
    k_scan_top<<<1, 1024, 0, s>>>(tile_sums, tiles);
    k_scan_apply<<<(int)tiles, 1024, 0, s>>>(in, n, tile_sums, out);
    return cudaGetLastError();
}

// Shuffle keys (opp_shuffle): bucket = hash(index, seed) mod nc (+ cell_base,
// so the cell-keyed counting sort can consume them), -1 for holes.
__global__ void k_shuffle_keys(const int32_t *__restrict__ p2c, const DevCounters *c,
                               unsigned long long seed, long long nb, int cell_base,
                               int32_t *__restrict__ keys) {
    const unsigned long long n = c->n;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        unsigned long long z = seed + (i + 1ull) * 0x9E3779B97F4A7C15ull;
        z ^= z >> 30;
        z *= 0xBF58476D1CE4E5B9ull;
        z ^= z >> 27;
        z *= 0x94D049BB133111EBull;
        z ^= z >> 31;
        keys[i] = p2c[i] < 0 ? -1 : cell_base + (int32_t)(z % (unsigned long long)nb);
    }
}

cudaError_t launch_shuffle_keys(const int32_t *p2c, const DevCounters *c, unsigned long long seed,
                                long long nb, int cell_base, int32_t *keys, int grid, cudaStream_t s) {
    k_shuffle_keys<<<grid, 256, 0, s>>>(p2c, c, seed, nb, cell_base, keys);
    return cudaGetLastError();
}

cudaError_t launch_sort_count(const int32_t *p2c, DevCounters *c, int cell_base, long long nc,
                              const uint32_t *skey, unsigned *hist, unsigned *start,
                              unsigned long long *tile_sums, int grid, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(hist, 0, sizeof(unsigned) * (nc + 1), s);
    if (e != cudaSuccess) return e;
    k_cell_hist<<<grid, 256, 0, s>>>(p2c, c, cell_base, skey, hist);
    return scan_exclusive(hist, start, nc + 1, tile_sums, s);
}

cudaError_t launch_sort_rank(const int32_t *p2c, DevCounters *c, int cell_base, const uint32_t *skey,
                             unsigned *start, uint32_t *dest, uint32_t *src_of, int rank_grid,
                             cudaStream_t s) {
    k_sort_rank<<<rank_grid, 256, 0, s>>>(p2c, c, cell_base, skey, start, dest, src_of);
    return cudaGetLastError();
}

cudaError_t launch_scatter_cols(const ColSet &src, const ColSet &dst, const uint32_t *dest,
                                const DevCounters *c, int grid, cudaStream_t s) {
    if (src.n == 0) return cudaSuccess;
    k_scatter_cols<<<grid, 256, 0, s>>>(src, dst, dest, c);
    return cudaGetLastError();
}

cudaError_t launch_sort_move(const ColSet &src, const ColSet &dst, const int32_t *p2c,
                             DevCounters *c, int cell_base, long long nc, const uint32_t *skey,
                             unsigned *start, uint32_t *dest, uint32_t *src_of, int grid,
                             int rank_grid, cudaStream_t s) {
    // the scan left the total in start[nc]; the rank pass consumes start[] as
    // cursors but never touches start[nc].  One thread per particle: every
    // warp waits on its cursor atomics once, so the round trips overlap.
    k_sort_rank<<<rank_grid, 256, 0, s>>>(p2c, c, cell_base, skey, start, nullptr, src_of);
    // column passes: each pass moves a group of components so that the
    // source window it re-reads stays resident in L2 (OPP_SORT_PASSES)
    int nu = 0;
    for (int j = 0; j < src.n; j++) nu += src.c[j].dim;
    // defaults measured on C2 (sort_move 0.36 -> 0.315 ms/step at sort_every 5):
    // two passes, 4 blocks per SM
    static const int passes = [] {
        const char *e = getenv("OPP_SORT_PASSES");
        return e ? atoi(e) : 2;
    }();
    static const int gmul = [] {
        const char *e = getenv("OPP_SORT_GRID");
        return e ? atoi(e) : 4;
    }();
    if (gmul > 0) {
        int dev = 0, nsm = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        grid = nsm * gmul;
    }
    const int np = passes < 1 ? 1 : (passes > nu ? nu : passes);
    for (int q = 0; q < np; q++)
        k_sort_gather<<<grid, 256, 0, s>>>(src, dst, src_of, start + nc, q * nu / np,
                                           (q + 1) * nu / np);
    k_sort_commit<<<1, 1, 0, s>>>(c, start + nc);
    return cudaGetLastError();
}

template <int DEP, int DH, bool MULTI, bool REFILL, int MINB>
static cudaError_t launch_tiled_b(const StepArgs &a, int grid, cudaStream_t s) {
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_push_move_deposit_tiled<DEP, DH, MULTI, REFILL, MINB>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, kTiledSmem);
        if (e != cudaSuccess) return e;
        // shared-memory carveout (percent of the unified L1/shared array);
        // what the stages do not take is L1 for the walk lines (OPP_CARVEOUT)
        if (const char *cv = getenv("OPP_CARVEOUT")) {
            e = cudaFuncSetAttribute(k_push_move_deposit_tiled<DEP, DH, MULTI, REFILL, MINB>,
                                     cudaFuncAttributePreferredSharedMemoryCarveout, atoi(cv));
            if (e != cudaSuccess) return e;
        }
        attr = true;
    }
    k_push_move_deposit_tiled<DEP, DH, MULTI, REFILL, MINB><<<grid, kTiledThreads, kTiledSmem, s>>>(a);
    k_push_move_deposit_tail<DEP, DH, MULTI><<<1, 256, 0, s>>>(a);
    return cudaGetLastError();
}

template <int DEP, int DH, bool MULTI, bool REFILL>
static cudaError_t launch_tiled(const StepArgs &a, int grid, cudaStream_t s) {
    return a.minb >= 3 ? launch_tiled_b<DEP, DH, MULTI, REFILL, OPP_MINB_HI>(a, grid, s)
                       : launch_tiled_b<DEP, DH, MULTI, REFILL, 1>(a, grid, s);
}

template <int DEP, int DH, bool CONT, bool MULTI>
static cudaError_t launch_pmd_t(const StepArgs &a, int grid, bool tiled, cudaStream_t s) {
    if (!CONT && tiled) {
        return a.refill ? launch_tiled<DEP, DH, MULTI, true>(a, grid, s)
                        : launch_tiled<DEP, DH, MULTI, false>(a, grid, s);
    } else if (CONT) {
        k_walk_refill<DEP, MULTI><<<grid, 256, 0, s>>>(a);
    } else {
        k_push_move_deposit<DEP, DH, CONT, MULTI><<<grid, 256, 0, s>>>(a);
    }
    return cudaGetLastError();
}

template <bool CONT>
static cudaError_t launch_pmd_c(int dep, int dh, bool multi, const StepArgs &a, int grid,
                                bool tiled, cudaStream_t s) {
    if (CONT) dh = 0;   // the continuation resumes walks: no seeding
#define OPP_CASE(D, H, M) \
    if (dep == D && dh == H && multi == M) return launch_pmd_t<D, H, CONT, M>(a, grid, tiled, s);
#define OPP_CASES(H) \
    OPP_CASE(0, H, false) OPP_CASE(1, H, false) OPP_CASE(2, H, false) \
    OPP_CASE(0, H, true) OPP_CASE(1, H, true) OPP_CASE(2, H, true)
    OPP_CASES(0)
    if (!CONT) {
        OPP_CASES(1)
        OPP_CASES(2)
    }
#undef OPP_CASES
#undef OPP_CASE
    return cudaErrorInvalidValue;
}

cudaError_t launch_push_move_deposit(int dep, int dh, bool multi, bool cont, bool tiled,
                                     const StepArgs &a, int grid, cudaStream_t s) {
    return cont ? launch_pmd_c<true>(dep, dh, multi, a, grid, tiled, s)
                : launch_pmd_c<false>(dep, dh, multi, a, grid, tiled, s);
}

int pmd_blocks_per_sm(bool tiled, int minb) {
    int nb = 0;
    cudaError_t e;
    if (tiled) {
        if (minb >= 3) {
            cudaFuncSetAttribute(k_push_move_deposit_tiled<0, 0, false, false, OPP_MINB_HI>,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, kTiledSmem);
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                &nb, k_push_move_deposit_tiled<0, 0, false, false, OPP_MINB_HI>, kTiledThreads, kTiledSmem);
        } else {
            cudaFuncSetAttribute(k_push_move_deposit_tiled<0, 0, false, false, 1>,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, kTiledSmem);
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                &nb, k_push_move_deposit_tiled<0, 0, false, false, 1>, kTiledThreads, kTiledSmem);
        }
    } else {
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            &nb, k_push_move_deposit<0, 0, false, false>, 256, 0);
    }
    return (e == cudaSuccess && nb > 0) ? nb : 1;
}

cudaError_t launch_mig_count(const int32_t *mig_cell, const DevCounters *c, const RankRanges &rr,
                             unsigned long long *counts, int grid, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(counts, 0, sizeof(unsigned long long) * rr.n, s);
    if (e != cudaSuccess) return e;
    k_mig_count<<<grid, 256, 0, s>>>(mig_cell, c, rr, counts);
    return cudaGetLastError();
}

cudaError_t launch_mig_pack(const ColSet &cols, int p2c_col, const uint32_t *mig,
                            const int32_t *mig_cell, const int32_t *mig_hops, const DevCounters *c,
                            const RankRanges &rr, unsigned long long *cursor, char *sendbuf,
                            int rec_bytes, int grid, cudaStream_t s) {
    k_mig_pack<<<grid, 256, 0, s>>>(cols, p2c_col, mig, mig_cell, mig_hops, c, rr, cursor, sendbuf,
                                    rec_bytes);
    return cudaGetLastError();
}

cudaError_t launch_mig_unpack(const ColSet &cols, const char *recvbuf, long long R, int rec_bytes,
                              DevCounters *c, uint32_t *work, int32_t *work_hops, int grid,
                              cudaStream_t s) {
    k_mig_unpack<<<grid, 256, 0, s>>>(cols, recvbuf, R, rec_bytes, c, work, work_hops);
    return cudaGetLastError();
}

cudaError_t launch_halo_pack(const double *Q, const int32_t *idx, long long m, double *out,
                             cudaStream_t s) {
    int g = (int)std::min<long long>(1184, (m + 255) / 256);
    k_halo_pack<<<g > 0 ? g : 1, 256, 0, s>>>(Q, idx, m, out);
    return cudaGetLastError();
}

cudaError_t launch_halo_add(double *Q, const int32_t *idx, long long m, const double *in,
                            cudaStream_t s) {
    int g = (int)std::min<long long>(1184, (m + 255) / 256);
    k_halo_add<<<g > 0 ? g : 1, 256, 0, s>>>(Q, idx, m, in);
    return cudaGetLastError();
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

// Compact overlay: per 4x4x4 brick, base = the lowest tet id, offsets int16;
// *overflow set if some brick spans more than 32767 ids (then the int32 map
// stays in use).
__global__ void k_overlay_compact(const int32_t *__restrict__ map, Overlay ov, int16_t *off,
                                  int32_t *base, unsigned *overflow) {
    const long long nbt = (long long)ov.nbc[0] * ov.nbc[1] * ov.nbc[2];
    for (long long b = (long long)blockIdx.x * blockDim.x + threadIdx.x; b < nbt;
         b += (long long)gridDim.x * blockDim.x) {
        const int bx = (int)(b % ov.nbc[0]), by = (int)((b / ov.nbc[0]) % ov.nbc[1]),
                  bz = (int)(b / ((long long)ov.nbc[0] * ov.nbc[1]));
        int v[64];
        int lo = INT_MAX, hi = -1;
        for (int e = 0; e < 64; e++) {
            const int ix = 4 * bx + (e & 3), iy = 4 * by + ((e >> 2) & 3), iz = 4 * bz + (e >> 4);
            int t = -1;
            if (ix < ov.n[0] && iy < ov.n[1] && iz < ov.n[2]) t = map[ov_slot32(ov, ix, iy, iz)];
            v[e] = t;
            if (t >= 0) {
                lo = min(lo, t);
                hi = max(hi, t);
            }
        }
        if (hi >= 0 && hi - lo > 32767) atomicOr(overflow, 1u);
        const int bs = hi >= 0 ? lo : 0;
        base[b] = bs;
        for (int e = 0; e < 64; e++) off[b * 64 + e] = (int16_t)(v[e] >= 0 ? v[e] - bs : -32768);
    }
}

cudaError_t launch_overlay_compact(const int32_t *map, const Overlay &ov, int16_t *off, int32_t *base,
                                   unsigned *overflow, cudaStream_t s) {
    const long long nbt = (long long)ov.nbc[0] * ov.nbc[1] * ov.nbc[2];
    cudaError_t e = cudaMemsetAsync(overflow, 0, sizeof(unsigned), s);
    if (e != cudaSuccess) return e;
    long long g = (nbt + 127) / 128;
    k_overlay_compact<<<(unsigned)(g > 0 ? (g < 65535 ? g : 65535) : 1), 128, 0, s>>>(map, ov, off, base,
                                                                                  overflow);
    return cudaGetLastError();
}

cudaError_t launch_overlay(const WalkLine *lines, const double *xyz, long long nc, int cell_base,
                           const Overlay &ov, int32_t *map, cudaStream_t s) {
    long long tot = (long long)ov.nb[0] * ov.nb[1] * ov.nb[2] * 32;   // bricks incl. padding
    int g1 = (int)((tot + 255) / 256), g2 = (int)((nc + 255) / 256);
    k_overlay_init<<<g1 > 0 ? g1 : 1, 256, 0, s>>>(map, tot);
    k_overlay_build<<<g2 > 0 ? g2 : 1, 256, 0, s>>>(lines, xyz, nc, cell_base, ov, map);
    k_overlay_finish<<<g1 > 0 ? g1 : 1, 256, 0, s>>>(map, tot);
    return cudaGetLastError();
}

cudaError_t launch_sr(const StepArgs &a, long long nc, long long nn, unsigned *hist,
                      unsigned *start, unsigned long long *tile_sums, double *sorted,
                      double *cellsum, const int32_t *n2cs_ptr, const int32_t *n2cs, int grid,
                      cudaStream_t s) {
    cudaMemsetAsync(hist, 0, sizeof(unsigned) * (nc + 1), s);
    k_sr_hist<<<grid, 256, 0, s>>>(a.sr_cell, a.cnt, hist);
    cudaError_t e = scan_exclusive(hist, start, nc + 1, tile_sums, s);
    if (e != cudaSuccess) return e;
    cudaMemcpyAsync(hist, start, sizeof(unsigned) * (nc + 1), cudaMemcpyDeviceToDevice, s);
    k_sr_scatter<<<grid, 256, 0, s>>>(a.sr_cell, a.sr_val, a.cap, a.cnt, hist, sorted);
    int gc = (int)((nc + 255) / 256), gn = (int)((nn + 255) / 256);
    k_sr_cell_reduce<<<gc > 0 ? gc : 1, 256, 0, s>>>(start, sorted, nc, cellsum);
    k_sr_node_gather<<<gn > 0 ? gn : 1, 256, 0, s>>>(n2cs_ptr, n2cs, cellsum, nn, a.Q);
    return cudaGetLastError();
}

}  // namespace opp
