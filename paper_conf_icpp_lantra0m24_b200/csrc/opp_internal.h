// opp_internal.h -- device data layouts shared by the host library and the
// sm_100a kernels of libopp.  Nothing here is visible through include/opp.h.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace opp {

// One 128-byte, 128-byte-aligned "walk line" per cell: everything one cell
// visit of the walk and the deposit needs, in a single L2 line (SURVEY.md
// §8(a)).  lambda_i = g_i . (x - p0), i = 1..3; lambda_0 = 1 - (l1+l2+l3)
// (node-relative form: keeps absolute accuracy far from the origin).
struct __align__(128) WalkLine {
    double g[9];      // rows: grad lambda_1, grad lambda_2, grad lambda_3
    double p0[3];     // local node 0
    int32_t c2c[4];   // neighbour across the face opposite local node i (global id), -1 boundary
    int32_t c2n[4];   // local node ids (for the deposit)
};
static_assert(sizeof(WalkLine) == 128, "walk line must be one 128-B line");

// Device-resident counters: the particle count lives on the device so a
// whole step can be enqueued without a host round trip.
struct DevCounters {
    unsigned long long n;            // committed particle count
    unsigned long long n_before;     // count entering the last push
    unsigned long long n_injected;   // injected since the last push
    unsigned long long n_inj_last;   // snapshot of n_injected at the last push
    unsigned long long n_holes;      // holes recorded by the last push (R)
    unsigned long long n_work;       // deferred walks (continuation worklist)
    unsigned long long n_deferred;   // snapshot of n_work for stats
    unsigned long long total_hops;
    unsigned long long n_capped;
    unsigned long long n_head, n_tail;   // hole-fill pairing lists
    unsigned long long n_removed_last;   // R of the last fill
    unsigned long long n_removed;        // REMOVE count of the last push
    unsigned long long n_mig_out, n_mig_in;
    unsigned long long inj_done_blocks;  // last-block-commit ticket for k_inject
    unsigned long long n_sr;             // SR deposit: number of stored records
    unsigned long long cum_pushed;       // sum of n_before over all steps
    unsigned long long cum_steps;
    unsigned long long n_mig;            // migrants recorded (current round)
    unsigned long long work_cursor;      // continuation: next worklist entry to claim
    unsigned long long unpack_done_blocks;
    unsigned int max_hops;
    unsigned int err_flags;              // bit 0: non-positive tet, bit 1: SR overflow
    unsigned long long pad[8];
};

constexpr int kMaxCols = 16;

// Generic particle column (a particle dat or the p2c map) for inject /
// hole fill / growth: SoA, elem_bytes in {4, 8}, dim components of stride
// `cap` elements each.
struct ColDesc {
    char *ptr;
    long long cap;
    int elem_bytes;
    int dim;
};
struct ColSet {
    ColDesc c[kMaxCols];
    const char *src[kMaxCols];   // k_inject: AoS source per column
    int n;
};

// One launch of the sort's gather: columns of equal capacity, each gathered
// from src into its spare dst.
struct GatherCols {
    const char *src[kMaxCols];
    char *dst[kMaxCols];
    int dim[kMaxCols];
    int eb[kMaxCols];
    int n;
    long long cap;
};

// Direct-hop overlay.
struct Overlay {
    double x0[3];
    double dx;
    double inv_dx;        // 1.0 / dx, rounded once on the host
    int n[3];
    int nb[3];            // bricks of 4x4x2 overlay cells (see ov_slot32)
    const int32_t *map;   // nb[0]*nb[1]*nb[2]*32 slots, -1 = no tet / padding
    // compact form (used when every 4x4x4 brick's tets lie within 32767 ids
    // of the brick's lowest): one 128-B line of 64 int16 offsets per brick +
    // an int32 base per brick -- twice the overlay cells per line, so the
    // lookups of a warp (particles of one or two tets) touch about half the
    // lines.  -32768 = no tet.
    int compact;
    int nbc[3];           // bricks of 4x4x4 overlay cells
    const int16_t *off;   // nbc[0]*nbc[1]*nbc[2]*64
    const int32_t *base;  // nbc[0]*nbc[1]*nbc[2]
};

struct StepArgs {
    double *pos;      // SoA [3][cap]
    double *vel;      // SoA [3][cap]
    int32_t *p2c;     // [cap], global cell ids; -1 = hole
    long long cap;
    const WalkLine *lines;     // local cells
    const double4 *ef;         // local cells, padded
    double *Q;                 // node charge (local nodes)
    DevCounters *cnt;
    uint32_t *holes;           // [cap]
    uint32_t *work;            // [cap] deferred particle indices
    int32_t *work_hops;        // [cap]
    int32_t *sr_cell;          // SR records (cell, 4 values)
    double *sr_val;            // [4][cap]
    uint32_t *mig;             // migrants: particle index, target global cell, hops
    int32_t *mig_cell;
    int32_t *mig_hops;
    double c1, dt, w;
    int cell_base, n_cells;    // global id of local cell 0, local cell count
    int hpass, hcap;
    int tile_group;            // consecutive 256-particle tiles per block visit (>= 1)
    int dcache;                // per-warp node-charge cache (opp_init_params.deposit_cache)
    Overlay ov;
    int n_nodes;               // local nodes (bounds of Q; checked builds)
    double *cacc;              // ATOMIC_WARPAGG: per-cell node-slot sums [4 * n_cells] (zeroed per
                               // step, gathered into Q after the move); null = reduce into Q
    int32_t *pcell;            // non-null on the step before a sort: the sort-key cell of
                               // every pushed particle (overlay tet of x + lead_dt v, -1 none)
    double lead_dt;
};

// Slab partition: rank r owns global cells [lo[r], hi[r]).
constexpr int kMaxRanks = 64;
struct RankRanges {
    int lo[kMaxRanks];
    int hi[kMaxRanks];
    int n;
};

}  // namespace opp
