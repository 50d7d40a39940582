/*
 * opp.h -- C ABI of the B200-native OP-PIC particle-loop library (libopp.so).
 *
 * The library implements the one data-parallel hot path of OP-PIC's
 * unstructured-mesh PIC method (Lantra, Wright, Mudalige, ICPP '24): the
 * per-timestep electrostatic particle loop on a tetrahedral mesh --
 * inject, gather the cell field, leap-frog push, multi-hop / direct-hop cell
 * walk, charge deposit to the cell's 4 nodes, hole-filling compaction, and
 * (nranks > 1) slab migration and node-charge halo over NCCL.
 * Citations are PAPER.md line ranges (section / figure / equation).
 *
 * Conventions (all entry points):
 *  - Every function returns an opp_status (0 = OPP_OK, < 0 = error) unless
 *    stated otherwise; on error opp_last_error() returns a thread-local
 *    message.  A failing call leaves the context unchanged, except that an
 *    asynchronous CUDA/NCCL failure is sticky and reported by the next call.
 *  - Handles (opp_set, opp_map, opp_dat) are small integers valid for the
 *    lifetime of the context that issued them.
 *  - Host pointers passed to opp_decl_* / opp_inject(on_device = 0) are read
 *    during the call (or, for opp_inject, before the call's stream work
 *    completes if the memory is pinned: keep it alive until the next
 *    synchronising call); the library copies, the caller keeps ownership.
 *    Device pointers (on_device = 1) must be valid device memory of
 *    params.device, ordered before the call on params.cuda_stream.
 *  - All work is enqueued on params.cuda_stream.  Calls that return data to
 *    the host (opp_get_*, opp_push_move_deposit with stats != NULL,
 *    opp_fill_holes with n_after != NULL) synchronise that stream.
 *  - Layouts: mesh dats are stored AoS ([n][dim], "dim" contiguous);
 *    particle dats and the particle->cell map are stored SoA on the device
 *    ([dim][capacity]) for coalesced per-component streaming.  Host-side
 *    arrays exchanged through this ABI are always AoS [n][dim].
 *  - One host thread per context; one context (process) per GPU.
 */
#ifndef OPP_H
#define OPP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct opp_ctx_s *opp_ctx;
typedef int32_t opp_set;
typedef int32_t opp_map;
typedef int32_t opp_dat;

enum opp_status {
    OPP_OK = 0,
    OPP_ERR_ARG = -1,      /* bad handle, size, type or pointer            */
    OPP_ERR_STATE = -2,    /* call not valid now (e.g. dats contain holes) */
    OPP_ERR_NOMEM = -3,    /* device / host allocation failed              */
    OPP_ERR_CAPACITY = -4, /* particle capacity exceeded, growth disabled  */
    OPP_ERR_CUDA = -5,     /* CUDA runtime / kernel error                  */
    OPP_ERR_NCCL = -6,     /* NCCL error, or NCCL not available            */
    OPP_ERR_MESH = -7      /* invalid mesh: non-positive tet, bad c2c      */
};

/* opp_decl_dat types (Fig. 4: OPP_REAL ...) */
enum opp_type { OPP_REAL = 0 /* fp64 */, OPP_INT = 1 /* int32 */, OPP_INT64 = 2 };

/* Per-particle move status (Fig. 6; 1336-1340 "marked
 * for communication" -> NEED_MIGRATE). */
enum opp_move_status { OPP_MOVE_DONE = 0, OPP_NEED_MOVE = 1, OPP_NEED_REMOVE = 2,
                       OPP_NEED_MIGRATE = 3 };

/* Deposit race handling (§3.3 and Fig. 3):
 * ATOMIC        one fp64 atomic add per (particle, node)              ("AT")
 * ATOMIC_WARPAGG same-cell contributions of a warp summed by shuffles
 *                before one set of 4 atomics per distinct cell, into the
 *                cell's 4 node slots (32 contiguous bytes); after the
 *                step's walks every node adds its slots in a fixed order
 *                (Eq. 10 unchanged: the same w*lambda_i, summed per cell
 *                first)
 * SORT_SEGRED   store (cell, w*lambda[4]) per particle, counting-sort by
 *                cell, reduce per cell, then per node               ("SR")
 * AUTO          library choice by measurement: ATOMIC_WARPAGG (fastest on
 *               C2, C4 and the clustered C5)                */
enum opp_deposit_mode { OPP_DEP_ATOMIC = 0, OPP_DEP_ATOMIC_WARPAGG = 1,
                        OPP_DEP_SORT_SEGRED = 2, OPP_DEP_AUTO = 3 };

typedef void *(*opp_alloc_fn)(size_t bytes, void *cuda_stream, void *user);
typedef void (*opp_free_fn)(void *ptr, size_t bytes, void *cuda_stream, void *user);

typedef struct {
    int device;                 /* CUDA device ordinal                               */
    void *cuda_stream;          /* cudaStream_t; NULL = the legacy default stream    */
    int rank, nranks;           /* slab partition index / count (nranks >= 1)        */
    const void *nccl_unique_id; /* 128-byte ncclUniqueId, required iff nranks > 1    */
    opp_alloc_fn alloc;         /* optional device allocator (e.g. torch's caching   */
    opp_free_fn free;           /*  allocator); NULL = cudaMalloc / cudaFree         */
    void *alloc_user;
    int deposit_mode;           /* enum opp_deposit_mode                             */
    int direct_hop;             /* DH: 0 = multi-hop only;
                                   1 = every particle's walk starts at the overlay
                                   seed of its pushed position; 2 = only a particle
                                   no longer inside its cell takes the seed
                                   (reading S19''); else OPP_ERR_ARG    */
    double overlay_spacing;     /* DH overlay cell size (mesh units); <= 0: auto     */
    int hop_budget_per_pass;    /* H_pass: hops in the fused kernel before a particle
                                   is deferred to the continuation pass (>= 0;
                                   0 = the fused kernel tests the start cell only) */
    int hop_cap;                /* H_cap: hops after which the current cell is
                                   accepted as final and counted (S4)               */
    int allow_growth;           /* 1 = grow particle capacity x1.5 on injection     */
    int sort_every;             /* > 0: every sort_every-th step the hole fill is a
                                   counting sort by cell (also compacts), 0 = never */
    int tma_pipeline;           /* 1 = stream particle tiles through shared memory
                                   with cp.async.bulk (default), 0 = direct loads   */
    int transport;              /* nranks > 1: 0 = NCCL (one process per GPU),
                                   1 = in-process loopback (contexts in one process,
                                   one host thread each; testing on one GPU)        */
    double sort_axis[3];        /* principal direction of motion
                                   used as the sort-by-cell locality key: cells are
                                   ordered by transverse bin, then along the axis;
                                   (0,0,0) = plain cell-id order                    */
    int deposit_cache;          /* ATOMIC_WARPAGG in the TMA pipeline: 1 = cell sums
                                   accumulate in a per-warp shared-memory cache
                                   across slices and leave with 4 node reductions
                                   when evicted (instead of the per-cell node
                                   slots); measured slower than the default on C2,
                                   C4 and the clustered C5; 0 = off
                                   (default)                                        */
    double sort_lead;           /* periodic sort (sort_every > 0) keyed at the
                                   ballistic extrapolation x + sort_lead*dt*v of each
                                   particle (the DH overlay's tet of that point, else
                                   the particle's cell) instead of its cell: the
                                   order is then best sort_lead steps after the sort
                                   (sort_every/2 centres it on the interval) rather
                                   than right after it.  The order of the set is
                                   implementation-defined (an
                                   auxiliary sort; reading S10), so results
                                   do not depend on it.  Needs direct_hop != 0;
                                   0 = key at the current cell (default)            */
} opp_init_params;

/* Per-step arguments of opp_push_move_deposit. */
typedef struct {
    double dt;          /* time step                                                */
    double qm;          /* charge / mass; the push uses c1 = qm * dt (one host mult) */
    double weight;      /* macro-particle charge Q_p of Eq. 10   */
    int zero_charge;    /* 1 = node charge := 0 before depositing                   */
    int fill_inline;    /* 1 = also run the hole fill (opp_fill_holes) in this call */
} opp_step_params;

/* Step statistics (filled when a stats pointer is given; one D2H copy). */
typedef struct {
    int64_t n_before;       /* particles entering the push (incl. injected)   */
    int64_t n_injected;     /* injected since the previous push               */
    int64_t n_removed;      /* left through a boundary face (NEED_REMOVE)     */
    int64_t n_after;        /* n_before - n_removed - migrated out + in        */
    int64_t n_migrated_out, n_migrated_in;
    int64_t total_hops;     /* sum over particles of cell hops this step      */
    int64_t n_hop_capped;   /* walks stopped by H_cap (must be 0 on valid meshes) */
    int64_t n_deferred;     /* particles handed to the continuation pass      */
    int32_t max_hops;
    int32_t migrate_rounds;
    int64_t cum_pushed;     /* sum of n_before over every step of this set so far */
    int64_t cum_steps;      /* number of steps of this set so far              */
} opp_step_stats;

/* Fill *p with defaults: device 0, default stream, 1 rank, cudaMalloc,
 * OPP_DEP_ATOMIC, MH only, overlay_spacing 0 (auto = 0.5 * mean edge),
 * H_pass = 4, H_cap = 1024, growth allowed, no periodic sort, TMA pipeline on. */
void opp_init_params_default(opp_init_params *p);

/* Create a context on params->device (nranks > 1: joins the NCCL clique). */
int opp_init(const opp_init_params *params, opp_ctx *out);
/* Free every device allocation and the NCCL communicator. */
int opp_finalize(opp_ctx ctx);

/* Rank 0 calls this and broadcasts the 128 bytes (e.g. via torch.distributed);
 * returns OPP_ERR_NCCL if the library was built without NCCL. */
int opp_get_nccl_unique_id(void *out128);

/* opp_decl_set (Fig. 4 l.2-3): a mesh set of `size` elements. */
int opp_decl_set(opp_ctx ctx, int64_t size, const char *name, opp_set *out);

/* opp_decl_particle_set (Fig. 4 l.6-7): a particle set
 * living on mesh set `cells` with n_init particles whose data follow in
 * opp_decl_dat / opp_decl_map; `capacity` (>= n_init, 0 = auto) is the
 * initial allocation. */
int opp_decl_particle_set(opp_ctx ctx, const char *name, opp_set cells, int64_t n_init,
                          int64_t capacity, opp_set *out);

/* opp_decl_map (Fig. 4 l.12-15): `dim` int32
 * entries per element of `from` pointing into `to` (-1 = none).
 * Mesh maps: c2n (dim 4) and c2c (dim 4; c2c[c][i] = the cell across the
 * face opposite local node c2n[c][i], -1 = domain boundary; validated,
 * OPP_ERR_MESH otherwise).  Particle maps: p2c (dim 1, from a particle set);
 * host may be NULL iff the set has n_init == 0.  Global
 * cell ids when nranks > 1. */
int opp_decl_map(opp_ctx ctx, opp_set from, opp_set to, int dim, const int32_t *host,
                 const char *name, opp_map *out);

/* opp_decl_dat (Fig. 4 l.20-30): `dim` values of
 * `type` per element of `set`, initialised from host (AoS [n][dim]) or zero
 * if host == NULL (NULL allowed for node/cell dats and empty particle sets). */
int opp_decl_dat(opp_ctx ctx, opp_set set, int dim, int type, const void *host,
                 const char *name, opp_dat *out);

/* Slab partition (the user provides the rank of one set
 * "via an opp_dat"; the library derives the rest).  Collective: every rank
 * calls it.  rank_of_cell[g] for every GLOBAL cell g (n_global_cells
 * entries); each rank's cells must form one contiguous global range, and
 * this context's `cells` set holds exactly its range, in order (so local
 * cell k is global cell base + k; c2c and p2c carry global ids).  node_gid
 * gives a global id for each of this rank's `nodes` (required iff
 * nranks > 1): nodes with equal ids on two ranks form the charge halo. */
int opp_set_partition(opp_ctx ctx, opp_set cells, int64_t n_global_cells,
                      const int32_t *rank_of_cell, opp_set nodes, const int64_t *node_gid);

/* opp_inject (PAPER.md:1014-1018 OPP_ITERATE_INJECTED, 1502-1508): append n
 * particles at [N, N+n).  cols lists EVERY particle dat / the p2c map of the
 * set (any order) and data[k] points to that column's n*dim values (AoS),
 * host (on_device = 0, copied H2D on the stream; pinned memory makes it
 * asynchronous) or device (on_device = 1).  Grows capacity if needed. */
int opp_inject(opp_ctx ctx, opp_set parts, int64_t n, int ncols, const int32_t *cols,
               const void *const *data, int on_device);

/* The fused electrostatic particle loop -- one time step (PAPER.md:398-410
 * Fig. 1 steps 2-4; CalcPosVel + Move + DepositCharge of 1586-1604):
 *   [zero node_charge]
 *   for every particle p (any order):
 *     E = cell_ef[p2c[p]]                      (cell-constant, 1576-1585)
 *     v += (qm*dt) * E ; x += v * dt           (leap-frog, 569-583)
 *     [DH] seed cell from the overlay          (1356-1370)
 *     walk: lambda = barycentric(x, cell); inside iff all lambda in [0,1];
 *           else cross the face opposite argmin lambda via c2c (595-603);
 *           -1 -> NEED_REMOVE (1508-1510); H_cap -> accept (S4)
 *     DONE: node_charge[c2n[cell][i]] += weight * lambda_i   (Eq. 10, 637-660)
 *     NEED_REMOVE: recorded as a hole (filled by opp_fill_holes)
 *   nranks > 1: migrants exchanged over NCCL until no rank has any; then the
 *   interface-node charge halo is summed (1280-1300, 1336-1354).
 * pos, vel: particle dats dim 3 OPP_REAL; p2c: particle map dim 1;
 * c2c, c2n: cell maps dim 4; node_pos: node dat dim 3 OPP_REAL;
 * cell_ef: cell dat dim 3 OPP_REAL; node_charge: node dat dim 1 OPP_REAL.
 * Between this call and opp_fill_holes the particle dats contain holes
 * (opp_get_dat returns OPP_ERR_STATE) unless params->fill_inline.
 * stats may be NULL (no host synchronisation).
 * A particle whose p2c entry is not one of this rank's cells (bad input to
 * opp_inject / opp_set_dat) is dropped as a hole without any memory access
 * through it; the next call that reads the step statistics (this one with
 * stats != NULL, or opp_get_step_stats) returns OPP_ERR_ARG once. */
int opp_push_move_deposit(opp_ctx ctx, opp_set parts, opp_dat pos, opp_dat vel, opp_map p2c,
                          opp_map c2c, opp_map c2n, opp_dat node_pos, opp_dat cell_ef,
                          opp_dat node_charge, const opp_step_params *params,
                          opp_step_stats *stats);

/* Statistics of the most recent opp_push_move_deposit on `parts` (and the
 * cumulative counters); synchronises.  Lets a caller run steps with
 * stats == NULL (no host round trip) and read the numbers afterwards. */
int opp_get_step_stats(opp_ctx ctx, opp_set parts, opp_step_stats *stats);

/* Hole filling ("shifting data from the end of the
 * opp_dats to fill the holes"): survivors at index >= N' = N - R move into the
 * holes below N'.  Particle order afterwards is implementation-defined.
 * n_after may be NULL (no host synchronisation). */
int opp_fill_holes(opp_ctx ctx, opp_set parts, int64_t *n_after);

/* Reorder the particle set by cell (counting sort; PAPER.md:1638-1644
 * "particle sorting is available as an auxiliary API call").  Drops holes
 * if a step left any (it then replaces opp_fill_holes).  Order within a cell
 * is implementation-defined. */
int opp_sort_by_cell(opp_ctx ctx, opp_set parts);

/* Random shuffle of the particle set -- the paper's "periodic shuffling"
 * (on its GPUs shuffling + hole fill beat sorting, since
 * it spreads same-cell particles and their atomics apart).  Every particle
 * draws a bucket from a counter-based hash of (index, seed); a counting sort
 * by bucket moves all columns (holes are dropped, like opp_sort_by_cell).
 * The permutation depends on seed and on the atomic order inside a bucket;
 * results of later steps are unchanged up to the deposit's summation order.
 * Call between steps.  Errors as opp_sort_by_cell. */
int opp_shuffle(opp_ctx ctx, opp_set parts, uint64_t seed);

/* Copy node charge (dim 1) to host_out[n]; synchronises. */
int opp_get_node_charge(opp_ctx ctx, opp_dat node_charge, double *host_out, int64_t n);

/* Copy the first n_elems elements of any dat or map to host (AoS); for
 * particle sets n_elems must equal the current count.  Synchronises. */
int opp_get_dat(opp_ctx ctx, int32_t dat_or_map, void *host_out, int64_t n_elems);

/* Overwrite the first n_elems elements of a dat (AoS source, host or device),
 * e.g. the per-step cell field.  Mesh maps are static. */
int opp_set_dat(opp_ctx ctx, opp_dat dat, const void *src, int64_t n_elems, int on_device);

/* Current particle count (synchronises). */
int opp_get_particle_count(opp_ctx ctx, opp_set parts, int64_t *n);

/* Device pointer + row stride (elements) of a dat/map column, for zero-copy
 * interop (read-only use); SoA for particle sets. */
int opp_get_dat_device_ptr(opp_ctx ctx, int32_t dat_or_map, void **ptr, int64_t *stride);

/* Phases of the step timed by opp_phase_timing (indices into ms_sum / count). */
enum opp_phase { OPP_PH_INJECT = 0, OPP_PH_BEGIN = 1, OPP_PH_PUSH_MOVE_DEPOSIT = 2,
                 OPP_PH_CONTINUE = 3, OPP_PH_SEGRED = 4, OPP_PH_FILL = 5, OPP_PH_MIGRATE = 6,
                 OPP_PH_HALO = 7, OPP_PH_SORT_COUNT = 8, OPP_PH_SORT_MOVE = 9,
                 OPP_PH_FIELD = 10, OPP_PH_EM_MOVE_DEPOSIT = 11, OPP_N_PHASES = 12 };

/* enable != 0: record CUDA events on the context stream around every phase
 * of the following calls (negligible overhead, no host synchronisation). */
int opp_phase_timing(opp_ctx ctx, int enable);

/* Sum of the recorded device time per phase (ms_sum[OPP_N_PHASES]) and the
 * number of recorded instances (count[OPP_N_PHASES]) since timing was
 * enabled or last read; synchronises, then resets the records. */
int opp_get_phase_times(opp_ctx ctx, double *ms_sum, int64_t *count);

/* Number of kernels this context has launched so far (evidence counter). */
int64_t opp_kernel_launch_count(opp_ctx ctx);

/* ---------------------------------------------------------------------------
 * Field solve: step 1 of the PIC loop (Fig. 1, Gauss' law
 * Eq. 1) by the finite-element method on the tetrahedral mesh.
 * Mini-FEM-PIC's ComputeJMatrix / ComputeF1Vector / linear solve /
 * ComputeElectricField (Fig. 6) in the
 * linear form north_star names ("a plain GPU conjugate-gradient on the FEM
 * Poisson system"; the Boltzmann-electron Newton solve is
 * opp_field_solve_boltzmann below):
 *   K phi = b,  K_ij = sum_e V_e grad(lambda_i) . grad(lambda_j)   (P1 Laplacian)
 *   b = rhs_scale * node_charge    (the consistent P1 load of the deposited
 *                                   point charges, Eq. 10; F2)
 *   phi = dirichlet_value on Dirichlet nodes; homogeneous Neumann elsewhere
 *   E_c = -sum_i phi[c2n[c][i]] grad(lambda_i)   (cell-constant, 1576-1585)
 * nranks > 1: every rank assembles its slab's cells; interface rows are
 * completed by the node halo exchange of the charge halo (opp_set_partition)
 * and dot products count each node once; every rank's dots are all-gathered
 * on the stream and summed in rank order on the device, which forms alpha,
 * beta and the stop test (the host reads one flag per batch of 8 iterations;
 * one rank runs one persistent kernel).
 * ------------------------------------------------------------------------- */
typedef struct {
    double rhs_scale;   /* b = rhs_scale * node_charge (q / eps0 per unit weight)       */
    double tol;         /* stop when ||r||_2 <= tol * ||b_F - K_FD phi_D||_2 (>= 0)      */
    int max_iter;       /* iteration cap (>= 0)                                          */
    int warm_start;     /* 1: free nodes start from node_potential's current values;
                           2: from 2 phi_{n-1} - phi_{n-2}, the linear extrapolation of the
                           last two solutions of warm-start-2 solves into this dat (the
                           first such solve starts like 1); 0: from 0                   */
    int precond;        /* 0: plain CG; 1: Jacobi (diagonal) preconditioned CG          */
    int slab_cg;        /* 1: run the slab (multi-rank) CG on one rank too (testing it);
                           0: one rank uses the persistent kernel                      */
} opp_field_params;

typedef struct {
    int32_t iterations; /* CG iterations of the last solve                              */
    int32_t converged;  /* 1 if the tolerance was met (0: max_iter reached)             */
    double rel_residual;/* ||r||_2 / ||b_F - K_FD phi_D||_2 (recursive residual)         */
    double rhs_norm;    /* ||b_F - K_FD phi_D||_2                                        */
} opp_field_stats;

/* Build the P1 system on the mesh of c2n (cells -> nodes, dim 4) with node
 * coordinates node_pos (dim 3 OPP_REAL): the sparsity (sliced ELLPACK, 32
 * rows per slice), the stiffness values (assembled on the device in a fixed
 * order: deterministic) and the Dirichlet data.  dirichlet_mask[n] != 0 marks
 * node n Dirichlet with value dirichlet_value[n] (host arrays of the node
 * count; copied).  Maps are static: call again to rebuild.
 * nranks > 1: collective, after opp_set_partition (node data are this rank's
 * nodes).  Errors: OPP_ERR_ARG (handles, NULL), OPP_ERR_MESH (c2n out of
 * range), OPP_ERR_NOMEM, OPP_ERR_STATE (nranks > 1 before the partition).
 * Synchronises. */
int opp_field_init(opp_ctx ctx, opp_map c2n, opp_dat node_pos, const int32_t *dirichlet_mask,
                   const double *dirichlet_value);

/* Solve for node_potential (node dat dim 1 OPP_REAL; in: warm start if
 * params->warm_start, out: phi) from node_charge (node dat dim 1 OPP_REAL,
 * e.g. after opp_push_move_deposit), then write cell_ef (cell dat dim 3
 * OPP_REAL; -1 = skip) = -grad(phi) per cell, which the next
 * opp_push_move_deposit gathers.  One rank: one persistent cooperative kernel
 * runs the whole CG, enqueued on the stream; stats may be NULL (no
 * synchronisation; read them later with opp_get_field_stats).  nranks > 1:
 * collective, synchronises once per iteration. */
int opp_field_solve(opp_ctx ctx, opp_dat node_charge, opp_dat node_potential, opp_dat cell_ef,
                    const opp_field_params *params, opp_field_stats *stats);

/* Statistics of the last opp_field_solve; synchronises. */
int opp_get_field_stats(opp_ctx ctx, opp_field_stats *stats);

/* ---------------------------------------------------------------------------
 * Boltzmann-electron field solve: the nonlinear
 * Poisson problem Mini-FEM-PIC solves by Newton's method with
 * ComputeF1Vector, ComputeJMatrix and a linear solver (PETSc KSP in the
 * paper; §4.1.1).  The paper names the routines only;
 * DESIGN.md §11 readings B1-B4 fix the formulas (normalised units):
 *   F_n(phi) = (K phi)_n - rhs_scale Q_n + ne_coef m_n exp((phi_n - phi0) / te)
 *   on free nodes (Dirichlet nodes hold dirichlet_value), m_n the lumped P1
 *   mass (sum over the node's cells of |V_e| / 4);
 *   J = K + diag(ne_coef m_n / te exp((phi_n - phi0) / te));
 *   Newton: J_FF delta_F = -F_F (Jacobi-)preconditioned CG to cg_tol relative
 *   to ||F_F||, phi_F += delta_F; start phi_F = phi0 (or the warm start);
 *   stop when ||F_F||_2 <= max(newton_tol ||F_F(phi_cold)||_2, newton_atol)
 *   or after max_newton steps, phi_cold = the cold start (phi0 on free
 *   nodes): a reference independent of the warm start.
 * Needs opp_field_init (same matrix, Dirichlet data and n2c).  node_charge /
 * node_potential / cell_ef as in opp_field_solve.  The loop is host-driven:
 * one ||F|| read-back per Newton step (synchronises).  nranks > 1 (slabs,
 * collective): K phi of interface rows is completed by the node halo, the
 * lumped mass likewise, the electron diagonal enters the Jacobian on the
 * owning rank's copy only, norms count each node once and are reduced across
 * ranks, and each Newton step runs the host-driven slab CG of
 * opp_field_solve.  Errors: OPP_ERR_ARG (te <= 0, ne_coef < 0,
 * tolerances < 0, max_newton / cg_max_iter < 0, NULL params), OPP_ERR_STATE,
 * OPP_ERR_NOMEM, OPP_ERR_CUDA.
 * ------------------------------------------------------------------------- */
typedef struct {
    double rhs_scale;   /* ion load b = rhs_scale * node_charge                          */
    double ne_coef;     /* electron term coefficient (n0 e / eps0 in solver units), >= 0 */
    double phi0;        /* reference potential (electron density = n0 at phi0)          */
    double te;          /* electron temperature in potential units (kTe / e), > 0       */
    double newton_tol;  /* relative stopping tolerance on ||F_F||_2 (>= 0)              */
    double newton_atol; /* absolute stopping tolerance on ||F_F||_2 (>= 0)              */
    double cg_tol;      /* inner CG: ||r|| <= cg_tol * ||F_F|| (>= 0); once ||F_F|| <= 1e-3
                           of the reference (the linear regime) the step solves only
                           as tightly as the stop needs: min(cg_tol, thr / (2 ||F_F||)) */
    int max_newton;     /* Newton step cap (>= 0)                                        */
    int cg_max_iter;    /* inner CG iteration cap per Newton step (>= 0)                 */
    int warm_start;     /* 1: free nodes start from node_potential's values; 2: from the
                           extrapolation of the last two warm-start-2 solutions (shared
                           with opp_field_solve); 0: phi0                              */
    int precond;        /* inner CG: 0 plain, 1 Jacobi (J's diagonal)                    */
} opp_boltzmann_params;

typedef struct {
    int32_t newton_steps;   /* Newton steps taken                                        */
    int32_t converged;      /* 1 if the stopping rule was met                            */
    int64_t cg_iterations;  /* inner CG iterations summed over the steps                 */
    double res_norm;        /* ||F_F(phi)||_2 at exit                                    */
    double res0_norm;       /* ||F_F(phi_start)||_2                                      */
    double ref_norm;        /* ||F_F(phi_cold)||_2, the stopping reference               */
} opp_boltzmann_stats;

int opp_field_solve_boltzmann(opp_ctx ctx, opp_dat node_charge, opp_dat node_potential,
                              opp_dat cell_ef, const opp_boltzmann_params *params,
                              opp_boltzmann_stats *stats);

/* ---------------------------------------------------------------------------
 * CabanaPIC-style electromagnetic particle loop (config C3; SURVEY.md §8(f)
 * NEXT-2): hex cells of a periodic nx*ny*nz grid declared as an unstructured
 * mesh through their cell-to-cell map.
 * All pointers are DEVICE pointers owned by the caller; calls are enqueued on
 * the context stream (no synchronisation unless stated).  Readings E1-E9 of
 * DESIGN.md §10 define what the paper leaves open.
 * ------------------------------------------------------------------------- */
typedef struct {
    double qdt_2mc;    /* q dt / (2 m c): E and B enter the push scaled by it            */
    double cdt_2h[3];  /* 2 c dt / h_a: offset units per unit u / gamma, per axis         */
    double qsp;        /* charge per unit weight (Q_p = qsp * w, Eq. 11)                  */
    int kcap;          /* face crossings allowed per particle and step (>= 0); at the cap
                          the particle stops on the face, inside its cell                 */
    int deposit_mode;  /* OPP_DEP_ATOMIC (12 fp64 reductions per segment) or
                          OPP_DEP_ATOMIC_WARPAGG (lanes sharing a cell summed in the warp) */
} opp_em_params;

typedef struct {
    int64_t n_crossings;   /* face crossings in the last opp_em_move_deposit             */
    int64_t n_capped;      /* particles stopped by kcap                                  */
    int32_t max_crossings;
    int32_t pad;
} opp_em_stats;

/* Interpolate: from edge E and face B of the periodic
 * grid to per-cell interpolators.  e[3][nc]: E_a on the cell's edge along a
 * at the (-,-) corner of its transverse offsets ((a+1)%3, (a+2)%3); the other
 * three edges of the cell are those of its transverse neighbours.  b[3][nc]:
 * B_a on the cell's face at offset -1 along a.  interp[nc][18]: ex, dexdy,
 * dexdz, d2exdydz, ey, deydz, deydx, d2eydzdx, ez, dezdx, dezdy, d2ezdxdy,
 * bx, dbxdx, by, dbydy, bz, dbzdz, so that E_a = f0 + s f1 + t (f2 + s f3)
 * with (s, t) the transverse offsets and B_a = f + x_a df.  Cell id =
 * i + nx (j + ny k).  Errors: OPP_ERR_ARG (sizes < 1, NULL). */
int opp_em_interpolate(opp_ctx ctx, int nx, int ny, int nz, const double *e, const double *b,
                       double *interp);

/* Move_Deposit: for particles [0, n) -- SoA columns of
 * row stride `stride` (elements): off[3][stride] offsets in [-1, 1]^3 of the
 * particle in its cell, u[3][stride] momenta gamma v / c, w[stride] weights,
 * cell[stride] -- interpolate E, B from interp[cell] (layout above), Boris-push
 * u (relativistic, exact rotation with t = qdt_2mc B / gamma), then move the
 * particle along its streak d_a = cdt_2h[a] u_a / gamma through the faces it
 * crosses, in order (first face hit; ties -> lowest axis; landing exactly on
 * a face is inside), the next cell from c2c[cell][f] (f = -x,+x,-y,+y,-z,+z;
 * n_cells rows), and add to acc[cell][12] the Eq. 11 current of every segment
 * (PAPER.md:637-680): for the edges along axis a, acc[4a + k] += Q_p *
 * integral of (1 + sb b)(1 + sc c)/4 d(offset_a) along the segment, edge k =
 * (sb, sc) in the order (-,-), (+,-), (-,+), (+,+) over the transverse
 * offsets (b, c) = ((a+1)%3, (a+2)%3).  off, u, cell are updated in place.
 * cell values must lie in [0, n_cells) and c2c must map into it (not
 * checked: out-of-range ids are undefined behaviour).  stats may be NULL (no
 * synchronisation); otherwise the call synchronises and fills it.
 * Errors: OPP_ERR_ARG (NULL, n < 0, stride < n, kcap < 0, bad mode). */
int opp_em_move_deposit(opp_ctx ctx, int64_t n, int64_t stride, double *off, double *u,
                        const double *w, int32_t *cell, const double *interp,
                        const int32_t *c2c, int64_t n_cells, double *acc,
                        const opp_em_params *params, opp_em_stats *stats);

/* Counting sort of the EM particles by cell (the auxiliary sort of
 * PAPER.md:1638-1644 applied to Move_Deposit: lanes of a warp then share a cell,
 * so the warp-aggregated current deposit sums one group): the n particles of
 * the input columns (row stride `stride`) are written, grouped by ascending
 * cell, to the output columns (same stride; must not alias the inputs).  The
 * order inside a cell is unspecified (any order is a correct sort).  Enqueued,
 * no synchronisation.  Errors: OPP_ERR_ARG (NULL, n < 0, stride < n),
 * OPP_ERR_NOMEM (scratch: 4 B per particle + 8 B per cell). */
int opp_em_sort_by_cell(opp_ctx ctx, int64_t n, int64_t stride, const double *off, const double *u,
                        const double *w, const int32_t *cell, int64_t n_cells, double *off_out,
                        double *u_out, double *w_out, int32_t *cell_out);

/* Field side of the EM loop ("the accumulator data is
 * processed in the AccumulateCurrent routine to obtain the current density
 * necessary for field solving.  Field solving follows a kernel based
 * leap-frog approach, with AdvanceE and AdvanceB"), normalised units
 * (c = eps0 = 1), Yee staggering matching opp_em_interpolate's layout: E_a and
 * J_a on the cell's edge along a at the (-,-) corner of its transverse
 * offsets, B_a on its face at offset -1; neighbours read through
 * c2c[n_cells][6]; h[3] the cell sizes; all arrays [3][n_cells] device
 * memory.  Enqueued, no synchronisation.  Errors: OPP_ERR_ARG (NULL,
 * n_cells < 1, h or dt not positive).
 *
 * AccumulateCurrent: J_a(edge) = (sum of the 4 adjacent cells' accumulator
 * entries for that edge) / (2 dt h_b h_c) -- with it the discrete continuity
 * equation (and so Gauss's law) holds exactly for the Eq. 11 deposit. */
int opp_em_accumulate_current(opp_ctx ctx, const double *acc, const int32_t *c2c, int64_t n_cells,
                              const double *h, double dt, double *J);
/* AdvanceB: B -= frac_dt * curl E (the leap-frog's half steps). */
int opp_em_advance_b(opp_ctx ctx, const double *e, double *b, const int32_t *c2c, int64_t n_cells,
                     const double *h, double frac_dt);
/* AdvanceE: E += dt * (curl B - J). */
int opp_em_advance_e(opp_ctx ctx, double *e, const double *b, const double *J, const int32_t *c2c,
                     int64_t n_cells, const double *h, double dt);

/* Statistics of the last opp_em_move_deposit; synchronises. */
int opp_em_get_stats(opp_ctx ctx, opp_em_stats *stats);

/* ---- CabanaPIC over slabs (config C3 on several GPUs; PAPER.md:1794-1800:
 * Update_Ghosts is the halo exchange of the CabanaPIC field side).  Each rank
 * (opp_init nranks / rank / transport) owns the z-layers [k0, k1) of the
 * periodic nx x ny x nz grid, i.e. cells [k0 nx ny, k1 nx ny); the ranks'
 * ranges must tile [0, nz) in rank order, so the neighbours are rank -+ 1
 * (mod nranks).  Collective.  Field arrays stay global-sized (nc cells) on
 * every rank: a rank computes its own cells and keeps the ghost layers it
 * reads current.  Errors: OPP_ERR_ARG (ranges do not tile). */
int opp_em_set_partition(opp_ctx ctx, int nx, int ny, int nz, int k0, int k1);

/* Move_Deposit over slabs: opp_em_move_deposit for this rank's particles
 * [0, *n) (columns of stride cap; id[cap] int64, may be NULL, travels with
 * its particle).  A particle whose path enters another rank's cell stops on
 * that face -- its deposits so far are this rank's -- and migrates with the
 * rest of its streak (96-B records over the transport, appended behind the
 * receiver's particles, which walks and deposits the rest); rounds repeat
 * until no rank has migrants; the departed particles' slots are filled from
 * the end.  On return *n = this rank's new count.
 * Collective.  Requires kcap >= 1.  Errors: OPP_ERR_STATE (no partition),
 * OPP_ERR_CAPACITY (arrivals beyond cap), OPP_ERR_ARG.  Synchronises once per
 * migration round (the message sizes). */
int opp_em_move_deposit_slab(opp_ctx ctx, int64_t *n, int64_t cap, double *off, double *u, double *w,
                             int32_t *cell, int64_t *id, const double *interp, const int32_t *c2c,
                             int64_t n_cells, double *acc, const opp_em_params *params,
                             opp_em_stats *stats);

/* The field side over slabs, one leap-frog step on this rank's cells:
 * AccumulateCurrent, AdvanceB(dt/2), AdvanceE(dt), AdvanceB(dt/2),
 * Interpolate, then acc := 0 on this rank's cells -- with Update_Ghosts
 * before each kernel that reads a neighbour's layer: acc and B of layer
 * k0 - 1 from rank - 1, E and B of layer k1 from rank + 1.  Collective;
 * global-sized arrays as above.  Errors as opp_em_accumulate_current. */
int opp_em_field_step_slab(opp_ctx ctx, double *e, double *b, double *J, double *acc, double *interp,
                           const int32_t *c2c, int64_t n_cells, const double *h, double dt);

/* Synchronise the context's stream; reports sticky asynchronous errors. */
int opp_sync(opp_ctx ctx);

/* Thread-local message describing the last error. */
const char *opp_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* OPP_H */
