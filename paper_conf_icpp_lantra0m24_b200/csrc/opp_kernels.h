// opp_kernels.h -- launchers of the sm_100a kernels (internal to libopp).
#pragma once
#include "opp_internal.h"

namespace opp {

cudaError_t launch_push_move_deposit(int dep, int dh, bool multi, bool cont, bool tiled,
                                     const StepArgs &a, int grid, cudaStream_t s);
int pmd_blocks_per_sm(bool tiled);
cudaError_t launch_step_begin(double *Q, long long nn, DevCounters *c, int zero, int grid,
                              cudaStream_t s);
cudaError_t launch_fill(const ColSet &cols, DevCounters *c, const uint32_t *holes,
                        const int32_t *p2c, uint32_t *head, uint32_t *tail, int grid,
                        cudaStream_t s);
cudaError_t launch_inject(const ColSet &cols, long long n, DevCounters *c, int grid,
                          cudaStream_t s);
cudaError_t launch_build_lines(const double *xyz, const int32_t *c2n, const int32_t *c2c,
                               long long nc, WalkLine *out, DevCounters *cnt, cudaStream_t s);
cudaError_t launch_pack_field(const double *ef, long long nc, double4 *out, cudaStream_t s);
cudaError_t launch_overlay(const WalkLine *lines, const double *xyz, long long nc, int cell_base,
                           const Overlay &ov, int32_t *map, cudaStream_t s);
cudaError_t launch_overlay_compact(const int32_t *map, const Overlay &ov, int16_t *off, int32_t *base,
                                   unsigned *overflow, cudaStream_t s);
// Q[v] += sum of cellsum[n2cs[k]] over node v's (cell, slot) entries (fixed order)
cudaError_t launch_cell_to_nodes(const int32_t *n2cs_ptr, const int32_t *n2cs, const double *cellsum,
                                 long long nn, double *Q, cudaStream_t s);
cudaError_t launch_sr(const StepArgs &a, long long nc, long long nn, unsigned *hist,
                      unsigned *start, unsigned long long *tile_sums, double *sorted,
                      double *cellsum, const int32_t *n2cs_ptr, const int32_t *n2cs, int grid,
                      cudaStream_t s);

long long scan_tiles(long long n);
cudaError_t scan_exclusive(const unsigned *in, unsigned *out, long long n,
                           unsigned long long *tile_sums, cudaStream_t s);
cudaError_t launch_shuffle_keys(const int32_t *p2c, const DevCounters *c, unsigned long long seed,
                                long long nb, int cell_base, int32_t *keys, int grid, cudaStream_t s);
cudaError_t launch_sort_count(const int32_t *p2c, DevCounters *c, int cell_base, long long nc,
                              const uint32_t *skey, unsigned *hist, unsigned *start,
                              unsigned long long *tile_sums, int grid, cudaStream_t s,
                              const int32_t *pcell = nullptr);
// pcell: optional predicted sort cell per particle (StepArgs::pcell); nc: local cells
cudaError_t launch_sort_rank(const int32_t *p2c, DevCounters *c, int cell_base, const uint32_t *skey,
                             unsigned *start, uint32_t *src_of, int rank_grid, cudaStream_t s,
                             const int32_t *pcell = nullptr, long long nc = 0);
cudaError_t launch_sort_gather(const GatherCols &g, const uint32_t *src_of, const unsigned *total_p,
                               int nsm, cudaStream_t s);
cudaError_t launch_sort_commit(DevCounters *c, const unsigned *start_total, cudaStream_t s);

cudaError_t launch_mig_count(const int32_t *mig_cell, const DevCounters *c, const RankRanges &rr,
                             unsigned long long *counts, int grid, cudaStream_t s);
cudaError_t launch_mig_pack(const ColSet &cols, int p2c_col, const uint32_t *mig,
                            const int32_t *mig_cell, const int32_t *mig_hops, const DevCounters *c,
                            const RankRanges &rr, unsigned long long *cursor, char *sendbuf,
                            int rec_bytes, int grid, cudaStream_t s);
cudaError_t launch_mig_unpack(const ColSet &cols, const char *recvbuf, long long R, int rec_bytes,
                              DevCounters *c, uint32_t *work, int32_t *work_hops, int grid,
                              cudaStream_t s);
cudaError_t launch_halo_pack(const double *Q, const int32_t *idx, long long m, double *out,
                             cudaStream_t s);
cudaError_t launch_halo_combine(double *Q, const int32_t *node, const int32_t *ptr, const int32_t *ent,
                                long long m, const double *in, cudaStream_t s);

cudaError_t launch_check_cells(const int32_t *cell, long long n, long long nc, unsigned *flag,
                               int grid, cudaStream_t s);

}  // namespace opp
