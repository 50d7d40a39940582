// opp_kernels.h -- launchers of the sm_100a kernels (internal to libopp).
#pragma once
#include "opp_internal.h"

namespace opp {

cudaError_t launch_push_move_deposit(int dep, bool dh, bool multi, bool cont, const StepArgs &a,
                                     int grid, cudaStream_t s);
int pmd_blocks_per_sm(int dep, bool dh);
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
cudaError_t launch_sr(const StepArgs &a, long long nc, long long nn, unsigned *hist,
                      unsigned *start, double *sorted, double *cellsum, const int32_t *n2cs_ptr,
                      const int32_t *n2cs, int grid, cudaStream_t s);

}  // namespace opp
