// opp_comm.h -- multi-GPU plumbing of libopp (slab partition, particle
// migration, node-charge halo).  Internal.
#pragma once
#include <string>
#include "opp_internal.h"

namespace opp {

struct Comm;

int comm_unique_id(void *out128, std::string &err);
int comm_init(Comm **out, const void *uid, int rank, int nranks, int device, std::string &err);
void comm_free(Comm *c);
int comm_set_partition(Comm *c, int rank, int nranks, long long n_local_cells,
                       const int32_t *rank_of_cell, int *cell_base, std::string &err);
int comm_migrate(Comm *c, StepArgs *a, cudaStream_t s, std::string &err);

}  // namespace opp
