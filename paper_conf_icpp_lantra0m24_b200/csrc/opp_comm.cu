// opp_comm.cu -- multi-GPU plumbing (single-rank stub).
#include "opp.h"
#include "opp_comm.h"

namespace opp {

struct Comm {
    int rank = 0, nranks = 1;
};

int comm_unique_id(void *, std::string &err) {
    err = "multi-GPU transport not built in this version";
    return OPP_ERR_NCCL;
}

int comm_init(Comm **out, const void *, int, int, int, std::string &err) {
    *out = nullptr;
    err = "multi-GPU transport not built in this version";
    return OPP_ERR_NCCL;
}

void comm_free(Comm *c) { delete c; }

int comm_set_partition(Comm *, int, int nranks, long long, const int32_t *, int *cell_base,
                       std::string &err) {
    if (nranks != 1) {
        err = "multi-GPU transport not built in this version";
        return OPP_ERR_NCCL;
    }
    *cell_base = 0;
    return OPP_OK;
}

int comm_migrate(Comm *, StepArgs *, cudaStream_t, std::string &err) {
    err = "multi-GPU transport not built in this version";
    return OPP_ERR_NCCL;
}

}  // namespace opp
