// opp_comm.h -- multi-GPU plumbing of libopp: the transport under the slab
// partition (particle migration, node-charge halo, termination).  Internal.
//
// Two transports implement the same three collectives:
//   NCCL      one process per GPU, NVLink/NVSwitch (production);
//   loopback  several contexts inside ONE process (one host thread each),
//             data moved with device-to-device copies -- lets the whole
//             multi-rank protocol run and be tested on a single GPU.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "opp_internal.h"

namespace opp {

struct Transport {
    int rank = 0, nranks = 1;
    virtual ~Transport() {}
    // all[r * n + k] = rank r's mine[k]  (host arrays)
    virtual int allgather_i64(const int64_t *mine, int n, int64_t *all, cudaStream_t s,
                              std::string &err) = 0;
    // point-to-point exchange of device byte buffers: to peer p send
    // sbytes[p] bytes at sendbuf + soff[p]; from peer p receive rbytes[p]
    // bytes into recvbuf + roff[p].  Enqueued on / completed w.r.t. stream s.
    virtual int exchange(const char *sendbuf, const std::vector<int64_t> &soff,
                         const std::vector<int64_t> &sbytes, char *recvbuf,
                         const std::vector<int64_t> &roff, const std::vector<int64_t> &rbytes,
                         cudaStream_t s, std::string &err) = 0;
    // device all-gather: out[r * bytes .. (r+1) * bytes) = rank r's in (device
    // buffers), enqueued on stream s (NCCL: no host synchronisation)
    virtual int allgather_dev(const void *in, size_t bytes, void *out, cudaStream_t s,
                              std::string &err) = 0;
};

struct Comm {
    Transport *t = nullptr;
    int rank = 0, nranks = 1;
    RankRanges rr{};
    bool partitioned = false;
    // halo: local node indices shared with each peer, ordered by global id
    std::vector<int64_t> halo_off, halo_cnt;   // per peer, in elements
    int32_t *d_halo_idx = nullptr;
    double *d_halo_send = nullptr, *d_halo_recv = nullptr;
    int64_t halo_n = 0;
    // combine plan: per distinct shared local node, its holders' values in
    // global rank order (own value: entry -1, a peer's: its recv slot), so
    // every rank sums a node's copies in the same order (bit-identical copies
    // for any number of ranks sharing a node)
    int32_t *d_hc_node = nullptr, *d_hc_ptr = nullptr, *d_hc_ent = nullptr;
    int64_t hc_n = 0;
    // migration
    unsigned long long *d_counts = nullptr;    // nranks
    unsigned long long *d_cursor = nullptr;    // nranks
    unsigned long long *d_allcounts = nullptr; // nranks * nranks (all ranks' count rows)
    char *sendbuf = nullptr, *recvbuf = nullptr;
    size_t send_cap = 0, recv_cap = 0;
    std::vector<int64_t> counts_host;          // nranks * nranks
};

enum { OPP_TRANSPORT_NCCL = 0, OPP_TRANSPORT_LOOPBACK = 1 };

int comm_unique_id(void *out128, std::string &err);
int comm_init(Comm **out, int transport, const void *uid, int rank, int nranks, int device,
              std::string &err);
void comm_free(Comm *c);
// Slab partition + halo plan (collective over all ranks).
int comm_set_partition(Comm *c, long long n_global_cells, const int32_t *rank_of_cell,
                       long long n_local_cells, long long n_local_nodes, const int64_t *node_gid,
                       int *cell_base, cudaStream_t s, std::string &err);
int comm_reserve(char **buf, size_t *cap, size_t need, std::string &err);

}  // namespace opp
