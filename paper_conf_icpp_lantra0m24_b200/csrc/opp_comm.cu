// opp_comm.cu -- transports (NCCL, in-process loopback) and the slab
// partition / halo plan.
#include "opp.h"
#include "opp_comm.h"

#include <algorithm>
#include <condition_variable>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>

#ifdef OPP_WITH_NCCL
#include <nccl.h>
#endif

namespace opp {

static int cuda_fail(cudaError_t e, const char *what, std::string &err) {
    err = std::string(what) + ": " + cudaGetErrorString(e);
    return OPP_ERR_CUDA;
}

int comm_reserve(char **buf, size_t *cap, size_t need, std::string &err) {
    if (need <= *cap) return OPP_OK;
    size_t ncap = std::max(need, *cap + *cap / 2);
    ncap = (ncap + 255) & ~(size_t)255;
    if (*buf) cudaFree(*buf);
    *buf = nullptr;
    *cap = 0;
    cudaError_t e = cudaMalloc(buf, ncap);
    if (e != cudaSuccess) return cuda_fail(e, "comm buffer", err);
    *cap = ncap;
    return OPP_OK;
}

// ---------------------------------------------------------------------------
// Loopback transport: ranks are contexts in one process, one host thread
// each; they meet at a hub keyed by the 128-byte id.
// ---------------------------------------------------------------------------
namespace {

struct Hub {
    std::mutex m;
    std::condition_variable cv;
    int nranks = 0;
    int arrived = 0;
    long gen = 0;
    std::vector<const void *> ptr;
    std::vector<std::vector<int64_t>> rows;
    std::vector<int> device;

    void barrier() {
        std::unique_lock<std::mutex> lk(m);
        long g = gen;
        if (++arrived == nranks) {
            arrived = 0;
            gen++;
            cv.notify_all();
        } else {
            cv.wait(lk, [&] { return gen != g; });
        }
    }
};

std::mutex g_hubs_m;
std::map<std::string, std::shared_ptr<Hub>> g_hubs;

struct LoopTransport : Transport {
    std::shared_ptr<Hub> hub;
    std::string key;

    ~LoopTransport() override {
        std::lock_guard<std::mutex> lk(g_hubs_m);
        hub.reset();
        auto it = g_hubs.find(key);
        if (it != g_hubs.end() && it->second.use_count() == 1) g_hubs.erase(it);
    }

    int allgather_i64(const int64_t *mine, int n, int64_t *all, cudaStream_t,
                      std::string &) override {
        hub->rows[rank].assign(mine, mine + n);
        hub->barrier();
        for (int r = 0; r < nranks; r++) std::memcpy(all + (size_t)r * n, hub->rows[r].data(), 8 * n);
        hub->barrier();
        return OPP_OK;
    }

    int exchange(const char *sendbuf, const std::vector<int64_t> &soff, const std::vector<int64_t> &,
                 char *recvbuf, const std::vector<int64_t> &roff, const std::vector<int64_t> &rbytes,
                 cudaStream_t s, std::string &err) override {
        cudaError_t e = cudaStreamSynchronize(s);   // the send buffer is complete
        if (e != cudaSuccess) return cuda_fail(e, "loopback sync", err);
        hub->ptr[rank] = sendbuf;
        hub->rows[rank] = soff;
        hub->barrier();
        for (int p = 0; p < nranks; p++) {
            if (p == rank || rbytes[p] == 0) continue;
            const char *src = (const char *)hub->ptr[p] + hub->rows[p][rank];
            e = cudaMemcpyPeerAsync(recvbuf + roff[p], hub->device[rank], src, hub->device[p],
                                    (size_t)rbytes[p], s);
            if (e != cudaSuccess) return cuda_fail(e, "loopback copy", err);
        }
        e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return cuda_fail(e, "loopback sync", err);
        hub->barrier();                             // peers finished reading my buffer
        return OPP_OK;
    }

    int allgather_dev(const void *in, size_t bytes, void *out, cudaStream_t s, std::string &err) override {
        cudaError_t e = cudaStreamSynchronize(s);   // my input is complete
        if (e != cudaSuccess) return cuda_fail(e, "loopback sync", err);
        hub->ptr[rank] = in;
        hub->barrier();
        for (int p = 0; p < nranks; p++) {
            e = cudaMemcpyPeerAsync((char *)out + (size_t)p * bytes, hub->device[rank], hub->ptr[p],
                                    hub->device[p], bytes, s);
            if (e != cudaSuccess) return cuda_fail(e, "loopback copy", err);
        }
        e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return cuda_fail(e, "loopback sync", err);
        hub->barrier();                             // peers finished reading my input
        return OPP_OK;
    }
};

#ifdef OPP_WITH_NCCL
struct NcclTransport : Transport {
    ncclComm_t comm = nullptr;
    int64_t *dbuf = nullptr;
    int dcap = 0;

    ~NcclTransport() override {
        if (comm) ncclCommDestroy(comm);
        if (dbuf) cudaFree(dbuf);
    }

    static int nccl_fail(ncclResult_t r, const char *what, std::string &err) {
        err = std::string(what) + ": " + ncclGetErrorString(r);
        return OPP_ERR_NCCL;
    }

    int allgather_i64(const int64_t *mine, int n, int64_t *all, cudaStream_t s,
                      std::string &err) override {
        int need = n * (nranks + 1);
        if (need > dcap) {
            if (dbuf) cudaFree(dbuf);
            cudaError_t e = cudaMalloc(&dbuf, 8 * (size_t)need);
            if (e != cudaSuccess) return cuda_fail(e, "allgather buffer", err);
            dcap = need;
        }
        cudaError_t e = cudaMemcpyAsync(dbuf, mine, 8 * (size_t)n, cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return cuda_fail(e, "allgather h2d", err);
        ncclResult_t r = ncclAllGather(dbuf, dbuf + n, (size_t)n, ncclInt64, comm, s);
        if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather", err);
        e = cudaMemcpyAsync(all, dbuf + n, 8 * (size_t)n * nranks, cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) return cuda_fail(e, "allgather d2h", err);
        e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return cuda_fail(e, "allgather sync", err);
        return OPP_OK;
    }

    int exchange(const char *sendbuf, const std::vector<int64_t> &soff,
                 const std::vector<int64_t> &sbytes, char *recvbuf, const std::vector<int64_t> &roff,
                 const std::vector<int64_t> &rbytes, cudaStream_t s, std::string &err) override {
        ncclResult_t r = ncclGroupStart();
        if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart", err);
        for (int p = 0; p < nranks; p++) {
            if (p == rank) continue;
            if (sbytes[p] > 0) {
                r = ncclSend(sendbuf + soff[p], (size_t)sbytes[p], ncclChar, p, comm, s);
                if (r != ncclSuccess) return nccl_fail(r, "ncclSend", err);
            }
            if (rbytes[p] > 0) {
                r = ncclRecv(recvbuf + roff[p], (size_t)rbytes[p], ncclChar, p, comm, s);
                if (r != ncclSuccess) return nccl_fail(r, "ncclRecv", err);
            }
        }
        r = ncclGroupEnd();
        if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd", err);
        return OPP_OK;
    }

    int allgather_dev(const void *in, size_t bytes, void *out, cudaStream_t s, std::string &err) override {
        ncclResult_t r = ncclAllGather(in, out, bytes, ncclChar, comm, s);
        if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather", err);
        return OPP_OK;
    }
};
#endif

}  // namespace

int comm_unique_id(void *out128, std::string &err) {
#ifdef OPP_WITH_NCCL
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) {
        err = std::string("ncclGetUniqueId: ") + ncclGetErrorString(r);
        return OPP_ERR_NCCL;
    }
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(out128, &id, 128);
    return OPP_OK;
#else
    (void)out128;
    err = "libopp was built without NCCL";
    return OPP_ERR_NCCL;
#endif
}

int comm_init(Comm **out, int transport, const void *uid, int rank, int nranks, int device,
              std::string &err) {
    *out = nullptr;
    if (!uid) {
        err = "nranks > 1 needs a 128-byte unique id";
        return OPP_ERR_ARG;
    }
    if (nranks > kMaxRanks) {
        err = "too many ranks";
        return OPP_ERR_ARG;
    }
    std::unique_ptr<Comm> c(new Comm());
    c->rank = rank;
    c->nranks = nranks;
    if (transport == OPP_TRANSPORT_LOOPBACK) {
        auto *t = new LoopTransport();
        t->key.assign((const char *)uid, 128);
        {
            std::lock_guard<std::mutex> lk(g_hubs_m);
            auto &h = g_hubs[t->key];
            if (!h) {
                h = std::make_shared<Hub>();
                h->nranks = nranks;
                h->ptr.assign(nranks, nullptr);
                h->rows.assign(nranks, {});
                h->device.assign(nranks, 0);
            }
            if (h->nranks != nranks) {
                delete t;
                err = "loopback: nranks differs between ranks";
                return OPP_ERR_ARG;
            }
            t->hub = h;
        }
        t->hub->device[rank] = device;
        t->rank = rank;
        t->nranks = nranks;
        c->t = t;
        t->hub->barrier();   // everybody joined
    } else {
#ifdef OPP_WITH_NCCL
        auto *t = new NcclTransport();
        ncclUniqueId id;
        std::memcpy(&id, uid, 128);
        ncclResult_t r = ncclCommInitRank(&t->comm, nranks, id, rank);
        if (r != ncclSuccess) {
            delete t;
            err = std::string("ncclCommInitRank: ") + ncclGetErrorString(r);
            return OPP_ERR_NCCL;
        }
        t->rank = rank;
        t->nranks = nranks;
        c->t = t;
#else
        err = "libopp was built without NCCL";
        return OPP_ERR_NCCL;
#endif
    }
    cudaError_t e = cudaMalloc(&c->d_counts, sizeof(unsigned long long) * (2 + (size_t)nranks) * nranks);
    if (e != cudaSuccess) {
        delete c->t;
        return cuda_fail(e, "comm counters", err);
    }
    c->d_cursor = c->d_counts + nranks;
    c->d_allcounts = c->d_counts + 2 * nranks;
    c->counts_host.assign((size_t)nranks * nranks, 0);
    *out = c.release();
    return OPP_OK;
}

void comm_free(Comm *c) {
    if (!c) return;
    delete c->t;
    if (c->d_counts) cudaFree(c->d_counts);
    if (c->d_halo_idx) cudaFree(c->d_halo_idx);
    if (c->d_halo_send) cudaFree(c->d_halo_send);
    if (c->d_halo_recv) cudaFree(c->d_halo_recv);
    if (c->d_hc_node) cudaFree(c->d_hc_node);
    if (c->d_hc_ptr) cudaFree(c->d_hc_ptr);
    if (c->d_hc_ent) cudaFree(c->d_hc_ent);
    if (c->sendbuf) cudaFree(c->sendbuf);
    if (c->recvbuf) cudaFree(c->recvbuf);
    delete c;
}

// Partition: each rank's cells form one contiguous global range (the
// "principal direction of motion" slabs).  Halo plan:
// every rank learns every other rank's node global ids and keeps, per peer,
// the local indices of the shared nodes ordered by global id, so both sides
// of an interface list the same nodes in the same order.
int comm_set_partition(Comm *c, long long n_global_cells, const int32_t *rank_of_cell,
                       long long n_local_cells, long long n_local_nodes, const int64_t *node_gid,
                       int *cell_base, cudaStream_t s, std::string &err) {
    const int R = c->nranks;
    std::vector<long long> lo(R, -1), hi(R, -1);
    for (long long g = 0; g < n_global_cells; g++) {
        int r = rank_of_cell[g];
        if (r < 0 || r >= R) {
            err = "rank_of_cell out of range";
            return OPP_ERR_ARG;
        }
        if (lo[r] < 0) lo[r] = g;
        else if (hi[r] != g) {
            err = "each rank's cells must form one contiguous global range";
            return OPP_ERR_ARG;
        }
        hi[r] = g + 1;
    }
    if (n_global_cells > 0x7ffffff0ll) {
        err = "global cell ids must fit int32";
        return OPP_ERR_ARG;
    }
    for (int r = 0; r < R; r++) {
        c->rr.lo[r] = (int)std::max(lo[r], 0ll);
        c->rr.hi[r] = (int)std::max(hi[r], 0ll);
    }
    c->rr.n = R;
    if ((long long)(c->rr.hi[c->rank] - c->rr.lo[c->rank]) != n_local_cells) {
        err = "the local cell set size differs from this rank's range";
        return OPP_ERR_ARG;
    }
    *cell_base = c->rr.lo[c->rank];
    if (R == 1 || !c->t) {
        c->partitioned = true;
        return OPP_OK;
    }
    // ---- halo plan: allgather node counts, then every list to every rank
    int64_t mine = n_local_nodes;
    std::vector<int64_t> cnt(R);
    int rc = c->t->allgather_i64(&mine, 1, cnt.data(), s, err);
    if (rc != OPP_OK) return rc;
    std::vector<int64_t> soff(R, 0), sbytes(R, 8 * n_local_nodes), roff(R), rbytes(R);
    int64_t tot = 0;
    for (int p = 0; p < R; p++) {
        roff[p] = tot;
        rbytes[p] = p == c->rank ? 0 : 8 * cnt[p];
        tot += rbytes[p];
        if (p == c->rank) sbytes[p] = 0;
    }
    char *dsend = nullptr, *drecv = nullptr;
    cudaError_t e = cudaMalloc(&dsend, std::max<int64_t>(8 * n_local_nodes, 8));
    if (e != cudaSuccess) return cuda_fail(e, "halo plan", err);
    e = cudaMalloc(&drecv, std::max<int64_t>(tot, 8));
    if (e != cudaSuccess) {
        cudaFree(dsend);
        return cuda_fail(e, "halo plan", err);
    }
    cudaMemcpyAsync(dsend, node_gid, 8 * n_local_nodes, cudaMemcpyHostToDevice, s);
    rc = c->t->exchange(dsend, soff, sbytes, drecv, roff, rbytes, s, err);
    std::vector<int64_t> all(tot / 8);
    if (rc == OPP_OK) {
        cudaMemcpyAsync(all.data(), drecv, tot, cudaMemcpyDeviceToHost, s);
        e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) rc = cuda_fail(e, "halo plan sync", err);
    }
    cudaFree(dsend);
    cudaFree(drecv);
    if (rc != OPP_OK) return rc;
    // my nodes sorted by gid
    std::vector<std::pair<int64_t, int32_t>> my(n_local_nodes);
    for (long long k = 0; k < n_local_nodes; k++) my[k] = {node_gid[k], (int32_t)k};
    std::sort(my.begin(), my.end());
    std::vector<int32_t> idx;
    c->halo_off.assign(R, 0);
    c->halo_cnt.assign(R, 0);
    for (int p = 0; p < R; p++) {
        c->halo_off[p] = (int64_t)idx.size();
        if (p == c->rank) continue;
        std::vector<int64_t> theirs(all.begin() + roff[p] / 8, all.begin() + (roff[p] + rbytes[p]) / 8);
        std::sort(theirs.begin(), theirs.end());
        size_t a = 0, b = 0;
        while (a < my.size() && b < theirs.size()) {
            if (my[a].first < theirs[b]) a++;
            else if (theirs[b] < my[a].first) b++;
            else {
                idx.push_back(my[a].second);
                a++;
                b++;
            }
        }
        c->halo_cnt[p] = (int64_t)idx.size() - c->halo_off[p];
    }
    c->halo_n = (int64_t)idx.size();
    if (c->d_halo_idx) cudaFree(c->d_halo_idx);
    if (c->d_halo_send) cudaFree(c->d_halo_send);
    if (c->d_halo_recv) cudaFree(c->d_halo_recv);
    c->d_halo_idx = nullptr;
    c->d_halo_send = c->d_halo_recv = nullptr;
    size_t hb = std::max<size_t>(idx.size(), 1);
    if (cudaMalloc(&c->d_halo_idx, 4 * hb) != cudaSuccess ||
        cudaMalloc(&c->d_halo_send, 8 * hb) != cudaSuccess ||
        cudaMalloc(&c->d_halo_recv, 8 * hb) != cudaSuccess) {
        err = "halo buffers";
        return OPP_ERR_NOMEM;
    }
    if (!idx.empty())
        cudaMemcpyAsync(c->d_halo_idx, idx.data(), 4 * idx.size(), cudaMemcpyHostToDevice, s);
    // combine plan: for each distinct shared local node, (rank, entry) pairs
    // of every holder sorted by rank (entry -1 = this rank's own value)
    std::map<int32_t, std::vector<std::pair<int, int32_t>>> holders;
    for (int p = 0; p < R; p++)
        for (int64_t k = c->halo_off[p]; k < c->halo_off[p] + c->halo_cnt[p]; k++)
            holders[idx[k]].push_back({p, (int32_t)k});
    std::vector<int32_t> hnode, hptr(1, 0), hent;
    for (auto &kv : holders) {
        kv.second.push_back({c->rank, -1});
        std::sort(kv.second.begin(), kv.second.end());
        hnode.push_back(kv.first);
        for (auto &pe : kv.second) hent.push_back(pe.second);
        hptr.push_back((int32_t)hent.size());
    }
    c->hc_n = (int64_t)hnode.size();
    if (c->d_hc_node) cudaFree(c->d_hc_node);
    if (c->d_hc_ptr) cudaFree(c->d_hc_ptr);
    if (c->d_hc_ent) cudaFree(c->d_hc_ent);
    c->d_hc_node = c->d_hc_ptr = c->d_hc_ent = nullptr;
    if (cudaMalloc(&c->d_hc_node, 4 * std::max<size_t>(hnode.size(), 1)) != cudaSuccess ||
        cudaMalloc(&c->d_hc_ptr, 4 * hptr.size()) != cudaSuccess ||
        cudaMalloc(&c->d_hc_ent, 4 * std::max<size_t>(hent.size(), 1)) != cudaSuccess) {
        err = "halo combine plan";
        return OPP_ERR_NOMEM;
    }
    if (!hnode.empty()) {
        cudaMemcpyAsync(c->d_hc_node, hnode.data(), 4 * hnode.size(), cudaMemcpyHostToDevice, s);
        cudaMemcpyAsync(c->d_hc_ent, hent.data(), 4 * hent.size(), cudaMemcpyHostToDevice, s);
    }
    cudaMemcpyAsync(c->d_hc_ptr, hptr.data(), 4 * hptr.size(), cudaMemcpyHostToDevice, s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "halo plan upload", err);
    c->partitioned = true;
    return OPP_OK;
}

}  // namespace opp
