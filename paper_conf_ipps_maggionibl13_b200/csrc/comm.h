// NCCL glue for the row-sharded multi-GPU Jacobi.
#pragma once
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#include "cme.h"

struct cme_comm_s;

namespace cme {

// Who sends which contiguous x range to whom after every step.  Offsets are
// x-span indices of the local buffers (send: own rows; recv: halo slots).
struct HaloPlan {
    std::vector<int> send_peer, recv_peer;
    std::vector<int64_t> send_off, send_cnt, recv_off, recv_cnt;
    int64_t volume() const {
        int64_t v = 0;
        for (auto c : recv_cnt) v += c;
        return v;
    }
};

enum { kTransportNccl = 0, kTransportP2P = 1, kTransportIpc = 2 };
constexpr int kMaxPeers = 8;

// One rank's device buffers, published to the group by the peer-memory
// transport: the two x-span iterate buffers, the sync flags, the check
// gather array and the output staging vector (+ geometry to address them).
struct P2PRank {
    double* xb[2] = {nullptr, nullptr};
    int64_t* flags = nullptr;   // [nranks] latest sync epoch signalled by each rank
    double* gather = nullptr;   // [nranks][B][8]
    double* io = nullptr;       // [n_global * B] reordered staging
    int64_t span_lo = 0;        // first global row of the x-span
    int device = 0;
    unsigned char uuid[16] = {};  // physical GPU (cudaDeviceProp::uuid)
    int32_t fused_ok = 0;       // can run the fused in-kernel halo sync (tile-record kernel)
};

int comm_transport(const cme_comm_s* c);
inline bool transport_is_peer(int t) { return t == kTransportP2P || t == kTransportIpc; }
// Publish `mine`, block until every rank of the group has, return all ranks'.
cme_status comm_p2p_exchange(cme_comm_s* c, const P2PRank& mine, std::vector<P2PRank>& all);
// Host-side barrier over the group (setup / teardown only).
void comm_p2p_host_barrier(cme_comm_s* c);

int comm_rank(const cme_comm_s* c);
int comm_nranks(const cme_comm_s* c);
int comm_device(const cme_comm_s* c);
cme_status comm_halo(cme_comm_s* c, const HaloPlan& p, double* xspan, cudaStream_t s);
// recv[r*count .. (r+1)*count) = send of rank r
cme_status comm_allgather(cme_comm_s* c, const double* send, double* recv, size_t count, cudaStream_t s);
// every rank r broadcasts buf[cuts[r], cuts[r+1]) (in doubles) to all ranks
cme_status comm_bcast_segments(cme_comm_s* c, double* buf, const std::vector<int64_t>& cuts,
                               cudaStream_t s);

}  // namespace cme
