// NCCL communicator for the row-sharded Jacobi.
//
// The paper is single-GPU (clusters are future work).  Across the
// GPUs of one NVSwitch box each iteration exchanges only the contiguous halo
// ranges of the iterate (grouped ncclSend/ncclRecv, captured into the same CUDA
// graph as the fused steps) and, every C iterations, an allgather of one
// 8-double partial record per rank that every rank reduces in rank order
// (deterministic, identical stop decisions everywhere).
//
// libnccl is loaded with dlopen: the copy torch already mapped into the
// process if there is one (RTLD_NOLOAD), else $CME_NCCL_LIB, else
// libnccl.so.2 -- so the process never holds two NCCL libraries.
#include <dlfcn.h>
#include <cstdlib>
#include <cstring>
#include <condition_variable>
#include <memory>
#include <mutex>
#include <vector>
#include <string>

#include <nccl.h>

#include "cme_internal.h"
#include "comm.h"

namespace cme {
namespace {

struct NcclApi {
    void* lib = nullptr;
    decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
    decltype(&ncclCommInitRank) CommInitRank = nullptr;
    decltype(&ncclCommDestroy) CommDestroy = nullptr;
    decltype(&ncclSend) Send = nullptr;
    decltype(&ncclRecv) Recv = nullptr;
    decltype(&ncclGroupStart) GroupStart = nullptr;
    decltype(&ncclGroupEnd) GroupEnd = nullptr;
    decltype(&ncclAllGather) AllGather = nullptr;
    decltype(&ncclBroadcast) Broadcast = nullptr;
    decltype(&ncclGetErrorString) GetErrorString = nullptr;
};

NcclApi g_api;
std::mutex g_mu;

cme_status load_nccl() {
    std::lock_guard<std::mutex> lk(g_mu);
    if (g_api.lib) return CME_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h && std::getenv("CME_NCCL_LIB")) h = dlopen(std::getenv("CME_NCCL_LIB"), RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        set_error(std::string("cannot load libnccl.so.2: ") + dlerror());
        return CME_ERR_NCCL;
    }
    NcclApi a;
    a.lib = h;
#define SYM(f)                                                              \
    a.f = reinterpret_cast<decltype(a.f)>(dlsym(h, "nccl" #f));             \
    if (!a.f) {                                                             \
        set_error("libnccl lacks nccl" #f);                                 \
        return CME_ERR_NCCL;                                                \
    }
    SYM(GetUniqueId) SYM(CommInitRank) SYM(CommDestroy) SYM(Send) SYM(Recv) SYM(GroupStart)
    SYM(GroupEnd) SYM(AllGather) SYM(Broadcast) SYM(GetErrorString)
#undef SYM
    g_api = a;
    return CME_OK;
}

}  // namespace
}  // namespace cme

namespace cme {
// In-process group of the peer-memory transport: ranks are host threads that
// publish their buffers here; a generation barrier orders setup/teardown.
struct LocalGroup {
    int n = 0;
    std::mutex mu;
    std::condition_variable cv;
    int count = 0;
    uint64_t gen = 0;
    std::vector<P2PRank> slots;
    void barrier() {
        std::unique_lock<std::mutex> lk(mu);
        const uint64_t g = gen;
        if (++count == n) {
            count = 0;
            ++gen;
            cv.notify_all();
        } else {
            cv.wait(lk, [&] { return gen != g; });
        }
    }
};
}  // namespace cme

struct cme_comm_s {
    int transport = cme::kTransportNccl;
    ncclComm_t comm = nullptr;
    int nranks = 1, rank = 0, device = 0;
    std::shared_ptr<cme::LocalGroup> group;   // P2P transport
};

namespace cme {

#define NCCL_TRY(expr)                                                               \
    do {                                                                             \
        ncclResult_t _r = (expr);                                                    \
        if (_r != ncclSuccess) {                                                     \
            set_error(std::string(#expr) + ": " + g_api.GetErrorString(_r));         \
            return CME_ERR_NCCL;                                                     \
        }                                                                            \
    } while (0)

int comm_transport(const cme_comm_s* c) { return c->transport; }

cme_status comm_p2p_exchange(cme_comm_s* c, const P2PRank& mine, std::vector<P2PRank>& all) {
    if (c->transport != kTransportP2P || !c->group) return CME_ERR_INVALID_ARG;
    {
        std::lock_guard<std::mutex> lk(c->group->mu);
        c->group->slots[c->rank] = mine;
    }
    c->group->barrier();
    {
        std::lock_guard<std::mutex> lk(c->group->mu);
        all = c->group->slots;
    }
    c->group->barrier();   // nobody republishes before everyone has read
    return CME_OK;
}

void comm_p2p_host_barrier(cme_comm_s* c) {
    if (c->group) c->group->barrier();
}

int comm_rank(const cme_comm_s* c) { return c->rank; }
int comm_nranks(const cme_comm_s* c) { return c->nranks; }
int comm_device(const cme_comm_s* c) { return c->device; }

cme_status comm_halo(cme_comm_s* c, const HaloPlan& p, double* xspan, cudaStream_t s) {
    if (p.send_peer.empty() && p.recv_peer.empty()) return CME_OK;
    NCCL_TRY(g_api.GroupStart());
    for (size_t i = 0; i < p.send_peer.size(); ++i)
        NCCL_TRY(g_api.Send(xspan + p.send_off[i], (size_t)p.send_cnt[i], ncclFloat64, p.send_peer[i], c->comm, s));
    for (size_t i = 0; i < p.recv_peer.size(); ++i)
        NCCL_TRY(g_api.Recv(xspan + p.recv_off[i], (size_t)p.recv_cnt[i], ncclFloat64, p.recv_peer[i], c->comm, s));
    NCCL_TRY(g_api.GroupEnd());
    return CME_OK;
}

cme_status comm_allgather(cme_comm_s* c, const double* send, double* recv, size_t count, cudaStream_t s) {
    NCCL_TRY(g_api.AllGather(send, recv, count, ncclFloat64, c->comm, s));
    return CME_OK;
}

cme_status comm_bcast_segments(cme_comm_s* c, double* buf, const std::vector<int64_t>& cuts, cudaStream_t s) {
    NCCL_TRY(g_api.GroupStart());
    for (int r = 0; r < c->nranks; ++r) {
        const size_t cnt = (size_t)(cuts[r + 1] - cuts[r]);
        if (cnt) NCCL_TRY(g_api.Broadcast(buf + cuts[r], buf + cuts[r], cnt, ncclFloat64, r, c->comm, s));
    }
    NCCL_TRY(g_api.GroupEnd());
    return CME_OK;
}

}  // namespace cme

extern "C" cme_status cme_comm_unique_id(uint8_t id[128]) {
    if (!id) return CME_ERR_INVALID_ARG;
    if (cme_status s = cme::load_nccl(); s != CME_OK) return s;
    ncclUniqueId u;
    ncclResult_t r = cme::g_api.GetUniqueId(&u);
    if (r != ncclSuccess) {
        cme::set_error(std::string("ncclGetUniqueId: ") + cme::g_api.GetErrorString(r));
        return CME_ERR_NCCL;
    }
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(id, &u, 128);
    return CME_OK;
}

extern "C" cme_status cme_comm_init(int nranks, int rank, const uint8_t id[128], int device, cme_comm* out) {
    if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks) return CME_ERR_INVALID_ARG;
    *out = nullptr;
    if (cme_status s = cme::load_nccl(); s != CME_OK) return s;
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        cme::set_error("no CUDA device visible");
        return CME_ERR_NO_DEVICE;
    }
    if (device < 0 && cudaGetDevice(&device) != cudaSuccess) return CME_ERR_CUDA;
    if (cudaSetDevice(device) != cudaSuccess) return CME_ERR_CUDA;
    ncclUniqueId u;
    std::memcpy(&u, id, 128);
    auto* c = new cme_comm_s();
    c->nranks = nranks;
    c->rank = rank;
    c->device = device;
    ncclResult_t r = cme::g_api.CommInitRank(&c->comm, nranks, u, rank);
    if (r != ncclSuccess) {
        cme::set_error(std::string("ncclCommInitRank: ") + cme::g_api.GetErrorString(r));
        delete c;
        return CME_ERR_NCCL;
    }
    *out = c;
    return CME_OK;
}

extern "C" cme_status cme_comm_init_local(int nranks, const int* devices, cme_comm* comms_out) {
    if (nranks < 1 || nranks > cme::kMaxPeers + 1 || !devices || !comms_out) return CME_ERR_INVALID_ARG;
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        cme::set_error("no CUDA device visible");
        return CME_ERR_NO_DEVICE;
    }
    for (int r = 0; r < nranks; ++r)
        if (devices[r] < 0 || devices[r] >= count) return CME_ERR_INVALID_ARG;
    // peer access between distinct devices (NVLink / NVSwitch); same device needs none
    for (int a = 0; a < nranks; ++a)
        for (int b = 0; b < nranks; ++b) {
            if (devices[a] == devices[b]) continue;
            int ok = 0;
            cudaDeviceCanAccessPeer(&ok, devices[a], devices[b]);
            if (!ok) {
                cme::set_error("devices without peer access");
                return CME_ERR_NCCL;
            }
            cudaSetDevice(devices[a]);
            cudaError_t e = cudaDeviceEnablePeerAccess(devices[b], 0);
            if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
                cme::set_error(std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorString(e));
                return CME_ERR_CUDA;
            }
            cudaGetLastError();
        }
    auto group = std::make_shared<cme::LocalGroup>();
    group->n = nranks;
    group->slots.resize(nranks);
    for (int r = 0; r < nranks; ++r) {
        auto* c = new cme_comm_s();
        c->transport = cme::kTransportP2P;
        c->nranks = nranks;
        c->rank = r;
        c->device = devices[r];
        c->group = group;
        comms_out[r] = c;
    }
    return CME_OK;
}

extern "C" cme_status cme_comm_init_ipc(int nranks, int rank, int device, cme_comm* out) {
    if (!out || nranks < 1 || nranks > cme::kMaxPeers + 1 || rank < 0 || rank >= nranks) return CME_ERR_INVALID_ARG;
    *out = nullptr;
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        cme::set_error("no CUDA device visible");
        return CME_ERR_NO_DEVICE;
    }
    if (device < 0 && cudaGetDevice(&device) != cudaSuccess) return CME_ERR_CUDA;
    if (device >= count) return CME_ERR_INVALID_ARG;
    auto* c = new cme_comm_s();
    c->transport = cme::kTransportIpc;
    c->nranks = nranks;
    c->rank = rank;
    c->device = device;
    *out = c;
    return CME_OK;
}

extern "C" void cme_comm_destroy(cme_comm c) {
    if (!c) return;
    if (c->comm && cme::g_api.CommDestroy) cme::g_api.CommDestroy(c->comm);
    delete c;
}
