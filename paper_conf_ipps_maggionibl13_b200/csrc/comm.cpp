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
#include <mutex>
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

struct cme_comm_s {
    ncclComm_t comm = nullptr;
    int nranks = 1, rank = 0, device = 0;
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

extern "C" void cme_comm_destroy(cme_comm c) {
    if (!c) return;
    if (c->comm) cme::g_api.CommDestroy(c->comm);
    delete c;
}
