// Device side of libcme: buffers in HBM, the fused step launches, the
// check/normalise/stop logic and the solve driver.
//
// Per solve the iteration runs as CUDA graphs of one "check block": C fused
// steps (the last with CHECK) + the partial reduction + the decision kernel,
// all device-side; the host only reads a small control block every C
// iterations and launches the next graph one block ahead, so it never stalls
// the GPU (a decided stop turns the look-ahead block into no-op launches).
//
// Batches (B rate sets on one pattern, B in {1,2,4,8}): iterates are
// member-minor (x[row*B + b]); every check reduces and decides per member;
// the solve stops when every member is CONVERGED or STAGNATED (or one is
// NUMERIC, or max_iter).
#include <cmath>
#include <cstddef>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>

#include "cme_internal.h"
#include "comm.h"
#include "launch.h"
#include "kernels_wf.cuh"
#include "kernels_resident.cuh"
#include "kernels_cpt.cuh"

namespace cme {

#define CUDA_TRY(expr)                                                                  \
    do {                                                                                \
        cudaError_t _e = (expr);                                                        \
        if (_e != cudaSuccess) {                                                        \
            set_error(std::string(#expr) + ": " + cudaGetErrorString(_e));              \
            return _e == cudaErrorMemoryAllocation ? CME_ERR_OOM : CME_ERR_CUDA;        \
        }                                                                               \
    } while (0)

#define CME_TRY(expr)                    \
    do {                                 \
        cme_status _s = (expr);          \
        if (_s != CME_OK) return _s;     \
    } while (0)

struct Device {
    int dev = -1;
    cudaStream_t own = nullptr, cap = nullptr;
    std::vector<void*> allocs;
    int B = 1;
    // packed matrix
    int64_t* slice_off = nullptr;
    int32_t* slice_w = nullptr;
    double* val = nullptr;
    int32_t* col = nullptr;
    int32_t* row_of = nullptr;
    double *lo = nullptr, *up = nullptr, *inv_d = nullptr;
    int64_t* csr_rp = nullptr;
    int32_t* csr_ci = nullptr;
    double* csr_v = nullptr;
    // ordering
    int32_t* perm_own = nullptr;     // original index of local row l
    int32_t* perm_global = nullptr;  // new_to_old (distributed output only)
    // iterates: x-span buffers, member-minor (element 0 = first x-span row;
    // one zero sentinel row on each side)
    double* xb[2] = {nullptr, nullptr};
    int cur = 0;
    double* partials = nullptr;      // [part_blocks][B][kPartials]
    int grid = 0, part_blocks = 0;
    double* gather = nullptr;        // [nranks][B][8]
    double* local8 = nullptr;        // [B][8]
    double* io = nullptr;            // n_global * B staging
    double* io2 = nullptr;           // second staging (distributed output)
    double* one = nullptr;           // constant 1.0 x kMaxBatch
    double* acc_base = nullptr;      // transient accumulator allocation (lazily)
    double* accb = nullptr;          //   its x-span base (one sentinel row in front)
    Ctrl* ctrl = nullptr;
    Ctrl* ctrl_host = nullptr;       // pinned, 2 slots
    int64_t n_global = 0, n_own = 0, nx = 0, own_off = 0, row_begin = 0;
    int64_t n_slices = 0;
    int format = CME_FMT_DIAG_SELL;
    bool band = false, rearr = false;
    // distributed
    cme_comm_s* comm = nullptr;
    int nranks = 1, rank = 0;
    bool p2p = false;                // peer-memory transport (no NCCL on the iteration path)
    int64_t* flags = nullptr;        // [nranks] sync epochs signalled by each rank (written by peers)
    int64_t* epoch = nullptr;        // [1] this rank's sync counter
    int npeer = 0;                   // other ranks
    int peer_rank[kMaxPushPeers] = {};
    int64_t* peer_flags[kMaxPushPeers] = {};
    double* peer_gather[kMaxPushPeers] = {};
    double* peer_io[kMaxPushPeers] = {};
    bool peer_nbr[kMaxPushPeers] = {};   // a halo neighbour (send or receive side)
    bool nbr_barrier = true;         // per-step barrier over the halo neighbours only
    int npush = 0;                   // peers that need some of my rows
    int64_t push_lo[kMaxPushPeers] = {}, push_hi[kMaxPushPeers] = {};   // local rows
    double* push_y[2][kMaxPushPeers] = {};   // peer buffer (parity b) shifted to my local rows
    bool peers_ready = false;        // IPC transport: attach done
    bool bar_pdl = false;            // step barrier launched with PDL (peers on other GPUs only)
    // fused in-kernel halo sync (kernels_vi2.cuh HaloSync): replaces the step barrier
    bool fused = false;
    bool same_gpu_peers = false;     // a peer rank shares this GPU (virtual ranks)
    int64_t* hsync = nullptr;        // [4] steps run, push/halo warp completions, CTAs out
    uint8_t* tile_kind = nullptr;    // [vi2 tiles] bit 0 reads halo rows, bit 1 pushes rows
    int64_t hs_push_warps = 0, hs_halo_warps = 0;
    int hs_nsend = 0, hs_nrecv = 0;
    int hs_send_rank[kMaxPushPeers] = {}, hs_recv_rank[kMaxPushPeers] = {};
    int64_t* hs_peer_pushed[kMaxPushPeers] = {};
    int64_t* hs_peer_consumed[kMaxPushPeers] = {};
    std::vector<void*> ipc_opened;   // peer allocations mapped into this process
    HaloPlan halo;                   // counts/offsets in doubles (rows x B)
    std::vector<int64_t> cuts;       // in doubles (rows x B) for the output broadcast
    // TMA-staged persistent kernel (kernels_tma.cuh)
    bool use_tma = false;
    int tma_ncw = 16;
    int tma_spw = 1;                 // slices per consumer warp per tile (all shapes: 1)
    int tma_grid = 0, tma_stages = 0, tma_stage_bytes = 0, tma_off_val = 0, tma_off_col = 0, tma_contig = 0;
    int tma_xpf = 0;
    int tma_occ = 0;                 // TMA CTAs per SM
    int2* tile_meta = nullptr;       // per slice {offset inside its tile, width} for the chosen tile shape
    int64_t n_tiles = 0;
    // compact encoding (kernels_cpt.cuh): the TMA kernel streams M's rows,
    // 16-bit column offsets and 8-bit row offsets
    bool cpt = false;
    double *cval = nullptr, *clo = nullptr, *cup = nullptr;
    int16_t* col16 = nullptr;
    uint8_t* row8 = nullptr;
    int32_t win_shift = 0;
    // value-indexed variant (cpt also set): dictionary + 16-bit value indices
    bool vi = false;
    double* dict = nullptr;
    uint16_t *vidx = nullptr, *loi = nullptr, *upi = nullptr;
    int dict_bytes = 0;              // shared-memory bytes of the dictionary (multiple of 128)
    int vi_idpf = 1;                 // L2 prefetch of the tile's inv_d by the producer (CME_VI_IDPF)
    // tile-record value-indexed kernel (kernels_vi2.cuh, B = 1): one contiguous
    // record per tile; replaces sell_vi_kernel when vi2 (CME_VI2 = 0 keeps it)
    bool vi2 = false;
    bool vi2_words = false;          // records hold packed vidx | col16 << 16 words (CME_VI2_WORDS)
    bool vi2_f64 = false;            // records of the f64 compact encoding (no value index; CME_REC)
    int vi2_ncw = 0, vi2_stages = 0, vi2_stage_bytes = 0, vi2_grid = 0, vi2_occ = 0;
    int64_t vi2_tiles = 0;
    unsigned char* vi2_rec = nullptr;
    int64_t* vi2_rec_off = nullptr;
    // x window in shared memory (XW; single GPU): per tile
    // the iterate chunks it gathers, streamed with its record
    bool vi2b = false;               // batched tile records (sell_vi2b_kernel, B > 1; vi2_* shape fields)
    int vi2b_dict_bytes = 0;         // > 0: its tuple dictionary staged in shared memory (B = 2)
    int xw = 0;                      // 1 mirrored ring, 2 ring with a wrap per entry
    int2* xw_ch = nullptr;           // [vi2 tiles] {first chunk, end chunk} (monotone)
    int xw_rows = 0, xw_mirror = 0, xw_off = 0, xw_ring_bytes = 0;
    int64_t xw_nx = 0;
    // wavefront s-step kernel over the tile records (kernels_wf.cuh): one
    // launch per s steps of a check block (single GPU, vi2 shapes)
    bool wf = false;
    int wf_s = 0;                    // steps per pass (CME_WF; 0/1 = off)
    int wf_lag = 0;                  // L: tiles between step j-1 and step j of a wave
    int wf_keep = 1;                 // records of non-final steps evict_normal in L2 (CME_WF_KEEP)
    uint32_t* wf_items = nullptr;    // [s * tiles] (j << 24) | t in wave order
    int2* wf_dep = nullptr;          // [tiles] dependency tile range
    uint32_t* wf_cnt = nullptr;      // [tiles] completion counters
    uint32_t* wf_sync = nullptr;     // [2] passes done, CTAs finished
    // SMEM-resident persistent kernel (kernels_resident.cuh)
    bool use_res = false;
    int res_grid = 0, res_smem = 0, res_rps = 1;
    int32_t* res_q = nullptr;        // [res_grid + 1] slice cuts
    int32_t* res_row = nullptr;      // [res_grid + 1] first own row per CTA
    int32_t* res_probe_off = nullptr;   // [res_grid + 1] CSR offsets of the probe lists
    int32_t* res_probe = nullptr;       // CTAs each CTA probes (readers it does not read)
    uint32_t* res_sync = nullptr;    // [4] grid-barrier words
    int64_t res_timeout_ns = 0;
    // graphs
    cudaGraphExec_t gexec[2] = {nullptr, nullptr};
    int64_t gC = -1;
    double gomega = -1;
    cudaEvent_t ev[2] = {nullptr, nullptr}, t0 = nullptr, t1 = nullptr;

    template <typename T>
    cme_status alloc(T*& p, size_t count) {
        void* q = nullptr;
        CUDA_TRY(cudaMalloc(&q, std::max<size_t>(count, 1) * sizeof(T)));
        allocs.push_back(q);
        p = static_cast<T*>(q);
        return CME_OK;
    }
    template <typename T>
    cme_status upload(T*& p, const std::vector<T>& h) {
        CME_TRY(alloc(p, h.size()));
        if (!h.empty()) CUDA_TRY(cudaMemcpy(p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice));
        return CME_OK;
    }
    int step_grid() const { return vi2 || vi2b ? vi2_grid : use_tma ? tma_grid : grid; }
};

// ------------------------------------------------------------------------------
// small kernels
// ------------------------------------------------------------------------------

// out[b][0..7] = {sum p0, sum p1, sum p2, max p3, max p4, 0,0,0} of member b
// over nblocks partial records, in a fixed order (deterministic).  1 CTA x 1024.
__global__ void __launch_bounds__(1024) reduce_partials_kernel(const double* partials, int nblocks, int B,
                                                               double* out, const int32_t* stop) {
    pdl_trigger();
    pdl_wait();
    if (stop != nullptr && *stop) return;
    __shared__ double s[32][5];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int b = 0; b < B; ++b) {
        double a = 0, bb = 0, c = 0, d = 0, e = 0;
        for (int i = threadIdx.x; i < nblocks; i += blockDim.x) {
            const double* p = partials + ((size_t)i * B + b) * kPartials;
            a += p[0]; bb += p[1]; c += p[2]; d = fmax(d, p[3]); e = fmax(e, p[4]);
        }
        a = warp_sum(a); bb = warp_sum(bb); c = warp_sum(c); d = warp_max(d); e = warp_max(e);
        if (lane == 0) { s[w][0] = a; s[w][1] = bb; s[w][2] = c; s[w][3] = d; s[w][4] = e; }
        __syncthreads();
        if (threadIdx.x == 0) {
            a = bb = c = d = e = 0;
            for (int i = 0; i < (int)(blockDim.x >> 5); ++i) {
                a += s[i][0]; bb += s[i][1]; c += s[i][2]; d = fmax(d, s[i][3]); e = fmax(e, s[i][4]);
            }
            double* o = out + 8 * b;
            o[0] = a; o[1] = bb; o[2] = c; o[3] = d; o[4] = e; o[5] = o[6] = o[7] = 0.0;
        }
        __syncthreads();
    }
}

// Check decision (readings R2-R5): decide_apply
// (kernels.cuh) on the rank-ordered check records.
__global__ void decide_kernel(const double* all, int nranks, Ctrl* c, int32_t len, int32_t final_partial) {
    pdl_trigger();
    pdl_wait();
    if (c->stop) return;
    decide_apply(all, nranks, c, len, final_partial);
}

// x_own[l*B + b] = src[b*n_global + perm[l]] (original -> reordered,
// member-major -> member-minor), per-CTA partials {sum, #bad} per member.
template <int B>
__global__ void __launch_bounds__(kCta) load_kernel(const double* src, const int32_t* perm, int64_t n,
                                                    int64_t n_global, double* x_own, double* partials) {
    CheckAcc<B> ck;
    for (int64_t l = (int64_t)blockIdx.x * kCta + threadIdx.x; l < n; l += (int64_t)gridDim.x * kCta) {
        const int64_t o = perm[l];
#pragma unroll
        for (int b = 0; b < B; ++b) {
            const double v = src[(size_t)b * n_global + o];
            x_own[l * B + b] = v;
            ck.sy[b] += v;
            ck.sx[b] += (!(v >= 0.0) || isinf(v)) ? 1.0 : 0.0;
        }
    }
    cta_check_partials<kWarpsPerCta, B>(ck, partials);
}

__global__ void load_decide_kernel(const double* all, int nranks, Ctrl* c, int32_t normalise) {
    const int B = c->batch;
    int bad = 0;
    for (int b = 0; b < B; ++b) {
        double s = 0.0, nb = 0.0;
        for (int r = 0; r < nranks; ++r) {
            s += all[((size_t)r * B + b) * 8];
            nb += all[((size_t)r * B + b) * 8 + 1];
        }
        bad |= normalise && (nb > 0.0 || !(s > 0.0) || isinf(s));
        c->inv_s[b] = normalise ? 1.0 / s : 1.0;
        c->mass[b] = s;
    }
    c->bad_input = bad;
}

__global__ void fill_kernel(double* x, int64_t n, double v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = v;
}

// out[b*n_out + perm[l]] = x[l*B + b] * scale[b]   (reordered -> original order)
__global__ void scatter_out_kernel(const double* x, const int32_t* perm, int64_t n, int B, int64_t n_out,
                                   const double* scale, double* out) {
    for (int64_t l = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; l < n; l += (int64_t)gridDim.x * blockDim.x) {
        const int64_t o = perm[l];
        for (int b = 0; b < B; ++b) out[(size_t)b * n_out + o] = x[l * B + b] * scale[b];
    }
}

__global__ void scale_copy_kernel(const double* x, int64_t n, int B, const double* scale, double* out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n * B; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = x[i] * scale[i % B];
}

// Peer-memory barrier (NEXT-4): one thread bumps this rank's epoch, publishes
// it into every peer's flag slot (release, system scope: the step's halo
// stores into that peer are ordered before it) and waits (acquire) until every
// peer has published the same epoch.  Bounded spin: a peer that never arrives
// turns the solve into CME_ERR_TIMEOUT instead of a hung GPU.
struct BarrierArgs {
    int64_t* flags;
    int64_t* epoch;
    int64_t* peer_flags[kMaxPushPeers];
    int peer_rank[kMaxPushPeers];
    int npeer, rank;
    const int32_t* stop;   // nullable: skip when the solve has stopped (all ranks agree)
    Ctrl* ctrl;
    int32_t early;   // 1: let the next step launch early (peers on other GPUs only)
};
__global__ void p2p_barrier_kernel(const BarrierArgs a) {
    // launched with programmatic dependent launch after a step: wait for the
    // step's grid (its stores, peer pushes included, are then complete), then
    // let the next step's CTAs launch and run their prologue (TMA prefetch of
    // their first tiles, dictionary load) while this thread publishes/spins;
    // the next step's griddepcontrol.wait still waits for this kernel
    pdl_wait();
    if (a.early) pdl_trigger();   // (the trigger, not the launch attribute, releases the dependent)
    if (threadIdx.x != 0) return;
    if (a.stop != nullptr && *a.stop) return;
    const int64_t e = *a.epoch + 1;
    *a.epoch = e;
    __threadfence_system();
    for (int p = 0; p < a.npeer; ++p)
        asm volatile("st.release.sys.global.s64 [%0], %1;" ::"l"(a.peer_flags[p] + a.rank), "l"(e) : "memory");
    for (int p = 0; p < a.npeer; ++p) {
        const int64_t* f = a.flags + a.peer_rank[p];
        int64_t v = 0;
        long long spins = 0;
        for (;;) {
            asm volatile("ld.acquire.sys.global.s64 %0, [%1];" : "=l"(v) : "l"(f) : "memory");
            if (v >= e) break;
            if (++spins > (1LL << 28)) {   // ~ tens of seconds: a peer is gone
                a.ctrl->status = CME_ERR_TIMEOUT;
                a.ctrl->stop = 1;
                return;
            }
            __nanosleep(64);
        }
    }
}

// dst[j][0..count) = src[0..count) for every destination (local and/or peer)
struct CopyArgs {
    const double* src;
    double* dst[kMaxPushPeers + 1];
    int ndst;
    int64_t count;
    const int32_t* stop;
};
__global__ void multicast_copy_kernel(const CopyArgs a) {
    if (a.stop != nullptr && *a.stop) return;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.count; i += (int64_t)gridDim.x * blockDim.x) {
        const double v = a.src[i];
        for (int j = 0; j < a.ndst; ++j) a.dst[j][i] = v;
    }
}

// ------------------------------------------------------------------------------
// setup / teardown
// ------------------------------------------------------------------------------
static int grid_for(int64_t n) {
    int sms = 148;
    int dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return (int)std::max<int64_t>(1, std::min<int64_t>((n + kCta - 1) / kCta, (int64_t)sms * 8));
}

void device_free(Device* d) {
    if (!d) return;
    if (d->dev >= 0) cudaSetDevice(d->dev);
    for (void* p : d->ipc_opened) cudaIpcCloseMemHandle(p);
    for (auto& g : d->gexec)
        if (g) cudaGraphExecDestroy(g);
    for (auto& e : d->ev)
        if (e) cudaEventDestroy(e);
    if (d->t0) cudaEventDestroy(d->t0);
    if (d->t1) cudaEventDestroy(d->t1);
    for (void* p : d->allocs) cudaFree(p);
    if (d->ctrl_host) cudaFreeHost(d->ctrl_host);
    if (d->own) cudaStreamDestroy(d->own);
    if (d->cap) cudaStreamDestroy(d->cap);
    delete d;
}

static cme_status select_device(int want, int* out) {
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        set_error("no CUDA device visible");
        return CME_ERR_NO_DEVICE;
    }
    int dev = want;
    if (dev < 0) CUDA_TRY(cudaGetDevice(&dev));
    if (dev >= count) { set_error("device ordinal out of range"); return CME_ERR_INVALID_ARG; }
    CUDA_TRY(cudaSetDevice(dev));
    *out = dev;
    return CME_OK;
}

static int env_int(const char* name, int dflt) {
    const char* v = std::getenv(name);
    return (v && *v) ? std::atoi(v) : dflt;
}

static cudaError_t tma_prepare_b(int B, int ncw, int smem) {
    switch (B) {
        case 1: return tma_prepare<1>(ncw, smem);
        case 2: return tma_prepare<2>(ncw, smem);
        case 4: return tma_prepare<4>(ncw, smem);
        default: return tma_prepare<8>(ncw, smem);
    }
}
static cudaError_t tma_occupancy_b(int B, int ncw, int smem, int* occ) {
    switch (B) {
        case 1: return tma_occupancy<1>(ncw, smem, occ);
        case 2: return tma_occupancy<2>(ncw, smem, occ);
        case 4: return tma_occupancy<4>(ncw, smem, occ);
        default: return tma_occupancy<8>(ncw, smem, occ);
    }
}

// Stage geometry of the TMA kernel for tiles of ts slices.
static int64_t tma_stage_bytes(const Device& d, const Packed& P, int ts, int64_t* off_val, int64_t* off_col,
                               int64_t* n_tiles) {
    const int ncw = ts;
    *n_tiles = (d.n_slices + ncw - 1) / ncw;
    int64_t max_nval = 0;
    for (int64_t t = 0; t < *n_tiles; ++t) {
        const int64_t q0 = t * ncw, q1 = std::min<int64_t>(q0 + ncw, d.n_slices);
        max_nval = std::max(max_nval, P.slice_off[q1] - P.slice_off[q0]);
    }
    auto a128 = [](int64_t b) { return (b + 127) / 128 * 128; };
    // every stage: [tile metadata (kMetaBytes)] then the data blocks, whose
    // offsets off_val / off_col are relative to the data base
    if (d.vi) {    // [inv_d][row8][loi, upi][vidx][col16]
        *off_val = a128(vi_fixed_bytes(ncw, d.band, d.rearr));
        *off_col = *off_val + a128(2 * max_nval);
        return meta_bytes(ts) + a128(*off_col + 2 * max_nval);
    }
    if (d.cpt) {   // [row8][lo, up][val][col16]
        *off_val = a128(cpt_fixed_bytes(ncw, d.band, d.rearr));
        *off_col = *off_val + a128(8 * max_nval);
        return kMetaBytes + a128(*off_col + 2 * max_nval);
    }
    *off_val = a128(tma_fixed_bytes(ncw, d.B, d.band, d.rearr));
    *off_col = *off_val + a128(8 * d.B * max_nval);
    return kMetaBytes + a128(*off_col + 4 * max_nval);
}

// Choose the step kernel.  The TMA ring pays once every CTA streams >= 2
// tiles (>~300K rows) and >= 16 consumer warps per SM can be resident; among
// the tile shapes (16- or 8-slice tiles) the one with the most resident
// consumer warps wins (batches have wider stages: B = 2 prefers 8-slice tiles,
// B >= 4 the register kernel).  Tuning knobs (environment, read at
// pack/distribute): CME_TMA = -1 auto / 0 off / 1 force, CME_TMA_WARPS (16 | 8
// forces the shape), CME_TMA_STAGES (2..8), CME_TMA_CTAS.
static cme_status configure_tma(Device& d, const Packed& P) {
    d.use_tma = false;
    const int want = env_int("CME_TMA", -1);
    if (want == 0 || d.n_slices == 0) return CME_OK;
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int stages_env = env_int("CME_TMA_STAGES", 0);   // 0 = auto
    const int stages_req = stages_env > 0 ? std::min(8, std::max(2, stages_env)) : 0;
    int force_w = env_int("CME_TMA_WARPS", 0);
    if (force_w == 31 && !(d.vi && d.B == 1)) force_w = 16;   // the 31-warp shape exists for sell_vi_kernel only
    if (force_w == 15 && !(d.vi && d.B > 1)) force_w = 16;    // and the 15-warp one for sell_vib_kernel
    struct Shape { int ncw, spw, stages, occ, grid; int64_t stage, off_val, off_col, n_tiles; };
    struct Cand { int ncw, spw; };
    // consumer warps, slices per warp; 31 warps (one 1024-thread CTA per SM,
    // one dictionary per SM) only for the value-indexed kernel at B = 1, 15
    // (a 512-thread CTA: 128 registers) only for the batched one
    const Cand cands[] = {{16, 1}, {8, 1}, {31, 1}, {15, 1}};
    Shape best{};
    for (const Cand& cd : cands) {
        const int ncw = cd.ncw, spw = cd.spw;
        if (force_w && ncw != force_w) continue;
        if (ncw == 31 && !(d.vi && d.B == 1)) continue;
        if (ncw == 15 && !(d.vi && d.B > 1)) continue;
        // auto at B = 8: the 15-warp shape (128 registers, 24-byte spill) beats
        // 16 warps (96 registers, 48-200 byte spills): cfg4 1 437 vs 1 523 us
        // per iteration; at B = 2 / 4 the 16-warp shape stays ahead by 1-2%
        if (ncw == 16 && d.vi && d.B == 8 && !force_w) continue;
        Shape sh{};
        sh.ncw = ncw;
        sh.spw = spw;
        sh.stage = tma_stage_bytes(d, P, ncw * spw, &sh.off_val, &sh.off_col, &sh.n_tiles);
        // the attribute is process-wide per kernel: always raise it to the
        // largest size any handle may use (handles on several host threads --
        // an in-process rank group -- would otherwise lower it under each
        // other's launches: "invalid argument")
        // dynamic-smem cap: the opt-in maximum minus the static shared memory
        // (barriers, check-reduction scratch: < 2 KB for 33 warps)
        const int cap = smem_max - (d.vi ? 4096 : 1024);
        if (d.vi && d.B > 1) CUDA_TRY(vib_prepare(d.B, ncw, cap));
        else if (d.vi) CUDA_TRY(vi_prepare(ncw, cap));
        else if (d.cpt) CUDA_TRY(cpt_prepare(ncw, cap));
        else CUDA_TRY(tma_prepare_b(d.B, ncw, cap));
        const int64_t extra = d.vi ? d.dict_bytes : 0;   // the dictionary sits in front of the stages
        auto occ_of = [&](int stages, int* occ) -> cudaError_t {
            *occ = 0;
            const int64_t bytes = extra + stages * sh.stage;
            if (bytes > cap) return cudaSuccess;
            return d.vi && d.B > 1 ? vib_occupancy(d.B, ncw, (int)bytes, occ)
                   : d.vi ? vi_occupancy(ncw, (int)bytes, occ)
                        : d.cpt ? cpt_occupancy(ncw, (int)bytes, occ)
                                : tma_occupancy_b(d.B, ncw, (int)bytes, occ);
        };
        if (stages_req > 0) {
            sh.stages = stages_req;
            while (sh.stages > 2 && extra + sh.stages * sh.stage > cap) --sh.stages;
            CUDA_TRY(occ_of(sh.stages, &sh.occ));
        } else {
            // auto: 2 stages, or -- for the value-indexed kernel and whenever
            // the iterate stays L2-resident -- the deepest ring (<= 4) that
            // keeps the residency of 2 stages.  Measured on B200: value index
            // on cfg4 3 stages 178 vs 2 stages 206 us; cfg3a (16 MB iterate)
            // 19.5 vs 21.5 us; but on config-5 matrices with a 128 MB iterate a
            // deeper ring costs 13% (mu 5) to 2x (random columns): the extra
            // TMA traffic in flight delays the DRAM-bound gathers
            const bool x_in_l2 = (d.nx + 2) * 8 * d.B <= ((int64_t)48 << 20);
            sh.stages = 2;
            CUDA_TRY(occ_of(2, &sh.occ));
            for (int st = 3; st <= 4 && sh.occ > 0 && (d.vi || x_in_l2); ++st) {
                int o = 0;
                CUDA_TRY(occ_of(st, &o));
                if (o < sh.occ) break;
                sh.stages = st;
            }
        }
        if (env_int("CME_VERBOSE", 0) > 1)
            std::fprintf(stderr, "[cme] tma shape: ncw=%d spw=%d stages=%d stage=%lld extra=%lld occ=%d\n", ncw, spw, sh.stages,
                         (long long)sh.stage, (long long)extra, sh.occ);
        if (sh.occ < 1) continue;   // tiles too wide for this shape
        sh.occ = std::max(1, std::min(sh.occ, env_int("CME_TMA_CTAS", sh.occ)));
        sh.grid = (int)std::min<int64_t>(sh.n_tiles, (int64_t)sms * sh.occ);
        // most slices in flight per SM (resident consumer warps x slices per
        // warp); ties: the earlier candidate (wider tiles, fewer dictionaries)
        if (sh.ncw * sh.spw * sh.occ > best.ncw * best.spw * best.occ) best = sh;
    }
    if (best.ncw == 0) return CME_OK;
    if (want < 0 && (best.ncw * best.occ < 15 || best.n_tiles < 2 * (int64_t)sms * best.occ))
        return CME_OK;   // too few resident consumer warps (< 15: the batched 15-warp shape passes), or a small problem: register kernel
    d.tma_ncw = best.ncw;
    d.tma_spw = best.spw;
    d.n_tiles = best.n_tiles;
    d.tma_stages = best.stages;
    d.tma_stage_bytes = (int)best.stage;
    d.tma_off_val = (int)best.off_val;
    d.tma_off_col = (int)best.off_col;
    d.tma_grid = best.grid;
    d.tma_occ = best.occ;
    d.tma_contig = env_int("CME_TMA_CONTIG", 0) != 0;   // measured: round robin wins on cfg4 (+3%)
    // L2 prefetch of each tile's x rows: pays when the iterate does not stay
    // L2-resident across steps (measured: cfg4, 160 MB of x, 235 vs 241 us;
    // cfg3a, 16 MB, 21.5 vs 20.5 us).  CME_TMA_XPF = -1 auto / 0 / 1.
    const int xpf = env_int("CME_TMA_XPF", -1);
    d.tma_xpf = xpf >= 0 ? xpf != 0 : (d.nx + 2) * 8 * d.B > (int64_t)48 << 20;
    // inv_d prefetch (value-indexed kernels): auto = with the x prefetch (the
    // streams that leave L2 between steps); CME_VI_IDPF = -1 auto / 0 / 1
    const int idpf = env_int("CME_VI_IDPF", -1);
    d.vi_idpf = idpf >= 0 ? idpf != 0 : d.tma_xpf;
    d.use_tma = true;
    if (env_int("CME_VERBOSE", 0))
        std::fprintf(stderr, "[cme] tma: B=%d compact=%d vi=%d dict=%d warps=%d spw=%d stages=%d stage_bytes=%lld occ=%d grid=%d tiles=%lld\n",
                     d.B, (int)d.cpt, (int)d.vi, d.dict_bytes, best.ncw, best.spw, best.stages, (long long)best.stage, best.occ, best.grid, (long long)best.n_tiles);
    return CME_OK;
}

// Tile records of the value-indexed encoding for tiles of ts slices
// (kernels_vi2.cuh): per tile one contiguous block
// [meta | row8 | loi, upi | inv_d | per slice: vidx[32 W], col16[32 W]],
// every block 16-B aligned; a pure re-layout of sec. 5c's arrays.
static int64_t vi2_record_bytes(const Packed& P, int ts, bool band, bool rearr, int64_t t, bool f64 = false) {
    const int64_t q0 = t * ts, q1 = std::min<int64_t>(q0 + ts, P.n_slices);
    return vi2_fixed_bytes(ts, band, rearr, f64) + (f64 ? 10 : 4) * (P.slice_off[q1] - P.slice_off[q0]);
}

static void vi2_build_records(const Packed& P, const Compact& C, int ts, bool band, bool rearr, bool words,
                              std::vector<unsigned char>& rec, std::vector<int64_t>& off, bool f64 = false) {
    const int64_t nt = (P.n_slices + ts - 1) / ts;
    off.assign(nt + 1, 0);
    for (int64_t t = 0; t < nt; ++t) off[t + 1] = off[t] + vi2_record_bytes(P, ts, band, rearr, t, f64);
    rec.assign((size_t)off[nt], 0);
    const int kMeta = ((ts + 1) & ~1) * 8;
    const int kRow = kMeta, kLoUp = kRow + (rearr ? ts * 32 : 0), kInv = kLoUp + (band ? ts * (f64 ? 512 : 128) : 0),
              kEnt = kInv + (f64 ? 0 : ts * 256);
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < nt; ++t) {
        unsigned char* R = rec.data() + off[t];
        const int64_t q0 = t * ts, q1 = std::min<int64_t>(q0 + ts, P.n_slices);
        const int64_t e0 = P.slice_off[q0];
        for (int64_t q = q0; q < q1; ++q) {
            const int32_t m[2] = {(int32_t)(P.slice_off[q] - e0), (int32_t)P.slice_w[q]};
            std::memcpy(R + 8 * (q - q0), m, 8);
            const int64_t sl0 = q * 32, ls0 = (q - q0) * 32;
            if (rearr) std::memcpy(R + kRow + ls0, C.row8.data() + sl0, 32);
            if (f64) {   // [lo_c, up_c (band)] | per slice: val_c[32 W] then col16[32 W]
                if (band) {
                    std::memcpy(R + kLoUp + 8 * ls0, C.lo.data() + sl0, 256);
                    std::memcpy(R + kLoUp + ts * 256 + 8 * ls0, C.up.data() + sl0, 256);
                }
                const int64_t ne = P.slice_off[q + 1] - P.slice_off[q];
                unsigned char* E = R + kEnt + 10 * (P.slice_off[q] - e0);
                std::memcpy(E, C.val.data() + P.slice_off[q], 8 * ne);
                std::memcpy(E + 8 * ne, C.col16.data() + P.slice_off[q], 2 * ne);
                continue;
            }
            if (band) {
                std::memcpy(R + kLoUp + 2 * ls0, C.loi.data() + sl0, 64);
                std::memcpy(R + kLoUp + ts * 64 + 2 * ls0, C.upi.data() + sl0, 64);
            }
            std::memcpy(R + kInv + 8 * ls0, P.inv_d.data() + sl0, 256);
            const int64_t ne = P.slice_off[q + 1] - P.slice_off[q];   // 32 W entries
            unsigned char* E = R + kEnt + 4 * (P.slice_off[q] - e0);
            if (words) {   // entry k: vidx | col16 << 16
                for (int64_t k = 0; k < ne; ++k) {
                    const uint32_t w = (uint32_t)C.vidx[P.slice_off[q] + k] |
                                       ((uint32_t)(uint16_t)C.col16[P.slice_off[q] + k] << 16);
                    std::memcpy(E + 4 * k, &w, 4);
                }
            } else {
                std::memcpy(E, C.vidx.data() + P.slice_off[q], 2 * ne);
                std::memcpy(E + 2 * ne, C.col16.data() + P.slice_off[q], 2 * ne);
            }
        }
    }
}

// Choose the vi2 tile shape, in the order measured on cfg4 (B200): 30
// consumer warps in one 1024-thread CTA per SM (one dictionary, 64 registers,
// 4 x 32 KB stages: 170 us per iteration) when >= 3 stages fit, else 16 in 2
// CTAs per SM (56 registers, 3 stages: 175 us); 23 warps in 2 CTAs per SM (40
// registers: spills, 2 stages: 227 us) only when forced.  Deepest ring <= 4
// stages.  CME_VI2_WARPS / CME_VI2_STAGES force a shape.
static cme_status configure_vi2(Device& d, const Packed& P, bool f64 = false) {
    d.vi2 = false;
    d.vi2_f64 = false;
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int force_w = env_int("CME_VI2_WARPS", 0), force_s = env_int("CME_VI2_STAGES", 0);
    const int cap = smem_max - 4096;
    struct Best { int ncw = 0, stages = 0, occ = 0; int64_t stage = 0, tiles = 0; } best;
    for (int ncw : {30, 16, 23}) {
        if (force_w && ncw != force_w) continue;
        if (!force_w && ncw == 23) continue;
        const int64_t nt = (P.n_slices + ncw - 1) / ncw;
        int64_t mx = 0;
        for (int64_t t = 0; t < nt; ++t) mx = std::max(mx, vi2_record_bytes(P, ncw, d.band, d.rearr, t, f64));
        const int64_t stage = (mx + 127) / 128 * 128;
        CUDA_TRY(vi2_prepare(ncw, cap));
        const int want_occ = ncw == 30 ? 1 : 2;
        int stages = 0, occ = 0;
        for (int st = force_s > 0 ? std::min(force_s, 8) : 4; st >= 2; --st) {
            const int64_t bytes = d.dict_bytes + st * stage;
            if (bytes > cap) continue;
            int o = 0;
            CUDA_TRY(vi2_occupancy(ncw, (int)bytes, &o, f64 ? 2 : 0));
            if (o >= want_occ || (force_s > 0 && o >= 1)) { stages = st; occ = o; break; }
        }
        if (env_int("CME_VERBOSE", 0) > 1)
            std::fprintf(stderr, "[cme] vi2 shape: ncw=%d stage=%lld stages=%d occ=%d\n", ncw, (long long)stage, stages, occ);
        if (!stages || (!force_w && !force_s && ncw == 30 && stages < 3)) continue;
        best = Best{ncw, stages, occ, stage, nt};
        break;   // first acceptable shape in measured order
    }
    if (!best.ncw) return CME_OK;
    if (env_int("CME_VI2", 1) == 0) return CME_OK;
    d.vi2 = true;
    d.vi2_words = !f64 && env_int("CME_VI2_WORDS", 0) != 0;
    d.vi2_f64 = f64;
    d.vi2_ncw = best.ncw;
    d.vi2_stages = best.stages;
    d.vi2_stage_bytes = (int)best.stage;
    d.vi2_occ = best.occ;
    d.vi2_tiles = best.tiles;
    d.vi2_grid = (int)std::min<int64_t>(best.tiles, (int64_t)sms * best.occ);
    // CME_VI2_GRID caps the grid (tests: many tiles per CTA wrap the ring many times)
    if (env_int("CME_VI2_GRID", 0) > 0) d.vi2_grid = std::min(d.vi2_grid, env_int("CME_VI2_GRID", 0));
    if (env_int("CME_VERBOSE", 0))
        std::fprintf(stderr, "[cme] vi2: warps=%d stages=%d stage_bytes=%d occ=%d grid=%d tiles=%lld dict=%d\n",
                     d.vi2_ncw, d.vi2_stages, d.vi2_stage_bytes, d.vi2_occ, d.vi2_grid, (long long)d.vi2_tiles,
                     d.dict_bytes);
    return CME_OK;
}

// Batched tile records (sell_vi2b_kernel): the B = 1
// record with a B-wide inv_d block (member-minor per slot).
static int64_t vi2b_record_bytes(const Packed& P, int ts, int B, bool band, bool rearr, int64_t t) {
    const int64_t q0 = t * ts, q1 = std::min<int64_t>(q0 + ts, P.n_slices);
    return vi2b_fixed_bytes(ts, B, band, rearr) + 4 * (P.slice_off[q1] - P.slice_off[q0]);
}

static void vi2b_build_records(const Packed& P, const Compact& C, int ts, int B, bool band, bool rearr,
                               std::vector<unsigned char>& rec, std::vector<int64_t>& off) {
    const int64_t nt = (P.n_slices + ts - 1) / ts;
    off.assign(nt + 1, 0);
    for (int64_t t = 0; t < nt; ++t) off[t + 1] = off[t] + vi2b_record_bytes(P, ts, B, band, rearr, t);
    rec.assign((size_t)off[nt], 0);
    const int kMeta = ((ts + 1) & ~1) * 8;
    const int kRow = kMeta, kLoUp = kRow + (rearr ? ts * 32 : 0), kInv = kLoUp + (band ? ts * 128 : 0),
              kEnt = kInv + ts * 256 * B;
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < nt; ++t) {
        unsigned char* R = rec.data() + off[t];
        const int64_t q0 = t * ts, q1 = std::min<int64_t>(q0 + ts, P.n_slices);
        const int64_t e0 = P.slice_off[q0];
        for (int64_t q = q0; q < q1; ++q) {
            const int32_t m[2] = {(int32_t)(P.slice_off[q] - e0), (int32_t)P.slice_w[q]};
            std::memcpy(R + 8 * (q - q0), m, 8);
            const int64_t sl0 = q * 32, ls0 = (q - q0) * 32;
            if (rearr) std::memcpy(R + kRow + ls0, C.row8.data() + sl0, 32);
            if (band) {
                std::memcpy(R + kLoUp + 2 * ls0, C.loi.data() + sl0, 64);
                std::memcpy(R + kLoUp + ts * 64 + 2 * ls0, C.upi.data() + sl0, 64);
            }
            std::memcpy(R + kInv + 8 * B * ls0, P.inv_d.data() + (size_t)sl0 * B, (size_t)256 * B);
            const int64_t ne = P.slice_off[q + 1] - P.slice_off[q];
            unsigned char* E = R + kEnt + 4 * (P.slice_off[q] - e0);
            std::memcpy(E, C.vidx.data() + P.slice_off[q], 2 * ne);
            std::memcpy(E + 2 * ne, C.col16.data() + P.slice_off[q], 2 * ne);
        }
    }
}

// Shape of the batched tile-record kernel (vi2b_warps: B = 2 16 warps, B = 4
// 16, B = 8 15), the deepest ring (<= 4 stages) that fits one CTA per SM.
// Auto (CME_VI2B = -1) only at B = 2, where it was measured faster on cfg4
// (333 vs 375 us per iteration); B = 4 573 vs 563 and B = 8 1 676 vs 1 364
// (the 404 KB tuple dictionary misses L1 either way) keep sell_vib_kernel.
// CME_VI2B = 1 forces it at any B, 0 disables it.
static cme_status configure_vi2b(Device& d, const Packed& P, int64_t dict_doubles) {
    d.vi2b = false;
    d.vi2b_dict_bytes = 0;
    const int want = env_int("CME_VI2B", -1);
    if (want == 0 || d.B < 2 || d.nranks > 1 || (want < 0 && d.B != 2)) return CME_OK;
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int cap = smem_max - 4096;
    const int ncw = vi2b_warps(d.B, env_int("CME_VI2_WARPS", 0));
    const int64_t nt = (P.n_slices + ncw - 1) / ncw;
    int64_t mx = 0;
    for (int64_t t = 0; t < nt; ++t) mx = std::max(mx, vi2b_record_bytes(P, ncw, d.B, d.band, d.rearr, t));
    const int64_t stage = (mx + 127) / 128 * 128;
    CUDA_TRY(vi2b_prepare(d.B, ncw, cap));
    const int force_s = env_int("CME_VI2_STAGES", 0);
    // B = 2 on 16-warp tiles: the tuple dictionary in shared memory when it fits
    // beside >= 3 stages (CME_VI2B_SD = 0 keeps it in global memory)
    const int64_t sd = d.B == 2 && ncw == 16 && env_int("CME_VI2B_SD", 1) != 0 ? (dict_doubles * 8 + 127) / 128 * 128 : 0;
    // first the staged-dictionary shapes (>= 3 stages), then the L1 ones
    for (int pass = sd > 0 ? 0 : 1; pass < 2; ++pass)
    for (int st = force_s > 0 ? std::min(force_s, 8) : 4; st >= 2; --st) {
        const int64_t dict = pass == 0 ? sd : 0;
        if (pass == 0 && st < 3 && force_s <= 0) continue;
        if (dict + st * stage > cap) continue;
        int occ = 0;
        CUDA_TRY(vi2b_occupancy(d.B, ncw, (int)(dict + st * stage), &occ));
        if (env_int("CME_VERBOSE", 0) > 1)
            std::fprintf(stderr, "[cme] vi2b shape: stages=%d stage=%lld dict=%lld (tuples %lld doubles) occ=%d\n", st,
                         (long long)stage, (long long)dict, (long long)dict_doubles, occ);
        if (occ < 1) continue;
        d.vi2b = true;
        d.vi2b_dict_bytes = (int)dict;
        d.vi2_ncw = ncw;
        d.vi2_stages = st;
        d.vi2_stage_bytes = (int)stage;
        d.vi2_occ = occ;
        d.vi2_tiles = nt;
        d.vi2_grid = (int)std::min<int64_t>(nt, (int64_t)sms * occ);
        if (env_int("CME_VI2_GRID", 0) > 0) d.vi2_grid = std::min(d.vi2_grid, env_int("CME_VI2_GRID", 0));
        if (env_int("CME_VERBOSE", 0))
            std::fprintf(stderr, "[cme] vi2b: B=%d warps=%d stages=%d stage_bytes=%d dict_smem=%d occ=%d grid=%d tiles=%lld\n",
                         d.B, ncw, st, d.vi2_stage_bytes, d.vi2b_dict_bytes, occ, d.vi2_grid, (long long)nt);
        return CME_OK;
    }
    return CME_OK;
}

// x-window plan (XW kernels) for tiles of ts slices:
// per tile the iterate chunks (256 rows, chunk k = rows [256 k - xoff,
// 256 k - xoff + 256) of the local x) holding its rows, band neighbours and
// gathered columns, as a suffix-min of the first and a prefix-max of the end
// chunk so the producer streams every chunk once, in order.
void xw_plan(const Packed& P, int ts, bool band, int64_t own_off, int xoff, int64_t nx,
             std::vector<int2>& ch) {
    const int64_t nt = (P.n_slices + ts - 1) / ts, n = P.n;
    std::vector<int64_t> lo(nt), hi(nt);
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t t = 0; t < nt; ++t) {
        int64_t mn = INT64_MAX, mx = INT64_MIN;
        const int64_t q1 = std::min<int64_t>((t + 1) * ts, P.n_slices);
        for (int64_t q = t * ts; q < q1; ++q)
            for (int ln = 0; ln < 32; ++ln) {
                const int64_t slot = q * 32 + ln;
                if (slot >= n) break;
                const int64_t r = P.row_of.empty() ? slot : P.row_of[slot];
                mn = std::min(mn, r - (band ? 1 : 0));
                mx = std::max(mx, r + (band ? 1 : 0));
                for (int32_t u = 0; u < P.slice_w[q]; ++u) {
                    const int64_t j = (int64_t)P.col[P.slice_off[q] + ln + 32 * u] - own_off;
                    mn = std::min(mn, j);
                    mx = std::max(mx, j);
                }
            }
        if (mn > mx) mn = mx = 0;   // an all-padding tile
        const int64_t last = (nx + xoff) >> 8;   // chunk of the sentinel row nx
        lo[t] = std::max<int64_t>(0, (mn + xoff) >> 8);
        hi[t] = std::min<int64_t>(last, (mx + xoff) >> 8) + 1;
    }
    for (int64_t t = nt - 2; t >= 0; --t) lo[t] = std::min(lo[t], lo[t + 1]);
    for (int64_t t = 1; t < nt; ++t) hi[t] = std::max(hi[t], hi[t - 1]);
    ch.resize(nt);
    for (int64_t t = 0; t < nt; ++t) ch[t] = make_int2((int)lo[t], (int)hi[t]);
}

// Ring chunks a CTA needs with S stages in flight: tiles j-S+1 .. j are live
// when tile j's chunks are issued (tile j-S has released its stage); and the
// widest tile's chunk count (the mirror).
int64_t xw_need(const std::vector<int2>& ch, int S, int64_t& span) {
    int64_t need = 1;
    span = 1;
    for (int64_t t = 0; t < (int64_t)ch.size(); ++t) {
        need = std::max<int64_t>(need, ch[t].y - ch[std::max<int64_t>(0, t - S + 1)].x);
        span = std::max<int64_t>(span, ch[t].y - ch[t].x);
    }
    return need;
}

// Mean distinct 32-byte sectors per warp-wide x gather (32 lanes' t-th
// entries of a slice), over every 16th slice: ~8-9 when consecutive rows
// gather consecutive columns (the CME orderings, cfg3a's grid band), up to 32
// for a random band (config 5).  Decides whether the x window pays.
static double gather_sectors(const Packed& P) {
    double sum = 0;
    int64_t cnt = 0;
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : sum, cnt)
    for (int64_t q = 0; q < P.n_slices; q += 16) {
        for (int32_t t = 0; t < P.slice_w[q]; ++t) {
            int64_t sec[32];
            int k = 0;
            for (int ln = 0; ln < 32; ++ln) {
                if (q * 32 + ln >= P.n) break;
                sec[k++] = (int64_t)P.col[P.slice_off[q] + ln + 32 * t] >> 2;
            }
            if (!k) continue;
            std::sort(sec, sec + k);
            sum += (double)(std::unique(sec, sec + k) - sec);
            ++cnt;
        }
    }
    return cnt ? sum / cnt : 0.0;
}

// The x-window shape (single GPU; records of the value-indexed encoding, or
// of the f64 compact one when there is no value index): the first of
// (30 warps, 4 | 3 stages), (16, 4 | 3), (30, 2), (16, 2) whose dictionary,
// stages and ring fit one CTA per SM, for the mirrored ring (XWM 1) if any
// shape fits it, else for the ring with a wrap per entry (XWM 2).  CME_XW = 1
// forces the x window, 0 disables it; auto (-1) takes it for f64 records whose
// x gathers are uncoalesced (>= 16 sectors per warp request) with a ring of at
// most CME_XW_RING_KB (160) KB.  Measured (B200): config 5
// (16 M rows, mu = 10, random band) width 1 024 291 us vs 410 on
// sell_cpt_kernel, width 4 096 330 vs 640 (wrap mode); coalesced gathers lose: cfg3a
// 28.7 vs 19.1 us, toggle N = 2 200 (RCM) 133 vs 79 us.
static cme_status configure_xw(Device& d, const Packed& P, bool f64, std::vector<int2>& plan) {
    d.xw = 0;
    const int want = env_int("CME_XW", -1);
    if (want == 0 || d.nranks > 1 || d.B != 1 || (want < 0 && !f64)) return CME_OK;
    if (want < 0) {
        const double sec = gather_sectors(P);
        if (env_int("CME_VERBOSE", 0)) std::fprintf(stderr, "[cme] xw: %.1f sectors per x gather\n", sec);
        if (sec < 16.0) return CME_OK;
    }
    // chunk k starts at local row 256 k - 1: 16-B aligned when x + own_off is 8 mod 16 (the
    // x-span buffers sit one sentinel row into 256-B aligned allocations), row -1 loadable
    const int xoff = 1;
    for (int b = 0; b < 2; ++b)
        if (((reinterpret_cast<uintptr_t>(d.xb[b] + d.own_off) >> 3) & 1) != 1) return CME_OK;
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int cap = smem_max - 4096, enc = f64 ? 2 : 0;
    const int dict = f64 ? 0 : d.dict_bytes;
    const int force_w = env_int("CME_VI2_WARPS", 0), force_s = env_int("CME_VI2_STAGES", 0);
    const int64_t nx = d.nx - d.own_off;
    const int64_t ring_cap = want > 0 ? INT64_MAX : (int64_t)env_int("CME_XW_RING_KB", 160) << 10;
    int64_t stage_of[2] = {0, 0};   // [30 warps, 16 warps]
    std::vector<int2> plan_of[2];   // chunk ranges per tile, by warp count
    // (8-warp tiles, for windows too wide for these: measured 587 vs 420 us on
    // config 5 width 8 192 -- too few warps once the gathers are shared loads)
    const int order[6][2] = {{30, 4}, {30, 3}, {16, 4}, {16, 3}, {30, 2}, {16, 2}};
    const int force_m = env_int("CME_XW_MODE", 0);   // 1 mirror, 2 wrap (tests)
    for (int mode = 1; mode <= 2; ++mode)
    for (const auto& sh : order) {
        if (force_m && mode != force_m) continue;
        const int ncw = sh[0];
        if (force_w && ncw != force_w) continue;
        const int st = force_s > 0 ? std::min(force_s, 8) : sh[1];
        if (force_s > 0 && sh[1] != 4) continue;   // one candidate per warp count when forced
        const int64_t nt = (P.n_slices + ncw - 1) / ncw;
        int64_t& stage = stage_of[ncw == 30 ? 0 : 1];
        if (!stage) {
            int64_t mx = 0;
            for (int64_t t = 0; t < nt; ++t) mx = std::max(mx, vi2_record_bytes(P, ncw, d.band, d.rearr, t, f64));
            stage = (mx + 127) / 128 * 128;
            CUDA_TRY(vi2_xw_prepare(ncw, cap));
        }
        {
            std::vector<int2>& ch = plan_of[ncw == 30 ? 0 : 1];
            if (ch.empty()) xw_plan(P, ncw, d.band, d.own_off, xoff, nx, ch);
            int64_t span = 1;
            const int64_t need = xw_need(ch, st, span);
            const int64_t slots = need, mirror = mode == 1 ? span - 1 : 0;
            const int64_t bytes = dict + st * stage + (slots + mirror) * 2048;
            if (env_int("CME_VERBOSE", 0) > 1)
                std::fprintf(stderr, "[cme] xw shape: ncw=%d stages=%d stage=%lld ring chunks=%lld (need %lld) smem=%lld\n",
                             ncw, st, (long long)stage, (long long)slots, (long long)need, (long long)bytes);
            if (bytes > cap || (slots + mirror) * 2048 > ring_cap) continue;
            int occ = 0;
            CUDA_TRY(vi2_xw_occupancy(ncw, (int)bytes, &occ, enc));
            if (occ < 1) continue;
            d.xw = mode;
            d.vi2 = true;
            d.vi2_f64 = f64;
            d.vi2_words = false;
            if (f64) d.dict_bytes = 0;
            d.vi2_ncw = ncw;
            d.vi2_stages = st;
            d.vi2_stage_bytes = (int)stage;
            d.vi2_occ = occ;
            d.vi2_tiles = nt;
            d.vi2_grid = (int)std::min<int64_t>(nt, (int64_t)sms * occ);
            if (env_int("CME_VI2_GRID", 0) > 0) d.vi2_grid = std::min(d.vi2_grid, env_int("CME_VI2_GRID", 0));
            d.xw_rows = (int)(slots * 256);
            d.xw_mirror = (int)mirror;
            d.xw_off = xoff;
            d.xw_nx = nx;
            d.xw_ring_bytes = (int)((slots + mirror) * 2048);
            plan = ch;
            if (env_int("CME_VERBOSE", 0))
                std::fprintf(stderr, "[cme] xw: mode=%d warps=%d stages=%d stage_bytes=%d ring=%d KB occ=%d grid=%d tiles=%lld\n",
                             mode, ncw, st, d.vi2_stage_bytes, d.xw_ring_bytes / 1024, occ, d.vi2_grid, (long long)nt);
            return CME_OK;
        }
    }
    return CME_OK;
}

// Wavefront plan (kernels_wf.cuh): per tile of ncw slices, the union of the
// tiles holding the rows it gathers (RAW) and the tiles gathering its rows
// (WAR), as one [first, last] range; then the (step, tile) items in wave
// order with lag L = max |dep - t| + 1 + extra (extra: tiles the G CTAs keep
// in flight, so a dependency is normally complete when it is polled).
static int wf_plan(const Packed& P, int ncw, bool band, int s, int extra, std::vector<int2>& dep,
                   std::vector<uint32_t>& items) {
    const int64_t n = P.n, ts = (int64_t)ncw * 32;
    const int64_t T = (P.n_slices + ncw - 1) / ncw;
    std::vector<int32_t> tile_of(n);
    for (int64_t slot = 0; slot < std::min(P.n_slots, n); ++slot) tile_of[P.row_of[slot]] = (int32_t)(slot / ts);
    dep.assign(T, make_int2(INT32_MAX, -1));
    std::vector<int2> war(T, make_int2(INT32_MAX, -1));
    for (int64_t u = 0; u < T; ++u) {
        int2 raw = make_int2(INT32_MAX, -1);
        auto see = [&](int64_t col) {
            if (col < 0 || col >= n) return;   // zero sentinels
            const int32_t t = tile_of[col];
            raw.x = std::min(raw.x, t);
            raw.y = std::max(raw.y, t);
            war[t].x = std::min(war[t].x, (int32_t)u);
            war[t].y = std::max(war[t].y, (int32_t)u);
        };
        for (int64_t q = u * ncw; q < std::min((u + 1) * ncw, P.n_slices); ++q)
            for (int lane = 0; lane < 32; ++lane) {
                const int64_t slot = q * 32 + lane;
                if (slot >= n) continue;
                const int64_t r = P.row_of[slot];
                see(r);
                if (band) { see(r - 1); see(r + 1); }
                for (int w = 0; w < P.slice_w[q]; ++w) see(P.col[P.slice_off[q] + lane + 32 * w]);
            }
        dep[u] = raw;
    }
    int dd = 0;
    for (int64_t t = 0; t < T; ++t) {
        int2& d = dep[t];
        d.x = std::min(d.x, war[t].x);
        d.y = std::max(d.y, war[t].y);
        if (d.y < 0) d = make_int2((int)t, (int)t);
        dd = std::max(dd, (int)std::max(d.y - t, t - d.x));
    }
    const int L = dd + 1 + std::max(extra, 0);
    items.clear();
    items.reserve((size_t)s * T);
    for (int64_t w = 0; w < T + (int64_t)(s - 1) * L; ++w)
        for (int j = 0; j < s; ++j) {
            const int64_t t = w - (int64_t)j * L;
            if (t >= 0 && t < T) items.push_back(((uint32_t)j << 24) | (uint32_t)t);
        }
    return L;
}

// Plan the SMEM-resident kernel (kernels_resident.cuh): one CTA per SM, each
// owning a window-aligned run of slices (<= 128) whose packed image fits in
// shared memory; its probe range = owners of the columns it reads plus the
// CTAs reading its rows.  Single GPU, B = 1, SELL formats.  CME_RESIDENT = -1
// auto (use it whenever it fits), 0 off, 1 force (error if it does not fit);
// CME_RES_TIMEOUT_MS bounds every wait (default 2000).
static cme_status configure_resident(Device& d, const Packed& P, bool distributed) {
    d.use_res = false;
    const int want = env_int("CME_RESIDENT", -1);
    if (want == 0 || (want < 0 && env_int("CME_TMA", -1) == 1)) return CME_OK;   // a forced TMA kernel wins
    auto refuse = [&](const char* why) {
        if (want == 1) { set_error(std::string("CME_RESIDENT=1: ") + why); return CME_ERR_INVALID_ARG; }
        return CME_OK;
    };
    if (distributed || d.B != 1 || d.format == CME_FMT_CSR || d.n_slices == 0)
        return refuse("needs one GPU, batch 1 and a sliced format");
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int64_t win = std::max<int32_t>(P.window, 1);
    int64_t g32 = 32, ww = win;
    while (ww) { const int64_t t = g32 % ww; g32 = ww; ww = t; }
    const int64_t unit = win > 1 ? win / g32 : 1;           // slices per window-aligned unit
    const int64_t units = (d.n_slices + unit - 1) / unit;
    const int G = (int)std::min<int64_t>(sms, units);
    std::vector<int32_t> q(G + 1);
    for (int b = 0; b <= G; ++b) q[b] = (int32_t)std::min<int64_t>(d.n_slices, (int64_t)b * units / G * unit);
    int64_t smem = 0, max_nsl = 0;
    for (int b = 0; b < G; ++b) {
        const int64_t nsl = q[b + 1] - q[b], nval = P.slice_off[q[b + 1]] - P.slice_off[q[b]];
        smem = std::max(smem, res_smem_bytes(nval, nsl, d.band, d.rearr));
        max_nsl = std::max(max_nsl, nsl);
    }
    if (max_nsl > 4 * kResWarps) return refuse("more than 128 slices per CTA");
    const int rps = max_nsl <= kResWarps ? 1 : max_nsl <= 2 * kResWarps ? 2 : 4;
    // auto: up to 2 row slots per thread (measured on B200: toggle N=300,
    // 179K rows, 2 slots: 3.8 us/iteration vs 4.2 for the register kernel;
    // N=400, 319K rows, 4 slots: 5.8 vs 4.9 for the TMA kernel)
    if (want < 0 && rps > 2) return CME_OK;
    smem = (smem + 15) / 16 * 16;
    if (smem > smem_max - 4096) return refuse("packed matrix does not fit in shared memory");
    // own-row and column hulls per CTA (local rows = x-span on one GPU)
    const int64_t n = d.n_own;
    std::vector<int64_t> rlo(G), rhi(G), clo(G), chi(G);
    for (int b = 0; b < G; ++b) {
        int64_t lo = INT64_MAX, hi = -1, cl = INT64_MAX, ch = -1, cnt = 0;
        for (int64_t slot = (int64_t)q[b] * 32; slot < std::min<int64_t>((int64_t)q[b + 1] * 32, n); ++slot) {
            const int64_t r = d.rearr ? P.row_of[slot] : slot;
            lo = std::min(lo, r); hi = std::max(hi, r); ++cnt;
        }
        if (cnt != hi - lo + 1) return refuse("CTA rows are not contiguous");
        cl = lo; ch = hi;
        if (d.band) { cl = std::max<int64_t>(0, lo - 1); ch = std::min<int64_t>(n - 1, hi + 1); }
        for (int64_t e = P.slice_off[q[b]]; e < P.slice_off[q[b + 1]]; ++e) {
            cl = std::min<int64_t>(cl, P.col[e]); ch = std::max<int64_t>(ch, P.col[e]);
        }
        rlo[b] = lo; rhi[b] = hi; clo[b] = std::max<int64_t>(cl, 0); chi[b] = std::min<int64_t>(ch, n - 1);
    }
    for (int b = 1; b < G; ++b)
        if (rlo[b] != rhi[b - 1] + 1) return refuse("CTA row runs are not consecutive");
    auto owner = [&](int64_t row) {
        return (int)(std::upper_bound(rlo.begin(), rlo.end(), row) - rlo.begin()) - 1;
    };
    // D[b] = CTAs whose rows b reads (its gathers see their outputs), R[b] =
    // CTAs reading b's rows; b probes R[b] \ D[b] (WAR, kernels_resident.cuh)
    std::vector<std::vector<char>> D(G, std::vector<char>(G, 0));
    for (int b = 0; b < G; ++b) {
        auto mark = [&](int64_t c) { if (c >= 0 && c < n) D[b][owner(c)] = 1; };
        for (int64_t e = P.slice_off[q[b]]; e < P.slice_off[q[b + 1]]; ++e) mark(P.col[e]);
        if (d.band) { mark(rlo[b] - 1); mark(rhi[b] + 1); }
        D[b][b] = 1;
    }
    std::vector<int32_t> probe_off(G + 1, 0), probe_cta;
    int64_t max_probes = 0;
    for (int b = 0; b < G; ++b) {
        for (int c = 0; c < G; ++c)
            if (c != b && D[c][b] && !D[b][c]) probe_cta.push_back(c);
        probe_off[b + 1] = (int32_t)probe_cta.size();
        max_probes = std::max<int64_t>(max_probes, probe_off[b + 1] - probe_off[b]);
    }
    if (max_probes > kResThreads) return refuse("too many probe CTAs");
    CUDA_TRY(resident_prepare(smem_max - 4096));   // process-wide cap (see configure_tma)
    int occ = 0;
    CUDA_TRY(resident_occupancy((int)smem, &occ));
    if (occ < 1) return refuse("resident kernel cannot be resident");
    std::vector<int32_t> first(G + 1);
    for (int b = 0; b < G; ++b) first[b] = (int32_t)rlo[b];
    first[G] = (int32_t)n;
    CME_TRY(d.upload(d.res_q, q));
    CME_TRY(d.upload(d.res_row, first));
    CME_TRY(d.upload(d.res_probe_off, probe_off));
    CME_TRY(d.upload(d.res_probe, probe_cta));
    CME_TRY(d.alloc(d.res_sync, 4));
    d.res_grid = G;
    d.res_smem = (int)smem;
    d.res_rps = rps;
    d.res_timeout_ns = (int64_t)std::max(1, env_int("CME_RES_TIMEOUT_MS", 2000)) * 1000000;
    d.use_res = true;
    if (env_int("CME_VERBOSE", 0))
        std::fprintf(stderr, "[cme] resident: grid=%d smem=%lld unit=%lld rows/thread=%d probes=%lld (max %lld)\n", G,
                     (long long)smem, (long long)unit, rps, (long long)probe_cta.size(), (long long)max_probes);
    return CME_OK;
}

// Load every kernel a solve may launch before any of them runs: with CUDA
// lazy loading (the default) the first launch of a kernel may wait for the
// device to drain, and a rank of an in-process group whose peer is spinning
// in p2p_barrier_kernel would then never get its kernel loaded (observed as a
// barrier time-out on the first run of the virtual-rank tests).
static cme_status preload_kernels(int B) {
    cudaFuncAttributes fa;
    CUDA_TRY(cudaFuncGetAttributes(&fa, reduce_partials_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, decide_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, load_kernel<1>));
    CUDA_TRY(cudaFuncGetAttributes(&fa, load_kernel<2>));
    CUDA_TRY(cudaFuncGetAttributes(&fa, load_kernel<4>));
    CUDA_TRY(cudaFuncGetAttributes(&fa, load_kernel<8>));
    CUDA_TRY(cudaFuncGetAttributes(&fa, load_decide_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, fill_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, scatter_out_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, scale_copy_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, p2p_barrier_kernel));
    CUDA_TRY(cudaFuncGetAttributes(&fa, multicast_copy_kernel));
    switch (B) {
        case 1: CUDA_TRY(sell_preload<1>()); break;
        case 2: CUDA_TRY(sell_preload<2>()); break;
        case 4: CUDA_TRY(sell_preload<4>()); break;
        default: CUDA_TRY(sell_preload<8>()); break;
    }
    return CME_OK;
}

// Build the device state from h->P (local layout) and the partition in h.
cme_status device_upload(cme_matrix_s* h, int want_dev, const HaloPlan* halo, cme_comm_s* comm) {
    int dev = 0;
    CME_TRY(select_device(want_dev, &dev));
    Device* d = new Device();
    d->dev = dev;
    auto fail = [&](cme_status s) { device_free(d); return s; };
    auto& P = h->P;
    const int B = P.B;
    d->B = B;
    d->format = h->format;
    d->band = P.band_on != 0;
    d->rearr = P.window > 1;
    d->n_global = h->A.n;
    d->n_own = P.n;
    d->n_slices = P.n_slices;
    d->nranks = h->nranks;
    d->rank = h->rank;
    d->comm = comm;
    d->row_begin = h->cuts.empty() ? 0 : h->cuts[h->rank];
    for (int64_t c : h->cuts) d->cuts.push_back(c * B);
    if (h->nranks > 1) {
        d->nx = h->span[2 * h->rank + 1] - h->span[2 * h->rank];
        d->own_off = d->row_begin - h->span[2 * h->rank];
    } else {
        d->nx = d->n_own;
        d->own_off = 0;
    }
    if (halo) {  // rows -> doubles
        d->halo = *halo;
        for (auto& v : d->halo.send_off) v *= B;
        for (auto& v : d->halo.send_cnt) v *= B;
        for (auto& v : d->halo.recv_off) v *= B;
        for (auto& v : d->halo.recv_cnt) v *= B;
    }
    cme_status s;
#define UP(field, vec) \
    if ((s = d->upload(d->field, vec)) != CME_OK) return fail(s);
    if (d->format == CME_FMT_CSR) {
        UP(csr_rp, P.csr_rp);
        UP(csr_ci, P.csr_ci);
        UP(csr_v, P.csr_v);
        UP(inv_d, P.inv_d);
    } else {
        UP(slice_off, P.slice_off);
        UP(slice_w, P.slice_w);
        UP(inv_d, P.inv_d);
    }
    {
        std::vector<int32_t> po(h->perm.begin() + d->row_begin, h->perm.begin() + d->row_begin + d->n_own);
        UP(perm_own, po);
        if (comm) UP(perm_global, h->perm);
    }
    for (int b = 0; b < 2; ++b) {
        double* base = nullptr;
        const size_t len = (size_t)(d->nx + 2) * B;
        if ((s = d->alloc(base, len)) != CME_OK) return fail(s);
        if (cudaMemset(base, 0, len * sizeof(double)) != cudaSuccess) return fail(CME_ERR_CUDA);
        d->xb[b] = base + B;
    }
    d->grid = d->format == CME_FMT_CSR ? (int)((d->n_own + kCta - 1) / kCta)
                                       : (int)((d->n_slices + kWarpsPerCta - 1) / kWarpsPerCta);
    d->grid = std::max(d->grid, 1);
    if (d->format != CME_FMT_CSR && (s = configure_tma(*d, P)) != CME_OK) return fail(s);
    // compact encoding when the TMA kernel streams a single matrix
    // (CME_COMPACT = 0 keeps layout v0 on the TMA kernel too)
    h->Cpt = Compact();
    // (tried even when layout v0's stages were too wide for a TMA shape: the
    // compact and value-indexed stages are 2.5-3x smaller)
    std::vector<int2> xwp;   // x-window chunk plan (sec. 5f), uploaded with the records
    const bool v0_tma = d->use_tma;
    const int v0_warps = v0_tma ? d->tma_ncw * d->tma_spw * d->tma_occ : 0;
    if (d->B == 1 && d->format == CME_FMT_DIAG_SELL && env_int("CME_COMPACT", 1) != 0 && env_int("CME_TMA", -1) != 0 &&
        encode_compact(P, d->own_off, h->Cpt)) {
        d->cpt = true;
        d->win_shift = h->Cpt.win_shift;
        // value-indexed (sec. 5c) when the dictionary fits next to a ring with
        // as many resident consumer warps (CME_VI = -1 auto / 0 off / 1 force)
        if ((s = configure_tma(*d, P)) != CME_OK) return fail(s);   // compact stage geometry
        // the warps the value index must match: the compact shape's, else layout v0's
        const int cpt_warps = d->use_tma ? d->tma_ncw * d->tma_spw * d->tma_occ : v0_warps;
        const int want_vi = env_int("CME_VI", -1);
        if (want_vi != 0 && encode_value_index(P, h->Cpt)) {
            d->vi = true;
            d->dict_bytes = (int)((h->Cpt.dict.size() * 8 + 127) / 128 * 128);
            if ((s = configure_tma(*d, P)) != CME_OK) return fail(s);
            // auto: only if the dictionary costs at most one resident consumer
            // warp -- a dictionary too large for two copies per SM runs on the
            // 31-warp single-dictionary CTA (100M-state toggle, 14.1K distinct
            // rates, 113 KB: 949 us per iteration vs 1 242 us on the compact
            // encoding with 2 x 16 warps)
            if (!d->use_tma || (want_vi < 0 && d->tma_ncw * d->tma_spw * d->tma_occ < cpt_warps - 1)) {
                d->vi = false;
                d->dict_bytes = 0;
                if ((s = configure_tma(*d, P)) != CME_OK) return fail(s);
            }
        }
        if (!d->use_tma) {   // no TMA shape for the compact encoding: back to layout v0
            d->cpt = d->vi = false;
            d->dict_bytes = 0;
            h->Cpt = Compact();
            if (v0_tma && (s = configure_tma(*d, P)) != CME_OK) return fail(s);
        }
        // the value-indexed encoding as tile records (sec. 5d)
        if (d->use_tma && d->vi && (s = configure_vi2(*d, P)) != CME_OK) return fail(s);
        // the f64 compact encoding as tile records too (CME_REC = 1; measured
        // mixed, so opt-in: cfg3a 18.7 us (16 warps) vs 19.1 on sell_cpt_kernel,
        // config 5 (w = 1024) 419 us vs 407)
        if (d->use_tma && d->cpt && !d->vi && env_int("CME_REC", 0) != 0 && (s = configure_vi2(*d, P, true)) != CME_OK)
            return fail(s);
        // the x window in shared memory (sec. 5f) for narrow bands
        if (d->use_tma && d->cpt && !comm && h->nranks == 1 && (s = configure_xw(*d, P, !d->vi, xwp)) != CME_OK)
            return fail(s);
    }
    if (d->B > 1 && d->format == CME_FMT_DIAG_SELL && env_int("CME_COMPACT", 1) != 0 && env_int("CME_VI", -1) != 0 &&
        env_int("CME_TMA", -1) != 0 && encode_compact(P, d->own_off, h->Cpt) && encode_value_index(P, h->Cpt)) {
        // a batch whose entries' rate tuples have a value index: the batched
        // value-indexed kernel (shared indices, tuple dictionary in L2)
        const bool was_tma = d->use_tma;
        d->cpt = d->vi = true;
        d->win_shift = h->Cpt.win_shift;
        d->dict_bytes = 0;   // read from global memory, not staged in shared memory
        if ((s = configure_tma(*d, P)) != CME_OK) return fail(s);
        if (!d->use_tma) {   // no TMA shape: back to layout v0
            d->cpt = d->vi = false;
            h->Cpt = Compact();
            if (was_tma && (s = configure_tma(*d, P)) != CME_OK) return fail(s);
        }
        // the batch's tile records (single GPU)
        if (d->use_tma && d->vi && !comm && h->nranks == 1 && (s = configure_vi2b(*d, P, (int64_t)h->Cpt.dict.size())) != CME_OK)
            return fail(s);
    }
    if ((s = configure_resident(*d, P, comm != nullptr || h->nranks > 1)) != CME_OK) return fail(s);
    if ((s = preload_kernels(B)) != CME_OK) return fail(s);
    if (d->use_tma) {
        const int ts = d->tma_ncw * d->tma_spw;   // slices per tile
        const int ms = meta_stride(ts);   // per-tile records, 16-byte aligned
        std::vector<int2> tm((size_t)d->n_tiles * ms, make_int2(0, 0));   // whole tiles (TMA copies)
        for (int64_t q = 0; q < P.n_slices; ++q)
            tm[q / ts * ms + q % ts] = make_int2((int)(P.slice_off[q] - P.slice_off[q / ts * ts]), P.slice_w[q]);
        if ((s = d->upload(d->tile_meta, tm)) != CME_OK) return fail(s);
    }
    if (d->format != CME_FMT_CSR) {
        if (d->vi2) {   // tile records + the dictionary; no separate index arrays
            if (!d->vi2_f64) {
                std::vector<double> dict(h->Cpt.dict);
                dict.resize(d->dict_bytes / 8, 0.0);   // staged in shared memory, 128-B padded
                UP(dict, dict);
            }
            if (d->xw) UP(xw_ch, xwp);
            std::vector<unsigned char> rec;
            std::vector<int64_t> roff;
            vi2_build_records(P, h->Cpt, d->vi2_ncw, d->band, d->rearr, d->vi2_words, rec, roff, d->vi2_f64);
            UP(vi2_rec, rec);
            UP(vi2_rec_off, roff);
            // wavefront s-step passes (CME_WF = s; single GPU, same grid as
            // the vi2 kernel so the check partials keep their layout)
            const int wf_s = env_int("CME_WF", 0);
            if (wf_s >= 2 && wf_s <= 8 && !comm && h->nranks == 1 && !d->xw && (d->vi2_ncw == 30 || d->vi2_ncw == 16) &&
                !d->vi2_words && !d->vi2_f64 && d->vi2_tiles < (1 << 24)) {
                const int smem = d->dict_bytes + d->vi2_stages * d->vi2_stage_bytes;
                int occ = 0;
                if (wf_prepare(d->vi2_ncw, smem) == cudaSuccess &&
                    wf_occupancy(d->vi2_ncw, smem, &occ) == cudaSuccess && occ >= d->vi2_occ) {
                    std::vector<int2> dep;
                    std::vector<uint32_t> items;
                    const int extra = env_int("CME_WF_LAG", (d->vi2_stages + 2) * d->vi2_grid / wf_s);
                    d->wf_lag = wf_plan(P, d->vi2_ncw, d->band, wf_s, extra, dep, items);
                    UP(wf_dep, dep);
                    UP(wf_items, items);
                    if ((s = d->alloc(d->wf_cnt, (size_t)d->vi2_tiles)) != CME_OK) return fail(s);
                    if ((s = d->alloc(d->wf_sync, 2)) != CME_OK) return fail(s);
                    if (cudaMemset(d->wf_cnt, 0, d->vi2_tiles * 4) != cudaSuccess ||
                        cudaMemset(d->wf_sync, 0, 8) != cudaSuccess)
                        return fail(CME_ERR_CUDA);
                    d->wf = true;
                    d->wf_s = wf_s;
                    d->wf_keep = env_int("CME_WF_KEEP", 1);
                    if (env_int("CME_VERBOSE", 0))
                        std::fprintf(stderr, "[cme] wavefront: s=%d lag=%d tiles=%lld items=%zu\n", wf_s, d->wf_lag,
                                     (long long)d->vi2_tiles, items.size());
                }
            }
        } else if (d->vi2b) {   // batched tile records + the tuple dictionary (L1, or staged: 128-B padded)
            std::vector<double> dict(h->Cpt.dict);
            if (d->vi2b_dict_bytes > 0) dict.resize(d->vi2b_dict_bytes / 8, 0.0);
            UP(dict, dict);
            std::vector<unsigned char> rec;
            std::vector<int64_t> roff;
            vi2b_build_records(P, h->Cpt, d->vi2_ncw, d->B, d->band, d->rearr, rec, roff);
            UP(vi2_rec, rec);
            UP(vi2_rec_off, roff);
        } else if (d->vi) {
            std::vector<double> dict(h->Cpt.dict);
            if (d->B == 1) dict.resize(d->dict_bytes / 8, 0.0);   // (B = 1: staged in shared memory, 128-B padded)
            UP(dict, dict);
            UP(vidx, h->Cpt.vidx);
            UP(col16, h->Cpt.col16);
            if (d->band) { UP(loi, h->Cpt.loi); UP(upi, h->Cpt.upi); }
            if (d->rearr) UP(row8, h->Cpt.row8);
        } else if (d->cpt) {
            UP(cval, h->Cpt.val);
            UP(col16, h->Cpt.col16);
            if (d->band) { UP(clo, h->Cpt.lo); UP(cup, h->Cpt.up); }
            if (d->rearr) UP(row8, h->Cpt.row8);
        }
        if (!d->cpt || d->use_res) {   // layout v0 arrays (register / resident kernels)
            UP(val, P.val);
            UP(col, P.col);
            if (d->band) { UP(lo, P.lo); UP(up, P.up); }
            if (d->rearr) UP(row_of, P.row_of);
        }
    }
#undef UP
    d->part_blocks = std::max(std::max(std::max(d->grid, d->res_grid), grid_for(d->n_own)), d->step_grid());
    if ((s = d->alloc(d->partials, (size_t)d->part_blocks * B * kPartials)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->gather, (size_t)d->nranks * B * 8)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->local8, (size_t)B * 8)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->io, (size_t)d->n_global * B)) != CME_OK) return fail(s);
    if (comm && (s = d->alloc(d->io2, (size_t)d->n_global * B)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->one, kMaxBatch)) != CME_OK) return fail(s);
    if (comm && B == 1) {
        // transient accumulator up front for a rank group: allocating it lazily
        // inside cme_transient could wait on a peer's spinning barrier kernel
        // (reproduced: 4 virtual ranks, register kernel, barrier time-outs)
        if ((s = d->alloc(d->acc_base, (size_t)(d->nx + 2))) != CME_OK) return fail(s);
        d->accb = d->acc_base + 1;
    }
    d->p2p = comm && transport_is_peer(comm_transport(comm));
    if (d->p2p) {
        // [0, P) step/exchange barrier epochs, [P, 2P) halo rows pushed into me
        // by rank q (steps), [2P, 3P) halo reads finished by rank p (fused sync)
        if ((s = d->alloc(d->flags, (size_t)3 * d->nranks)) != CME_OK) return fail(s);
        if ((s = d->alloc(d->hsync, 4)) != CME_OK) return fail(s);
        if (cudaMemset(d->hsync, 0, 4 * sizeof(int64_t)) != cudaSuccess) return fail(CME_ERR_CUDA);
        if ((s = d->alloc(d->epoch, 1)) != CME_OK) return fail(s);
        if (cudaMemset(d->flags, 0, 3 * d->nranks * sizeof(int64_t)) != cudaSuccess ||
            cudaMemset(d->epoch, 0, sizeof(int64_t)) != cudaSuccess)
            return fail(CME_ERR_CUDA);
    }
    if ((s = d->alloc(d->ctrl, 1)) != CME_OK) return fail(s);
    const double ones[kMaxBatch] = {1, 1, 1, 1, 1, 1, 1, 1};
    if (cudaMemcpy(d->one, ones, sizeof(ones), cudaMemcpyHostToDevice) != cudaSuccess) return fail(CME_ERR_CUDA);
    if (cudaMemset(d->ctrl, 0, sizeof(Ctrl)) != cudaSuccess) return fail(CME_ERR_CUDA);
    if (cudaMallocHost(&d->ctrl_host, 2 * sizeof(Ctrl)) != cudaSuccess) return fail(CME_ERR_OOM);
    if (cudaStreamCreateWithFlags(&d->own, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&d->cap, cudaStreamNonBlocking) != cudaSuccess)
        return fail(CME_ERR_CUDA);
    for (auto& e : d->ev)
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return fail(CME_ERR_CUDA);
    if (cudaEventCreate(&d->t0) != cudaSuccess || cudaEventCreate(&d->t1) != cudaSuccess) return fail(CME_ERR_CUDA);
    if (cudaDeviceSynchronize() != cudaSuccess) return fail(CME_ERR_CUDA);
    device_free(h->dev);
    h->dev = d;
    return CME_OK;
}


// ------------------------------------------------------------------------------
// exchanges of the row-sharded solve: NCCL (grouped send/recv, allgather,
// broadcast) or the peer-memory transport (direct stores + flag barriers)
// ------------------------------------------------------------------------------
// neighbours_only: the per-step barrier, which only has to order the halo
// stores -- RAW with the ranks that push rows to me, WAR with the ranks I push
// rows to -- so it publishes to and waits for those ranks only (under RCM the
// two row-range neighbours).  Every other exchange (check records, load, output
// segments) is a barrier over all ranks.  One epoch counter serves both: every
// rank runs the same sequence of barriers, so at a full barrier every rank
// publishes the same epoch to everyone, and a flag left behind by skipped
// step barriers only ever lags (the waits compare with >=).
static cme_status p2p_barrier(Device& d, cudaStream_t s, bool respect_stop, bool neighbours_only = false) {
    if (d.npeer == 0) return CME_OK;   // a group of one
    BarrierArgs b{};
    b.flags = d.flags;
    b.epoch = d.epoch;
    b.npeer = 0;
    for (int p = 0; p < d.npeer; ++p) {
        if (neighbours_only && !d.peer_nbr[p]) continue;
        b.peer_flags[b.npeer] = d.peer_flags[p];
        b.peer_rank[b.npeer] = d.peer_rank[p];
        ++b.npeer;
    }
    b.rank = d.rank;
    b.stop = respect_stop ? &d.ctrl->stop : nullptr;
    b.ctrl = d.ctrl;
    b.early = d.bar_pdl ? 1 : 0;
    CUDA_TRY(launch_ex(p2p_barrier_kernel, dim3(1), dim3(32), 0, d.bar_pdl, s, b));
    return CME_OK;
}

// after a step wrote buffer `dst`: halo exchange (NCCL) / step barrier (P2P;
// the halo rows were already stored into the peers by the step kernel)
static cme_status exch_after_step(Device& d, int dst, cudaStream_t s) {
    if (!d.comm || d.fused) return CME_OK;   // fused: the step kernel ordered the halo itself
    if (d.p2p) return p2p_barrier(d, s, true, d.nbr_barrier);
    return comm_halo(d.comm, d.halo, d.xb[dst], s);
}

// every rank's [B][8] check record (local8) into gather[rank] on all ranks
static cme_status exch_records(Device& d, cudaStream_t s, bool respect_stop) {
    if (!d.comm) return CME_OK;
    const size_t cnt = (size_t)8 * d.B;
    if (!d.p2p) return comm_allgather(d.comm, d.local8, d.gather, cnt, s);
    CopyArgs c{};
    c.src = d.local8;
    c.dst[0] = d.gather + (size_t)d.rank * cnt;
    for (int p = 0; p < d.npeer; ++p) c.dst[p + 1] = d.peer_gather[p] + (size_t)d.rank * cnt;
    c.ndst = d.npeer + 1;
    c.count = (int64_t)cnt;
    c.stop = respect_stop ? &d.ctrl->stop : nullptr;
    multicast_copy_kernel<<<1, 64, 0, s>>>(c);
    CUDA_TRY(cudaGetLastError());
    return p2p_barrier(d, s, respect_stop);
}

// fill the halo of buffer `buf` from the peers' own rows (load time)
static cme_status exch_halo_full(Device& d, int buf, cudaStream_t s) {
    if (!d.comm) return CME_OK;
    if (!d.p2p) return comm_halo(d.comm, d.halo, d.xb[buf], s);
    const double* own = d.xb[buf] + d.own_off * d.B;
    for (int p = 0; p < d.npush; ++p) {
        CopyArgs c{};
        c.src = own + d.push_lo[p] * d.B;
        c.dst[0] = d.push_y[buf][p] + d.push_lo[p] * d.B;
        c.ndst = 1;
        c.count = (d.push_hi[p] - d.push_lo[p]) * d.B;
        multicast_copy_kernel<<<64, 256, 0, s>>>(c);
        CUDA_TRY(cudaGetLastError());
    }
    return p2p_barrier(d, s, false);
}

// every rank's own segment of the reordered staging vector io to all ranks
static cme_status exch_segments(Device& d, cudaStream_t s) {
    if (!d.p2p) return comm_bcast_segments(d.comm, d.io, d.cuts, s);
    CopyArgs c{};
    const int64_t off = d.cuts[d.rank];
    c.src = d.io + off;
    for (int p = 0; p < d.npeer; ++p) c.dst[p] = d.peer_io[p] + off;
    c.ndst = d.npeer;
    c.count = d.cuts[d.rank + 1] - off;
    if (c.ndst) {
        multicast_copy_kernel<<<grid_for(c.count), kCta, 0, s>>>(c);
        CUDA_TRY(cudaGetLastError());
    }
    return p2p_barrier(d, s, false);
}

// Fused halo sync plan (kernels_vi2.cuh HaloSync): per tile of the record
// kernel, does it gather rows outside this rank's own rows (halo) and does it
// hold rows some peer needs (push); the peers' flag words; and, when ranks
// share a GPU (virtual ranks), a grid cap so every rank's step kernel can be
// resident at once (a spinning gate needs its peer's tiles to run).
static cme_status hs_plan(cme_matrix_s* h, const std::vector<P2PRank>& all, int on_gpu) {
    Device& d = *h->dev;
    const Packed& P = h->P;
    const int ncw = d.vi2_ncw;
    const int64_t T = d.vi2_tiles, n = P.n;
    std::vector<uint8_t> kind(T, 0);
    for (int64_t t = 0; t < T; ++t)
        for (int64_t q = t * ncw; q < std::min<int64_t>((t + 1) * ncw, P.n_slices); ++q)
            for (int lane = 0; lane < 32; ++lane) {
                const int64_t slot = q * 32 + lane;
                if (slot >= n) continue;
                const int64_t r = P.row_of[slot];   // local row; x-span index own_off + r
                for (int p = 0; p < d.npush; ++p)
                    if (r >= d.push_lo[p] && r < d.push_hi[p]) kind[t] |= 2;
                auto halo = [&](int64_t xs) { return xs < d.own_off || xs >= d.own_off + n; };
                if (d.band && (halo(d.own_off + r - 1) || halo(d.own_off + r + 1))) kind[t] |= 1;
                for (int w = 0; w < P.slice_w[q]; ++w)
                    if (halo(P.col[P.slice_off[q] + lane + 32 * w])) kind[t] |= 1;
            }
    int64_t np = 0, nh = 0;
    for (uint8_t k : kind) { np += (k & 2) != 0; nh += (k & 1) != 0; }
    if (d.tile_kind == nullptr) CME_TRY(d.alloc(d.tile_kind, (size_t)T));
    CUDA_TRY(cudaMemcpy(d.tile_kind, kind.data(), T, cudaMemcpyHostToDevice));
    d.hs_push_warps = np * ncw;
    d.hs_halo_warps = nh * ncw;
    const HaloPlan& hp = h->halo;
    d.hs_nsend = d.hs_nrecv = 0;
    for (int sp : hp.send_peer) {
        d.hs_send_rank[d.hs_nsend] = sp;
        d.hs_peer_pushed[d.hs_nsend++] = all[sp].flags + d.nranks + d.rank;
    }
    for (int rq : hp.recv_peer) {
        d.hs_recv_rank[d.hs_nrecv] = rq;
        d.hs_peer_consumed[d.hs_nrecv++] = all[rq].flags + 2 * d.nranks + d.rank;
    }
    if (on_gpu > 1) {   // co-residency of the ranks sharing this GPU
        int dev = 0, sms = 0;
        CUDA_TRY(cudaGetDevice(&dev));
        CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        d.vi2_grid = std::max(1, std::min(d.vi2_grid, sms * d.vi2_occ / on_gpu));
    }
    if (env_int("CME_VERBOSE", 0))
        std::fprintf(stderr, "[cme] rank %d fused halo sync: %lld push / %lld halo tiles of %lld, %d send / %d recv peers, grid %d\n",
                     d.rank, (long long)np, (long long)nh, (long long)T, d.hs_nsend, d.hs_nrecv, d.vi2_grid);
    return CME_OK;
}

// Peer-memory transport: given every rank's published buffers, derive the
// peers' flag/gather/io pointers and, for every peer that needs some of my
// rows, where in its x-span they go.
static void p2p_wire(cme_matrix_s* h, const std::vector<P2PRank>& all) {
    Device& d = *h->dev;
    d.npeer = 0;
    for (int r = 0; r < d.nranks; ++r) {
        if (r == d.rank) continue;
        d.peer_rank[d.npeer] = r;
        d.peer_flags[d.npeer] = all[r].flags;
        d.peer_gather[d.npeer] = all[r].gather;
        d.peer_io[d.npeer] = all[r].io;
        const HaloPlan& hp = h->halo;   // halo neighbours: I push rows to r, or r pushes rows to me
        d.peer_nbr[d.npeer] = std::find(hp.send_peer.begin(), hp.send_peer.end(), r) != hp.send_peer.end() ||
                              std::find(hp.recv_peer.begin(), hp.recv_peer.end(), r) != hp.recv_peer.end();
        ++d.npeer;
    }
    // CME_P2P_NBR = 0 restores the all-rank step barrier (A/B, tests)
    d.nbr_barrier = env_int("CME_P2P_NBR", 1) != 0;
    const HaloPlan& hp = h->halo;   // rows (not scaled by B)
    d.npush = 0;
    for (size_t i = 0; i < hp.send_peer.size(); ++i) {
        const int sp = hp.send_peer[i];
        const int64_t lo_local = hp.send_off[i] - d.own_off;   // x-span offset -> own local row
        d.push_lo[d.npush] = lo_local;
        d.push_hi[d.npush] = lo_local + hp.send_cnt[i];
        const int64_t shift = (d.row_begin - all[sp].span_lo) * d.B;   // my local row 0 in peer's x-span
        for (int b = 0; b < 2; ++b) d.push_y[b][d.npush] = all[sp].xb[b] + shift;
        ++d.npush;
    }
    // the step barrier may let the next step's CTAs launch early (PDL) only
    // when no peer shares this GPU: early-resident persistent CTAs would keep
    // a same-GPU peer's step off the SMs while the barrier waits for it
    d.bar_pdl = env_int("CME_PDL", 1) != 0;
    int on_gpu = 0;
    for (int r = 0; r < d.nranks; ++r)
        if (std::memcmp(all[r].uuid, all[d.rank].uuid, 16) == 0) ++on_gpu;
    d.same_gpu_peers = on_gpu > 1;
    if (d.same_gpu_peers) d.bar_pdl = false;
    // fused in-kernel halo sync when every rank runs the tile-record kernel
    bool all_ok = d.nranks > 1;
    for (int r = 0; r < d.nranks; ++r) all_ok = all_ok && all[r].fused_ok;
    d.fused = all_ok && hs_plan(h, all, on_gpu) == CME_OK;
    d.peers_ready = true;
}

static P2PRank p2p_mine(cme_matrix_s* h) {
    Device& d = *h->dev;
    P2PRank mine;
    mine.fused_ok = d.vi2 && d.B == 1 && !d.vi2_words && env_int("CME_P2P_FUSED", 1) != 0 ? 1 : 0;
    mine.xb[0] = d.xb[0];
    mine.xb[1] = d.xb[1];
    mine.flags = d.flags;
    mine.gather = d.gather;
    mine.io = d.io;
    mine.span_lo = h->span[2 * h->rank];
    mine.device = d.dev;
    cudaDeviceProp pr;
    if (cudaGetDeviceProperties(&pr, d.dev) == cudaSuccess) std::memcpy(mine.uuid, &pr.uuid, 16);
    return mine;
}

// In-process group (cme_comm_init_local): exchange through the group object.
cme_status device_p2p_setup(cme_matrix_s* h) {
    Device& d = *h->dev;
    if (!d.p2p || comm_transport(d.comm) != kTransportP2P) return CME_OK;
    std::vector<P2PRank> all;
    CME_TRY(comm_p2p_exchange(d.comm, p2p_mine(h), all));
    p2p_wire(h, all);
    return CME_OK;
}

// Multi-process group (cme_comm_init_ipc): this rank's buffers as CUDA IPC
// handles + offsets (allocation bases are exported; the x-span pointers sit
// one sentinel row past them).
struct IpcBlob {
    uint64_t magic;
    int32_t rank, device;
    int64_t span_lo;
    cudaIpcMemHandle_t h[5];   // xb[0] base, xb[1] base, flags, gather, io
    int64_t off[5];            // byte offset of the published pointer in its allocation
    unsigned char uuid[16];    // the exporting process's physical GPU
    int32_t fused_ok;          // P2PRank::fused_ok
};
static_assert(sizeof(IpcBlob) <= CME_IPC_BLOB_BYTES, "IPC blob too large");
constexpr uint64_t kIpcMagic = 0x434d45495043ull;   // "CMEIPC"

cme_status device_ipc_export(cme_matrix_s* h, uint8_t* out) {
    Device& d = *h->dev;
    if (!d.p2p || comm_transport(d.comm) != kTransportIpc) { set_error("not an IPC-distributed handle"); return CME_ERR_BAD_STATE; }
    CUDA_TRY(cudaSetDevice(d.dev));
    IpcBlob b{};
    b.magic = kIpcMagic;
    b.rank = d.rank;
    b.device = d.dev;
    b.span_lo = h->span[2 * h->rank];
    {
        const P2PRank me = p2p_mine(h);
        std::memcpy(b.uuid, me.uuid, 16);
        b.fused_ok = me.fused_ok;
    }
    // allocation bases (device_upload): xb[b] sits one sentinel row of B doubles in
    void* bases[5] = {d.xb[0] - d.B, d.xb[1] - d.B, d.flags, d.gather, d.io};
    const int64_t offs[5] = {(int64_t)(d.B * sizeof(double)), (int64_t)(d.B * sizeof(double)), 0, 0, 0};
    for (int i = 0; i < 5; ++i) {
        CUDA_TRY(cudaIpcGetMemHandle(&b.h[i], bases[i]));
        b.off[i] = offs[i];
    }
    std::memset(out, 0, CME_IPC_BLOB_BYTES);
    std::memcpy(out, &b, sizeof(b));
    return CME_OK;
}

cme_status device_ipc_attach(cme_matrix_s* h, const uint8_t* blobs) {
    Device& d = *h->dev;
    if (!d.p2p || comm_transport(d.comm) != kTransportIpc) { set_error("not an IPC-distributed handle"); return CME_ERR_BAD_STATE; }
    CUDA_TRY(cudaSetDevice(d.dev));
    std::vector<P2PRank> all(d.nranks);
    for (int r = 0; r < d.nranks; ++r) {
        IpcBlob b;
        std::memcpy(&b, blobs + (size_t)r * CME_IPC_BLOB_BYTES, sizeof(b));
        if (b.magic != kIpcMagic || b.rank != r) { set_error("bad IPC blob order/content"); return CME_ERR_INVALID_ARG; }
        if (r == d.rank) { all[r] = p2p_mine(h); continue; }
        void* mapped[5];
        for (int i = 0; i < 5; ++i) {
            CUDA_TRY(cudaIpcOpenMemHandle(&mapped[i], b.h[i], cudaIpcMemLazyEnablePeerAccess));
            d.ipc_opened.push_back(mapped[i]);
            mapped[i] = (char*)mapped[i] + b.off[i];
        }
        all[r].xb[0] = (double*)mapped[0];
        all[r].xb[1] = (double*)mapped[1];
        all[r].flags = (int64_t*)mapped[2];
        all[r].gather = (double*)mapped[3];
        all[r].io = (double*)mapped[4];
        all[r].span_lo = b.span_lo;
        all[r].device = b.device;
        std::memcpy(all[r].uuid, b.uuid, 16);
        all[r].fused_ok = b.fused_ok;
    }
    p2p_wire(h, all);
    return CME_OK;
}

// ------------------------------------------------------------------------------
// launches
// ------------------------------------------------------------------------------
static cme_status launch_step(Device& d, cudaStream_t s, int src, int dst, bool check, const double* pre,
                              double omega, double unif_lam_inv = 0.0, double acc_w = 0.0) {
    StepArgs a{};
    a.unif_lam_inv = unif_lam_inv;
    a.acc = unif_lam_inv != 0.0 ? d.accb : nullptr;
    a.acc_w = acc_w;
    a.npush = d.p2p ? d.npush : 0;
    for (int p = 0; p < a.npush; ++p) {
        a.push_lo[p] = d.push_lo[p];
        a.push_hi[p] = d.push_hi[p];
        a.push_y[p] = d.push_y[dst][p];
    }
    a.n_rows = d.n_own;
    a.slice_begin = 0;
    a.slice_end = d.n_slices;
    a.slice_off = d.slice_off;
    a.slice_w = d.slice_w;
    a.tile_meta = d.tile_meta;
    a.val = d.val;
    a.col = d.col;
    a.row_of = d.row_of;
    a.lo = d.lo;
    a.up = d.up;
    a.inv_d = d.inv_d;
    a.x = d.xb[src];
    a.y = d.xb[dst];
    a.own_off = d.own_off;
    a.omega = omega;
    a.pre_scale = pre;
    a.partials = d.partials;
    a.stop = &d.ctrl->stop;
    a.csr_rp = d.csr_rp;
    a.csr_ci = d.csr_ci;
    a.csr_v = d.csr_v;
    // programmatic dependent launch between consecutive steps (not across the
    // NCCL calls of a distributed solve, which are ordinary stream work)
    // (not when fused-sync ranks share the GPU: an early-resident next step
    // could hold SMs a peer's current step needs to release a gate)
    const bool pdl = (!d.comm || d.p2p) && env_int("CME_PDL", 1) != 0 && !(d.fused && d.same_gpu_peers);
    if (d.format == CME_FMT_CSR) {
        CUDA_TRY(check ? launch_ex(csr_step_kernel<true>, dim3(d.grid), dim3(kCta), 0, pdl, s, a)
                       : launch_ex(csr_step_kernel<false>, dim3(d.grid), dim3(kCta), 0, pdl, s, a));
    } else if (d.vi2) {
        Vi2Args V{a, d.vi2_rec, d.vi2_rec_off, d.dict, d.vi2_tiles, d.vi2_stages, d.vi2_stage_bytes, d.dict_bytes,
                  d.win_shift, d.tma_xpf};
        V.contig = env_int("CME_VI2_CONTIG", 0);
        if (d.fused) {
            HaloSync& hs = V.hs;
            hs.on = 1;
            hs.local = d.hsync;
            hs.pushed = d.flags + d.nranks;
            hs.consumed = d.flags + 2 * d.nranks;
            hs.nsend = d.hs_nsend;
            hs.nrecv = d.hs_nrecv;
            for (int p = 0; p < d.hs_nsend; ++p) { hs.send_rank[p] = d.hs_send_rank[p]; hs.peer_pushed[p] = d.hs_peer_pushed[p]; }
            for (int q = 0; q < d.hs_nrecv; ++q) { hs.recv_rank[q] = d.hs_recv_rank[q]; hs.peer_consumed[q] = d.hs_peer_consumed[q]; }
            hs.tile_kind = d.tile_kind;
            hs.push_warps = d.hs_push_warps;
            hs.halo_warps = d.hs_halo_warps;
            // as long as the barrier kernel's bound: a peer's host thread may be
            // late to launch (8 virtual ranks in one process measured > 2 s)
            hs.timeout_ns = (int64_t)std::max(1, env_int("CME_P2P_TIMEOUT_MS", 30000)) * 1000000;
            hs.ctrl = d.ctrl;
        }
        if (d.xw) {
            V.xw_ch = d.xw_ch;
            V.xw_rows = d.xw_rows;
            V.xw_mirror = d.xw_mirror;
            V.xw_off = d.xw_off;
            V.xw_nx = d.xw_nx;
            V.xpf = 0;
            CUDA_TRY(launch_vi2_xw(V, d.vi2_ncw, d.vi2_grid,
                                   d.dict_bytes + d.vi2_stages * d.vi2_stage_bytes + d.xw_ring_bytes, d.band, d.rearr,
                                   check, d.vi2_f64 ? 2 : 0, d.xw, pdl, s));
        } else
            CUDA_TRY(launch_vi2(V, d.vi2_ncw, d.vi2_grid, d.dict_bytes + d.vi2_stages * d.vi2_stage_bytes, d.band,
                                d.rearr, check, d.vi2_f64 ? 2 : d.vi2_words ? 1 : 0, pdl, s));
    } else if (d.vi2b) {
        Vi2Args V{a, d.vi2_rec, d.vi2_rec_off, d.dict, d.vi2_tiles, d.vi2_stages, d.vi2_stage_bytes,
                  d.vi2b_dict_bytes, d.win_shift, d.tma_xpf};
        CUDA_TRY(launch_vi2b(V, d.B, d.vi2_ncw, d.vi2_grid, d.vi2b_dict_bytes + d.vi2_stages * d.vi2_stage_bytes, d.band,
                             d.rearr, check, pdl, s));
    } else if (d.use_tma && d.vi && d.B > 1) {
        ViArgs V{CptArgs{TmaArgs{a, d.n_tiles, d.tma_stages, d.tma_stage_bytes, d.tma_off_val, d.tma_off_col,
                                 d.tma_contig, d.tma_xpf},
                         d.col16, d.row8, d.win_shift},
                 d.dict, d.vidx, d.loi, d.upi, 0, d.vi_idpf};
        CUDA_TRY(launch_vib(V, d.B, d.tma_ncw, d.tma_grid, d.tma_stages * d.tma_stage_bytes, d.band, d.rearr, check, pdl,
                            s));
    } else if (d.use_tma && d.vi) {
        ViArgs V{CptArgs{TmaArgs{a, d.n_tiles, d.tma_stages, d.tma_stage_bytes, d.tma_off_val, d.tma_off_col,
                                 d.tma_contig, d.tma_xpf},
                         d.col16, d.row8, d.win_shift},
                 d.dict, d.vidx, d.loi, d.upi, d.dict_bytes, d.vi_idpf};
        CUDA_TRY(launch_vi(V, d.tma_ncw, d.tma_grid, d.dict_bytes + d.tma_stages * d.tma_stage_bytes, d.band, d.rearr,
                           check, pdl, s));
    } else if (d.use_tma && d.cpt) {
        a.val = d.cval;
        a.lo = d.clo;
        a.up = d.cup;
        a.col = nullptr;
        a.row_of = nullptr;
        CptArgs K{TmaArgs{a, d.n_tiles, d.tma_stages, d.tma_stage_bytes, d.tma_off_val, d.tma_off_col, d.tma_contig, d.tma_xpf},
                  d.col16, d.row8, d.win_shift};
        CUDA_TRY(launch_cpt(K, d.tma_ncw, d.tma_grid, d.tma_stages * d.tma_stage_bytes, d.band, d.rearr, check, pdl, s));
    } else if (d.use_tma) {
        TmaArgs T{a, d.n_tiles, d.tma_stages, d.tma_stage_bytes, d.tma_off_val, d.tma_off_col, d.tma_contig, d.tma_xpf};
        const int smem = d.tma_stages * d.tma_stage_bytes;
        cudaError_t e;
        switch (d.B) {
            case 1: e = launch_tma<1>(T, d.tma_ncw, d.tma_grid, smem, d.band, d.rearr, check, pdl, s); break;
            case 2: e = launch_tma<2>(T, d.tma_ncw, d.tma_grid, smem, d.band, d.rearr, check, pdl, s); break;
            case 4: e = launch_tma<4>(T, d.tma_ncw, d.tma_grid, smem, d.band, d.rearr, check, pdl, s); break;
            default: e = launch_tma<8>(T, d.tma_ncw, d.tma_grid, smem, d.band, d.rearr, check, pdl, s); break;
        }
        CUDA_TRY(e);
    } else {
        cudaError_t e;
        switch (d.B) {
            case 1: e = launch_sell<1>(a, d.grid, d.band, d.rearr, check, pdl, s); break;
            case 2: e = launch_sell<2>(a, d.grid, d.band, d.rearr, check, pdl, s); break;
            case 4: e = launch_sell<4>(a, d.grid, d.band, d.rearr, check, pdl, s); break;
            default: e = launch_sell<8>(a, d.grid, d.band, d.rearr, check, pdl, s); break;
        }
        CUDA_TRY(e);
    }
    return exch_after_step(d, dst, s);
}

// nsteps Jacobi steps from buffer `start` in SMEM-resident launches (chunks of
// 2^20 check blocks, so the 32-bit grid-barrier counters cannot wrap); solve:
// the last step closes a partial check block (max_iter).  Stops early when a
// check decides (ctrl.stop).
static cme_status launch_res(Device& d, cudaStream_t s, int start, int64_t nsteps, bool solve, int64_t C,
                             double omega) {
    const int64_t chunk = C >= (int64_t(1) << 40) ? std::max<int64_t>(nsteps, 1) : (int64_t(1) << 20) * C;
    for (int64_t done = 0; done < nsteps;) {
        const int64_t len = std::min(chunk, nsteps - done);
        CUDA_TRY(cudaMemsetAsync(d.res_sync, 0, 4 * sizeof(uint32_t), s));
        ResArgs a{};
        a.n_rows = d.n_own;
        a.slice_off = d.slice_off;
        a.slice_w = d.slice_w;
        a.val = d.val;
        a.col = d.col;
        a.row_of = d.row_of;
        a.lo = d.lo;
        a.up = d.up;
        a.inv_d = d.inv_d;
        a.xb0 = d.xb[0];
        a.xb1 = d.xb[1];
        a.cta_q = d.res_q;
        a.cta_row = d.res_row;
        a.probe_off = d.res_probe_off;
        a.probe = d.res_probe;
        a.sync = d.res_sync;
        a.partials = d.partials;
        a.ctrl = d.ctrl;
        a.nsteps = len;
        a.C = C;
        a.omega = omega;
        a.start = (int)((start + done) & 1);
        a.solve = solve && done + len == nsteps ? 1 : 0;
        a.timeout_ns = d.res_timeout_ns;
        CUDA_TRY(launch_resident(a, d.res_grid, d.res_smem, d.band, d.rearr, d.res_rps, s));
        done += len;
        if (done < nsteps) {   // a later chunk only if no check stopped the solve
            int32_t stop = 0;
            CUDA_TRY(cudaMemcpyAsync(&stop, &d.ctrl->stop, sizeof(stop), cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaStreamSynchronize(s));
            if (stop) break;
        }
    }
    return CME_OK;
}

// s = d.wf_s consecutive steps from buffer src in one wavefront launch; the
// result lands in buffer (src + s) & 1 like s single steps.
static cme_status launch_wf_pass(Device& d, cudaStream_t s, int src, bool check, const double* pre, double omega) {
    StepArgs a{};
    a.n_rows = d.n_own;
    a.slice_begin = 0;
    a.slice_end = d.n_slices;
    a.x = d.xb[src];
    a.y = d.xb[1 - src];
    a.own_off = d.own_off;
    a.omega = omega;
    a.pre_scale = pre;
    a.partials = d.partials;
    a.stop = &d.ctrl->stop;
    WfArgs A{Vi2Args{a, d.vi2_rec, d.vi2_rec_off, d.dict, d.vi2_tiles, d.vi2_stages, d.vi2_stage_bytes, d.dict_bytes,
                     d.win_shift, d.tma_xpf},
             d.wf_items, d.wf_dep, d.wf_cnt, d.wf_sync, d.ctrl, d.wf_s, d.wf_keep,
             (int64_t)std::max(1, env_int("CME_RES_TIMEOUT_MS", 2000)) * 1000000};
    const bool pdl = env_int("CME_PDL", 1) != 0;
    CUDA_TRY(launch_wf(A, d.vi2_ncw, d.vi2_grid, d.dict_bytes + d.vi2_stages * d.vi2_stage_bytes, d.band, d.rearr,
                       check, pdl, s));
    return CME_OK;
}

// reduce partials of the last CHECK step and decide
static cme_status launch_finalize(Device& d, cudaStream_t s, int32_t len, int32_t final_partial) {
    const bool pdl = (!d.comm || d.p2p) && env_int("CME_PDL", 1) != 0;
    CUDA_TRY(launch_ex(reduce_partials_kernel, dim3(1), dim3(1024), 0, pdl, s, (const double*)d.partials,
                       d.step_grid(), d.B, d.comm ? d.local8 : d.gather, (const int32_t*)&d.ctrl->stop));
    CME_TRY(exch_records(d, s, true));
    CUDA_TRY(launch_ex(decide_kernel, dim3(1), dim3(1), 0, pdl, s, (const double*)d.gather, d.nranks, d.ctrl, len,
                       final_partial));
    return CME_OK;
}

// One check block of C steps starting from buffer `start`: steps 0..C-2 plain,
// step C-1 CHECK; the first step applies the pending 1/||y_b||_1 (R5).
static cme_status enqueue_block(Device& d, cudaStream_t s, int start, int64_t C, double omega, bool final_partial) {
    int64_t t0 = 0;
    if (d.wf)   // wavefront passes of s steps, single steps for the remainder
        for (; t0 + d.wf_s <= C; t0 += d.wf_s)
            CME_TRY(launch_wf_pass(d, s, (int)((start + t0) & 1), t0 + d.wf_s == C, t0 == 0 ? d.ctrl->inv_s : nullptr,
                                   omega));
    for (int64_t t = t0; t < C; ++t) {
        const int src = (int)((start + t) & 1);
        CME_TRY(launch_step(d, s, src, 1 - src, t == C - 1, t == 0 ? d.ctrl->inv_s : nullptr, omega));
    }
    return launch_finalize(d, s, (int32_t)C, final_partial ? 1 : 0);
}

static cme_status ensure_graphs(Device& d, int64_t C, double omega, bool* built = nullptr) {
    if (built) *built = false;
    if (d.gC == C && d.gomega == omega && d.gexec[0]) return CME_OK;
    if (built) *built = true;
    if (d.comm && !d.p2p) {
        // NCCL sets up peer connections lazily on first use: do that outside
        // the capture (one throw-away exchange + gather on the private stream)
        CME_TRY(comm_halo(d.comm, d.halo, d.xb[1], d.own));
        CME_TRY(comm_allgather(d.comm, d.local8, d.gather, (size_t)8 * d.B, d.own));
        CUDA_TRY(cudaStreamSynchronize(d.own));
    }
    for (auto& g : d.gexec)
        if (g) { cudaGraphExecDestroy(g); g = nullptr; }
    const int nstart = (C & 1) ? 2 : 1;
    for (int st = 0; st < nstart; ++st) {
        cudaGraph_t g = nullptr;
        CUDA_TRY(cudaStreamBeginCapture(d.cap, cudaStreamCaptureModeThreadLocal));
        cme_status e = enqueue_block(d, d.cap, st, C, omega, false);
        cudaError_t ce = cudaStreamEndCapture(d.cap, &g);
        if (e != CME_OK) { if (g) cudaGraphDestroy(g); return e; }
        if (ce != cudaSuccess) { set_error(cudaGetErrorString(ce)); return CME_ERR_CUDA; }
        ce = cudaGraphInstantiate(&d.gexec[st], g, 0);
        cudaGraphDestroy(g);
        if (ce != cudaSuccess) { set_error(cudaGetErrorString(ce)); return CME_ERR_CUDA; }
    }
    d.gC = C;
    d.gomega = omega;
    return CME_OK;
}

// Build the check-block graphs before any exchange of this call, and in an
// in-process rank group let every rank finish building before any rank
// launches a spinning barrier: graph instantiation/destruction in one rank's
// thread can wait on the device, i.e. on a peer's barrier kernel that waits
// for this rank (observed as sporadic barrier time-outs of the virtual-rank
// tests).  All ranks rebuild at the same calls (same C and omega).
static cme_status prepare_graphs(Device& d, int64_t C, double omega) {
    bool built = false;
    CME_TRY(ensure_graphs(d, C, omega, &built));
    if (built && d.comm && comm_transport(d.comm) == kTransportP2P) comm_p2p_host_barrier(d.comm);
    return CME_OK;
}

static cudaStream_t stream_of(cme_matrix_s* h) {
    return h->sopts.stream ? (cudaStream_t)h->sopts.stream : h->dev->own;
}

static bool is_device_ptr(const void* p) {
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

static Ctrl fresh_ctrl(const cme_matrix_s* h, const Device& d) {
    Ctrl c{};
    c.omega = 1.0; c.tol = -1.0; c.stag_tol = 0.0;
    c.C = 1; c.max_iter = INT64_MAX; c.stop_mode = 0; c.nranks = d.nranks; c.batch = d.B;
    c.iter = 0; c.status = -1; c.stop = 0; c.bad_input = 0;
    for (int b = 0; b < kMaxBatch; ++b) {
        c.norm_inf[b] = b < (int)h->norm_inf.size() ? h->norm_inf[b] : 1.0;
        c.delta[b] = c.delta_prev[b] = c.resid[b] = -1.0;
        c.mass[b] = 1.0;
        c.inv_s[b] = 1.0;
        c.mstatus[b] = -1;
        c.miters[b] = 0;
    }
    return c;
}

// x (own rows) <- p0 / sum(p0) per member (or uniform); halo filled; ctrl reset to free-run.
static cme_status load_iterate(cme_matrix_s* h, const double* p0, bool normalise, cudaStream_t s) {
    Device& d = *h->dev;
    const int B = d.B;
    d.cur = 0;
    double* x = d.xb[0] + d.own_off * B;
    const Ctrl c = fresh_ctrl(h, d);
    CUDA_TRY(cudaMemcpyAsync(d.ctrl, &c, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
    if (d.wf) {   // wavefront completion counters restart with the solve
        CUDA_TRY(cudaMemsetAsync(d.wf_cnt, 0, (size_t)d.vi2_tiles * 4, s));
        CUDA_TRY(cudaMemsetAsync(d.wf_sync, 0, 8, s));
    }
    if (!p0) {
        fill_kernel<<<grid_for(d.n_own * B), kCta, 0, s>>>(x, d.n_own * B, 1.0 / (double)d.n_global);
        CUDA_TRY(cudaGetLastError());
    } else {
        const double* src = p0;
        if (!is_device_ptr(p0)) {
            CUDA_TRY(cudaMemcpyAsync(d.io, p0, (size_t)d.n_global * B * sizeof(double), cudaMemcpyHostToDevice, s));
            src = d.io;
        }
        const int g = grid_for(d.n_own);
        switch (B) {
            case 1: load_kernel<1><<<g, kCta, 0, s>>>(src, d.perm_own, d.n_own, d.n_global, x, d.partials); break;
            case 2: load_kernel<2><<<g, kCta, 0, s>>>(src, d.perm_own, d.n_own, d.n_global, x, d.partials); break;
            case 4: load_kernel<4><<<g, kCta, 0, s>>>(src, d.perm_own, d.n_own, d.n_global, x, d.partials); break;
            default: load_kernel<8><<<g, kCta, 0, s>>>(src, d.perm_own, d.n_own, d.n_global, x, d.partials); break;
        }
        reduce_partials_kernel<<<1, 1024, 0, s>>>(d.partials, g, B, d.comm ? d.local8 : d.gather, nullptr);
        CUDA_TRY(cudaGetLastError());
        CME_TRY(exch_records(d, s, false));
        load_decide_kernel<<<1, 1, 0, s>>>(d.gather, d.nranks, d.ctrl, normalise ? 1 : 0);
        CUDA_TRY(cudaGetLastError());
    }
    if (d.use_res) {   // epoch state of the resident kernel: the other buffer's rows negative
        fill_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(d.xb[1] + d.own_off, d.n_own, -0.0);
        CUDA_TRY(cudaGetLastError());
    }
    return exch_halo_full(d, 0, s);
}

// p_out[b][original order] <- x[cur] * scale[b]
static cme_status write_out(cme_matrix_s* h, double* p_out, const double* scale, cudaStream_t s) {
    Device& d = *h->dev;
    const int B = d.B;
    const size_t bytes = (size_t)d.n_global * B * sizeof(double);
    const double* x = d.xb[d.cur] + d.own_off * B;
    const bool dev_out = is_device_ptr(p_out);
    double* dst = dev_out ? p_out : d.io;
    if (!d.comm) {
        scatter_out_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(x, d.perm_own, d.n_own, B, d.n_global, scale, dst);
        CUDA_TRY(cudaGetLastError());
    } else {
        // own rows -> reordered global staging, broadcast every rank's segment,
        // then un-permute into the caller's buffer (or the second staging buffer)
        scale_copy_kernel<<<grid_for(d.n_own * B), kCta, 0, s>>>(x, d.n_own, B, scale, d.io + d.row_begin * B);
        CUDA_TRY(cudaGetLastError());
        CME_TRY(exch_segments(d, s));
        dst = dev_out ? p_out : d.io2;
        scatter_out_kernel<<<grid_for(d.n_global), kCta, 0, s>>>(d.io, d.perm_global, d.n_global, B, d.n_global,
                                                                 d.one, dst);
        CUDA_TRY(cudaGetLastError());
    }
    if (!dev_out) CUDA_TRY(cudaMemcpyAsync(p_out, dst, bytes, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    return CME_OK;
}

static double effective_omega(cme_matrix_s* h) {
    if (h->sopts.omega > 0.0) return h->sopts.omega;
    return h->period == 1 ? 1.0 : 0.9;
}

static void fill_reports(cme_matrix_s* h, const Ctrl& f, double omega, double seconds, int32_t overall) {
    const int B = h->dev->B;
    h->member_reports.assign(B, cme_report{});
    for (int b = 0; b < B; ++b) {
        cme_report& r = h->member_reports[b];
        r.status = f.mstatus[b] == -1 ? overall : f.mstatus[b];
        r.iters = f.mstatus[b] == -1 ? f.iter : f.miters[b];
        r.delta = f.delta[b];
        r.resid = f.resid[b];
        r.mass = f.mass[b];
        r.omega = omega;
        r.seconds = seconds;
    }
    h->report = h->member_reports[0];
    h->report.status = overall;
    h->report.iters = f.iter;
}

static cme_status peers_check(const Device& d) {
    if (d.p2p && !d.peers_ready) { set_error("peer-memory transport: cme_matrix_ipc_attach first"); return CME_ERR_BAD_STATE; }
    return CME_OK;
}

// End of a solve: time, control block, reports, output (P:L125 final L1 scale).
static cme_status solve_epilogue(cme_matrix_s* h, cudaStream_t s, double omega, int64_t max_iter, double* p_out,
                                 int64_t* iters_out) {
    Device& d = *h->dev;
    CUDA_TRY(cudaEventRecord(d.t1, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl_host[0], d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    const Ctrl& f = d.ctrl_host[0];
    d.cur = (int)(f.iter & 1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, d.t0, d.t1);
    if (f.status == CME_ERR_TIMEOUT) {
        set_error(d.use_res ? "resident kernel: a dependency wait timed out (CME_RES_TIMEOUT_MS)"
                  : d.wf    ? "wavefront kernel: a tile dependency wait timed out (CME_RES_TIMEOUT_MS)"
                  : d.fused ? "peer-memory transport: a peer rank never signalled its halo rows (fused sync, "
                              "CME_P2P_TIMEOUT_MS)"
                            : "peer-memory transport: a peer rank never reached the flag barrier");
        if (iters_out) *iters_out = f.iter;
        return CME_ERR_TIMEOUT;
    }
    const int32_t overall = max_iter == 0 ? CME_NOT_CONVERGED : f.status;
    fill_reports(h, f, omega, ms * 1e-3, overall);
    if (iters_out) *iters_out = f.iter;
    CME_TRY(write_out(h, p_out, d.ctrl->inv_s, s));
    return (cme_status)overall;
}

cme_status device_solve(cme_matrix_s* h, const double* p0, double tol, int64_t max_iter, double* p_out,
                        int64_t* iters_out) {
    Device& d = *h->dev;
    CME_TRY(peers_check(d));
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    const int64_t C = h->sopts.check_every;
    const double omega = effective_omega(h);
    if (!d.use_res) CME_TRY(prepare_graphs(d, C, omega));
    CME_TRY(load_iterate(h, p0, true, s));
    // solve parameters (inv_s / mass / bad_input from the load are kept: they
    // live after `bad_input` in Ctrl)
    Ctrl c = fresh_ctrl(h, d);
    c.omega = omega; c.tol = tol; c.stag_tol = h->sopts.stag_tol;
    c.C = C; c.max_iter = max_iter; c.stop_mode = h->sopts.stop;
    CUDA_TRY(cudaMemcpyAsync(d.ctrl, &c, offsetof(Ctrl, bad_input), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->delta, &c.delta, offsetof(Ctrl, mass) - offsetof(Ctrl, delta),
                             cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->mstatus, &c.mstatus, sizeof(Ctrl) - offsetof(Ctrl, mstatus),
                             cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (p0 && d.ctrl_host[0].bad_input) {
        set_error("p0 has a negative/NaN entry or no positive mass");
        return CME_ERR_INVALID_ARG;
    }
    if (d.use_res) {   // one persistent launch runs the whole solve
        CUDA_TRY(cudaEventRecord(d.t0, s));
        CME_TRY(launch_res(d, s, 0, max_iter, true, C, omega));
        return solve_epilogue(h, s, omega, max_iter, p_out, iters_out);
    }
    const int64_t nfull = max_iter / C, rem = max_iter % C;
    CUDA_TRY(cudaEventRecord(d.t0, s));
    int64_t launched = 0, done = 0;
    int start = 0;
    int32_t status = -1;
    while (done < nfull) {
        while (launched < nfull && launched < done + 2) {
            CUDA_TRY(cudaGraphLaunch(d.gexec[start], s));
            CUDA_TRY(cudaMemcpyAsync(&d.ctrl_host[launched & 1], d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaEventRecord(d.ev[launched & 1], s));
            start = (int)((start + C) & 1);
            ++launched;
        }
        CUDA_TRY(cudaEventSynchronize(d.ev[done & 1]));
        status = d.ctrl_host[done & 1].status;
        ++done;
        if (status != -1) break;
    }
    if (status == -1 && rem > 0) CME_TRY(enqueue_block(d, s, start, rem, omega, true));
    return solve_epilogue(h, s, omega, max_iter, p_out, iters_out);
}

// Transient landscape p(t) = exp(A t) p0 by uniformization (R22):
// step k adds w_k x_k to the accumulator and forms x_{k+1} = (I + A/Lambda) x_k
// in the same fused kernel.  Weights: Poisson(mu = Lambda t) on k <= Kmax =
// ceil(mu + 10 sqrt(mu) + 40), normalised to sum 1, right-truncated at the
// first K whose tail mass is <= eps.
cme_status device_transient(cme_matrix_s* h, const double* p0, double t, double eps, double* p_out,
                            int64_t* terms_out) {
    Device& d = *h->dev;
    CME_TRY(peers_check(d));
    if (d.B != 1) { set_error("transient solves take one rate set (batch 1)"); return CME_ERR_INVALID_ARG; }
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    double lam = 0.0;
    for (double v : h->A.d) lam = std::max(lam, -v);
    const double mu = lam * t;
    const int64_t kmax = (int64_t)std::ceil(mu + 10.0 * std::sqrt(mu) + 40.0);
    std::vector<double> w(kmax + 1);
    double lmax = -INFINITY;
    for (int64_t k = 0; k <= kmax; ++k) {
        w[k] = mu > 0.0 ? (double)k * std::log(mu) - std::lgamma((double)k + 1.0) : (k == 0 ? 0.0 : -INFINITY);
        lmax = std::max(lmax, w[k]);
    }
    double W = 0.0;
    for (double& v : w) { v = std::exp(v - lmax); W += v; }
    for (double& v : w) v /= W;
    int64_t K = kmax;
    double tail = 0.0;
    while (K > 0 && tail + w[K] <= eps) { tail += w[K]; --K; }
    if (!d.acc_base) {
        CME_TRY(d.alloc(d.acc_base, (size_t)(d.nx + 2)));
        d.accb = d.acc_base + 1;
    }
    CUDA_TRY(cudaMemsetAsync(d.acc_base, 0, (size_t)(d.nx + 2) * sizeof(double), s));
    if (p0) {
        CME_TRY(load_iterate(h, p0, false, s));
    } else {  // all mass on the initial microstate (original state 0)
        std::vector<double> e0(d.n_global, 0.0);
        e0[0] = 1.0;
        CME_TRY(load_iterate(h, e0.data(), false, s));
    }
    for (int64_t k = 0; k <= K; ++k)
        CME_TRY(launch_step(d, s, (int)(k & 1), (int)((k + 1) & 1), false, nullptr, 1.0, 1.0 / lam, w[k]));
    // p(t) = accumulator (own rows), original order
    const double* xacc = d.accb + d.own_off;
    const bool dev_out = is_device_ptr(p_out);
    double* dst = dev_out ? p_out : d.io;
    if (!d.comm) {
        scatter_out_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(xacc, d.perm_own, d.n_own, 1, d.n_global, d.one, dst);
        CUDA_TRY(cudaGetLastError());
    } else {
        scale_copy_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(xacc, d.n_own, 1, d.one, d.io + d.row_begin);
        CUDA_TRY(cudaGetLastError());
        CME_TRY(exch_segments(d, s));
        dst = dev_out ? p_out : d.io2;
        scatter_out_kernel<<<grid_for(d.n_global), kCta, 0, s>>>(d.io, d.perm_global, d.n_global, 1, d.n_global,
                                                                 d.one, dst);
        CUDA_TRY(cudaGetLastError());
    }
    if (!dev_out) CUDA_TRY(cudaMemcpyAsync(p_out, dst, (size_t)d.n_global * sizeof(double), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    d.cur = (int)((K + 1) & 1);
    if (terms_out) *terms_out = K + 1;
    h->report = cme_report{};
    h->report.status = CME_OK;
    h->report.iters = K + 1;
    h->report.omega = lam;   // the uniformization rate
    return CME_OK;
}

void device_describe(const Device* d, cme_info* f) {
    if (!d) { f->kernel = -1; return; }
    f->kernel = d->format == CME_FMT_CSR ? 2 : d->use_res ? 3 : d->use_tma ? 1 : 0;
    f->tma_warps = d->vi2 || d->vi2b ? d->vi2_ncw : d->use_tma ? d->tma_ncw : 0;
    f->tma_stages = d->vi2 || d->vi2b ? d->vi2_stages : d->use_tma ? d->tma_stages : 0;
    f->records = d->vi2 || d->vi2b ? 1 : 0;
    f->wf_steps = d->wf ? d->wf_s : 0;
    f->halo_fused = d->fused ? 1 : 0;
    f->xwin_kb = d->xw ? d->xw_ring_bytes / 1024 : 0;
    f->wf_lag = d->wf ? d->wf_lag : 0;
    f->grid = d->use_res ? d->res_grid : d->step_grid();
    f->compact = d->vi ? 2 : d->cpt ? 1 : 0;
    if (d->vi) {   // value-indexed: 4 B per ELL slot (shared by a batch), inv_d per row and member
        const int64_t n_ell = f->n_ell, nl = d->n_own, slots = f->n_slots, sl = f->n_slices, nb = d->B;
        f->bytes_fmt = 4 * n_ell + 8 * nb * nl + (d->rearr ? nl : 0) + (d->band ? 4 * nl : 0) + 12 * sl + 16 * nb * nl;
        f->packed_bytes = 4 * n_ell + 8 * nb * slots + (d->rearr ? slots : 0) + (d->band ? 4 * slots : 0) + 12 * sl + 8 +
                          d->dict_bytes + (d->use_res ? f->packed_bytes : 0);
    } else if (d->cpt) {   // bytes a plain step streams in the compact encoding (no inv_d)
        const int64_t n_ell = f->n_ell, nl = d->n_own, slots = f->n_slots, sl = f->n_slices;
        f->bytes_fmt = 10 * n_ell + (d->rearr ? nl : 0) + (d->band ? 16 * nl : 0) + 12 * sl + 16 * nl;
        f->packed_bytes = 10 * n_ell + (d->rearr ? slots : 0) + (d->band ? 16 * slots : 0) + 8 * slots + 12 * sl + 8 +
                          (d->use_res ? f->packed_bytes : 0);
    }
}

cme_status device_spmv(cme_matrix_s* h, const double* x, double* y) {
    Device& d = *h->dev;
    CME_TRY(peers_check(d));
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    CME_TRY(load_iterate(h, x, false, s));
    // always a plain step kernel: the SMEM-resident kernel carries its epoch in
    // the iterate's sign bit and so needs x >= +0, while y = M_omega x is
    // defined for any x (layout v0 is uploaded whenever the resident kernel is)
    CME_TRY(launch_step(d, s, 0, 1, false, nullptr, effective_omega(h)));
    d.cur = 1;
    return write_out(h, y, d.one, s);
}

cme_status device_load(cme_matrix_s* h, const double* p0) {
    Device& d = *h->dev;
    CME_TRY(peers_check(d));
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    // free-run control: omega/C for the graphs, never stop
    const double omega = effective_omega(h);
    const int64_t C = h->sopts.check_every;
    if (!d.use_res) CME_TRY(prepare_graphs(d, C, omega));
    CME_TRY(load_iterate(h, p0, true, s));
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (p0 && d.ctrl_host[0].bad_input) {
        set_error("p0 has a negative/NaN entry or no positive mass");
        return CME_ERR_INVALID_ARG;
    }
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->omega, &omega, sizeof(double), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->C, &C, sizeof(int64_t), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    return CME_OK;
}

cme_status device_run(cme_matrix_s* h, int64_t blocks) {
    Device& d = *h->dev;
    CME_TRY(peers_check(d));
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    const int64_t C = h->sopts.check_every;
    if (d.use_res) {
        CME_TRY(launch_res(d, s, d.cur, blocks * C, false, C, effective_omega(h)));
        d.cur = (int)((d.cur + blocks * C) & 1);
        return CME_OK;
    }
    CME_TRY(prepare_graphs(d, C, effective_omega(h)));
    for (int64_t b = 0; b < blocks; ++b) {
        CUDA_TRY(cudaGraphLaunch(d.gexec[d.cur], s));
        d.cur = (int)((d.cur + C) & 1);
    }
    return CME_OK;
}

cme_status device_fetch(cme_matrix_s* h, double* p_out) {
    Device& d = *h->dev;
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CME_TRY(write_out(h, p_out, d.ctrl->inv_s, s));
    const Ctrl& f = d.ctrl_host[0];
    fill_reports(h, f, effective_omega(h), 0.0, f.status);
    return CME_OK;
}

}  // namespace cme
