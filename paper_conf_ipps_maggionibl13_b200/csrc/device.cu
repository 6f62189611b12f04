// Device side of libcme: buffers in HBM, the fused step launches, the
// check/normalise/stop logic and the solve driver.
//
// Per solve the iteration runs as CUDA graphs of one "check block": C fused
// steps (the last with CHECK) + the partial reduction + the decision kernel,
// all device-side; the host only reads a ~100-byte control block every C
// iterations and launches the next graph one block ahead, so it never stalls
// the GPU (a decided stop turns the look-ahead block into no-op launches).
#include <cmath>
#include <cstddef>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>

#include "cme_internal.h"
#include "comm.h"
#include "kernels.cuh"
#include "kernels_tma.cuh"
#include "kernels_persist.cuh"

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
    // iterates: x-span buffers (element 0 = first x-span entry; [-1], [nx] zero)
    double* xb[2] = {nullptr, nullptr};
    int cur = 0;
    double* partials = nullptr;
    int grid = 0, part_blocks = 0;
    double* gather = nullptr;        // [nranks * 8]
    double* local8 = nullptr;        // [8]
    double* io = nullptr;            // n_global staging
    double* io2 = nullptr;           // second staging (distributed output)
    double* one = nullptr;           // constant 1.0
    Ctrl* ctrl = nullptr;
    Ctrl* ctrl_host = nullptr;       // pinned, 2 slots
    int64_t n_global = 0, n_own = 0, nx = 0, own_off = 0, row_begin = 0;
    int64_t n_slices = 0;
    int format = CME_FMT_DIAG_SELL;
    bool band = false, rearr = false;
    // distributed
    cme_comm_s* comm = nullptr;
    int nranks = 1, rank = 0;
    HaloPlan halo;
    std::vector<int64_t> cuts;
    // TMA-staged persistent kernel (kernels_tma.cuh)
    bool use_tma = false;
    int tma_ncw = 8;
    int tma_grid = 0, tma_stages = 0, tma_stage_bytes = 0, tma_off_val = 0, tma_off_col = 0;
    int64_t n_tiles = 0;
    // persistent cooperative kernel for small problems (kernels_persist.cuh)
    bool use_persist = false;
    int p_grid = 0;
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
};

// ------------------------------------------------------------------------------
// small kernels
// ------------------------------------------------------------------------------

// out8 = {sum p0, sum p1, sum p2, max p3, max p4, 0,0,0} over nblocks partial
// records, in a fixed order (deterministic).  One CTA of 1024 threads.
__global__ void __launch_bounds__(1024) reduce_partials_kernel(const double* partials, int nblocks,
                                                               double* out8, const int32_t* stop) {
    if (stop != nullptr && *stop) return;
    double a = 0, b = 0, c = 0, d = 0, e = 0;
    for (int i = threadIdx.x; i < nblocks; i += blockDim.x) {
        const double* p = partials + (size_t)i * kPartials;
        a += p[0]; b += p[1]; c += p[2]; d = fmax(d, p[3]); e = fmax(e, p[4]);
    }
    __shared__ double s[32][5];
    a = warp_sum(a); b = warp_sum(b); c = warp_sum(c); d = warp_max(d); e = warp_max(e);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (lane == 0) { s[w][0] = a; s[w][1] = b; s[w][2] = c; s[w][3] = d; s[w][4] = e; }
    __syncthreads();
    if (threadIdx.x == 0) {
        a = b = c = d = e = 0;
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) {
            a += s[i][0]; b += s[i][1]; c += s[i][2]; d = fmax(d, s[i][3]); e = fmax(e, s[i][4]);
        }
        out8[0] = a; out8[1] = b; out8[2] = c; out8[3] = d; out8[4] = e;
        out8[5] = out8[6] = out8[7] = 0.0;
    }
}

// Check decision (readings R2-R5).  all8 holds one
// 8-double record per rank, combined in rank order.
__global__ void decide_kernel(const double* all8, int nranks, Ctrl* c, int32_t len, int32_t final_partial) {
    if (c->stop) return;
    double s = 0, sx = 0, sd = 0, md = 0, mx = 0;
    for (int r = 0; r < nranks; ++r) {
        const double* p = all8 + 8 * r;
        s += p[0]; sx += p[1]; sd += p[2]; md = fmax(md, p[3]); mx = fmax(mx, p[4]);
    }
    const int64_t k = c->iter + len;
    c->iter = k;
    const double delta = sd / sx;
    const double resid = md / (c->omega * c->norm_inf * mx);
    c->red[0] = s; c->red[1] = sx; c->red[2] = sd; c->red[3] = md; c->red[4] = mx;
    c->mass = s;
    c->delta = delta;
    c->resid = resid;
    if (!(s > 0.0) || isinf(s) || isnan(delta)) { c->status = CME_ERR_NUMERIC; c->stop = 1; return; }
    c->inv_s = 1.0 / s;  // L1 normalisation, applied by the next step (R5)
    if (final_partial) { c->status = CME_NOT_CONVERGED; c->stop = 1; return; }
    const double crit = c->stop_mode == CME_STOP_DELTA_L1 ? delta : resid;
    if (crit <= c->tol) { c->status = CME_OK; c->stop = 1; return; }
    if (c->stag_tol > 0.0 && k >= 2 * c->C && fabs(delta - c->delta_prev) <= c->stag_tol * c->delta_prev) {
        c->status = CME_STAGNATED; c->stop = 1; return;
    }
    c->delta_prev = delta;
    if (k >= c->max_iter) { c->status = CME_NOT_CONVERGED; c->stop = 1; }
}

// x_own[l] = src[perm[l]] (original -> reordered), per-CTA partials {sum, #bad}.
__global__ void __launch_bounds__(kCta) load_kernel(const double* src, const int32_t* perm, int64_t n,
                                                    double* x_own, double* partials) {
    double s = 0.0, bad = 0.0;
    for (int64_t l = (int64_t)blockIdx.x * kCta + threadIdx.x; l < n; l += (int64_t)gridDim.x * kCta) {
        const double v = src[perm[l]];
        x_own[l] = v;
        s += v;
        bad += !(v >= 0.0) || isinf(v);
    }
    cta_check_partials<kWarpsPerCta>(s, bad, 0.0, 0.0, 0.0, partials);
}

__global__ void load_decide_kernel(const double* all8, int nranks, Ctrl* c, int32_t normalise) {
    double s = 0.0, bad = 0.0;
    for (int r = 0; r < nranks; ++r) { s += all8[8 * r]; bad += all8[8 * r + 1]; }
    c->bad_input = normalise && (bad > 0.0 || !(s > 0.0) || isinf(s));
    c->inv_s = normalise ? 1.0 / s : 1.0;
    c->mass = s;
}

__global__ void fill_kernel(double* x, int64_t n, double v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = v;
}

// out[perm[l]] = x[l] * scale  (reordered -> original order)
__global__ void scatter_out_kernel(const double* x, const int32_t* perm, int64_t n, const double* scale,
                                   double* out) {
    const double sc = *scale;
    for (int64_t l = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; l < n; l += (int64_t)gridDim.x * blockDim.x)
        out[perm[l]] = x[l] * sc;
}

__global__ void scale_copy_kernel(const double* x, int64_t n, const double* scale, double* out) {
    const double sc = *scale;
    for (int64_t l = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; l < n; l += (int64_t)gridDim.x * blockDim.x)
        out[l] = x[l] * sc;
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

template <int W, bool B, bool R, bool D, bool C>
static cudaError_t tma_attr(int smem) {
    return cudaFuncSetAttribute(sell_tma_kernel<W, B, R, D, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
}

template <int W>
static cudaError_t tma_attr_all(int smem) {
    cudaError_t e = cudaSuccess;
#define A(b, r, dd, c) if (e == cudaSuccess) e = tma_attr<W, b, r, dd, c>(smem);
    A(0,0,0,0) A(0,0,0,1) A(0,0,1,0) A(0,0,1,1) A(0,1,0,0) A(0,1,0,1) A(0,1,1,0) A(0,1,1,1)
    A(1,0,0,0) A(1,0,0,1) A(1,0,1,0) A(1,0,1,1) A(1,1,0,0) A(1,1,0,1) A(1,1,1,0) A(1,1,1,1)
#undef A
    return e;
}

template <int W>
static void launch_tma(const Device& d, const TmaArgs& T, bool damp, bool check, cudaStream_t s) {
    const int smem = d.tma_stages * d.tma_stage_bytes;
    const int key = (d.band ? 8 : 0) | (d.rearr ? 4 : 0) | (damp ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K(b, r, dd, c) \
    case (b * 8 + r * 4 + dd * 2 + c): sell_tma_kernel<W, b, r, dd, c><<<d.tma_grid, TmaShape<W>::kThreads, smem, s>>>(T); break;
        K(0, 0, 0, 0) K(0, 0, 0, 1) K(0, 0, 1, 0) K(0, 0, 1, 1)
        K(0, 1, 0, 0) K(0, 1, 0, 1) K(0, 1, 1, 0) K(0, 1, 1, 1)
        K(1, 0, 0, 0) K(1, 0, 0, 1) K(1, 0, 1, 0) K(1, 0, 1, 1)
        K(1, 1, 0, 0) K(1, 1, 0, 1) K(1, 1, 1, 0) K(1, 1, 1, 1)
#undef K
    }
}

// Choose stages / CTAs per SM for the TMA kernel.  Tuning knobs (environment,
// read at pack/distribute time): CME_TMA=0 forces the register kernel,
// CME_TMA_STAGES, CME_TMA_CTAS override the defaults (4 stages, max resident).
static cme_status configure_tma(Device& d, const Packed& P) {
    d.use_tma = false;
    const int want = env_int("CME_TMA", -1);   // -1 auto, 0 off, 1 force
    if (want == 0 || d.n_slices == 0) return CME_OK;
    const int ncw = env_int("CME_TMA_WARPS", 16) == 8 ? 8 : 16;
    d.tma_ncw = ncw;
    d.n_tiles = (d.n_slices + ncw - 1) / ncw;
    int64_t max_nval = 0;
    for (int64_t t = 0; t < d.n_tiles; ++t) {
        const int64_t q0 = t * ncw, q1 = std::min<int64_t>(q0 + ncw, d.n_slices);
        max_nval = std::max(max_nval, P.slice_off[q1] - P.slice_off[q0]);
    }
    auto a128 = [](int64_t b) { return (b + 127) / 128 * 128; };
    const int64_t off_val = a128(tma_fixed_bytes(ncw, d.band, d.rearr));
    const int64_t off_col = off_val + a128(8 * max_nval);
    const int64_t stage = a128(off_col + 4 * max_nval);
    int dev = 0, smem_max = 0, sms = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    int stages = std::min(8, std::max(2, env_int("CME_TMA_STAGES", 2)));
    while (stages > 2 && stages * stage > smem_max - 1024) --stages;
    if (stages * stage > smem_max - 1024) return CME_OK;  // tiles too wide: register kernel
    const int smem = (int)(stages * stage);
    CUDA_TRY(ncw == 16 ? tma_attr_all<16>(smem) : tma_attr_all<8>(smem));
    int occ = 0;
    if (ncw == 16)
        CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sell_tma_kernel<16, false, true, true, true>,
                                                               TmaShape<16>::kThreads, smem));
    else
        CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sell_tma_kernel<8, false, true, true, true>,
                                                               TmaShape<8>::kThreads, smem));
    occ = std::max(1, std::min(occ, env_int("CME_TMA_CTAS", occ)));
    d.tma_stages = stages;
    d.tma_stage_bytes = (int)stage;
    d.tma_off_val = (int)off_val;
    d.tma_off_col = (int)off_col;
    d.tma_grid = (int)std::min<int64_t>(d.n_tiles, (int64_t)sms * occ);
    // the ring only pays when every CTA streams >= 2 tiles; small problems
    // (<~300K rows) run faster on the register kernel
    if (want < 0 && d.n_tiles < 2 * (int64_t)sms * occ) return CME_OK;
    if (env_int("CME_VERBOSE", 0))
        std::fprintf(stderr, "[cme] tma: warps=%d stages=%d stage_bytes=%lld occ=%d grid=%d tiles=%lld\n", ncw,
                     stages, (long long)stage, occ, d.tma_grid, (long long)d.n_tiles);
    d.use_tma = true;
    return CME_OK;
}

template <bool B, bool R, bool D>
static cudaError_t launch_persist_t(const PersistArgs& P, int grid, cudaStream_t s) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kCta);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, sell_persistent_kernel<B, R, D>, P);
}

// Persistent cooperative kernel for L2-resident problems: one launch per check
// block.  CME_PERSIST: -1 auto (<= 1M local rows, single GPU), 0 off, 1 force.
static cme_status configure_persist(Device& d) {
    d.use_persist = false;
    const int want = env_int("CME_PERSIST", -1);
    if (want == 0 || d.comm || d.format == CME_FMT_CSR || d.n_slices == 0) return CME_OK;
    if (want < 0 && (d.use_tma || d.n_own > (1 << 20))) return CME_OK;
    int dev = 0, sms = 0, occ = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sell_persistent_kernel<true, true, true>, kCta, 0));
    int occ2 = 0;
    CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, sell_persistent_kernel<false, false, false>, kCta, 0));
    occ = std::max(1, std::min(occ, occ2));
    const int64_t need = (d.n_slices + kWarpsPerCta - 1) / kWarpsPerCta;
    d.p_grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * occ));
    d.use_persist = true;
    d.use_tma = false;
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
    d->format = h->format;
    d->band = P.band_on != 0;
    d->rearr = P.window > 1;
    d->n_global = h->A.n;
    d->n_own = P.n;
    d->n_slices = P.n_slices;
    d->nranks = h->nranks;
    d->rank = h->rank;
    d->comm = comm;
    d->cuts = h->cuts;
    d->row_begin = h->cuts.empty() ? 0 : h->cuts[h->rank];
    if (h->nranks > 1) {
        d->nx = h->span[2 * h->rank + 1] - h->span[2 * h->rank];
        d->own_off = d->row_begin - h->span[2 * h->rank];
        d->halo = *halo;
    } else {
        d->nx = d->n_own;
        d->own_off = 0;
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
        UP(val, P.val);
        UP(col, P.col);
        UP(inv_d, P.inv_d);
        if (d->band) { UP(lo, P.lo); UP(up, P.up); }
        if (d->rearr) UP(row_of, P.row_of);
    }
    {
        std::vector<int32_t> po(h->perm.begin() + d->row_begin, h->perm.begin() + d->row_begin + d->n_own);
        UP(perm_own, po);
        if (comm) UP(perm_global, h->perm);
    }
#undef UP
    for (int b = 0; b < 2; ++b) {
        double* base = nullptr;
        if ((s = d->alloc(base, d->nx + 2)) != CME_OK) return fail(s);
        if (cudaMemset(base, 0, (d->nx + 2) * sizeof(double)) != cudaSuccess) return fail(CME_ERR_CUDA);
        d->xb[b] = base + 1;
    }
    d->grid = d->format == CME_FMT_CSR ? (int)((d->n_own + kCta - 1) / kCta)
                                       : (int)((d->n_slices + kWarpsPerCta - 1) / kWarpsPerCta);
    d->grid = std::max(d->grid, 1);
    if (d->format != CME_FMT_CSR && (s = configure_tma(*d, P)) != CME_OK) return fail(s);
    if ((s = configure_persist(*d)) != CME_OK) return fail(s);
    d->part_blocks = std::max(d->grid, grid_for(d->n_own));
    if ((s = d->alloc(d->partials, (size_t)d->part_blocks * kPartials)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->gather, (size_t)d->nranks * 8)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->local8, 8)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->io, d->n_global)) != CME_OK) return fail(s);
    if (comm && (s = d->alloc(d->io2, d->n_global)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->one, 1)) != CME_OK) return fail(s);
    if ((s = d->alloc(d->ctrl, 1)) != CME_OK) return fail(s);
    const double one = 1.0;
    if (cudaMemcpy(d->one, &one, sizeof(double), cudaMemcpyHostToDevice) != cudaSuccess) return fail(CME_ERR_CUDA);
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
// launches
// ------------------------------------------------------------------------------
template <bool B, bool R, bool D, bool C>
static void launch_sell(const StepArgs& a, int grid, cudaStream_t s) {
    sell_step_kernel<B, R, D, C><<<grid, kCta, 0, s>>>(a);
}

static cme_status launch_step(Device& d, cudaStream_t s, int src, int dst, bool check, const double* pre,
                              double omega) {
    StepArgs a{};
    a.n_rows = d.n_own;
    a.slice_begin = 0;
    a.slice_end = d.n_slices;
    a.slice_off = d.slice_off;
    a.slice_w = d.slice_w;
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
    const bool damp = omega != 1.0;
    if (d.format == CME_FMT_CSR) {
        if (damp) { if (check) csr_step_kernel<true, true><<<d.grid, kCta, 0, s>>>(a); else csr_step_kernel<true, false><<<d.grid, kCta, 0, s>>>(a); }
        else { if (check) csr_step_kernel<false, true><<<d.grid, kCta, 0, s>>>(a); else csr_step_kernel<false, false><<<d.grid, kCta, 0, s>>>(a); }
    } else if (d.use_tma) {
        TmaArgs T{a, d.n_tiles, d.tma_stages, d.tma_stage_bytes, d.tma_off_val, d.tma_off_col};
        if (d.tma_ncw == 16) launch_tma<16>(d, T, damp, check, s);
        else launch_tma<8>(d, T, damp, check, s);
    } else {
        const int key = (d.band ? 8 : 0) | (d.rearr ? 4 : 0) | (damp ? 2 : 0) | (check ? 1 : 0);
        switch (key) {
#define K(b, r, dd, c) case (b * 8 + r * 4 + dd * 2 + c): launch_sell<b, r, dd, c>(a, d.grid, s); break;
            K(0, 0, 0, 0) K(0, 0, 0, 1) K(0, 0, 1, 0) K(0, 0, 1, 1)
            K(0, 1, 0, 0) K(0, 1, 0, 1) K(0, 1, 1, 0) K(0, 1, 1, 1)
            K(1, 0, 0, 0) K(1, 0, 0, 1) K(1, 0, 1, 0) K(1, 0, 1, 1)
            K(1, 1, 0, 0) K(1, 1, 0, 1) K(1, 1, 1, 0) K(1, 1, 1, 1)
#undef K
        }
    }
    CUDA_TRY(cudaGetLastError());
    if (d.comm) CME_TRY(comm_halo(d.comm, d.halo, d.xb[dst], s));
    return CME_OK;
}

// reduce partials of the last CHECK step and decide
static cme_status launch_finalize(Device& d, cudaStream_t s, int32_t len, int32_t final_partial) {
    reduce_partials_kernel<<<1, 1024, 0, s>>>(d.partials, d.use_persist ? d.p_grid : d.use_tma ? d.tma_grid : d.grid,
                                              d.comm ? d.local8 : d.gather, &d.ctrl->stop);
    CUDA_TRY(cudaGetLastError());
    if (d.comm) CME_TRY(comm_allgather8(d.comm, d.local8, d.gather, s));
    decide_kernel<<<1, 1, 0, s>>>(d.gather, d.nranks, d.ctrl, len, final_partial);
    CUDA_TRY(cudaGetLastError());
    return CME_OK;
}

// One check block of C steps starting from buffer `start`: steps 0..C-2 plain,
// step C-1 CHECK; the first step applies the pending 1/||y||_1 (R5).
static cme_status enqueue_block(Device& d, cudaStream_t s, int start, int64_t C, double omega, bool final_partial) {
    if (d.use_persist) {
        PersistArgs P{};
        P.a.n_rows = d.n_own;
        P.a.slice_begin = 0;
        P.a.slice_end = d.n_slices;
        P.a.slice_off = d.slice_off;
        P.a.slice_w = d.slice_w;
        P.a.val = d.val;
        P.a.col = d.col;
        P.a.row_of = d.row_of;
        P.a.lo = d.lo;
        P.a.up = d.up;
        P.a.inv_d = d.inv_d;
        P.a.own_off = d.own_off;
        P.a.omega = omega;
        P.a.pre_scale = &d.ctrl->inv_s;
        P.a.partials = d.partials;
        P.a.stop = &d.ctrl->stop;
        P.xb0 = d.xb[0];
        P.xb1 = d.xb[1];
        P.start = start;
        P.steps = (int32_t)C;
        const bool damp = omega != 1.0;
        const int key = (d.band ? 4 : 0) | (d.rearr ? 2 : 0) | (damp ? 1 : 0);
        cudaError_t e = cudaSuccess;
        switch (key) {
            case 0: e = launch_persist_t<false, false, false>(P, d.p_grid, s); break;
            case 1: e = launch_persist_t<false, false, true>(P, d.p_grid, s); break;
            case 2: e = launch_persist_t<false, true, false>(P, d.p_grid, s); break;
            case 3: e = launch_persist_t<false, true, true>(P, d.p_grid, s); break;
            case 4: e = launch_persist_t<true, false, false>(P, d.p_grid, s); break;
            case 5: e = launch_persist_t<true, false, true>(P, d.p_grid, s); break;
            case 6: e = launch_persist_t<true, true, false>(P, d.p_grid, s); break;
            case 7: e = launch_persist_t<true, true, true>(P, d.p_grid, s); break;
        }
        CUDA_TRY(e);
        return launch_finalize(d, s, (int32_t)C, final_partial ? 1 : 0);
    }
    for (int64_t t = 0; t < C; ++t) {
        const int src = (int)((start + t) & 1);
        CME_TRY(launch_step(d, s, src, 1 - src, t == C - 1, t == 0 ? &d.ctrl->inv_s : nullptr, omega));
    }
    return launch_finalize(d, s, (int32_t)C, final_partial ? 1 : 0);
}

static cme_status ensure_graphs(Device& d, int64_t C, double omega) {
    if (d.gC == C && d.gomega == omega && d.gexec[0]) return CME_OK;
    if (d.comm) {
        // NCCL sets up peer connections lazily on first use: do that outside
        // the capture (one throw-away exchange + gather on the private stream)
        CME_TRY(comm_halo(d.comm, d.halo, d.xb[1], d.own));
        CME_TRY(comm_allgather8(d.comm, d.local8, d.gather, d.own));
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

static cudaStream_t stream_of(cme_matrix_s* h) {
    return h->sopts.stream ? (cudaStream_t)h->sopts.stream : h->dev->own;
}

static bool is_device_ptr(const void* p) {
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

// x (own rows) <- p0 / sum(p0) (or uniform); halo filled; ctrl reset to free-run.
static cme_status load_iterate(cme_matrix_s* h, const double* p0, bool normalise, cudaStream_t s) {
    Device& d = *h->dev;
    d.cur = 0;
    double* x = d.xb[0] + d.own_off;
    Ctrl c{};
    c.omega = 1.0; c.tol = -1.0; c.stag_tol = 0.0; c.norm_inf = h->norm_inf;
    c.C = 1; c.max_iter = INT64_MAX; c.stop_mode = 0; c.nranks = d.nranks;
    c.iter = 0; c.delta = -1; c.delta_prev = -1; c.resid = -1; c.mass = 1.0; c.inv_s = 1.0;
    c.status = -1; c.stop = 0;
    CUDA_TRY(cudaMemcpyAsync(d.ctrl, &c, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
    if (!p0) {
        fill_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(x, d.n_own, 1.0 / (double)d.n_global);
        CUDA_TRY(cudaGetLastError());
    } else {
        const double* src = p0;
        if (!is_device_ptr(p0)) {
            CUDA_TRY(cudaMemcpyAsync(d.io, p0, d.n_global * sizeof(double), cudaMemcpyHostToDevice, s));
            src = d.io;
        }
        const int g = grid_for(d.n_own);
        load_kernel<<<g, kCta, 0, s>>>(src, d.perm_own, d.n_own, x, d.partials);
        reduce_partials_kernel<<<1, 1024, 0, s>>>(d.partials, g, d.comm ? d.local8 : d.gather, nullptr);
        CUDA_TRY(cudaGetLastError());
        if (d.comm) CME_TRY(comm_allgather8(d.comm, d.local8, d.gather, s));
        load_decide_kernel<<<1, 1, 0, s>>>(d.gather, d.nranks, d.ctrl, normalise ? 1 : 0);
        CUDA_TRY(cudaGetLastError());
    }
    if (d.comm) CME_TRY(comm_halo(d.comm, d.halo, d.xb[0], s));
    return CME_OK;
}

// p_out (original order) <- x[cur] * scale
static cme_status write_out(cme_matrix_s* h, double* p_out, const double* scale, cudaStream_t s) {
    Device& d = *h->dev;
    const double* x = d.xb[d.cur] + d.own_off;
    const bool dev_out = is_device_ptr(p_out);
    double* dst = dev_out ? p_out : d.io;
    if (!d.comm) {
        scatter_out_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(x, d.perm_own, d.n_own, scale, dst);
        CUDA_TRY(cudaGetLastError());
    } else {
        // own rows -> reordered global staging, broadcast every rank's segment,
        // then un-permute into the caller's buffer (or the second staging buffer)
        scale_copy_kernel<<<grid_for(d.n_own), kCta, 0, s>>>(x, d.n_own, scale, d.io + d.row_begin);
        CUDA_TRY(cudaGetLastError());
        CME_TRY(comm_bcast_segments(d.comm, d.io, d.cuts, s));
        double* out = dev_out ? p_out : d.io2;
        scatter_out_kernel<<<grid_for(d.n_global), kCta, 0, s>>>(d.io, d.perm_global, d.n_global, d.one, out);
        CUDA_TRY(cudaGetLastError());
        if (!dev_out)
            CUDA_TRY(cudaMemcpyAsync(p_out, d.io2, d.n_global * sizeof(double), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        return CME_OK;
    }
    if (!dev_out) CUDA_TRY(cudaMemcpyAsync(p_out, d.io, d.n_global * sizeof(double), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    return CME_OK;
}

static double effective_omega(cme_matrix_s* h) {
    if (h->sopts.omega > 0.0) return h->sopts.omega;
    return h->period == 1 ? 1.0 : 0.9;
}

cme_status device_solve(cme_matrix_s* h, const double* p0, double tol, int64_t max_iter, double* p_out,
                        int64_t* iters_out) {
    Device& d = *h->dev;
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    const int64_t C = h->sopts.check_every;
    const double omega = effective_omega(h);
    CME_TRY(load_iterate(h, p0, true, s));
    Ctrl c{};
    c.omega = omega; c.tol = tol; c.stag_tol = h->sopts.stag_tol; c.norm_inf = h->norm_inf;
    c.C = C; c.max_iter = max_iter; c.stop_mode = h->sopts.stop; c.nranks = d.nranks;
    c.iter = 0; c.delta = -1; c.delta_prev = -1; c.resid = -1; c.mass = 1.0;
    c.status = -1; c.stop = 0;
    // keep inv_s from the load (1/sum p0): patch every field but inv_s/mass/bad_input
    CUDA_TRY(cudaMemcpyAsync(d.ctrl, &c, offsetof(Ctrl, mass), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->status, &c.status, 2 * sizeof(int32_t), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (p0 && d.ctrl_host[0].bad_input) {
        set_error("p0 has a negative/NaN entry or no positive mass");
        return CME_ERR_INVALID_ARG;
    }
    CME_TRY(ensure_graphs(d, C, omega));
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
    if (status == -1 && rem > 0) {
        CME_TRY(enqueue_block(d, s, start, rem, omega, true));
    } else if (status == -1 && max_iter == 0) {
        // no iteration: the output is the normalised start vector
    }
    CUDA_TRY(cudaEventRecord(d.t1, s));
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl_host[0], d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    const Ctrl& f = d.ctrl_host[0];
    d.cur = (int)(f.iter & 1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, d.t0, d.t1);
    h->report.status = max_iter == 0 ? CME_NOT_CONVERGED : f.status;
    h->report.iters = f.iter;
    h->report.delta = f.delta;
    h->report.resid = f.resid;
    h->report.mass = f.mass;
    h->report.omega = omega;
    h->report.seconds = ms * 1e-3;
    if (iters_out) *iters_out = f.iter;
    CME_TRY(write_out(h, p_out, &d.ctrl->inv_s, s));
    return (cme_status)h->report.status;
}

void device_describe(const Device* d, cme_info* f) {
    if (!d) { f->kernel = -1; return; }
    f->kernel = d->format == CME_FMT_CSR ? 2 : d->use_persist ? 3 : d->use_tma ? 1 : 0;
    f->tma_warps = d->use_tma ? d->tma_ncw : 0;
    f->tma_stages = d->use_tma ? d->tma_stages : 0;
    f->grid = d->use_persist ? d->p_grid : d->use_tma ? d->tma_grid : d->grid;
}

cme_status device_spmv(cme_matrix_s* h, const double* x, double* y) {
    Device& d = *h->dev;
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    CME_TRY(load_iterate(h, x, false, s));
    CME_TRY(launch_step(d, s, 0, 1, false, nullptr, effective_omega(h)));
    d.cur = 1;
    return write_out(h, y, d.one, s);
}

cme_status device_load(cme_matrix_s* h, const double* p0) {
    Device& d = *h->dev;
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    CME_TRY(load_iterate(h, p0, true, s));
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (p0 && d.ctrl_host[0].bad_input) {
        set_error("p0 has a negative/NaN entry or no positive mass");
        return CME_ERR_INVALID_ARG;
    }
    // free-run control: omega for the graphs, never stop
    const double omega = effective_omega(h);
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->omega, &omega, sizeof(double), cudaMemcpyHostToDevice, s));
    const int64_t C = h->sopts.check_every;
    CUDA_TRY(cudaMemcpyAsync(&d.ctrl->C, &C, sizeof(int64_t), cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    return ensure_graphs(d, C, omega);
}

cme_status device_run(cme_matrix_s* h, int64_t blocks) {
    Device& d = *h->dev;
    CUDA_TRY(cudaSetDevice(d.dev));
    cudaStream_t s = stream_of(h);
    const int64_t C = h->sopts.check_every;
    CME_TRY(ensure_graphs(d, C, effective_omega(h)));
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
    CME_TRY(write_out(h, p_out, &d.ctrl->inv_s, s));
    const Ctrl& f = d.ctrl_host[0];
    h->report.iters = f.iter;
    h->report.delta = f.delta;
    h->report.resid = f.resid;
    h->report.mass = f.mass;
    h->report.status = f.status;
    return CME_OK;
}

}  // namespace cme
