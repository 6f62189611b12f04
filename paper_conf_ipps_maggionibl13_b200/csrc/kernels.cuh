// sm_100a kernels of the fused Jacobi step.
//
// One step computes, for every row r (slot s of the packed layout):
//   y_r = sc * [ (1-omega) x_r + omega * inv_d_s * ((lo_s x_{r-1} + up_s x_{r+1}) + sum_t val x[col]) ]
// = sc * M_omega x (eq. 8 with relaxation omega, R1; sc = pending
// 1/||y||_1 of the previous check, R5).  CHECK steps also emit per-CTA
// partials of sum y, sum x, sum |y - x|, max |a_ii||y - x| and max x, which
// are the L1 normalisation, delta (R2) and the paper's normalised
// residual (r_i = a_ii (x_i - (Mx)_i) = |a_ii| (y_i - x_i) / omega).
//
// Mapping: warp = one 32-row slice (slice size decoupled from the
// 256-thread CTA), lane = slot.  The slice's val/col block is contiguous and
// column-major, so each t-step of a warp reads 256 B of val and 128 B of col
// fully coalesced.  Streams are read with L1::no_allocate + an L2 evict-first
// policy so the gathered iterate x keeps L1/L2; all val/col loads of a chunk
// of up to 8 t-steps are issued before the dependent x gathers (ILP).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace cme {

constexpr int kWarpsPerCta = 8;
constexpr int kCta = 32 * kWarpsPerCta;
constexpr int kPartials = 8;  // doubles per CTA partial record
constexpr int kUnroll = 8;    // t-steps whose loads are issued together

// Device control block of a solve (host writes the inputs, finalize the rest).
struct Ctrl {
    double omega, tol, stag_tol, norm_inf;
    int64_t C, max_iter;
    int32_t stop_mode, nranks;
    int64_t iter;                 // iterations completed
    double delta, delta_prev, resid, mass, inv_s;
    int32_t status;               // -1 running, else cme_status
    int32_t stop;                 // 1 -> later step/finalize launches are no-ops
    int32_t bad_input, pad_;
    double red[kPartials];        // globally reduced check partials
};

struct StepArgs {
    int64_t n_rows;        // rows owned (slots >= n_rows are padding)
    int64_t slice_begin, slice_end;
    const int64_t* slice_off;
    const int32_t* slice_w;
    const double* val;
    const int32_t* col;    // x-span coordinates
    const int32_t* row_of; // slot -> local row (nullptr: identity)
    const double* lo;
    const double* up;
    const double* inv_d;
    const double* x;       // x-span base (x[-1], x[nx] are zero sentinels)
    double* y;             // x-span base of the output buffer
    int64_t own_off;       // own row r lives at x-span index own_off + r
    double omega;
    const double* pre_scale;  // nullable
    double* partials;         // CHECK: [gridDim.x][kPartials]
    const int32_t* stop;      // nullable
    // CSR arm
    const int64_t* csr_rp;
    const int32_t* csr_ci;
    const double* csr_v;
};

__device__ __forceinline__ uint64_t evict_first_policy() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ double ld_stream(const double* p, uint64_t pol) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int32_t ld_stream(const int32_t* p, uint64_t pol) {
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ double ld_x(const double* p) { return __ldg(p); }

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ double warp_max(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// CTA-level deterministic reduction of the 5 check quantities into
// partials[blockIdx.x]; NW = warps in the CTA (all must call it).
template <int NW = kWarpsPerCta>
__device__ __forceinline__ void cta_check_partials(double sy, double sx, double sd, double md,
                                                   double mx, double* partials) {
    __shared__ double red[NW][5];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    sy = warp_sum(sy); sx = warp_sum(sx); sd = warp_sum(sd);
    md = warp_max(md); mx = warp_max(mx);
    if (lane == 0) { red[w][0] = sy; red[w][1] = sx; red[w][2] = sd; red[w][3] = md; red[w][4] = mx; }
    __syncthreads();
    if (threadIdx.x == 0) {
        double a = 0, b = 0, c = 0, d = 0, e = 0;
        for (int i = 0; i < NW; ++i) {
            a += red[i][0]; b += red[i][1]; c += red[i][2];
            d = fmax(d, red[i][3]); e = fmax(e, red[i][4]);
        }
        double* o = partials + (size_t)blockIdx.x * kPartials;
        o[0] = a; o[1] = b; o[2] = c; o[3] = d; o[4] = e; o[5] = 0; o[6] = 0; o[7] = 0;
    }
}

// x loads: read-only path (.nc) when x is constant for the whole launch;
// L2-coherent (.cg) in the persistent kernel, whose x is rewritten by other
// CTAs between grid barriers.
template <bool COHERENT>
__device__ __forceinline__ double ld_xv(const double* p) {
    if (COHERENT) {
        double v;
        asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p));
        return v;
    }
    return __ldg(p);
}

// Check terms of one row: y, x (both scaled), inv_d.
struct SlotOut {
    double y, x, id;
    bool valid;
};
__device__ __forceinline__ void check_accum(const SlotOut& o, double& sy, double& sx, double& sd, double& md,
                                            double& mx) {
    if (!o.valid) return;
    const double df = fabs(o.y - o.x);
    sy += o.y; sx += o.x; sd += df; md = fmax(md, df / o.id); mx = fmax(mx, o.x);
}

// One slot (lane) of slice q: computes and stores y_r for its row r.
template <bool BAND, bool REARR, bool DAMP, bool NEEDX, bool COHERENT>
__device__ __forceinline__ SlotOut sell_slot(const StepArgs& a, int64_t q, int lane, uint64_t pol,
                                             const double* x, double* y, const double* pre_scale) {
    const int64_t slot = q * 32 + lane;
    const int w = __ldg(a.slice_w + q);
    const int64_t base = __ldg(a.slice_off + q) + lane;
    if (slot >= a.n_rows) return SlotOut{0.0, 0.0, 1.0, false};
    const int64_t r = REARR ? (int64_t)ld_stream(a.row_of + slot, pol) : slot;
    const double* xo = x + a.own_off;
    double acc = 0.0;
    for (int t0 = 0; t0 < w; t0 += kUnroll) {
        double v[kUnroll];
        int32_t c[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            if (t0 + u < w) {
                v[u] = ld_stream(a.val + base + 32 * (int64_t)(t0 + u), pol);
                c[u] = ld_stream(a.col + base + 32 * (int64_t)(t0 + u), pol);
            }
        }
        double xv[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
            if (t0 + u < w) xv[u] = ld_xv<COHERENT>(x + c[u]);
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
            if (t0 + u < w) acc = fma(v[u], xv[u], acc);
    }
    double s = acc;
    if (BAND) {
        const double l = ld_stream(a.lo + slot, pol), up = ld_stream(a.up + slot, pol);
        s = fma(l, ld_xv<COHERENT>(xo + r - 1), up * ld_xv<COHERENT>(xo + r + 1)) + acc;
    }
    const double id = ld_stream(a.inv_d + slot, pol);
    double xr = (DAMP || NEEDX) ? ld_xv<COHERENT>(xo + r) : 0.0;
    double yv = DAMP ? fma(1.0 - a.omega, xr, a.omega * (id * s)) : id * s;
    if (pre_scale != nullptr) {
        const double sc = *pre_scale;
        yv *= sc;
        xr *= sc;
    }
    y[a.own_off + r] = yv;
    return SlotOut{yv, xr, id, true};
}

template <bool BAND, bool REARR, bool DAMP, bool CHECK>
__global__ void __launch_bounds__(kCta) sell_step_kernel(const StepArgs a) {
    if (a.stop != nullptr && *a.stop) return;
    const uint64_t pol = evict_first_policy();
    const int lane = threadIdx.x & 31;
    const int64_t q = a.slice_begin + (int64_t)blockIdx.x * kWarpsPerCta + (threadIdx.x >> 5);
    double sy = 0.0, sx = 0.0, sd = 0.0, md = 0.0, mx = 0.0;
    if (q < a.slice_end) {
        const SlotOut o = sell_slot<BAND, REARR, DAMP, CHECK, false>(a, q, lane, pol, a.x, a.y, a.pre_scale);
        if (CHECK) check_accum(o, sy, sx, sd, md, mx);
    }
    if (CHECK) cta_check_partials<kWarpsPerCta>(sy, sx, sd, md, mx, a.partials);
}

// Plain CSR arm (ablation, CME_FMT_CSR): one thread per row.
template <bool DAMP, bool CHECK>
__global__ void __launch_bounds__(kCta) csr_step_kernel(const StepArgs a) {
    if (a.stop != nullptr && *a.stop) return;
    const int64_t r = a.slice_begin * 32 + (int64_t)blockIdx.x * kCta + threadIdx.x;
    double sy = 0.0, sx = 0.0, sd = 0.0, md = 0.0, mx = 0.0;
    if (r < a.n_rows && r < a.slice_end * 32) {
        const int64_t b = __ldg(a.csr_rp + r), e = __ldg(a.csr_rp + r + 1);
        double acc = 0.0;
        for (int64_t p = b; p < e; ++p) acc = fma(__ldg(a.csr_v + p), ld_x(a.x + __ldg(a.csr_ci + p)), acc);
        const double id = __ldg(a.inv_d + r);
        const double* xo = a.x + a.own_off;
        double xr = (DAMP || CHECK) ? ld_x(xo + r) : 0.0;
        double yv = DAMP ? fma(1.0 - a.omega, xr, a.omega * (id * acc)) : id * acc;
        if (a.pre_scale != nullptr) {
            const double sc = *a.pre_scale;
            yv *= sc;
            xr *= sc;
        }
        a.y[a.own_off + r] = yv;
        if (CHECK) {
            const double df = fabs(yv - xr);
            sy = yv; sx = xr; sd = df; md = df / id; mx = xr;
        }
    }
    if (CHECK) cta_check_partials<kWarpsPerCta>(sy, sx, sd, md, mx, a.partials);
}

}  // namespace cme
