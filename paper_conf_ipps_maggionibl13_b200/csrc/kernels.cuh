// sm_100a kernels of the fused Jacobi step.
//
// One step computes, for every row r (slot s of the packed layout) and every
// batch member b (B rate sets sharing one pattern; B = 1 is the plain solve):
//   y_rb = sc_b * [ (1-omega) x_rb + omega * inv_d_sb * ((lo_sb x_{r-1,b} + up_sb x_{r+1,b})
//                                                         + sum_t val_tb x[col_t, b]) ]
// = sc_b * M_omega x_b (eq. 8 with relaxation omega, R1; sc_b = the
// pending 1/||y_b||_1 of the previous check, R5).  CHECK steps also emit
// per-CTA partials of sum y, sum x, sum |y - x|, max |a_ii||y - x| and max x
// per member: the L1 normalisation, delta (R2) and the paper's
// normalised residual (r_i = |a_ii| (y_i - x_i) / omega, R21).
//
// Mapping: warp = one 32-row slice (slice size decoupled from the
// CTA), lane = slot.  The slice's val/col block is contiguous and
// column-major, so each t-step of a warp reads 256*B B of val and 128 B of col,
// fully coalesced; the iterate is member-minor (x[c*B + b]) so one gather
// fetches all B members of a column with one 8*B-byte load (B = 4: a 256-bit
// LDG).  Streams are read with L1::no_allocate + an L2 evict-first policy so
// the gathered iterate keeps L1/L2.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "cme.h"   // status codes (decide_apply)

namespace cme {

constexpr int kWarpsPerCta = 8;
constexpr int kCta = 32 * kWarpsPerCta;
constexpr int kPartials = 8;   // doubles per (CTA, member) partial record
constexpr int kMaxBatch = 8;
constexpr int kMaxPushPeers = 8;

// Device control block of a solve (host writes the inputs, decide_kernel the rest).
struct Ctrl {
    double omega, tol, stag_tol;
    int64_t C, max_iter;
    int32_t stop_mode, nranks, batch, pad0_;
    int64_t iter;                 // iterations completed
    int32_t status;               // -1 running, else overall cme_status
    int32_t stop;                 // 1 -> later step/finalize launches are no-ops
    int32_t bad_input, pad1_;
    double norm_inf[kMaxBatch];
    double delta[kMaxBatch], delta_prev[kMaxBatch], resid[kMaxBatch], mass[kMaxBatch];
    double inv_s[kMaxBatch];      // pending 1/sum(y_b), applied by the next step
    int32_t mstatus[kMaxBatch];   // per member: -1 running, else cme_status
    int64_t miters[kMaxBatch];    // iteration at which the member's status was set
};

struct StepArgs {
    int64_t n_rows;        // rows owned (slots >= n_rows are padding)
    int64_t slice_begin, slice_end;
    const int64_t* slice_off;
    const int32_t* slice_w;
    const int2* tile_meta;  // TMA kernels: per slice {slice_off[q] - slice_off[first slice of its tile], slice_w[q]}
    const double* val;     // [n_ell][B]
    const int32_t* col;    // x-span coordinates
    const int32_t* row_of; // slot -> local row (nullptr: identity)
    const double* lo;      // [n_slots][B]
    const double* up;
    const double* inv_d;
    const double* x;       // x-span base, member-minor; x[-B..-1], x[nx*B..] zero sentinels
    double* y;             // x-span base of the output buffer
    int64_t own_off;       // own row r lives at x-span index own_off + r
    double omega;
    const double* pre_scale;  // nullable: [B] pending scales
    double* partials;         // CHECK: [gridDim.x][B][kPartials]
    const int32_t* stop;      // nullable
    // CSR arm (B = 1)
    const int64_t* csr_rp;
    const int32_t* csr_ci;
    const double* csr_v;
    // transient mode (uniformization, R22): y = x + (A x)/Lambda and
    // acc += acc_w * x; unif_lam_inv = 0 selects the Jacobi step
    double unif_lam_inv;
    double* acc;           // x-span base of the accumulator (nullable)
    double acc_w;
    // peer-memory halo (NEXT-4): own rows [push_lo[p], push_hi[p]) are also
    // stored at push_y[p] + r*B, i.e. into peer p's output buffer (NVLink)
    int32_t npush;
    int64_t push_lo[kMaxPushPeers], push_hi[kMaxPushPeers];
    double* push_y[kMaxPushPeers];
};

// Programmatic dependent launch (the step kernels and the check kernels are
// launched with cudaLaunchAttributeProgrammaticStreamSerialization): let the
// next grid in the stream be scheduled early, and wait for the previous grid's
// results before touching anything it wrote (x, ctrl).  Both are no-ops for a
// normal launch.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

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

// B contiguous doubles (B*8-byte aligned): read-only path, vector loads.
template <int B>
__device__ __forceinline__ void ld_vec(const double* p, double* v) {
    if constexpr (B == 1) {
        v[0] = __ldg(p);
    } else if constexpr (B == 2) {
        const double2 t = __ldg(reinterpret_cast<const double2*>(p));
        v[0] = t.x; v[1] = t.y;
    } else {
#pragma unroll
        for (int k = 0; k < B; k += 4)
            asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
                         : "=d"(v[k]), "=d"(v[k + 1]), "=d"(v[k + 2]), "=d"(v[k + 3]) : "l"(p + k));
    }
}
// B contiguous stream doubles (no L1 allocation, L2 evict-first)
template <int B>
__device__ __forceinline__ void ld_stream_vec(const double* p, uint64_t pol, double* v) {
    if constexpr (B == 1) {
        v[0] = ld_stream(p, pol);
    } else if constexpr (B == 2) {
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;"
                     : "=d"(v[0]), "=d"(v[1]) : "l"(p), "l"(pol));
    } else {
#pragma unroll
        for (int k = 0; k < B; k += 4)
            asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f64 {%0,%1,%2,%3}, [%4], %5;"
                         : "=d"(v[k]), "=d"(v[k + 1]), "=d"(v[k + 2]), "=d"(v[k + 3]) : "l"(p + k), "l"(pol));
    }
}

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

// Per-thread check accumulators of B members.
template <int B>
struct CheckAcc {
    double sy[B], sx[B], sd[B], md[B], mx[B];
    __device__ __forceinline__ CheckAcc() {
#pragma unroll
        for (int b = 0; b < B; ++b) sy[b] = sx[b] = sd[b] = md[b] = mx[b] = 0.0;
    }
    __device__ __forceinline__ void add(int b, double y, double x, double id) {
        const double df = fabs(y - x);
        sy[b] += y; sx[b] += x; sd[b] += df; md[b] = fmax(md[b], df / id); mx[b] = fmax(mx[b], x);
    }
};

// CTA-level deterministic reduction of the check quantities of B members into
// partials[blockIdx.x][b]; NW = warps in the CTA (all threads must call it).
template <int NW, int B>
__device__ __forceinline__ void cta_check_partials(const CheckAcc<B>& c, double* partials) {
    __shared__ double red[NW][5];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll 1
    for (int b = 0; b < B; ++b) {
        const double sy = warp_sum(c.sy[b]), sx = warp_sum(c.sx[b]), sd = warp_sum(c.sd[b]);
        const double md = warp_max(c.md[b]), mx = warp_max(c.mx[b]);
        if (lane == 0) { red[w][0] = sy; red[w][1] = sx; red[w][2] = sd; red[w][3] = md; red[w][4] = mx; }
        __syncwarp();      // converged warps at the aligned CTA barrier (compute-sanitizer synccheck)
        __syncthreads();
        if (threadIdx.x == 0) {
            double a = 0, bb = 0, cc = 0, d = 0, e = 0;
            for (int i = 0; i < NW; ++i) {
                a += red[i][0]; bb += red[i][1]; cc += red[i][2];
                d = fmax(d, red[i][3]); e = fmax(e, red[i][4]);
            }
            double* o = partials + ((size_t)blockIdx.x * B + b) * kPartials;
            o[0] = a; o[1] = bb; o[2] = cc; o[3] = d; o[4] = e; o[5] = 0; o[6] = 0; o[7] = 0;
        }
        __syncwarp();
        __syncthreads();
    }
}

template <int B>
__device__ __forceinline__ void store_vec(double* dst, const double (&yv)[B]) {
    if constexpr (B == 1) {
        dst[0] = yv[0];
    } else if constexpr (B == 2) {
        *reinterpret_cast<double2*>(dst) = make_double2(yv[0], yv[1]);
    } else {
#pragma unroll
        for (int k = 0; k < B; k += 4)
            asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(dst + k), "d"(yv[k]), "d"(yv[k + 1]),
                         "d"(yv[k + 2]), "d"(yv[k + 3])
                         : "memory");
    }
}

// Epilogue of one row shared by all SELL kernels: band term, damping, pending
// scale, store, check terms.  acc = sum_t val x[col]; lo/up/id = the slot's
// B-vectors; xo/yo = x-span bases shifted to the own rows (member-minor).
// Own-row and band loads of row r (issued before the gathers by callers that
// want them in flight together).
template <int B, bool BAND>
struct RowX {
    double xl[B], xu[B], xr[B];
    __device__ __forceinline__ void load(const double* xo, int64_t r) {
        if (BAND) {
            ld_vec<B>(xo + (r - 1) * B, xl);
            ld_vec<B>(xo + (r + 1) * B, xu);
        }
        // x_r unconditionally: a guarded load could not be hoisted next to the
        // gathers (measured 3% slower on cfg4); it shares their L1/L2 lines
        ld_vec<B>(xo + r * B, xr);
    }
};

template <int B, bool BAND, bool CHECK>
__device__ __forceinline__ void finish_row_x(const StepArgs& a, int64_t r, double* yo, const double (&acc)[B],
                                             const double (&lo)[B], const double (&up)[B], const double (&id)[B],
                                             const double* pre_scale, CheckAcc<B>& ck, const RowX<B, BAND>& X) {
    const double(&xl)[B] = X.xl;
    const double(&xu)[B] = X.xu;
    const double(&xr)[B] = X.xr;
    const bool damp = a.omega != 1.0;
    double yv[B];
    const bool unif = a.unif_lam_inv != 0.0;
#pragma unroll
    for (int b = 0; b < B; ++b) {
        const double s = BAND ? fma(lo[b], xl[b], up[b] * xu[b]) + acc[b] : acc[b];
        double y = damp ? fma(1.0 - a.omega, xr[b], a.omega * (id[b] * s)) : id[b] * s;
        if (unif) {   // transient: (I + A/Lambda) x with a_rr = -1/id
            y = fma(a.unif_lam_inv, s - xr[b] / id[b], xr[b]);
            double* ac = a.acc + (a.own_off + r) * B + b;
            *ac = fma(a.acc_w, xr[b], *ac);
        }
        double x = (damp || CHECK) ? xr[b] : 0.0;
        if (pre_scale != nullptr) {
            const double sc = pre_scale[b];
            y *= sc;
            x *= sc;
        }
        yv[b] = y;
        if (CHECK) ck.add(b, y, x, id[b]);
    }
    store_vec<B>(yo + r * B, yv);
    for (int p = 0; p < a.npush; ++p)   // halo rows straight into the peer's buffer
        if (r >= a.push_lo[p] && r < a.push_hi[p]) store_vec<B>(a.push_y[p] + r * B, yv);
}

template <int B, bool BAND, bool CHECK>
__device__ __forceinline__ void finish_row(const StepArgs& a, int64_t r, const double* xo, double* yo,
                                           const double (&acc)[B], const double (&lo)[B], const double (&up)[B],
                                           const double (&id)[B], const double* pre_scale, CheckAcc<B>& ck) {
    RowX<B, BAND> X;
    X.load(xo, r);
    finish_row_x<B, BAND, CHECK>(a, r, yo, acc, lo, up, id, pre_scale, ck, X);
}

// Check decision (readings R2-R5), per member.
// all holds one [B][8] record per rank, combined in rank order.  Runs on one
// thread (decide_kernel, or the last-arriving CTA of the resident kernel).
static __device__ __noinline__ void decide_apply(const double* all, int nranks, Ctrl* c, int32_t len, int32_t final_partial) {
    const int B = c->batch;
    const int64_t k = c->iter + len;
    c->iter = k;
    bool numeric = false, running = false;
    for (int b = 0; b < B; ++b) {
        double s = 0, sx = 0, sd = 0, md = 0, mx = 0;
        for (int r = 0; r < nranks; ++r) {
            const double* p = all + ((size_t)r * B + b) * 8;
            s += p[0]; sx += p[1]; sd += p[2]; md = fmax(md, p[3]); mx = fmax(mx, p[4]);
        }
        const double delta = sd / sx;
        const double resid = md / (c->omega * c->norm_inf[b] * mx);
        c->mass[b] = s;
        c->delta[b] = delta;
        c->resid[b] = resid;
        if (!(s > 0.0) || isinf(s) || isnan(delta)) {
            c->mstatus[b] = CME_ERR_NUMERIC;
            c->miters[b] = k;
            numeric = true;
            continue;
        }
        c->inv_s[b] = 1.0 / s;  // L1 normalisation, applied by the next step (R5)
        if (final_partial || c->mstatus[b] != -1) continue;
        const double crit = c->stop_mode == CME_STOP_DELTA_L1 ? delta : resid;
        if (crit <= c->tol) {
            c->mstatus[b] = CME_OK;
            c->miters[b] = k;
        } else if (c->stag_tol > 0.0 && k >= 2 * c->C &&
                   fabs(delta - c->delta_prev[b]) <= c->stag_tol * c->delta_prev[b]) {
            c->mstatus[b] = CME_STAGNATED;
            c->miters[b] = k;
        } else {
            c->delta_prev[b] = delta;
            running = true;
        }
    }
    int32_t overall = -1;
    if (numeric) {
        overall = CME_ERR_NUMERIC;
    } else if (final_partial || (running && k >= c->max_iter)) {
        overall = CME_NOT_CONVERGED;
    } else if (!running) {
        overall = CME_OK;
        for (int b = 0; b < B; ++b)
            if (c->mstatus[b] == CME_STAGNATED) overall = CME_STAGNATED;
    }
    if (overall != -1) {
        for (int b = 0; b < B; ++b)
            if (c->mstatus[b] == -1) { c->mstatus[b] = CME_NOT_CONVERGED; c->miters[b] = k; }
        c->status = overall;
        c->stop = 1;
    }
}

// ILP chunk (t-steps whose loads are issued together) for a batch width.
template <int B>
struct Chunk {
    static constexpr int U = B >= 8 ? 1 : 8 / B;
};

// Sum over the W ELL entries of one slot: all stream loads, then all gathers,
// then the FMAs in t order (W known at compile time: no predicated-off slots).
template <int B, int W>
__device__ __forceinline__ void ell_row_global(const StepArgs& a, int64_t base, uint64_t pol, double (&acc)[B]) {
    double v[W][B], xv[W][B];
    int32_t c[W];
#pragma unroll
    for (int u = 0; u < W; ++u) {
        const int64_t e = base + 32 * (int64_t)u;
        ld_stream_vec<B>(a.val + e * B, pol, v[u]);
        c[u] = ld_stream(a.col + e, pol);
    }
#pragma unroll
    for (int u = 0; u < W; ++u) ld_vec<B>(a.x + (int64_t)c[u] * B, xv[u]);
#pragma unroll
    for (int u = 0; u < W; ++u)
#pragma unroll
        for (int b = 0; b < B; ++b) acc[b] = fma(v[u][b], xv[u][b], acc[b]);
}

template <int B, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(kCta) sell_step_kernel(const StepArgs a) {
    pdl_trigger();
    pdl_wait();
    if (a.stop != nullptr && *a.stop) return;
    const uint64_t pol = evict_first_policy();
    const int lane = threadIdx.x & 31;
    const int64_t q = a.slice_begin + (int64_t)blockIdx.x * kWarpsPerCta + (threadIdx.x >> 5);
    CheckAcc<B> ck;
    if (q < a.slice_end) {
        const int64_t slot = q * 32 + lane;
        const int w = __ldg(a.slice_w + q);
        const int64_t base = __ldg(a.slice_off + q) + lane;
        if (slot < a.n_rows) {
            const int64_t r = REARR ? (int64_t)ld_stream(a.row_of + slot, pol) : slot;
            double acc[B];
#pragma unroll
            for (int b = 0; b < B; ++b) acc[b] = 0.0;
            constexpr int U = Chunk<B>::U;
            switch (B == 1 ? w : -1) {   // warp-uniform exact widths for the common B = 1 case
                case 0: break;
                case 1: ell_row_global<B, 1>(a, base, pol, acc); break;
                case 2: ell_row_global<B, 2>(a, base, pol, acc); break;
                case 3: ell_row_global<B, 3>(a, base, pol, acc); break;
                case 4: ell_row_global<B, 4>(a, base, pol, acc); break;
                case 5: ell_row_global<B, 5>(a, base, pol, acc); break;
                case 6: ell_row_global<B, 6>(a, base, pol, acc); break;
                case 7: ell_row_global<B, 7>(a, base, pol, acc); break;
                case 8: ell_row_global<B, 8>(a, base, pol, acc); break;
                default:
                    for (int t0 = 0; t0 < w; t0 += U) {
                        double v[U][B], xv[U][B];
                        int32_t c[U];
#pragma unroll
                        for (int u = 0; u < U; ++u)
                            if (t0 + u < w) {
                                const int64_t e = base + 32 * (int64_t)(t0 + u);
                                ld_stream_vec<B>(a.val + e * B, pol, v[u]);
                                c[u] = ld_stream(a.col + e, pol);
                            }
#pragma unroll
                        for (int u = 0; u < U; ++u)
                            if (t0 + u < w) ld_vec<B>(a.x + (int64_t)c[u] * B, xv[u]);
#pragma unroll
                        for (int u = 0; u < U; ++u)
                            if (t0 + u < w)
#pragma unroll
                                for (int b = 0; b < B; ++b) acc[b] = fma(v[u][b], xv[u][b], acc[b]);
                    }
            }
            double lo[B], up[B], id[B];
            if (BAND) {
                ld_stream_vec<B>(a.lo + slot * B, pol, lo);
                ld_stream_vec<B>(a.up + slot * B, pol, up);
            }
            ld_stream_vec<B>(a.inv_d + slot * B, pol, id);
            finish_row<B, BAND, CHECK>(a, r, a.x + a.own_off * B, a.y + a.own_off * B, acc, lo, up, id,
                                       a.pre_scale, ck);
        }
    }
    if (CHECK) cta_check_partials<kWarpsPerCta, B>(ck, a.partials);
}

// Plain CSR arm (ablation, CME_FMT_CSR, B = 1): one thread per row.
template <bool CHECK>
__global__ void __launch_bounds__(kCta) csr_step_kernel(const StepArgs a) {
    pdl_trigger();
    pdl_wait();
    if (a.stop != nullptr && *a.stop) return;
    const int64_t r = a.slice_begin * 32 + (int64_t)blockIdx.x * kCta + threadIdx.x;
    CheckAcc<1> ck;
    if (r < a.n_rows && r < a.slice_end * 32) {
        const int64_t b = __ldg(a.csr_rp + r), e = __ldg(a.csr_rp + r + 1);
        double acc[1] = {0.0};
        for (int64_t p = b; p < e; ++p) acc[0] = fma(__ldg(a.csr_v + p), __ldg(a.x + __ldg(a.csr_ci + p)), acc[0]);
        const double id[1] = {__ldg(a.inv_d + r)}, z[1] = {0.0};
        finish_row<1, false, CHECK>(a, r, a.x + a.own_off, a.y + a.own_off, acc, z, z, id, a.pre_scale, ck);
    }
    if (CHECK) cta_check_partials<kWarpsPerCta, 1>(ck, a.partials);
}

}  // namespace cme
