// SMEM-resident persistent Jacobi kernel for problems whose packed matrix fits
// in the shared memory of the whole GPU (148 SMs x ~225 KB = 33 MB: up to
// ~450K CME states; config 2, the ~100K-state toggle switch, is 7 MB).
//
// Same arithmetic as sell_step_kernel (eq. 8 with relaxation omega, R1;
// FMAs in t order, identical rounding), but one launch runs many iterations:
//
// * each CTA (1024 threads, one per SM, cooperative launch => all resident)
//   owns a fixed, window-aligned, contiguous run of rows; it copies that run's
//   val/col/inv_d/row_of/lo/up into shared memory ONCE, so an iteration reads
//   only the iterate x from L2;
// * no barrier or flag between CTAs per iteration: the iterate carries its own
//   epoch.  Probabilities are >= +0 (every term of eq. 8 is non-negative), so
//   the sign bit is free: step k (of this launch) stores its y with the sign
//   of epoch m = (k+1)/2 -- the m-th write into that buffer of the double
//   buffer (m odd: negative).  A gather of x[c] for step k expects epoch k/2
//   and re-loads (ld.relaxed.gpu, L2) until the sign matches, then uses |x|.
//   RAW is thus carried by the data itself (an 8-byte store is single-copy
//   atomic).  WAR (step k overwrites the buffer neighbours read in step k-1)
//   holds because every CTA finishes ALL its gathers of a step (one CTA
//   barrier) before storing any row of it, and observes a step-(k-1) output
//   of every CTA that reads its rows -- which proves that CTA finished its
//   step-(k-1) gathers: through its own gathers when it also reads that
//   CTA's rows, else through one extra "probe" load of that CTA's first row;
// * every C-th step (and the last step of a solve cut short by max_iter) the
//   CTAs write their check partials and meet at one grid barrier whose last
//   arriver reduces the partials in CTA order and runs decide_apply (the same
//   decision code as decide_kernel), then releases the generation; all CTAs
//   read stop / the pending 1/sum(y) from the control block;
// * at the end of a launch (after one more grid barrier) each CTA rewrites its
//   own rows: the final iterate positive, the other buffer -0.0, which is the
//   state the next launch (or write_out) expects.
//
// Every spin is bounded by a %globaltimer deadline: a lost CTA turns the solve
// into CME_ERR_TIMEOUT ("resident kernel timed out"), never a hung GPU.
#pragma once
#include "kernels.cuh"

namespace cme {

constexpr int kResThreads = 1024;
constexpr int kResWarps = kResThreads / 32;

struct ResArgs {
    int64_t n_rows;
    const int64_t* slice_off;
    const int32_t* slice_w;
    const double* val;
    const int32_t* col;
    const int32_t* row_of;
    const double* lo;
    const double* up;
    const double* inv_d;
    double* xb0;             // iterate buffers (x-span bases, zero sentinel on each side)
    double* xb1;
    const int32_t* cta_q;    // [G+1] slice cuts
    const int32_t* cta_row;  // [G+1] first own row of each CTA (cta_row[G] = n)
    const int32_t* probe_off;   // [G+1] CSR offsets into probe
    const int32_t* probe;       // CTAs that read CTA b's rows but whose rows b does not read
    uint32_t* sync;          // [0] grid-barrier arrivals, [1] released generation (zeroed)
    double* partials;        // [G][kPartials]
    Ctrl* ctrl;
    int64_t nsteps;          // steps to run (stops earlier when ctrl->stop is set by a check)
    int64_t C;               // check interval
    double omega;
    int32_t start;           // buffer holding the current iterate (positive; the other is negative)
    int32_t solve;           // 1: the last step is a (partial) check block end (max_iter)
    int64_t timeout_ns;
};

__device__ __forceinline__ uint64_t global_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// iterate accesses: strong (relaxed, gpu scope) -- coherent in L2, no stale L1.
// CME_RES_LD (A/B builds only): 1 = ld.global.cg, 2 = ld.volatile.global.
#ifndef CME_RES_LD
#define CME_RES_LD 0
#endif
__device__ __forceinline__ double ld_x(const double* p) {
    double v;
    if (CME_RES_LD == 1)
        asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    else if (CME_RES_LD == 2)
        asm volatile("ld.volatile.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    else
        asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_x(double* p, double v) {
    asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
__device__ __forceinline__ bool neg_bit(double v) { return __double_as_longlong(v) < 0; }
__device__ __forceinline__ double with_sign(double v, bool neg) {
    const long long b = __double_as_longlong(v) & 0x7fffffffffffffffLL;
    return __longlong_as_double(neg ? (b | (long long)0x8000000000000000ULL) : b);
}
// |x[p]| once its epoch sign is `neg` (re-load until then; `bad` after
// `timeout` ns).  The clock is read only on the slow path: the fast path is
// one sign test.
__device__ __forceinline__ double settle(const double* p, double v, bool neg, uint64_t timeout, bool& bad) {
    if (neg_bit(v) != neg) {
        const uint64_t t0 = global_ns();
        do {
            v = ld_x(p);
            if (global_ns() - t0 > timeout) { bad = true; break; }
        } while (neg_bit(v) != neg);
    }
    return fabs(v);
}

// Shared-memory image of one CTA's run of slices.
struct ResSmem {
    double* val;      // [nval], slice-relative layout of the packed val
    double* inv_d;    // [rows]
    double* lo;       // [rows] (band)
    double* up;
    int32_t* col;     // [nval]
    int32_t* row_of;  // [rows] (rearrangement)
    int32_t* w;       // [nsl] slice width
    int32_t* off;     // [nsl] slice offset relative to the run
};

// Bytes of the shared-memory image (host and device agree).
__host__ __device__ inline int64_t res_smem_bytes(int64_t nval, int64_t nsl, bool band, bool rearr) {
    const int64_t rows = 32 * nsl;
    return 8 * nval + 8 * rows * (band ? 3 : 1) + 4 * nval + (rearr ? 4 * rows : 0) + 8 * nsl;
}

// sum_t val_t |x[col_t]| over W entries of a slot (W known: no predicated-off
// slots), all gathers in flight before the epoch checks and the FMAs (t
// order: the register kernel's rounding).
template <int W>
__device__ __forceinline__ double res_ell(const double* sval, const int32_t* scol, int base, const double* x,
                                          bool neg, uint64_t dl, bool& bad) {
    int32_t c[W];
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) c[u] = scol[base + 32 * u];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = ld_x(x + c[u]);
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(sval[base + 32 * u], settle(x + c[u], xv[u], neg, dl, bad), acc);
    return acc;
}

// y of row slot (local slice ql, lane) from the epoch-checked iterate x
// (dl = the per-spin timeout in ns).
template <bool BAND, bool REARR>
__device__ __forceinline__ double res_row(const ResArgs& a, const ResSmem& s, int ql, int64_t slot, const double* x,
                                          bool neg, double sc, uint64_t dl, bool& bad, int64_t& r, double& xr_out,
                                          double& id_out) {
    const int lane = threadIdx.x & 31;
    const int sl = ql * 32 + lane;
    const int w = s.w[ql];
    const int base = s.off[ql] + lane;
    r = REARR ? (int64_t)s.row_of[sl] : slot;
    // own/band loads first, in flight with the gathers (band rows outside
    // [0, n) are the zero sentinels: never written, never epoch-checked)
    const bool has_l = BAND && r > 0, has_u = BAND && r + 1 < a.n_rows;
    double xr = ld_x(x + r), xl = 0.0, xu = 0.0;
    if (has_l) xl = ld_x(x + r - 1);
    if (has_u) xu = ld_x(x + r + 1);
    double acc;
    switch (w) {   // warp-uniform
        case 0: acc = 0.0; break;
        case 1: acc = res_ell<1>(s.val, s.col, base, x, neg, dl, bad); break;
        case 2: acc = res_ell<2>(s.val, s.col, base, x, neg, dl, bad); break;
        case 3: acc = res_ell<3>(s.val, s.col, base, x, neg, dl, bad); break;
        case 4: acc = res_ell<4>(s.val, s.col, base, x, neg, dl, bad); break;
        case 5: acc = res_ell<5>(s.val, s.col, base, x, neg, dl, bad); break;
        case 6: acc = res_ell<6>(s.val, s.col, base, x, neg, dl, bad); break;
        case 7: acc = res_ell<7>(s.val, s.col, base, x, neg, dl, bad); break;
        case 8: acc = res_ell<8>(s.val, s.col, base, x, neg, dl, bad); break;
        default: {
            acc = 0.0;
            int t = 0;
            for (; t + 4 <= w; t += 4) {
                int32_t c[4];
                double xv[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) c[u] = s.col[base + 32 * (t + u)];
#pragma unroll
                for (int u = 0; u < 4; ++u) xv[u] = ld_x(x + c[u]);
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    acc = fma(s.val[base + 32 * (t + u)], settle(x + c[u], xv[u], neg, dl, bad), acc);
            }
            for (; t < w; ++t) {
                const double* p = x + s.col[base + 32 * t];
                acc = fma(s.val[base + 32 * t], settle(p, ld_x(p), neg, dl, bad), acc);
            }
        }
    }
    xr = settle(x + r, xr, neg, dl, bad);
    if (has_l) xl = settle(x + r - 1, xl, neg, dl, bad);
    if (has_u) xu = settle(x + r + 1, xu, neg, dl, bad);
    const double id = s.inv_d[sl];
    const double sm = BAND ? fma(s.lo[sl], xl, s.up[sl] * xu) + acc : acc;
    double yv = a.omega != 1.0 ? fma(1.0 - a.omega, xr, a.omega * (id * sm)) : id * sm;
    yv *= sc;
    xr_out = xr * sc;
    id_out = id;
    return yv;
}

// Grid barrier over the co-resident CTAs (generation `gen`, 1-based).  The
// last CTA to arrive runs `last(tid)` with the whole CTA, then releases.
// Returns false on timeout.  All threads of every CTA must call it.
template <typename Last>
__device__ __forceinline__ bool res_grid_barrier(uint32_t* sync, uint32_t gen, uint64_t deadline, int* s_flag,
                                                 Last last) {
    const int tid = threadIdx.x;
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        const uint32_t old = atomicAdd(sync, 1u);
        s_flag[0] = old == gen * gridDim.x - 1;
        s_flag[1] = 0;
    }
    __syncthreads();
    if (s_flag[0]) {
        __threadfence();
        last(tid);   // contains its own CTA barriers
        if (tid == 0) {
            __threadfence();
            st_release_u32(sync + 1, gen);
        }
    } else if (tid == 0) {
        int spins = 0;
        while (ld_acquire_u32(sync + 1) < gen)
            if ((++spins & 255) == 0 && global_ns() > deadline) { s_flag[1] = 1; break; }
    }
    __syncthreads();
    return s_flag[1] == 0;
}

// R = row slots per thread (slices per CTA <= 32 R).
template <bool BAND, bool REARR, int R>
__global__ void __launch_bounds__(kResThreads, 1) sell_resident_kernel(const ResArgs a) {
    extern __shared__ __align__(16) double res_smem[];
    __shared__ double s_rec[kPartials];
    __shared__ double s_red[kResWarps][5];
    __shared__ int s_flag[2];
    const int G = gridDim.x, b = blockIdx.x, tid = threadIdx.x, lane = tid & 31, wp = tid >> 5;
    const int64_t q0 = a.cta_q[b];
    const int nsl = a.cta_q[b + 1] - a.cta_q[b];
    const int64_t e0 = a.slice_off[q0];
    const int nval = (int)(a.slice_off[q0 + nsl] - e0);
    const int rows = 32 * nsl;
    ResSmem s;
    s.val = res_smem;
    s.inv_d = s.val + nval;
    s.lo = s.inv_d + rows;
    s.up = s.lo + (BAND ? rows : 0);
    s.col = reinterpret_cast<int32_t*>(s.up + (BAND ? rows : 0));
    s.row_of = s.col + nval;
    s.w = s.row_of + (REARR ? rows : 0);
    s.off = s.w + nsl;
    {   // the CTA's matrix run -> shared memory, once per launch
        const uint64_t pol = evict_first_policy();
        for (int i = tid; i < nval; i += kResThreads) {
            s.val[i] = ld_stream(a.val + e0 + i, pol);
            s.col[i] = ld_stream(a.col + e0 + i, pol);
        }
        const int64_t s0 = q0 * 32;
        for (int i = tid; i < rows; i += kResThreads) {
            s.inv_d[i] = __ldg(a.inv_d + s0 + i);
            if (BAND) { s.lo[i] = __ldg(a.lo + s0 + i); s.up[i] = __ldg(a.up + s0 + i); }
            if (REARR) s.row_of[i] = __ldg(a.row_of + s0 + i);
        }
        for (int i = tid; i < nsl; i += kResThreads) {
            s.w[i] = __ldg(a.slice_w + q0 + i);
            s.off[i] = (int32_t)(__ldg(a.slice_off + q0 + i) - e0);
        }
    }
    // probe: thread tid < nprobe checks the first row of one reader CTA that
    // this CTA's gathers do not already observe
    const int p0 = a.probe_off[b], nprobe = a.probe_off[b + 1] - p0;
    const int64_t probe = tid < nprobe ? (int64_t)a.cta_row[a.probe[p0 + tid]] : -1;
    const int64_t it0 = *(volatile const int64_t*)&a.ctrl->iter;
    double sc = *(volatile const double*)&a.ctrl->inv_s[0];   // pending 1/sum(y) (R5)
    uint32_t gen = 0;
    bool timed_out = false;
    __syncthreads();
    int64_t k = 0;
    while (k < a.nsteps) {
        const uint64_t dl = (uint64_t)a.timeout_ns;   // per-spin budget (settle)
        const int src = (int)((a.start + k) & 1);
        const double* x = src ? a.xb1 : a.xb0;
        double* y = src ? a.xb0 : a.xb1;
        const bool in_neg = (k >> 1) & 1, out_neg = ((k + 1) >> 1) & 1;
        const int64_t done = it0 + k + 1;
        const bool full = done % a.C == 0;
        const bool check = full || (a.solve && k + 1 == a.nsteps);
        bool bad = false;
#ifndef CME_RES_NOPROBE   // (A/B measurement only: without probes WAR is not guaranteed)
        if (probe >= 0) (void)settle(x + probe, ld_x(x + probe), in_neg, dl, bad);
#endif
        double yv[R], xr[R], id[R];
        int64_t rr[R];
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const int ql = wp + kResWarps * j;
            const int64_t slot = (q0 + ql) * 32 + lane;
            rr[j] = -1;
            if (ql < nsl && slot < a.n_rows)
                yv[j] = res_row<BAND, REARR>(a, s, ql, slot, x, in_neg, sc, dl, bad, rr[j], xr[j], id[j]);
        }
        // every gather/probe of this step done CTA-wide before any store (WAR)
        if (__syncthreads_or(bad)) { timed_out = true; break; }
        if (check) {
            CheckAcc<1> ck;
#pragma unroll
            for (int j = 0; j < R; ++j)
                if (rr[j] >= 0) ck.add(0, yv[j], xr[j], id[j]);
            cta_check_partials<kResWarps, 1>(ck, a.partials);
        }
#pragma unroll
        for (int j = 0; j < R; ++j)
            if (rr[j] >= 0) st_x(y + rr[j], with_sign(yv[j], out_neg));
        sc = 1.0;
        ++k;
        if (!check) continue;
        // grid-wide check: the last CTA to arrive reduces the partials in CTA
        // order and decides
        const int32_t len = full ? (int32_t)a.C : (int32_t)(done % a.C);
        const bool ok = res_grid_barrier(a.sync, ++gen, global_ns() + dl, s_flag, [&](int t) {
            double v0 = 0, v1 = 0, v2 = 0, v3 = 0, v4 = 0;
            for (int i = t; i < G; i += kResThreads) {
                const double* p = a.partials + (size_t)i * kPartials;
                v0 += __ldcg(p); v1 += __ldcg(p + 1); v2 += __ldcg(p + 2);
                v3 = fmax(v3, __ldcg(p + 3)); v4 = fmax(v4, __ldcg(p + 4));
            }
            v0 = warp_sum(v0); v1 = warp_sum(v1); v2 = warp_sum(v2); v3 = warp_max(v3); v4 = warp_max(v4);
            if ((t & 31) == 0) {
                s_red[t >> 5][0] = v0; s_red[t >> 5][1] = v1; s_red[t >> 5][2] = v2;
                s_red[t >> 5][3] = v3; s_red[t >> 5][4] = v4;
            }
            __syncthreads();
            if (t == 0) {
                double r0 = 0, r1 = 0, r2 = 0, r3 = 0, r4 = 0;
                for (int i = 0; i < kResWarps; ++i) {
                    r0 += s_red[i][0]; r1 += s_red[i][1]; r2 += s_red[i][2];
                    r3 = fmax(r3, s_red[i][3]); r4 = fmax(r4, s_red[i][4]);
                }
                s_rec[0] = r0; s_rec[1] = r1; s_rec[2] = r2; s_rec[3] = r3; s_rec[4] = r4;
                s_rec[5] = s_rec[6] = s_rec[7] = 0.0;
                if (!a.ctrl->stop) decide_apply(s_rec, 1, a.ctrl, len, full ? 0 : 1);
            }
        });
        if (!ok) { timed_out = true; break; }
        const int32_t stop = *(volatile const int32_t*)&a.ctrl->stop;
        sc = *(volatile const double*)&a.ctrl->inv_s[0];
        __syncthreads();   // everyone read stop/sc before the next check can rewrite them
        if (stop) break;
    }
    if (!timed_out) {
        // nobody reads the iterate any more: own rows of the final buffer
        // positive, of the other buffer -0.0 (the next launch's state)
        const uint64_t dl = global_ns() + (uint64_t)a.timeout_ns;
        if (res_grid_barrier(a.sync, ++gen, dl, s_flag, [](int) {})) {
            const int src = (int)((a.start + k) & 1);
            double* xf = src ? a.xb1 : a.xb0;
            double* xo = src ? a.xb0 : a.xb1;
            for (int64_t r = a.cta_row[b] + tid; r < a.cta_row[b + 1]; r += kResThreads) {
                st_x(xf + r, fabs(ld_x(xf + r)));
                st_x(xo + r, -0.0);
            }
        } else {
            timed_out = true;
        }
    }
    if (timed_out && tid == 0) {
        a.ctrl->status = CME_ERR_TIMEOUT;
        a.ctrl->stop = 1;
    }
}

}  // namespace cme
