// TMA-staged step kernel over the COMPACT encoding of layout v0 (B = 1;
// DESIGN.md sec. 5b).  Same operator as sell_tma_kernel -- y = M_omega x with
// M = |D|^-1 O (eq. 8, R1) -- but the packed matrix is stored as the
// rows of M itself, so a plain step streams
//   val_c  8 B / ELL slot   (a_rj / (-a_rr), one IEEE division at pack time)
//   col16  2 B / ELL slot   (j - r: the RCM / DFS bands of the CME networks
//                            keep every offset inside int16)
//   row8   1 B / row        (r - window base, rearranged packs only)
//   lo_c, up_c              (band only)
// instead of 12 B / slot + 12 B / row: inv_d is read only by CHECK steps (the
// paper residual needs |a_rr|, R21) and by transient steps.  The arithmetic
// order is the plain kernel's (gathers in t order, band term first), with the
// division moved from the row sum to the entries: per-row relative difference
// <= (k + 2) u, inside the per-SpMV bound of DESIGN.md sec. 6.
#pragma once
#include "kernels_tma.cuh"

#ifndef CME_ABL   // kernel ablation level for dev A/B builds only (tools/gpu_abl.sh); 0 = the product kernel
#define CME_ABL 0
#endif

namespace cme {

struct CptArgs {
    TmaArgs T;            // T.a.val / lo / up = the compact arrays, T.a.inv_d = 1/(-a_rr)
    const int16_t* col16;
    const uint8_t* row8;
    int32_t win_shift;    // log2(rearrangement window), 0 = identity slot -> row
};

// Stage layout: [row8 if REARR][lo, up if BAND][val][col16] for NCW*32 slots.
__host__ __device__ inline int cpt_fixed_bytes(int ncw, bool band, bool rearr) {
    return ncw * 32 * ((rearr ? 1 : 0) + (band ? 16 : 0));
}

template <int NCW, bool BAND, bool REARR>
__device__ __noinline__ void cpt_issue_call(unsigned char* st, uint64_t* bar, const int64_t* slice_off,
                                            int64_t slice_end, const uint8_t* row8, const double* lo,
                                            const double* up, const double* val, const int16_t* col16,
                                            int off_val, int off_col, int64_t tile, uint64_t pol,
                                            const int2* tile_meta) {
    constexpr int kSlots = NCW * 32;
    constexpr int kOffRow = 0, kOffLo = REARR ? kSlots : 0, kOffUp = kOffLo + 8 * kSlots;
    const int64_t q0 = tile * NCW;
    const int64_t q1 = min(q0 + NCW, slice_end);
    const int64_t e0 = slice_off[q0], e1 = slice_off[q1];
    const uint32_t slots = (uint32_t)(q1 - q0) * 32u;
    const uint32_t nval = (uint32_t)(e1 - e0);
    uint32_t bytes = nval * 10u + meta_stride(NCW) * 8u;
    if (REARR) bytes += slots;
    if (BAND) bytes += slots * 16u;
    mbar_expect_tx(bar, bytes);
    issue_meta(st, bar, tile_meta, tile, NCW, pol);
    st += kMetaBytes;
    if (REARR) bulk_g2s(st + kOffRow, row8 + q0 * 32, slots, bar, pol);
    if (BAND) {
        bulk_g2s(st + kOffLo, lo + q0 * 32, slots * 8u, bar, pol);
        bulk_g2s(st + kOffUp, up + q0 * 32, slots * 8u, bar, pol);
    }
    if (nval) {
        bulk_g2s(st + off_val, val + e0, nval * 8u, bar, pol);
        bulk_g2s(st + off_col, col16 + e0, nval * 2u, bar, pol);
    }
}

template <int NCW, bool BAND, bool REARR>
__device__ __forceinline__ void cpt_issue(const CptArgs& K, unsigned char* smem, uint64_t* full, int64_t tile, int s,
                                          uint64_t pol) {
    const StepArgs& a = K.T.a;
    if (K.T.xpf) {
        const int64_t r0 = tile * NCW * 32, r1 = min(r0 + NCW * 32, a.n_rows);
        if (r1 > r0) prefetch_l2(a.x + a.own_off + r0, (uint64_t)(r1 - r0) * 8);
    }
    cpt_issue_call<NCW, BAND, REARR>(smem + (size_t)s * K.T.stage_bytes, &full[s], a.slice_off, a.slice_end, K.row8,
                                     a.lo, a.up, a.val, K.col16, K.T.off_val, K.T.off_col, tile, pol, a.tile_meta);
}

// Sum over the W entries of one slot: all gathers x[r + dj] first, then the
// FMAs in t order.
template <int W>
__device__ __forceinline__ void ell_row_cpt(const int16_t* scol, const double* sval, const double* xr, double& acc) {
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = __ldg(xr + scol[32 * u]);
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(sval[32 * u], xv[u], acc);
}

template <int NCW, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(TmaShape<NCW>::kThreads, TmaShape<NCW>::kMinBlocks)
    sell_cpt_kernel(const CptArgs K) {
    constexpr int kConsumers = NCW, kTileSlices = NCW, kSlots = NCW * 32;
    constexpr int kOffRow = 0, kOffLo = REARR ? kSlots : 0, kOffUp = kOffLo + 8 * kSlots;
    const TmaArgs& T = K.T;
    const StepArgs& a = T.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int S = T.stages;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const bool producer = warp == kConsumers && lane == 0;
    uint64_t pol = 0;
    int64_t t_first, my_tiles, t_stride;
    tma_tile_range(T, &t_first, &my_tiles, &t_stride);
    const int64_t t_end = t_first + my_tiles * t_stride;
    const int pro = (int)(my_tiles < (int64_t)S ? my_tiles : (int64_t)S);
    if (producer) {   // the matrix is constant: prefetch while the previous step drains
        pol = evict_first_policy();
        for (int i = 0; i < pro; ++i) cpt_issue<NCW, BAND, REARR>(K, smem, full, t_first + (int64_t)i * t_stride, i, pol);
    }
    pdl_wait();
    if (a.stop != nullptr && *a.stop) {
        if (producer)
            for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        return;
    }
    CheckAcc<1> ck;
    if (warp == kConsumers) {
        if (lane == 0 && my_tiles > pro) {
            int s = 0;
            uint32_t phase = 1;
            for (int64_t tile = t_first + (int64_t)pro * t_stride; tile < t_end; tile += t_stride) {
                mbar_wait(&empty[s], phase ^ 1u);
                cpt_issue<NCW, BAND, REARR>(K, smem, full, tile, s, pol);
                if (++s == S) { s = 0; phase ^= 1u; }
            }
        }
    } else {
        // loop invariants hoisted and 32-bit slot/row indices, as in
        // sell_vi_kernel; the epilogue: y = (1-omega) x_r + omega (M x)_r, pending scale, check terms
        const double* xo = a.x + a.own_off;
        double* yo = a.y + a.own_off;
        const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end, ws = K.win_shift;
        const int stage_bytes = T.stage_bytes, off_val = T.off_val, off_col = T.off_col;
        const double om = a.omega, om1 = 1.0 - a.omega;
        const bool damp = om != 1.0, unif = a.unif_lam_inv != 0.0;
        const double sc = a.pre_scale != nullptr ? a.pre_scale[0] : 1.0;
        const int npush = a.npush;
        int s = 0;
        uint32_t phase = 0;
        for (int64_t tile = t_first; tile < t_end; tile += t_stride) {
            const unsigned char* st = smem + s * stage_bytes + kMetaBytes;
            mbar_wait(&full[s], phase);
            const int2 meta = reinterpret_cast<const int2*>(st - kMetaBytes)[warp];   // {offset in tile, width}
            const int q = (int)tile * kTileSlices + warp;
            const int slot = q * 32 + lane;
            if (q < slice_end && slot < n_rows) {
                const int ls = warp * 32 + lane;
                const double* sval = reinterpret_cast<const double*>(st + off_val) + meta.x + lane;
                const int16_t* scol = reinterpret_cast<const int16_t*>(st + off_col) + meta.x + lane;
                const int r = REARR ? ((slot >> ws) << ws) + st[kOffRow + ls] : slot;
                RowX<1, BAND> X;
                X.load(xo, r);
                const double* xr = xo + r;
                double acc = 0.0;
                switch (meta.y) {   // warp-uniform exact widths
                    case 0: break;
                    case 1: ell_row_cpt<1>(scol, sval, xr, acc); break;
                    case 2: ell_row_cpt<2>(scol, sval, xr, acc); break;
                    case 3: ell_row_cpt<3>(scol, sval, xr, acc); break;
                    case 4: ell_row_cpt<4>(scol, sval, xr, acc); break;
                    case 5: ell_row_cpt<5>(scol, sval, xr, acc); break;
                    case 6: ell_row_cpt<6>(scol, sval, xr, acc); break;
                    case 7: ell_row_cpt<7>(scol, sval, xr, acc); break;
                    case 8: ell_row_cpt<8>(scol, sval, xr, acc); break;
                    default:
                        for (int t0 = 0; t0 < meta.y; t0 += 8) {
                            double xv[8];
#pragma unroll
                            for (int u = 0; u < 8; ++u)
                                if (t0 + u < meta.y) xv[u] = __ldg(xr + scol[32 * (t0 + u)]);
#pragma unroll
                            for (int u = 0; u < 8; ++u)
                                if (t0 + u < meta.y) acc = fma(sval[32 * (t0 + u)], xv[u], acc);
                        }
                }
                const double sum = BAND ? fma(reinterpret_cast<const double*>(st + kOffLo)[ls], X.xl[0],
                                              reinterpret_cast<const double*>(st + kOffUp)[ls] * X.xu[0]) + acc
                                        : acc;
                const double x_r = X.xr[0];
                double y = damp ? fma(om1, x_r, om * sum) : sum;
                if (unif) {   // transient: x + (A x)_r / Lambda, (A x)_r = |a_rr| (s - x_r)
                    const double id = __ldg(a.inv_d + slot);
                    y = fma(a.unif_lam_inv, (sum - x_r) / id, x_r);
                    double* ac = a.acc + a.own_off + r;
                    *ac = fma(a.acc_w, x_r, *ac);
                }
                y *= sc;
                yo[r] = y;
                if (CHECK) ck.add(0, y, x_r * sc, __ldg(a.inv_d + slot));
                for (int p = 0; p < npush; ++p)   // halo rows straight into the peer's buffer
                    if (r >= a.push_lo[p] && r < a.push_hi[p]) a.push_y[p][r] = y;
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
            if (++s == S) { s = 0; phase ^= 1u; }
        }
    }
    if (CHECK) cta_check_partials<NCW + 1, 1>(ck, a.partials);
}

// ---------------------------------------------------------------------------
// Value-indexed variant (the CSR-VI idea): the rates of a
// mass-action CME take few distinct values (r_k times small binomials: 6 318
// on the 20M-state toggle switch), so an entry is a 16-bit index into a
// dictionary of O's distinct values held in shared memory plus the 16-bit
// column offset -- 4 B per ELL slot -- and inv_d stays a per-row stream.  The
// arithmetic is the layout-v0 kernel's exactly (same values, same FMA order,
// the row sum times inv_d), so results are bit-identical to it.
struct ViArgs {
    CptArgs K;             // K.T.a.inv_d per row; K.col16 / row8 / win_shift as the compact encoding
    const double* dict;    // [n_dict] ascending (padded to 16 B)
    const uint16_t* vidx;  // [n_ell]
    const uint16_t* loi;   // [n_slots] (band)
    const uint16_t* upi;
    int32_t dict_bytes;    // multiple of 128: stages start here in shared memory
    int32_t idpf;          // L2 prefetch of each tile's inv_d rows with the tile (CME_VI_IDPF)
};

// Stage layout: [row8 if REARR][loi, upi if BAND][vidx][col16].  inv_d is not
// staged: each lane streams its own 8 bytes from global memory next to its x
// loads, which keeps the stages small enough for a 4-deep ring next to the
// two dictionaries of an SM (measured: 3 stages 178 us vs 2 stages 206 us).
__host__ __device__ inline int vi_fixed_bytes(int ncw, bool band, bool rearr) {
    return ncw * 32 * ((rearr ? 1 : 0) + (band ? 4 : 0));
}

template <int TS, bool BAND, bool REARR>
__device__ __noinline__ void vi_issue_call(unsigned char* st, uint64_t* bar, const int64_t* slice_off,
                                           int64_t slice_end, const double* inv_d, const uint8_t* row8,
                                           const uint16_t* loi, const uint16_t* upi, const uint16_t* vidx,
                                           const int16_t* col16, int off_val, int off_col, int64_t tile,
                                           uint64_t pol, const int2* tile_meta) {
    constexpr int kSlots = TS * 32;
    constexpr int kOffRow = 0, kOffLo = kOffRow + (REARR ? kSlots : 0), kOffUp = kOffLo + 2 * kSlots;
    const int64_t q0 = tile * TS;
    const int64_t q1 = min(q0 + TS, slice_end);
    const int64_t e0 = slice_off[q0], e1 = slice_off[q1];
    const uint32_t slots = (uint32_t)(q1 - q0) * 32u;
    const uint32_t nval = (uint32_t)(e1 - e0);
    uint32_t bytes = nval * 4u + meta_stride(TS) * 8u;
    if (REARR) bytes += slots;
    if (BAND) bytes += slots * 4u;
    mbar_expect_tx(bar, bytes);
    issue_meta(st, bar, tile_meta, tile, TS, pol);
    st += meta_bytes(TS);
    if (REARR) bulk_g2s(st + kOffRow, row8 + q0 * 32, slots, bar, pol);
    if (BAND) {
        bulk_g2s(st + kOffLo, loi + q0 * 32, slots * 2u, bar, pol);
        bulk_g2s(st + kOffUp, upi + q0 * 32, slots * 2u, bar, pol);
    }
    if (nval) {
        bulk_g2s(st + off_val, vidx + e0, nval * 2u, bar, pol);
        bulk_g2s(st + off_col, col16 + e0, nval * 2u, bar, pol);
    }
}

template <int TS, bool BAND, bool REARR, int B = 1>
__device__ __forceinline__ void vi_issue(const ViArgs& V, unsigned char* stages, uint64_t* full, int64_t tile, int s,
                                         uint64_t pol) {
    const StepArgs& a = V.K.T.a;
    if (V.K.T.xpf || V.idpf) {
        const int64_t r0 = tile * TS * 32, r1 = min(r0 + TS * 32, a.n_rows);
        // the tile's own x rows (B members each, member-minor)
        if (V.K.T.xpf && r1 > r0) prefetch_l2(a.x + (a.own_off + r0) * B, (uint64_t)(r1 - r0) * 8 * B);
        // and its inv_d slots: each consumer lane loads its own inv_d next to
        // its x loads, and without the prefetch that load is a DRAM round trip
        // on every slice's critical path (ablation on cfg4)
        if (V.idpf && r1 > r0) prefetch_l2(a.inv_d + r0 * B, (uint64_t)(r1 - r0) * 8 * B);
    }
    vi_issue_call<TS, BAND, REARR>(stages + (size_t)s * V.K.T.stage_bytes, &full[s], a.slice_off, a.slice_end,
                                   a.inv_d, V.K.row8, V.loi, V.upi, V.vidx, V.K.col16, V.K.T.off_val, V.K.T.off_col,
                                   tile, pol, a.tile_meta);
}

// One slot's W entries: all x gathers and dictionary reads issued first, then
// the FMAs in t order (the layout-v0 order: acc = val * x + acc).
template <int W>
__device__ __forceinline__ double vi_row(const int16_t* scol, const uint16_t* svi, const double* sdict,
                                         const double* xr) {
    double xv[W], vv[W];
#if CME_ABL == 3
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = (double)scol[32 * u];   // (ablation: no gathers, no dictionary)
#pragma unroll
    for (int u = 0; u < W; ++u) vv[u] = (double)svi[32 * u];
#elif CME_ABL == 4
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = __ldg(xr + (scol[32 * u] & 1));   // (ablation: no gathers, no dictionary)
#pragma unroll
    for (int u = 0; u < W; ++u) vv[u] = (double)svi[32 * u];
#elif CME_ABL == 5
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = __ldg(xr + (scol[32 * u] & 1));   // (ablation: no gathers)
#pragma unroll
    for (int u = 0; u < W; ++u) vv[u] = sdict[svi[32 * u]];
#else
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = __ldg(xr + scol[32 * u]);
#pragma unroll
    for (int u = 0; u < W; ++u) vv[u] = sdict[svi[32 * u]];
#endif
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(vv[u], xv[u], acc);
    return acc;
}
// Slots wider than 8: chunks of 8, same order.
__device__ __forceinline__ double vi_row_wide(const int16_t* scol, const uint16_t* svi, const double* sdict,
                                              const double* xr, int w) {
    double acc = 0.0;
    for (int t0 = 0; t0 < w; t0 += 8) {
        double xc[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) xc[u] = __ldg(xr + scol[32 * (t0 + u)]);
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) acc = fma(sdict[svi[32 * (t0 + u)]], xc[u], acc);
    }
    return acc;
}

// NCW consumer warps, one slice each per tile.  (Measured and removed: two
// slices per warp with both slices' gathers in flight -- on one CTA per SM with
// a 5-stage ring 210-217 us, on two CTAs per SM with register spills 374 us,
// vs 185-189 us for this loop on cfg4.)
template <int NCW, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(TmaShape<NCW>::kThreads, TmaShape<NCW>::kMinBlocks)
    sell_vi_kernel(const ViArgs V) {
    constexpr int kConsumers = NCW, kTileSlices = NCW, kSlots = kTileSlices * 32;
    constexpr int kMeta = meta_bytes(kTileSlices);
    constexpr int kOffRow = 0, kOffLo = kOffRow + (REARR ? kSlots : 0), kOffUp = kOffLo + 2 * kSlots;
    const CptArgs& K = V.K;
    const TmaArgs& T = K.T;
    const StepArgs& a = T.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8], dbar;
    const double* sdict = reinterpret_cast<const double*>(smem);
    unsigned char* stages = smem + V.dict_bytes;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int S = T.stages;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers);
        }
        mbar_init(&dbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const bool producer = warp == kConsumers && lane == 0;
    uint64_t pol = 0;
    int64_t t_first, my_tiles, t_stride;
    tma_tile_range(T, &t_first, &my_tiles, &t_stride);
    const int64_t t_end = t_first + my_tiles * t_stride;
    const int pro = (int)(my_tiles < (int64_t)S ? my_tiles : (int64_t)S);
    if (producer) {   // dictionary and first tiles are constant: load while the previous step drains
        pol = evict_first_policy();
        uint64_t keep;   // every CTA reads the dictionary: keep it in L2
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(keep));
        mbar_expect_tx(&dbar, (uint32_t)V.dict_bytes);
        bulk_g2s(smem, V.dict, (uint32_t)V.dict_bytes, &dbar, keep);
        for (int i = 0; i < pro; ++i)
            vi_issue<kTileSlices, BAND, REARR>(V, stages, full, t_first + (int64_t)i * t_stride, i, pol);
    }
    pdl_wait();
    if (!CME_ABL && a.stop != nullptr && *a.stop) {   // (ablation builds run every launch)
        if (producer) {
            mbar_wait(&dbar, 0u);
            for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        }
        return;
    }
    CheckAcc<1> ck;
    if (warp == kConsumers) {
        if (lane == 0 && my_tiles > pro) {
            int s = 0;
            uint32_t phase = 1;
            for (int64_t tile = t_first + (int64_t)pro * t_stride; tile < t_end; tile += t_stride) {
                mbar_wait(&empty[s], phase ^ 1u);
                vi_issue<kTileSlices, BAND, REARR>(V, stages, full, tile, s, pol);
                if (++s == S) { s = 0; phase ^= 1u; }
            }
        }
        if (lane == 0 && my_tiles == 0) mbar_wait(&dbar, 0u);   // no tile ever waits on it
    } else {
        // one slice per warp: loop invariants hoisted (the ncu instruction
        // census found ~120 per-slice instructions, mostly kernel-parameter
        // reloads and 64-bit index arithmetic); 32-bit slot/row indices
        // (n < 2^31); the epilogue is finish_row_x's arithmetic, with the
        // pending scale (constant for this launch) read once
        const double* xo = a.x + a.own_off;
        double* yo = a.y + a.own_off;
        const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end, ws = K.win_shift;
        const int stage_bytes = T.stage_bytes, off_val = T.off_val, off_col = T.off_col;
        const double om = a.omega, om1 = 1.0 - a.omega;
        const bool damp = om != 1.0, unif = a.unif_lam_inv != 0.0;
        const double sc = a.pre_scale != nullptr ? a.pre_scale[0] : 1.0;
        const int npush = a.npush;
        const uint64_t pol_s = evict_first_policy();
        mbar_wait(&dbar, 0u);
        int s = 0;
        uint32_t phase = 0;
        for (int64_t tile = t_first; tile < t_end; tile += t_stride) {
            const unsigned char* st = stages + s * stage_bytes + kMeta;
            mbar_wait(&full[s], phase);
            const int2 meta = reinterpret_cast<const int2*>(st - kMeta)[warp];   // {offset in tile, width}
            const int q = (int)tile * kTileSlices + warp;
            const int slot = q * 32 + lane;
#if CME_ABL == 1   // (ablation: the ring alone)
            if (q < slice_end && slot < n_rows && meta.y == 12345) {
#else
            if (q < slice_end && slot < n_rows) {
#endif
                const int ls = warp * 32 + lane;
                const int r = REARR ? ((slot >> ws) << ws) + st[kOffRow + ls] : slot;
                const double id = ld_stream(a.inv_d + slot, pol_s);   // with the x loads, before the gathers
                RowX<1, BAND> X;
                X.load(xo, r);
                const double* xr = xo + r;
                const uint16_t* svi = reinterpret_cast<const uint16_t*>(st + off_val) + meta.x + lane;
                const int16_t* scol = reinterpret_cast<const int16_t*>(st + off_col) + meta.x + lane;
                double acc = 0.0;
#if CME_ABL == 2   // (ablation: the row stream without the entries)
                if (meta.y != 12345) {} else
#endif
                switch (meta.y) {   // warp-uniform exact widths
                    case 0: break;
                    case 1: acc = vi_row<1>(scol, svi, sdict, xr); break;
                    case 2: acc = vi_row<2>(scol, svi, sdict, xr); break;
                    case 3: acc = vi_row<3>(scol, svi, sdict, xr); break;
                    case 4: acc = vi_row<4>(scol, svi, sdict, xr); break;
                    case 5: acc = vi_row<5>(scol, svi, sdict, xr); break;
                    case 6: acc = vi_row<6>(scol, svi, sdict, xr); break;
                    case 7: acc = vi_row<7>(scol, svi, sdict, xr); break;
                    case 8: acc = vi_row<8>(scol, svi, sdict, xr); break;
                    default: acc = vi_row_wide(scol, svi, sdict, xr, meta.y);
                }
                const double sum = BAND ? fma(sdict[reinterpret_cast<const uint16_t*>(st + kOffLo)[ls]], X.xl[0],
                                              sdict[reinterpret_cast<const uint16_t*>(st + kOffUp)[ls]] * X.xu[0]) + acc
                                        : acc;
                const double x_r = X.xr[0];
                double y = damp ? fma(om1, x_r, om * (id * sum)) : id * sum;
                if (unif) {   // transient: (I + A/Lambda) x with a_rr = -1/id
                    y = fma(a.unif_lam_inv, sum - x_r / id, x_r);
                    double* ac = a.acc + a.own_off + r;
                    *ac = fma(a.acc_w, x_r, *ac);
                }
                y *= sc;   // = finish_row_x's pending-scale multiply (exact when sc = 1)
                yo[r] = y;
                if (CHECK) ck.add(0, y, ((damp || CHECK) ? x_r : 0.0) * sc, id);
                for (int p = 0; p < npush; ++p)   // halo rows straight into the peer's buffer
                    if (r >= a.push_lo[p] && r < a.push_hi[p]) a.push_y[p][r] = y;
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
            if (++s == S) { s = 0; phase ^= 1u; }
        }
    }
    if (CHECK) cta_check_partials<NCW + 1, 1>(ck, a.partials);
}

// ---------------------------------------------------------------------------
// Batched value-indexed kernel (B = 2, 4, 8 rate sets on one pattern; DESIGN.md
// sec. 5c): every stored entry's B-tuple of rates is one dictionary tuple, so
// the members share the 16-bit index and the 16-bit column offset -- 4/B bytes
// per entry per member.  The tuples (n_dict x B doubles, member-minor) are read
// from global memory (L1/L2) with one B-wide vector load, next to the B-wide x
// gather; inv_d is a per-lane B-wide stream.  Arithmetic = the layout-v0
// batched kernels' (same values, FMAs in t order per member, row sum x inv_d).
template <int NCW, int B, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(TmaShape<NCW>::kThreads, 1) sell_vib_kernel(const ViArgs V) {
    constexpr int kConsumers = NCW, kTileSlices = NCW, kSlots = kTileSlices * 32;
    constexpr int kMeta = meta_bytes(kTileSlices);
    constexpr int kOffRow = 0, kOffLo = kOffRow + (REARR ? kSlots : 0), kOffUp = kOffLo + 2 * kSlots;
    constexpr int U = Chunk<B>::U;   // entries whose loads are in flight together
    const CptArgs& K = V.K;
    const TmaArgs& T = K.T;
    const StepArgs& a = T.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8];
    unsigned char* stages = smem;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int S = T.stages;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const bool producer = warp == kConsumers && lane == 0;
    uint64_t pol = 0;
    int64_t t_first, my_tiles, t_stride;
    tma_tile_range(T, &t_first, &my_tiles, &t_stride);
    const int64_t t_end = t_first + my_tiles * t_stride;
    const int pro = (int)(my_tiles < (int64_t)S ? my_tiles : (int64_t)S);
    if (producer) {
        pol = evict_first_policy();
        for (int i = 0; i < pro; ++i)
            vi_issue<kTileSlices, BAND, REARR, B>(V, stages, full, t_first + (int64_t)i * t_stride, i, pol);
    }
    pdl_wait();
    if (a.stop != nullptr && *a.stop) {
        if (producer)
            for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        return;
    }
    CheckAcc<B> ck;
    if (warp == kConsumers) {
        if (lane == 0 && my_tiles > pro) {
            int s = 0;
            uint32_t phase = 1;
            for (int64_t tile = t_first + (int64_t)pro * t_stride; tile < t_end; tile += t_stride) {
                mbar_wait(&empty[s], phase ^ 1u);
                vi_issue<kTileSlices, BAND, REARR, B>(V, stages, full, tile, s, pol);
                if (++s == S) { s = 0; phase ^= 1u; }
            }
        }
    } else {
        const double* xo = a.x + a.own_off * B;
        double* yo = a.y + a.own_off * B;
        const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end, ws = K.win_shift;
        const int stage_bytes = T.stage_bytes, off_val = T.off_val, off_col = T.off_col;
        const uint64_t pol_s = evict_first_policy();
        const double* dict = V.dict;
        int s = 0;
        uint32_t phase = 0;
        for (int64_t tile = t_first; tile < t_end; tile += t_stride) {
            const unsigned char* st = stages + s * stage_bytes + kMeta;
            mbar_wait(&full[s], phase);
            const int2 meta = reinterpret_cast<const int2*>(st - kMeta)[warp];   // {offset in tile, width}
            const int q = (int)tile * kTileSlices + warp;
            const int slot = q * 32 + lane;
            if (q < slice_end && slot < n_rows) {
                const int ls = warp * 32 + lane;
                const int r = REARR ? ((slot >> ws) << ws) + st[kOffRow + ls] : slot;
                double id[B];
                ld_stream_vec<B>(a.inv_d + (int64_t)slot * B, pol_s, id);
                RowX<B, BAND> X;
                X.load(xo, r);
                const uint16_t* svi = reinterpret_cast<const uint16_t*>(st + off_val) + meta.x + lane;
                const int16_t* scol = reinterpret_cast<const int16_t*>(st + off_col) + meta.x + lane;
                double acc[B];
#pragma unroll
                for (int b = 0; b < B; ++b) acc[b] = 0.0;
                for (int t0 = 0; t0 < meta.y; t0 += U) {
                    double xv[U][B], vv[U][B];
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (t0 + u < meta.y) {
                            ld_vec<B>(xo + (int64_t)(r + scol[32 * (t0 + u)]) * B, xv[u]);
                            ld_vec<B>(dict + (int64_t)svi[32 * (t0 + u)] * B, vv[u]);
                        }
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (t0 + u < meta.y)
#pragma unroll
                            for (int b = 0; b < B; ++b) acc[b] = fma(vv[u][b], xv[u][b], acc[b]);
                }
                double lo[B], up[B];
                if (BAND) {
                    ld_vec<B>(dict + (int64_t)reinterpret_cast<const uint16_t*>(st + kOffLo)[ls] * B, lo);
                    ld_vec<B>(dict + (int64_t)reinterpret_cast<const uint16_t*>(st + kOffUp)[ls] * B, up);
                }
                finish_row_x<B, BAND, CHECK>(a, r, yo, acc, lo, up, id, a.pre_scale, ck, X);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
            if (++s == S) { s = 0; phase ^= 1u; }
        }
    }
    if (CHECK) cta_check_partials<NCW + 1, B>(ck, a.partials);
}

}  // namespace cme
