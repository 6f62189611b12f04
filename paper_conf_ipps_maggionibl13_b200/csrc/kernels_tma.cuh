// TMA-staged persistent variant of the fused Jacobi step (sm_100a).
//
// Same arithmetic and layout as sell_step_kernel (kernels.cuh); what changes
// is how the packed matrix reaches the SM.  A tile is NCW consecutive slices
// (NCW*32 rows, whole rearrangement windows); its val and col entries
// are ONE contiguous block each (layout v0), and its inv_d / row_of / lo / up
// entries are contiguous too.  A producer warp streams every tile of the CTA's
// round-robin share into a ring of S shared-memory stages with 1-D bulk copies
// (cp.async.bulk ... mbarrier::complete_tx, the TMA engine), each stage
// guarded by a full/empty mbarrier pair; NCW consumer warps (one slice each)
// read their rows from shared memory, gather x from global memory (L1/L2),
// and store y.  Default NCW = 16, S = 2, 2 CTAs/SM (56 regs): 32 consumer
// warps/SM and 4 x ~43 KB of tiles in flight per SM, so the kernel runs at
// the HBM limit (92% of the measured copy bandwidth on cfg4) where the
// register-only kernel was latency-bound at 62%.
#pragma once
#include "kernels.cuh"

namespace cme {

// NCW consumer warps (one slice each) + 1 producer warp; a tile = NCW slices.
template <int NCW>
struct TmaShape {
    static constexpr int kThreads = 32 * (NCW + 1);
    // register cap: 75 / 60 regs; 31 consumer warps = one 1024-thread CTA per SM (64 regs)
    static constexpr int kMinBlocks = NCW == 8 ? 3 : NCW == 31 ? 1 : 2;   // (23: 2 x 768 threads)
};

struct TmaArgs {
    StepArgs a;
    int64_t n_tiles;
    int32_t stages;
    int32_t stage_bytes;  // bytes per stage (multiple of 128)
    int32_t off_val;      // byte offsets inside a stage
    int32_t off_col;
    int32_t contig;       // 1: CTA b takes a contiguous run of tiles, 0: round robin (default, CME_TMA_CONTIG)
    int32_t xpf;          // 1: L2-prefetch a tile's own x rows when its matrix tile is issued (CME_TMA_XPF)
};

// Tile sequence of one CTA: contiguous runs keep consecutive tiles -- whose x
// gather windows overlap -- on the same SM, so the window stays in L1;
// round robin interleaves the CTAs.  Returns the first tile, the count and
// the stride.
__device__ __forceinline__ void tma_tile_range(const TmaArgs& T, int64_t* first, int64_t* count, int64_t* stride) {
    const int64_t b = blockIdx.x, G = gridDim.x;
    if (T.contig) {
        const int64_t lo = b * T.n_tiles / G, hi = (b + 1) * T.n_tiles / G;
        *first = lo;
        *count = hi - lo;
        *stride = 1;
    } else {
        *first = b;
        *count = b < T.n_tiles ? (T.n_tiles - 1 - b) / G + 1 : 0;
        *stride = G;
    }
}

// Every stage starts with the tile's slice metadata: per slice {entry offset
// inside the tile, width} (host-built tile_meta, padded to whole tiles), moved
// by the same TMA transaction as the tile.  Reading it from global memory put
// two dependent L2 round trips (slice_off[q], slice_off[q0]) at the head of
// every consumer's tile -- the top stall in the ncu source view (16.5%).
// bytes of the metadata block of a tile of ts slices (keeps the data 128-B aligned)
__host__ __device__ constexpr int meta_bytes(int ts) { return (ts * 8 + 127) / 128 * 128; }
constexpr int kMetaBytes = 128;   // = meta_bytes(NCW) for the NCW <= 16 one-slice-per-warp tiles


__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// try_wait with a suspend-time hint (ncu counted ~14 polls per tile wait in
// the value-indexed kernel; a nanosleep back-off between polls measured the
// same 187-188 us on cfg4, so the polls do not cost throughput).
#ifndef CME_MBAR_SUSPEND_NS
#define CME_MBAR_SUSPEND_NS 1000000
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(b)),
        "r"(parity), "n"(CME_MBAR_SUSPEND_NS)
        : "memory");
}
// L2 prefetch of [p, p + bytes) by the TMA engine (16-byte granules).  The
// iterate a tile's rows will gather is first touched by the tile itself (the
// RCM/DFS bands keep every gather within a few tiles of its row), so without
// it those first touches are DRAM round trips on the consumers' critical
// path.  L2 is the point of coherence: prefetching a line the previous step
// is still writing cannot produce a stale read.
__device__ __forceinline__ void prefetch_l2(const void* p, uint64_t bytes) {
    const uint64_t a = reinterpret_cast<uint64_t>(p) & ~uint64_t(15);
    const uint64_t e = (reinterpret_cast<uint64_t>(p) + bytes + 15) & ~uint64_t(15);
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"((uint32_t)(e - a)) : "memory");
}

// 1-D bulk copy global -> shared, completion counted on mbarrier `b`
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b,
                                         uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
            "r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(b)), "l"(pol)
        : "memory");
}

// Per-tile metadata stride in int2 entries: an even count keeps every tile's
// record 16-byte aligned and sized for the bulk copy (odd tile shapes: 31).
__host__ __device__ constexpr int meta_stride(int ts) { return (ts + 1) & ~1; }

__device__ __forceinline__ void issue_meta(unsigned char* st, uint64_t* bar, const int2* tile_meta, int64_t tile,
                                           int ncw, uint64_t pol) {
    const int ms = meta_stride(ncw);
    bulk_g2s(st, tile_meta + tile * ms, (uint32_t)ms * 8u, bar, pol);
}

// Stage layout: [inv_d][row_of if REARR][lo, up if BAND][val][col] for
// NCW*32 slots and B members; the host computes the same offsets from
// tma_fixed_bytes() and the widest tile.
__host__ __device__ inline int tma_fixed_bytes(int ncw, int B, bool band, bool rearr) {
    return ncw * 32 * (8 * B + (rearr ? 4 : 0) + (band ? 16 * B : 0));
}

// Sum over the W ELL entries of one slot from shared memory: all x gathers
// first, then the FMAs in t order (W known at compile time).
template <int B, int W>
__device__ __forceinline__ void ell_row_smem(const int32_t* scol, const double* sval, const double* x,
                                             double (&acc)[B]) {
    double xv[W][B];
#pragma unroll
    for (int u = 0; u < W; ++u) ld_vec<B>(x + (int64_t)scol[32 * u] * B, xv[u]);
#pragma unroll
    for (int u = 0; u < W; ++u)
#pragma unroll
        for (int b = 0; b < B; ++b) acc[b] = fma(sval[32 * u * B + b], xv[u][b], acc[b]);
}

// Producer: one tile -> one stage (inv_d, row_of, lo/up, val, col blocks, all
// contiguous in HBM), completion counted on `bar`.  Scalar arguments only, so
// the call neither copies the kernel parameters to local memory nor carries
// the producer's addressing into the consumers' register allocation.
#ifndef CME_TMA_PRODUCER_INLINE
#define CME_TMA_PRODUCER_INLINE 0
#endif
template <int NCW, int B, bool BAND, bool REARR>
__device__ __forceinline__ void tma_issue_body(unsigned char* st, uint64_t* bar, const int64_t* slice_off,
                                               int64_t slice_end, const double* inv_d, const int32_t* row_of,
                                               const double* lo, const double* up, const double* val,
                                               const int32_t* col, int off_val, int off_col, int64_t tile,
                                               uint64_t pol, const int2* tile_meta) {
    constexpr int kSlots = NCW * 32;
    constexpr int kOffInvd = 0, kOffRow = 8 * B * kSlots, kOffLo = kOffRow + (REARR ? 4 * kSlots : 0),
                  kOffUp = kOffLo + 8 * B * kSlots;
    const int64_t q0 = tile * NCW;
    const int64_t q1 = min(q0 + NCW, slice_end);
    const int64_t e0 = slice_off[q0], e1 = slice_off[q1];
    const uint32_t slots = (uint32_t)(q1 - q0) * 32u;
    const uint32_t nval = (uint32_t)(e1 - e0);
    uint32_t bytes = nval * (8u * B + 4u) + slots * 8u * B + meta_stride(NCW) * 8u;
    if (REARR) bytes += slots * 4u;
    if (BAND) bytes += slots * 16u * B;
    mbar_expect_tx(bar, bytes);
    issue_meta(st, bar, tile_meta, tile, NCW, pol);
    st += kMetaBytes;
    bulk_g2s(st + kOffInvd, inv_d + q0 * 32 * B, slots * 8u * B, bar, pol);
    if (REARR) bulk_g2s(st + kOffRow, row_of + q0 * 32, slots * 4u, bar, pol);
    if (BAND) {
        bulk_g2s(st + kOffLo, lo + q0 * 32 * B, slots * 8u * B, bar, pol);
        bulk_g2s(st + kOffUp, up + q0 * 32 * B, slots * 8u * B, bar, pol);
    }
    if (nval) {
        bulk_g2s(st + off_val, val + e0 * B, nval * 8u * B, bar, pol);
        bulk_g2s(st + off_col, col + e0, nval * 4u, bar, pol);
    }
}
template <int NCW, int B, bool BAND, bool REARR>
__device__ __noinline__ void tma_issue_call(unsigned char* st, uint64_t* bar, const int64_t* slice_off,
                                            int64_t slice_end, const double* inv_d, const int32_t* row_of,
                                            const double* lo, const double* up, const double* val,
                                            const int32_t* col, int off_val, int off_col, int64_t tile,
                                            uint64_t pol, const int2* tile_meta) {
    tma_issue_body<NCW, B, BAND, REARR>(st, bar, slice_off, slice_end, inv_d, row_of, lo, up, val, col, off_val,
                                        off_col, tile, pol, tile_meta);
}
template <int NCW, int B, bool BAND, bool REARR>
__device__ __forceinline__ void tma_issue(const TmaArgs& T, unsigned char* smem, uint64_t* full, int64_t tile, int s,
                                          uint64_t pol) {
    const StepArgs& a = T.a;
    unsigned char* st = smem + (size_t)s * T.stage_bytes;
    if (T.xpf) {
        const int64_t r0 = tile * NCW * 32, r1 = min(r0 + NCW * 32, a.n_rows);
        if (r1 > r0) prefetch_l2(a.x + (a.own_off + r0) * B, (uint64_t)(r1 - r0) * 8 * B);
    }
    if (CME_TMA_PRODUCER_INLINE)
        tma_issue_body<NCW, B, BAND, REARR>(st, &full[s], a.slice_off, a.slice_end, a.inv_d, a.row_of, a.lo, a.up,
                                            a.val, a.col, T.off_val, T.off_col, tile, pol, a.tile_meta);
    else
        tma_issue_call<NCW, B, BAND, REARR>(st, &full[s], a.slice_off, a.slice_end, a.inv_d, a.row_of, a.lo, a.up,
                                            a.val, a.col, T.off_val, T.off_col, tile, pol, a.tile_meta);
}

#ifndef CME_TMA_EXACT_WIDTHS
#define CME_TMA_EXACT_WIDTHS 1
#endif
constexpr bool kExactWidths = CME_TMA_EXACT_WIDTHS;
#ifndef CME_TMA_EARLY_X
#define CME_TMA_EARLY_X 1
#endif
constexpr bool kEarlyX = CME_TMA_EARLY_X;

template <int NCW, int B, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(TmaShape<NCW>::kThreads, TmaShape<NCW>::kMinBlocks)
    sell_tma_kernel(const TmaArgs T) {
    constexpr int kConsumers = NCW, kTileSlices = NCW, kSlots = NCW * 32;
    constexpr int kOffInvd = 0, kOffRow = 8 * B * kSlots, kOffLo = kOffRow + (REARR ? 4 * kSlots : 0),
                  kOffUp = kOffLo + 8 * B * kSlots;
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
    // Prologue: the packed matrix is constant across steps, so the first S
    // tiles stream in while the previous step (programmatic dependency) drains.
    int64_t t_first, my_tiles, t_stride;
    tma_tile_range(T, &t_first, &my_tiles, &t_stride);
    const int64_t t_end = t_first + my_tiles * t_stride;
    const int pro = (int)(my_tiles < (int64_t)S ? my_tiles : (int64_t)S);
    if (producer) {
        pol = evict_first_policy();
        for (int i = 0; i < pro; ++i)
            tma_issue<NCW, B, BAND, REARR>(T, smem, full, t_first + (int64_t)i * t_stride, i, pol);
    }
    pdl_wait();   // x / ctrl of the previous step are final from here on
    if (a.stop != nullptr && *a.stop) {
        // a decided solve: drain the prologue copies before the CTA exits
        if (producer)
            for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        return;
    }
    CheckAcc<B> ck;

    if (warp == kConsumers) {
        // ---------------- producer ----------------
        if (lane == 0 && my_tiles > pro) {
            // stage s and the parity of its current use, advanced incrementally
            int s = 0;
            uint32_t phase = 1;   // pro == S here: every stage holds its first use
            for (int64_t tile = t_first + (int64_t)pro * t_stride; tile < t_end; tile += t_stride) {
                mbar_wait(&empty[s], phase ^ 1u);   // consumers released the previous use
                tma_issue<NCW, B, BAND, REARR>(T, smem, full, tile, s, pol);
                if (++s == S) { s = 0; phase ^= 1u; }
            }
        }
    } else {
        // ---------------- consumers ----------------
        const double* xo = a.x + a.own_off * B;
        double* yo = a.y + a.own_off * B;
        int s = 0;
        uint32_t phase = 0;
        for (int64_t tile = t_first; tile < t_end; tile += t_stride) {
            const int64_t q0 = tile * kTileSlices;
            const int64_t q = q0 + warp;
            const unsigned char* st = smem + (size_t)s * T.stage_bytes + kMetaBytes;
            mbar_wait(&full[s], phase);
            const int2 meta = reinterpret_cast<const int2*>(st - kMetaBytes)[warp];   // {offset in tile, width}
            const int w = meta.y;
            const int64_t loff = meta.x;
            const int64_t slot = q * 32 + lane;
            if (q < a.slice_end && slot < a.n_rows) {
                const int ls = warp * 32 + lane;
                const double* sval = reinterpret_cast<const double*>(st + T.off_val) + (loff + lane) * B;
                const int32_t* scol = reinterpret_cast<const int32_t*>(st + T.off_col) + loff + lane;
                const int64_t r = REARR ? (int64_t) reinterpret_cast<const int32_t*>(st + kOffRow)[ls] : slot;
                // own/band x loads in flight with the gathers (CME_TMA_EARLY_X)
                RowX<B, BAND> X;
                if (kEarlyX) X.load(xo, r);
                double acc[B];
#pragma unroll
                for (int b = 0; b < B; ++b) acc[b] = 0.0;
                switch (kExactWidths && B <= 2 ? w : -1) {   // warp-uniform exact widths
                    case 0: break;
                    case 1: ell_row_smem<B, 1>(scol, sval, a.x, acc); break;
                    case 2: ell_row_smem<B, 2>(scol, sval, a.x, acc); break;
                    case 3: ell_row_smem<B, 3>(scol, sval, a.x, acc); break;
                    case 4: ell_row_smem<B, 4>(scol, sval, a.x, acc); break;
                    case 5: ell_row_smem<B, 5>(scol, sval, a.x, acc); break;
                    case 6: ell_row_smem<B, 6>(scol, sval, a.x, acc); break;
                    case 7: ell_row_smem<B, 7>(scol, sval, a.x, acc); break;
                    case 8: ell_row_smem<B, 8>(scol, sval, a.x, acc); break;
                    default: {
                        constexpr int U = Chunk<B>::U;
                        for (int t0 = 0; t0 < w; t0 += U) {
                            double xv[U][B];   // all gathers of the chunk in flight, then FMAs
#pragma unroll
                            for (int u = 0; u < U; ++u)
                                if (t0 + u < w) ld_vec<B>(a.x + (int64_t)scol[32 * (t0 + u)] * B, xv[u]);
#pragma unroll
                            for (int u = 0; u < U; ++u)
                                if (t0 + u < w)
#pragma unroll
                                    for (int b = 0; b < B; ++b)
                                        acc[b] = fma(sval[32 * (t0 + u) * B + b], xv[u][b], acc[b]);
                        }
                    }
                }
                double lo[B], up[B], id[B];
#pragma unroll
                for (int b = 0; b < B; ++b) {
                    id[b] = reinterpret_cast<const double*>(st + kOffInvd)[ls * B + b];
                    lo[b] = BAND ? reinterpret_cast<const double*>(st + kOffLo)[ls * B + b] : 0.0;
                    up[b] = BAND ? reinterpret_cast<const double*>(st + kOffUp)[ls * B + b] : 0.0;
                }
                if (!kEarlyX) X.load(xo, r);
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
