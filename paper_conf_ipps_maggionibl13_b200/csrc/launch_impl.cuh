// Definitions of the launchers declared in launch.h (included by step_b*.cu).
#pragma once
#include "launch.h"

namespace cme {

template <int B>
cudaError_t launch_sell(const StepArgs& a, int grid, bool band, bool rearr, bool check, bool pdl, cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K(bd, r, c) \
    case bd * 4 + r * 2 + c: return launch_ex(sell_step_kernel<B, bd, r, c>, dim3(grid), dim3(kCta), 0, pdl, s, a);
        K(0, 0, 0) K(0, 0, 1) K(0, 1, 0) K(0, 1, 1) K(1, 0, 0) K(1, 0, 1) K(1, 1, 0) K(1, 1, 1)
#undef K
    }
    return cudaErrorInvalidValue;
}

template <int W, int B>
static cudaError_t launch_tma_w(const TmaArgs& T, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                                cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K(bd, r, c)                                                                                          \
    case bd * 4 + r * 2 + c:                                                                                 \
        return launch_ex(sell_tma_kernel<W, B, bd, r, c>, dim3(grid), dim3(TmaShape<W>::kThreads), smem, pdl, s, T);
        K(0, 0, 0) K(0, 0, 1) K(0, 1, 0) K(0, 1, 1) K(1, 0, 0) K(1, 0, 1) K(1, 1, 0) K(1, 1, 1)
#undef K
    }
    return cudaErrorInvalidValue;
}

template <int B>
cudaError_t launch_tma(const TmaArgs& T, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                       cudaStream_t s) {
    return ncw == 16 ? launch_tma_w<16, B>(T, grid, smem, band, rearr, check, pdl, s)
                     : launch_tma_w<8, B>(T, grid, smem, band, rearr, check, pdl, s);
}

template <int W, int B>
static cudaError_t tma_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A(bd, r, c) \
    if (e == cudaSuccess)  \
        e = cudaFuncSetAttribute(sell_tma_kernel<W, B, bd, r, c>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    A(0, 0, 0) A(0, 0, 1) A(0, 1, 0) A(0, 1, 1) A(1, 0, 0) A(1, 0, 1) A(1, 1, 0) A(1, 1, 1)
#undef A
    return e;
}

template <int B>
cudaError_t tma_prepare(int ncw, int smem) {
    return ncw == 16 ? tma_prepare_w<16, B>(smem) : tma_prepare_w<8, B>(smem);
}

template <int B>
cudaError_t tma_occupancy(int ncw, int smem, int* occ) {
    // the heaviest variant (band + rearrangement + check) bounds the residency
    if (ncw == 16)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_tma_kernel<16, B, true, true, true>,
                                                             TmaShape<16>::kThreads, smem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_tma_kernel<8, B, true, true, true>,
                                                         TmaShape<8>::kThreads, smem);
}

// Force every register-kernel variant of width B (and the CSR arm) to load
// now: under CUDA lazy loading the first launch of a kernel can wait for the
// device to drain, which deadlocks against a peer's spinning barrier kernel
// in an in-process rank group.
template <int B>
cudaError_t sell_preload() {
    cudaFuncAttributes fa;
    cudaError_t e = cudaSuccess;
#define L(bd, r, c) \
    if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, sell_step_kernel<B, bd, r, c>);
    L(0, 0, 0) L(0, 0, 1) L(0, 1, 0) L(0, 1, 1) L(1, 0, 0) L(1, 0, 1) L(1, 1, 0) L(1, 1, 1)
#undef L
    if (e == cudaSuccess && B == 1) e = cudaFuncGetAttributes(&fa, csr_step_kernel<true>);
    if (e == cudaSuccess && B == 1) e = cudaFuncGetAttributes(&fa, csr_step_kernel<false>);
    return e;
}

#define CME_INSTANTIATE_LAUNCHERS(B)                                                                       \
    template cudaError_t launch_sell<B>(const StepArgs&, int, bool, bool, bool, bool, cudaStream_t);        \
    template cudaError_t launch_tma<B>(const TmaArgs&, int, int, int, bool, bool, bool, bool, cudaStream_t); \
    template cudaError_t tma_prepare<B>(int, int);                                                          \
    template cudaError_t tma_occupancy<B>(int, int, int*);                                                  \
    template cudaError_t sell_preload<B>();

}  // namespace cme
