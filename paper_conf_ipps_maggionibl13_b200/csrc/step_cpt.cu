// Launchers of the compact-encoding TMA step kernel (kernels_cpt.cuh, B = 1).
#include "kernels_cpt.cuh"
#include "launch.h"

namespace cme {

template <int W>
static cudaError_t launch_cpt_w(const CptArgs& K, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                                cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(bd, r, c)                                                                                       \
    case bd * 4 + r * 2 + c:                                                                               \
        return launch_ex(sell_cpt_kernel<W, bd, r, c>, dim3(grid), dim3(TmaShape<W>::kThreads), smem, pdl, s, K);
        K_(0, 0, 0) K_(0, 0, 1) K_(0, 1, 0) K_(0, 1, 1) K_(1, 0, 0) K_(1, 0, 1) K_(1, 1, 0) K_(1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_cpt(const CptArgs& K, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                       cudaStream_t s) {
    return ncw == 16 ? launch_cpt_w<16>(K, grid, smem, band, rearr, check, pdl, s)
                     : launch_cpt_w<8>(K, grid, smem, band, rearr, check, pdl, s);
}

template <int W>
static cudaError_t cpt_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c) \
    if (e == cudaSuccess) e = cudaFuncSetAttribute(sell_cpt_kernel<W, bd, r, c>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}

cudaError_t cpt_prepare(int ncw, int smem) { return ncw == 16 ? cpt_prepare_w<16>(smem) : cpt_prepare_w<8>(smem); }

cudaError_t cpt_occupancy(int ncw, int smem, int* occ) {
    // the heaviest variant (band + rearrangement + check) bounds the residency
    if (ncw == 16)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_cpt_kernel<16, true, true, true>,
                                                             TmaShape<16>::kThreads, smem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_cpt_kernel<8, true, true, true>,
                                                         TmaShape<8>::kThreads, smem);
}

template <int W>
static cudaError_t launch_vi_w(const ViArgs& V, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                               cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(bd, r, c)                                                                                      \
    case bd * 4 + r * 2 + c:                                                                              \
        return launch_ex(sell_vi_kernel<W, bd, r, c>, dim3(grid), dim3(TmaShape<W>::kThreads), smem, pdl, s, V);
        K_(0, 0, 0) K_(0, 0, 1) K_(0, 1, 0) K_(0, 1, 1) K_(1, 0, 0) K_(1, 0, 1) K_(1, 1, 0) K_(1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_vi(const ViArgs& V, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                      cudaStream_t s) {
    return ncw == 16   ? launch_vi_w<16>(V, grid, smem, band, rearr, check, pdl, s)
           : ncw == 31 ? launch_vi_w<31>(V, grid, smem, band, rearr, check, pdl, s)
                       : launch_vi_w<8>(V, grid, smem, band, rearr, check, pdl, s);
}

template <int W>
static cudaError_t vi_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c)                                                                                         \
    if (e == cudaSuccess)                                                                                    \
        e = cudaFuncSetAttribute(sell_vi_kernel<W, bd, r, c>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}

cudaError_t vi_prepare(int ncw, int smem) {
    return ncw == 16 ? vi_prepare_w<16>(smem) : ncw == 31 ? vi_prepare_w<31>(smem) : vi_prepare_w<8>(smem);
}

cudaError_t vi_occupancy(int ncw, int smem, int* occ) {
    // the heaviest variant (band + rearrangement + check) bounds the residency
    if (ncw == 16)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi_kernel<16, true, true, true>,
                                                             TmaShape<16>::kThreads, smem);
    if (ncw == 31)   // one 1024-thread CTA per SM: one dictionary copy per SM
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi_kernel<31, true, true, true>,
                                                             TmaShape<31>::kThreads, smem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi_kernel<8, true, true, true>,
                                                         TmaShape<8>::kThreads, smem);
}

template <int W, int B>
static cudaError_t launch_vib_w(const ViArgs& V, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                                cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(bd, r, c)                                                                                           \
    case bd * 4 + r * 2 + c:                                                                                   \
        return launch_ex(sell_vib_kernel<W, B, bd, r, c>, dim3(grid), dim3(TmaShape<W>::kThreads), smem, pdl, s, V);
        K_(0, 0, 0) K_(0, 0, 1) K_(0, 1, 0) K_(0, 1, 1) K_(1, 0, 0) K_(1, 0, 1) K_(1, 1, 0) K_(1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}
template <int B>
static cudaError_t launch_vib_b(const ViArgs& V, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                                bool pdl, cudaStream_t s) {
    // 15 consumer warps: 16 warps per CTA, so the one-CTA-per-SM register cap
    // is 128 (17 warps round up to 20 in the register allocation: 96, spills)
    return ncw == 16   ? launch_vib_w<16, B>(V, grid, smem, band, rearr, check, pdl, s)
           : ncw == 15 ? launch_vib_w<15, B>(V, grid, smem, band, rearr, check, pdl, s)
                       : launch_vib_w<8, B>(V, grid, smem, band, rearr, check, pdl, s);
}
cudaError_t launch_vib(const ViArgs& V, int B, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                       bool pdl, cudaStream_t s) {
    switch (B) {
        case 2: return launch_vib_b<2>(V, ncw, grid, smem, band, rearr, check, pdl, s);
        case 4: return launch_vib_b<4>(V, ncw, grid, smem, band, rearr, check, pdl, s);
        case 8: return launch_vib_b<8>(V, ncw, grid, smem, band, rearr, check, pdl, s);
    }
    return cudaErrorInvalidValue;
}

template <int W, int B>
static cudaError_t vib_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c)                                                                                          \
    if (e == cudaSuccess)                                                                                     \
        e = cudaFuncSetAttribute(sell_vib_kernel<W, B, bd, r, c>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}
cudaError_t vib_prepare(int B, int ncw, int smem) {
    switch (B) {
        case 2: return ncw == 16 ? vib_prepare_w<16, 2>(smem) : ncw == 15 ? vib_prepare_w<15, 2>(smem) : vib_prepare_w<8, 2>(smem);
        case 4: return ncw == 16 ? vib_prepare_w<16, 4>(smem) : ncw == 15 ? vib_prepare_w<15, 4>(smem) : vib_prepare_w<8, 4>(smem);
        case 8: return ncw == 16 ? vib_prepare_w<16, 8>(smem) : ncw == 15 ? vib_prepare_w<15, 8>(smem) : vib_prepare_w<8, 8>(smem);
    }
    return cudaErrorInvalidValue;
}
template <int W, int B>
static cudaError_t vib_occ_w(int smem, int* occ) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vib_kernel<W, B, true, true, true>,
                                                         TmaShape<W>::kThreads, smem);
}
cudaError_t vib_occupancy(int B, int ncw, int smem, int* occ) {
    switch (B) {
        case 2: return ncw == 16 ? vib_occ_w<16, 2>(smem, occ) : ncw == 15 ? vib_occ_w<15, 2>(smem, occ) : vib_occ_w<8, 2>(smem, occ);
        case 4: return ncw == 16 ? vib_occ_w<16, 4>(smem, occ) : ncw == 15 ? vib_occ_w<15, 4>(smem, occ) : vib_occ_w<8, 4>(smem, occ);
        case 8: return ncw == 16 ? vib_occ_w<16, 8>(smem, occ) : ncw == 15 ? vib_occ_w<15, 8>(smem, occ) : vib_occ_w<8, 8>(smem, occ);
    }
    return cudaErrorInvalidValue;
}

}  // namespace cme
