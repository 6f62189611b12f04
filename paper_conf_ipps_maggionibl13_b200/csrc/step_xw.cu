// Launchers of the x-window tile-record step kernel (kernels_vi2.cuh with
// XWM = 1 mirrored ring / 2 ring with a wrap per entry; B = 1, one GPU;
// DESIGN.md sec. 5f).
#include "kernels_vi2.cuh"
#include "launch.h"

namespace cme {

template <int W, int M>
static cudaError_t launch_xw_w(const Vi2Args& V, int grid, int smem, bool band, bool rearr, bool check, int enc,
                               bool pdl, cudaStream_t s) {
    const int key = (enc == 2 ? 8 : 0) | (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(e, bd, r, c)                                                                                        \
    case (e ? 8 : 0) + bd * 4 + r * 2 + c:                                                                     \
        return launch_ex(sell_vi2_kernel<W, bd, r, c, e, M>, dim3(grid), dim3(Vi2Shape<W>::kThreads), smem, pdl, \
                         s, V);
        K_(0, 0, 0, 0) K_(0, 0, 0, 1) K_(0, 0, 1, 0) K_(0, 0, 1, 1) K_(0, 1, 0, 0) K_(0, 1, 0, 1) K_(0, 1, 1, 0)
        K_(0, 1, 1, 1) K_(2, 0, 0, 0) K_(2, 0, 0, 1) K_(2, 0, 1, 0) K_(2, 0, 1, 1) K_(2, 1, 0, 0) K_(2, 1, 0, 1)
        K_(2, 1, 1, 0) K_(2, 1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_vi2_xw(const Vi2Args& V, int ncw, int grid, int smem, bool band, bool rearr, bool check, int enc,
                          int mode, bool pdl, cudaStream_t s) {
    if (enc == 1) return cudaErrorInvalidValue;
    if (mode == 2)
        return ncw == 30 ? launch_xw_w<30, 2>(V, grid, smem, band, rearr, check, enc, pdl, s)
                         : launch_xw_w<16, 2>(V, grid, smem, band, rearr, check, enc, pdl, s);
    return ncw == 30 ? launch_xw_w<30, 1>(V, grid, smem, band, rearr, check, enc, pdl, s)
                     : launch_xw_w<16, 1>(V, grid, smem, band, rearr, check, enc, pdl, s);
}

template <int W, int M>
static cudaError_t xw_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c)                                                                                            \
    if (e == cudaSuccess)                                                                                       \
        e = cudaFuncSetAttribute(sell_vi2_kernel<W, bd, r, c, 0, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                 smem);                                                                         \
    if (e == cudaSuccess)                                                                                       \
        e = cudaFuncSetAttribute(sell_vi2_kernel<W, bd, r, c, 2, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                 smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}

cudaError_t vi2_xw_prepare(int ncw, int smem) {
    cudaError_t e = ncw == 30 ? xw_prepare_w<30, 1>(smem) : xw_prepare_w<16, 1>(smem);
    if (e == cudaSuccess) e = ncw == 30 ? xw_prepare_w<30, 2>(smem) : xw_prepare_w<16, 2>(smem);
    return e;
}

template <int W>
static cudaError_t xw_occupancy_w(int enc, int smem, int* occ) {
    return enc == 2 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi2_kernel<W, true, true, true, 2, 2>,
                                                                     Vi2Shape<W>::kThreads, smem)
                    : cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi2_kernel<W, true, true, true, 0, 2>,
                                                                     Vi2Shape<W>::kThreads, smem);
}

cudaError_t vi2_xw_occupancy(int ncw, int smem, int* occ, int enc) {
    return ncw == 30 ? xw_occupancy_w<30>(enc, smem, occ) : xw_occupancy_w<16>(enc, smem, occ);
}

}  // namespace cme
