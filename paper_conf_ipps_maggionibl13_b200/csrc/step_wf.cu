// Launchers of the wavefront s-step kernel (kernels_wf.cuh, B = 1, one GPU).
#include "kernels_wf.cuh"
#include "launch.h"

namespace cme {

template <int W>
static cudaError_t launch_wf_w(const WfArgs& A, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                               cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(bd, r, c)                                                                                           \
    case bd * 4 + r * 2 + c:                                                                                   \
        return launch_ex(sell_wf_kernel<W, bd, r, c>, dim3(grid), dim3(Vi2Shape<W>::kThreads), smem, pdl, s, A);
        K_(0, 0, 0) K_(0, 0, 1) K_(0, 1, 0) K_(0, 1, 1) K_(1, 0, 0) K_(1, 0, 1) K_(1, 1, 0) K_(1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_wf(const WfArgs& A, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                      cudaStream_t s) {
    return ncw == 30 ? launch_wf_w<30>(A, grid, smem, band, rearr, check, pdl, s)
                     : launch_wf_w<16>(A, grid, smem, band, rearr, check, pdl, s);
}

template <int W>
static cudaError_t wf_prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c)                                                                                          \
    if (e == cudaSuccess)                                                                                     \
        e = cudaFuncSetAttribute(sell_wf_kernel<W, bd, r, c>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}

cudaError_t wf_prepare(int ncw, int smem) { return ncw == 30 ? wf_prepare_w<30>(smem) : wf_prepare_w<16>(smem); }

cudaError_t wf_occupancy(int ncw, int smem, int* occ) {
    if (ncw == 30)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_wf_kernel<30, true, true, true>,
                                                             Vi2Shape<30>::kThreads, smem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_wf_kernel<16, true, true, true>,
                                                         Vi2Shape<16>::kThreads, smem);
}

}  // namespace cme
