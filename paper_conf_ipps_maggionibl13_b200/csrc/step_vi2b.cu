// Launchers of the batched tile-record step kernel (kernels_vi2.cuh:
// sell_vi2b_kernel, B = 2, 4, 8).
#include "kernels_vi2.cuh"
#include "launch.h"

namespace cme {

// consumer warps per CTA (one CTA per SM) by batch width: B = 2 16 (30 at
// the 64-register cap measured 382 vs 333 us on cfg4), B = 4 16, B = 8 15 (the
// B-wide accumulators and in-flight loads need up to 128 registers); `force`
// (CME_VI2_WARPS) picks the alternative
int vi2b_warps(int B, int force) {
    if (B == 2) return force == 30 ? 30 : 16;
    if (B == 4) return force == 30 ? 30 : 16;
    return force == 8 ? 8 : 15;
}

template <int W, int B, bool SD = false>
static cudaError_t launch_w(const Vi2Args& V, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                            cudaStream_t s) {
    const int key = (band ? 4 : 0) | (rearr ? 2 : 0) | (check ? 1 : 0);
    switch (key) {
#define K_(bd, r, c)                                                                                           \
    case bd * 4 + r * 2 + c:                                                                                   \
        return launch_ex(sell_vi2b_kernel<W, B, bd, r, c, SD>, dim3(grid), dim3(Vi2bShape<W, B>::kThreads), smem, \
                         pdl, s, V);
        K_(0, 0, 0) K_(0, 0, 1) K_(0, 1, 0) K_(0, 1, 1) K_(1, 0, 0) K_(1, 0, 1) K_(1, 1, 0) K_(1, 1, 1)
#undef K_
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_vi2b(const Vi2Args& V, int B, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                        bool pdl, cudaStream_t s) {
    const bool sd = V.dict_bytes > 0;   // the tuple dictionary in shared memory (B = 2, 16 warps)
    if (B == 2 && sd) return ncw == 16 ? launch_w<16, 2, true>(V, grid, smem, band, rearr, check, pdl, s)
                                       : cudaErrorInvalidValue;
    if (B == 2) return ncw == 16 ? launch_w<16, 2>(V, grid, smem, band, rearr, check, pdl, s)
                                 : launch_w<30, 2>(V, grid, smem, band, rearr, check, pdl, s);
    if (B == 4) return ncw == 30 ? launch_w<30, 4>(V, grid, smem, band, rearr, check, pdl, s)
                                 : launch_w<16, 4>(V, grid, smem, band, rearr, check, pdl, s);
    if (B == 8) return ncw == 8 ? launch_w<8, 8>(V, grid, smem, band, rearr, check, pdl, s)
                                : launch_w<15, 8>(V, grid, smem, band, rearr, check, pdl, s);
    return cudaErrorInvalidValue;
}

template <int W, int B, bool SD = false>
static cudaError_t prepare_w(int smem) {
    cudaError_t e = cudaSuccess;
#define A_(bd, r, c)                                                                                       \
    if (e == cudaSuccess)                                                                                  \
        e = cudaFuncSetAttribute(sell_vi2b_kernel<W, B, bd, r, c, SD>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                 smem);
    A_(0, 0, 0) A_(0, 0, 1) A_(0, 1, 0) A_(0, 1, 1) A_(1, 0, 0) A_(1, 0, 1) A_(1, 1, 0) A_(1, 1, 1)
#undef A_
    return e;
}

cudaError_t vi2b_prepare(int B, int ncw, int smem) {
    if (B == 2 && ncw == 16) {
        const cudaError_t e = prepare_w<16, 2, true>(smem);
        if (e != cudaSuccess) return e;
    }
    if (B == 2) return ncw == 16 ? prepare_w<16, 2>(smem) : prepare_w<30, 2>(smem);
    if (B == 4) return ncw == 30 ? prepare_w<30, 4>(smem) : prepare_w<16, 4>(smem);
    if (B == 8) return ncw == 8 ? prepare_w<8, 8>(smem) : prepare_w<15, 8>(smem);
    return cudaErrorInvalidValue;
}

template <int W, int B>
static cudaError_t occ_w(int smem, int* occ) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_vi2b_kernel<W, B, true, true, true>,
                                                         Vi2bShape<W, B>::kThreads, smem);
}

cudaError_t vi2b_occupancy(int B, int ncw, int smem, int* occ) {
    if (B == 2) return ncw == 16 ? occ_w<16, 2>(smem, occ) : occ_w<30, 2>(smem, occ);
    if (B == 4) return ncw == 30 ? occ_w<30, 4>(smem, occ) : occ_w<16, 4>(smem, occ);
    if (B == 8) return ncw == 8 ? occ_w<8, 8>(smem, occ) : occ_w<15, 8>(smem, occ);
    return cudaErrorInvalidValue;
}

}  // namespace cme
