// Launchers of the SMEM-resident persistent Jacobi kernel (kernels_resident.cuh).
#include "kernels_resident.cuh"
#include "launch.h"

namespace cme {

#define CME_RES_VARIANTS(X) \
    X(0, 0, 1) X(0, 1, 1) X(1, 0, 1) X(1, 1, 1) X(0, 0, 2) X(0, 1, 2) X(1, 0, 2) X(1, 1, 2) \
    X(0, 0, 4) X(0, 1, 4) X(1, 0, 4) X(1, 1, 4)

cudaError_t resident_prepare(int smem) {
    cudaError_t e = cudaSuccess;
#define A(bd, r, R) \
    if (e == cudaSuccess) \
        e = cudaFuncSetAttribute(sell_resident_kernel<bd, r, R>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    CME_RES_VARIANTS(A)
#undef A
    return e;
}

cudaError_t resident_occupancy(int smem, int* occ) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, sell_resident_kernel<true, true, 4>, kResThreads, smem);
}

// Cooperative launch: the grid (<= one CTA per SM) is guaranteed co-resident,
// which the epoch waits and the grid barriers rely on.  rps = row slots per
// thread (1, 2 or 4).
cudaError_t launch_resident(const ResArgs& a, int grid, int smem, bool band, bool rearr, int rps, cudaStream_t s) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kResThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const int key = (band ? 1 : 0) * 100 + (rearr ? 1 : 0) * 10 + rps;
    switch (key) {
#define K(bd, r, R) \
    case bd * 100 + r * 10 + R: return cudaLaunchKernelEx(&cfg, sell_resident_kernel<bd, r, R>, a);
        CME_RES_VARIANTS(K)
#undef K
    }
    return cudaErrorInvalidValue;
}

}  // namespace cme
