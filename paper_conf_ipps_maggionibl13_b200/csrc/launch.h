// Host-side launchers of the step kernels, instantiated per batch width B in
// step_b{1,2,4,8}.cu (so nvcc compiles them in parallel).
#pragma once
#include <cuda_runtime.h>
#include <utility>

#include "kernels_tma.cuh"

namespace cme {

// pdl: launch with programmatic stream serialization (the kernel may start
// while the previous kernel in the stream drains; it waits in-kernel).
template <int B>
cudaError_t launch_sell(const StepArgs& a, int grid, bool band, bool rearr, bool check, bool pdl, cudaStream_t s);
template <int B>
cudaError_t launch_tma(const TmaArgs& T, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                       cudaStream_t s);

// cudaLaunchKernelEx with an optional programmatic-dependency attribute
template <typename... KArgs, typename... Args>
cudaError_t launch_ex(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, bool pdl, cudaStream_t s,
                      Args&&... args) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}
// cudaFuncSetAttribute(max dynamic smem) on every TMA variant of (B, ncw)
template <int B>
cudaError_t tma_prepare(int ncw, int smem);
template <int B>
cudaError_t tma_occupancy(int ncw, int smem, int* blocks_per_sm);
// load every register-kernel variant of width B now (see launch_impl.cuh)
template <int B>
cudaError_t sell_preload();

}  // namespace cme

namespace cme {
struct CptArgs;
// compact-encoding TMA step kernel (step_cpt.cu, B = 1)
cudaError_t launch_cpt(const CptArgs& K, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                       cudaStream_t s);
cudaError_t cpt_prepare(int ncw, int smem);
cudaError_t cpt_occupancy(int ncw, int smem, int* blocks_per_sm);
struct ViArgs;
// value-indexed TMA step kernel (step_cpt.cu, B = 1)
cudaError_t launch_vi(const ViArgs& V, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                      cudaStream_t s);
cudaError_t vi_prepare(int ncw, int smem);
cudaError_t vi_occupancy(int ncw, int smem, int* blocks_per_sm);
// batched value-indexed TMA step kernel (step_cpt.cu, B = 2, 4, 8)
cudaError_t launch_vib(const ViArgs& V, int B, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                       bool pdl, cudaStream_t s);
cudaError_t vib_prepare(int B, int ncw, int smem);
cudaError_t vib_occupancy(int B, int ncw, int smem, int* blocks_per_sm);
struct Vi2Args;
// tile-record TMA step kernel (step_vi2.cu, B = 1): ncw = 16, 23 or 30; enc 0 value
// index, 1 value index as packed words, 2 f64 compact values (no dictionary)
cudaError_t launch_vi2(const Vi2Args& V, int ncw, int grid, int smem, bool band, bool rearr, bool check, int enc,
                       bool pdl, cudaStream_t s);
cudaError_t vi2_prepare(int ncw, int smem);
cudaError_t vi2_occupancy(int ncw, int smem, int* blocks_per_sm, int enc = 0);
// batched tile records (step_vi2b.cu, B = 2, 4, 8)
int vi2b_warps(int B, int force);
cudaError_t launch_vi2b(const Vi2Args& V, int B, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                        bool pdl, cudaStream_t s);
cudaError_t vi2b_prepare(int B, int ncw, int smem);
cudaError_t vi2b_occupancy(int B, int ncw, int smem, int* blocks_per_sm);
// the x-window variant (step_xw.cu): ncw = 16 or 30, enc 0 or 2
cudaError_t launch_vi2_xw(const Vi2Args& V, int ncw, int grid, int smem, bool band, bool rearr, bool check, int enc,
                          int mode /* 1 mirrored ring, 2 wrap */, bool pdl, cudaStream_t s);
cudaError_t vi2_xw_prepare(int ncw, int smem);
cudaError_t vi2_xw_occupancy(int ncw, int smem, int* blocks_per_sm, int enc);
struct ResArgs;
// SMEM-resident persistent Jacobi kernel (resident.cu)
cudaError_t resident_prepare(int smem);
cudaError_t resident_occupancy(int smem, int* blocks_per_sm);
cudaError_t launch_resident(const ResArgs& a, int grid, int smem, bool band, bool rearr, int rps, cudaStream_t s);
}  // namespace cme
namespace cme {
struct WfArgs;
// wavefront s-step kernel over the tile records (step_wf.cu, B = 1, one GPU): ncw = 16 or 30
cudaError_t launch_wf(const WfArgs& A, int ncw, int grid, int smem, bool band, bool rearr, bool check, bool pdl,
                      cudaStream_t s);
cudaError_t wf_prepare(int ncw, int smem);
cudaError_t wf_occupancy(int ncw, int smem, int* blocks_per_sm);
}  // namespace cme
