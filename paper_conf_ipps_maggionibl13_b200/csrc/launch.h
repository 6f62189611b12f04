// Host-side launchers of the step kernels, instantiated per batch width B in
// step_b{1,2,4,8}.cu (so nvcc compiles them in parallel).
#pragma once
#include <cuda_runtime.h>

#include "kernels_tma.cuh"

namespace cme {

template <int B>
cudaError_t launch_sell(const StepArgs& a, int grid, bool band, bool rearr, bool check, cudaStream_t s);
template <int B>
cudaError_t launch_tma(const TmaArgs& T, int ncw, int grid, int smem, bool band, bool rearr, bool check,
                       cudaStream_t s);
// cudaFuncSetAttribute(max dynamic smem) on every TMA variant of (B, ncw)
template <int B>
cudaError_t tma_prepare(int ncw, int smem);
template <int B>
cudaError_t tma_occupancy(int ncw, int smem, int* blocks_per_sm);

}  // namespace cme
