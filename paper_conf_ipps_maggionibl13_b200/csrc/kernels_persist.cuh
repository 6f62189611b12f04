// Persistent cooperative variant for small (L2-resident) problems.
//
// Below ~1M rows an iteration moves only a few MB that sit in the 126 MB L2,
// and one kernel launch per iteration (graph node turnaround ~2 us) costs more
// than the arithmetic.  This kernel runs a whole check block -- C steps --
// in ONE cooperative launch: a grid of co-resident CTAs walks the slices
// grid-stride, then a grid-wide barrier (cooperative_groups grid.sync) swaps
// the buffers.  x is read L2-coherent (.cg) because other CTAs rewrite it
// between barriers; the packed matrix streams keep the L1::no_allocate path.
// Same arithmetic as sell_step_kernel (kernels.cuh), the CHECK partials of the
// block's last step go to partials[blockIdx.x].
#pragma once
#include <cooperative_groups.h>

#include "kernels.cuh"

namespace cme {

struct PersistArgs {
    StepArgs a;          // a.x / a.y unused; buffers below
    double* xb0;
    double* xb1;
    int32_t start;       // buffer holding the block's input iterate
    int32_t steps;       // C
};

template <bool BAND, bool REARR, bool DAMP>
__global__ void __launch_bounds__(kCta) sell_persistent_kernel(const PersistArgs P) {
    const StepArgs& a = P.a;
    if (a.stop != nullptr && *a.stop) return;
    cooperative_groups::grid_group grid = cooperative_groups::this_grid();
    const uint64_t pol = evict_first_policy();
    const int lane = threadIdx.x & 31;
    const int64_t wstride = (int64_t)gridDim.x * kWarpsPerCta;
    const int64_t w0 = (int64_t)blockIdx.x * kWarpsPerCta + (threadIdx.x >> 5);
    double sy = 0.0, sx = 0.0, sd = 0.0, md = 0.0, mx = 0.0;
    for (int t = 0; t < P.steps; ++t) {
        const int src = (P.start + t) & 1;
        const double* x = src ? P.xb1 : P.xb0;
        double* y = src ? P.xb0 : P.xb1;
        const double* pre = t == 0 ? a.pre_scale : nullptr;
        const bool last = t == P.steps - 1;
        for (int64_t q = a.slice_begin + w0; q < a.slice_end; q += wstride) {
            const SlotOut o = sell_slot<BAND, REARR, DAMP, true, true>(a, q, lane, pol, x, y, pre);
            if (last) check_accum(o, sy, sx, sd, md, mx);
        }
        if (!last) grid.sync();
    }
    cta_check_partials<kWarpsPerCta>(sy, sx, sd, md, mx, a.partials);
}

}  // namespace cme
