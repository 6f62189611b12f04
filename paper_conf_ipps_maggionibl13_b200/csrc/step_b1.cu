// Step-kernel launchers for batch width B = 1 (see launch.h).
#include "launch_impl.cuh"

namespace cme {
CME_INSTANTIATE_LAUNCHERS(1)
}  // namespace cme
