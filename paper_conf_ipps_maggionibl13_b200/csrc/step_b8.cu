// Step-kernel launchers for batch width B = 8 (see launch.h).
#include "launch_impl.cuh"

namespace cme {
CME_INSTANTIATE_LAUNCHERS(8)
}  // namespace cme
