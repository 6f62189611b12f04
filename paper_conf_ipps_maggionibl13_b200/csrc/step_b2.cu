// Step-kernel launchers for batch width B = 2 (see launch.h).
#include "launch_impl.cuh"

namespace cme {
CME_INSTANTIATE_LAUNCHERS(2)
}  // namespace cme
