// Step-kernel launchers for batch width B = 4 (see launch.h).
#include "launch_impl.cuh"

namespace cme {
CME_INSTANTIATE_LAUNCHERS(4)
}  // namespace cme
