// k_svg_async.cu -- staged SV instances, MODE 1 (cp.async / LDGSTS row staging, "_A1").
#include <cstring>

#include "k_svg_launch.cuh"

namespace ug {
template cudaError_t launch_svg_mode<1>(int, int, const GraphArgs &, const OpArgs &, int, int, const SplitPlan &,
                                        float *, cudaStream_t);
}  // namespace ug
