// k_svg_tma.cu -- staged SV instances, MODE 0 (TMA gather4 row staging, "_M1").
#include <cstring>

#include "k_svg_launch.cuh"

namespace ug {
template cudaError_t launch_svg_mode<0>(int, int, const GraphArgs &, const OpArgs &, int, int, const SplitPlan &,
                                        float *, cudaStream_t);
}  // namespace ug
