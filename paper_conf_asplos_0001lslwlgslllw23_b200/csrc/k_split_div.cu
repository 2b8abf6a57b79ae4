// k_split_div.cu -- SV instances for K_DIV (see k_split.cuh).
#include "k_split.cuh"

namespace ug {
UG_SV_INSTANTIATE(K_DIV)
}  // namespace ug
