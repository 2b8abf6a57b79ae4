// k_split_addsub.cu -- SV instances for K_ADD, K_SUB (see k_split.cuh).
#include "k_split.cuh"

namespace ug {
UG_SV_INSTANTIATE(K_ADD)
UG_SV_INSTANTIATE(K_SUB)
}  // namespace ug
