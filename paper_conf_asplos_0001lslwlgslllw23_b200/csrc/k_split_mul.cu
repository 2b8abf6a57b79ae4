// k_split_mul.cu -- SV instances for K_MUL (see k_split.cuh).
#include "k_split.cuh"

namespace ug {
UG_SV_INSTANTIATE(K_MUL)
}  // namespace ug
