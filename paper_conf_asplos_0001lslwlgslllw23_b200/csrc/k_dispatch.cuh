// k_dispatch.cuh -- runtime (edge_op, gather_op, vec) -> template instance.
// This is the paper's code-generation step done at compile time: the op
// set is closed (160 ops), so every (strategy template x device-function) pair is
// instantiated ahead of time instead of generated per call.
#pragma once
#include "k_common.cuh"

#define UG_DISPATCH_VEC(vec, VEC, ...)                         \
    switch (vec) {                                             \
    case 4: { constexpr int VEC = 4; __VA_ARGS__; } break;     \
    case 2: { constexpr int VEC = 2; __VA_ARGS__; } break;     \
    default: { constexpr int VEC = 1; __VA_ARGS__; } break;    \
    }

#define UG_DISPATCH_KE(ke, KE, ...)                            \
    switch (ke) {                                              \
    case K_COPY: { constexpr int KE = K_COPY; __VA_ARGS__; } break; \
    case K_ADD:  { constexpr int KE = K_ADD;  __VA_ARGS__; } break; \
    case K_SUB:  { constexpr int KE = K_SUB;  __VA_ARGS__; } break; \
    case K_MUL:  { constexpr int KE = K_MUL;  __VA_ARGS__; } break; \
    default:     { constexpr int KE = K_DIV;  __VA_ARGS__; } break; \
    }

// Reducers only (no assign).
#define UG_DISPATCH_RED(gop, GOP, ...)                                         \
    switch (gop) {                                                             \
    case UG_GATHER_SUM:  { constexpr int GOP = UG_GATHER_SUM;  __VA_ARGS__; } break; \
    case UG_GATHER_MAX:  { constexpr int GOP = UG_GATHER_MAX;  __VA_ARGS__; } break; \
    case UG_GATHER_MIN:  { constexpr int GOP = UG_GATHER_MIN;  __VA_ARGS__; } break; \
    default:             { constexpr int GOP = UG_GATHER_MEAN; __VA_ARGS__; } break; \
    }

// Reducers + assign.
#define UG_DISPATCH_GOP(gop, GOP, ...)                                         \
    switch (gop) {                                                             \
    case UG_GATHER_ASSIGN: { constexpr int GOP = UG_GATHER_ASSIGN; __VA_ARGS__; } break; \
    case UG_GATHER_SUM:  { constexpr int GOP = UG_GATHER_SUM;  __VA_ARGS__; } break; \
    case UG_GATHER_MAX:  { constexpr int GOP = UG_GATHER_MAX;  __VA_ARGS__; } break; \
    case UG_GATHER_MIN:  { constexpr int GOP = UG_GATHER_MIN;  __VA_ARGS__; } break; \
    default:             { constexpr int GOP = UG_GATHER_MEAN; __VA_ARGS__; } break; \
    }

namespace ug {
__host__ __forceinline__ int ilog2(int x) {
    int l = 0;
    while ((1 << l) < x) ++l;
    return l;
}
}  // namespace ug
