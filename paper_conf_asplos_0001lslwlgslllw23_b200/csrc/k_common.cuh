// k_common.cuh -- device functions shared by the schedule templates (the paper's
// "device function interface": global-function templates per strategy,
// device functions per arithmetic).  Compiled with -fmad=true but every message is formed
// with explicit _rn intrinsics so it is rounded once, exactly as a standalone
// message-creation op would (reading R11); accumulation order is the only freedom.
#pragma once
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>

#include "ug_internal.h"

namespace ug {

// ---------------------------------------------------------------- edge_op (Fig. 5 line 18)
template <int KE>
__device__ __forceinline__ float edge_fn(float a, float b) {
    if constexpr (KE == K_COPY) return a;
    else if constexpr (KE == K_ADD) return __fadd_rn(a, b);
    else if constexpr (KE == K_SUB) return __fsub_rn(a, b);
    else if constexpr (KE == K_MUL) return __fmul_rn(a, b);
    else return __fdiv_rn(a, b);
}

// ---------------------------------------------------------------- gather_op (Fig. 5 line 19)
// Total order with -0 < +0 and NaN-propagating (R12): max.NaN / min.NaN are IEEE 754-2019
// maximum / minimum -- the canonical NaN 0x7FFFFFFF if either input is NaN, and -0 < +0 (measured
// on this B200 by scripts/probes/minmax_zero.cu: max(-0, +0) = +0, min(-0, +0) = -0 in either
// argument order), so no explicit signed-zero tie rule is needed.
__device__ __forceinline__ float fmax_nan(float a, float b) {
    float m;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(m) : "f"(a), "f"(b));
    return m;
}
__device__ __forceinline__ float fmin_nan(float a, float b) {
    float m;
    asm("min.NaN.f32 %0, %1, %2;" : "=f"(m) : "f"(a), "f"(b));
    return m;
}
__device__ __forceinline__ float tmax(float a, float b) { return fmax_nan(a, b); }
__device__ __forceinline__ float tmin(float a, float b) { return fmin_nan(a, b); }
constexpr uint32_t UG_CANONICAL_NAN = 0x7FFFFFFFu;

template <int GOP>
__device__ __forceinline__ float g_init() {
    if constexpr (GOP == UG_GATHER_MAX) return -CUDART_INF_F;
    else if constexpr (GOP == UG_GATHER_MIN) return CUDART_INF_F;
    else return 0.0f;
}

template <int GOP>
__device__ __forceinline__ float g_combine(float acc, float m) {
    if constexpr (GOP == UG_GATHER_MAX) return tmax(acc, m);
    else if constexpr (GOP == UG_GATHER_MIN) return tmin(acc, m);
    else return __fadd_rn(acc, m);
}

// Final value of an owner-computed row (R7 zero in-degree -> 0; R8 mean = sum / deg with one
// IEEE division).
template <int GOP>
__device__ __forceinline__ float g_finalize(float acc, int64_t deg) {
    if (deg == 0) return 0.0f;
    if constexpr (GOP == UG_GATHER_MEAN) return __fdiv_rn(acc, (float)deg);
    else return acc;
}

// ---------------------------------------------------------------- vector loads
template <int VEC> struct VecT;
template <> struct VecT<1> { using T = float; };
template <> struct VecT<2> { using T = float2; };
template <> struct VecT<4> { using T = float4; };

template <int VEC>
__device__ __forceinline__ void ldg_vec(const float *__restrict__ p, float (&r)[VEC]) {
    if constexpr (VEC == 1) {
        r[0] = __ldg(p);
    } else if constexpr (VEC == 2) {
        float2 t = __ldg(reinterpret_cast<const float2 *>(p));
        r[0] = t.x; r[1] = t.y;
    } else {
        float4 t = __ldg(reinterpret_cast<const float4 *>(p));
        r[0] = t.x; r[1] = t.y; r[2] = t.z; r[3] = t.w;
    }
}

template <int VEC>
__device__ __forceinline__ void st_vec(float *p, const float (&r)[VEC]) {
    if constexpr (VEC == 1) {
        p[0] = r[0];
    } else if constexpr (VEC == 2) {
        *reinterpret_cast<float2 *>(p) = make_float2(r[0], r[1]);
    } else {
        *reinterpret_cast<float4 *>(p) = make_float4(r[0], r[1], r[2], r[3]);
    }
}

// ---------------------------------------------------------------- L2 cache-policy loads
// createpolicy + ld.global.nc.L2::cache_hint: keep the gathered feature slab resident
// (evict_last) while streaming index arrays through L2 (evict_first).
#ifndef UG_KEEP_FRACTION
#define UG_KEEP_FRACTION 1.0
#endif
#define UG_STR2(x) #x
#define UG_STR(x) UG_STR2(x)
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, " UG_STR(UG_KEEP_FRACTION) ";" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

template <int VEC>
__device__ __forceinline__ void ldg_vec_hint(const float *__restrict__ p, float (&r)[VEC], uint64_t pol) {
    if constexpr (VEC == 1) {
        asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(r[0]) : "l"(p), "l"(pol));
    } else if constexpr (VEC == 2) {
        asm("ld.global.nc.L2::cache_hint.v2.f32 {%0, %1}, [%2], %3;" : "=f"(r[0]), "=f"(r[1]) : "l"(p), "l"(pol));
    } else {
        asm("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
            : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]) : "l"(p), "l"(pol));
    }
}

template <int VEC>
__device__ __forceinline__ void st_vec_hint(float *p, const float (&r)[VEC], uint64_t pol) {
    if constexpr (VEC == 1) {
        asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(r[0]), "l"(pol) : "memory");
    } else if constexpr (VEC == 2) {
        asm volatile("st.global.L2::cache_hint.v2.f32 [%0], {%1, %2}, %3;" ::"l"(p), "f"(r[0]), "f"(r[1]), "l"(pol)
                     : "memory");
    } else {
        asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "f"(r[0]), "f"(r[1]),
                     "f"(r[2]), "f"(r[3]), "l"(pol) : "memory");
    }
}

__device__ __forceinline__ int32_t ldg_i32_hint(const int32_t *__restrict__ p, uint64_t pol) {
    int32_t r;
    asm("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}

template <int VEC>
__device__ __forceinline__ void fetch_hint(const Operand &x, int64_t row, int64_t col, float (&r)[VEC],
                                           uint64_t pol) {
    const float *p = x.p + row * x.ld + col;
    if (x.div == 1) {
        ldg_vec_hint<VEC>(p, r, pol);
    } else {
        float s = __ldg(p);
#pragma unroll
        for (int i = 0; i < VEC; ++i) r[i] = s;
    }
}

template <int KE, int VEC>
__device__ __forceinline__ void message_hint(const OpArgs &op, int64_t ra, int64_t ca, int64_t rb,
                                             int64_t cb, float (&m)[VEC], uint64_t pol) {
    float a[VEC];
    fetch_hint<VEC>(op.A, ra, ca, a, pol);
    if constexpr (KE == K_COPY) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) m[i] = a[i];
    } else {
        float b[VEC];
        fetch_hint<VEC>(op.B, rb, cb, b, pol);
#pragma unroll
        for (int i = 0; i < VEC; ++i) m[i] = edge_fn<KE>(a[i], b[i]);
    }
}

// Store the first n (<= VEC) lanes of a vector: the ragged tail of a row.
template <int VEC>
__device__ __forceinline__ void st_vec_n(float *p, const float (&r)[VEC], int n) {
    if (n >= VEC) { st_vec<VEC>(p, r); return; }
#pragma unroll
    for (int i = 0; i < VEC; ++i)
        if (i < n) p[i] = r[i];
}

// Store n (<= VEC) values into C whose rows only guarantee `cvec`-wide alignment (SV loads
// with a wider vector than C's layout allows: e.g. float4 loads, 8-byte-aligned output rows).
template <int VEC>
__device__ __forceinline__ void st_out(float *p, const float (&r)[VEC], int n, int cvec) {
    if (n >= VEC && cvec >= VEC) {
        st_vec<VEC>(p, r);
    } else if (VEC == 4 && n >= 4 && cvec >= 2) {
        *reinterpret_cast<float2 *>(p) = make_float2(r[0], r[1]);
        *reinterpret_cast<float2 *>(p + 2) = make_float2(r[VEC > 2 ? 2 : 0], r[VEC > 3 ? 3 : 0]);
    } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i)
            if (i < n) p[i] = r[i];
    }
}

// Row of an operand for the edge (src, dst, e): type_idx_dict.
__device__ __forceinline__ int64_t op_row(int32_t type, int64_t src, int64_t dst, int64_t e) {
    return type == UG_T_SRC_V ? src : (type == UG_T_DST_V ? dst : e);
}

// Column of feature f in an operand: full width -> f, per-head width -> f / D (R6).
__device__ __forceinline__ int64_t op_col(const Operand &x, int f) {
    return x.div == 1 ? (int64_t)f : (int64_t)(f / x.div);
}

// VEC features starting at column `col` of row `row` (broadcast when x.div > 1; the
// VEC features of one chunk always lie inside one head: the host guarantees D % VEC == 0).
template <int VEC>
__device__ __forceinline__ void fetch(const Operand &x, int64_t row, int64_t col, float (&r)[VEC]) {
    const float *p = x.p + row * x.ld + col;
    if (x.div == 1) {
        ldg_vec<VEC>(p, r);
    } else {
        float s = __ldg(p);
#pragma unroll
        for (int i = 0; i < VEC; ++i) r[i] = s;
    }
}

// Message vector for one edge (elementwise ops).
template <int KE, int VEC>
__device__ __forceinline__ void message(const OpArgs &op, int64_t ra, int64_t ca, int64_t rb,
                                        int64_t cb, float (&m)[VEC]) {
    float a[VEC];
    fetch<VEC>(op.A, ra, ca, a);
    if constexpr (KE == K_COPY) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) m[i] = a[i];
    } else {
        float b[VEC];
        fetch<VEC>(op.B, rb, cb, b);
#pragma unroll
        for (int i = 0; i < VEC; ++i) m[i] = edge_fn<KE>(a[i], b[i]);
    }
}

// Message when A is a full-width Src_V operand addressable with 32-bit element offsets
// (V * ld < 2^32): the row address is one IMAD + IMAD.WIDE from the column index.
template <int KE, int VEC>
__device__ __forceinline__ void message_fast(const OpArgs &op, uint32_t src, uint32_t f, int64_t rb,
                                             int64_t cb, float (&m)[VEC]) {
    ldg_vec<VEC>(op.A.p + (src * (uint32_t)op.A.ld + f), m);
    if constexpr (KE != K_COPY) {
        float b[VEC];
        fetch<VEC>(op.B, rb, cb, b);
#pragma unroll
        for (int i = 0; i < VEC; ++i) m[i] = edge_fn<KE>(m[i], b[i]);
    }
}

// Owner-computes gather of one destination row v over in-edge positions k0, k0+kstep, ... < k1
// into R register chunks of VEC features (chunk j at feature fb + j*stride, valid if < f_hi).
// U edges are processed per step so that U*R row loads are in flight per lane.
template <int KE, int GOP, int VEC, int R, int U>
__device__ __forceinline__ void gather_row(const GraphArgs &g, const OpArgs &op, int64_t v, int64_t k0,
                                           int64_t k1, int64_t kstep, const int64_t (&ca)[R],
                                           const int64_t (&cb)[R], int fb, int stride, int f_hi,
                                           float (&acc)[R][VEC]) {
    int64_t k = k0;
    for (; k + (U - 1) * kstep < k1; k += U * kstep) {
        int64_t ra[U], rb[U];
#pragma unroll
        for (int q = 0; q < U; ++q) {
            const int64_t kk = k + q * kstep;
            const int64_t src = g.col[kk];
            const int64_t e = g.eid ? (int64_t)g.eid[kk] : kk;
            ra[q] = op_row(op.A.type, src, v, e);
            rb[q] = op_row(op.B.type, src, v, e);
        }
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const int f = fb + j * stride;
            if (f < f_hi) {
                float m[U][VEC];
#pragma unroll
                for (int q = 0; q < U; ++q) message<KE, VEC>(op, ra[q], ca[j], rb[q], cb[j], m[q]);
#pragma unroll
                for (int q = 0; q < U; ++q)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[j][i] = g_combine<GOP>(acc[j][i], m[q][i]);
            }
        }
    }
    for (; k < k1; k += kstep) {
        const int64_t src = g.col[k];
        const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
        const int64_t ra = op_row(op.A.type, src, v, e);
        const int64_t rb = op_row(op.B.type, src, v, e);
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const int f = fb + j * stride;
            if (f < f_hi) {
                float m[VEC];
                message<KE, VEC>(op, ra, ca[j], rb, cb[j], m);
#pragma unroll
                for (int i = 0; i < VEC; ++i) acc[j][i] = g_combine<GOP>(acc[j][i], m[i]);
            }
        }
    }
}

// ---------------------------------------------------------------- atomics (pass 2)
// max/min on fp32 by the integer-order trick: non-negative floats order like signed ints,
// negative floats order reversed as unsigned ints; -0 (0x80000000) < +0 (0).
// NaN (R12) is absorbing: for max it is stored as 0x7FFFFFFF (the largest positive int: no later
// value replaces it); for min as 0xFFFFFFFF (the largest unsigned: no later value replaces it),
// which the epilogue rewrites to the canonical 0x7FFFFFFF.
__device__ __forceinline__ void atomic_max_f32(float *addr, float v) {
    if (isnan(v)) atomicMax(reinterpret_cast<int *>(addr), (int)UG_CANONICAL_NAN);
    else if (!signbit(v)) atomicMax(reinterpret_cast<int *>(addr), __float_as_int(v));
    else atomicMin(reinterpret_cast<unsigned int *>(addr), __float_as_uint(v));
}
__device__ __forceinline__ void atomic_min_f32(float *addr, float v) {
    if (isnan(v)) atomicMax(reinterpret_cast<unsigned int *>(addr), 0xFFFFFFFFu);
    else if (!signbit(v)) atomicMin(reinterpret_cast<int *>(addr), __float_as_int(v));
    else atomicMax(reinterpret_cast<unsigned int *>(addr), __float_as_uint(v));
}

template <int GOP, int VEC>
__device__ __forceinline__ void atomic_flush(float *p, const float (&acc)[VEC], int n) {
    if constexpr (GOP == UG_GATHER_SUM || GOP == UG_GATHER_MEAN) {
        if (n >= VEC) {
            if constexpr (VEC == 4) {
                atomicAdd(reinterpret_cast<float4 *>(p), make_float4(acc[0], acc[1], acc[2], acc[3]));
                return;
            } else if constexpr (VEC == 2) {
                atomicAdd(reinterpret_cast<float2 *>(p), make_float2(acc[0], acc[1]));
                return;
            }
        }
#pragma unroll
        for (int i = 0; i < VEC; ++i)
            if (i < n) atomicAdd(p + i, acc[i]);
    } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i) {
            if (i < n) {
                if constexpr (GOP == UG_GATHER_MAX) atomic_max_f32(p + i, acc[i]);
                else atomic_min_f32(p + i, acc[i]);
            }
        }
    }
}

// Release / acquire fence of the last-arriver merges (store partials; fence; relaxed atomicAdd
// on the arrival counter  ||  atomicAdd; fence; load partials): the PTX fence-based
// release-acquire pattern at gpu scope, lighter than __threadfence()'s fence.sc.gpu.
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

// Helpers for launch sizing.
__host__ __device__ __forceinline__ int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace ug
