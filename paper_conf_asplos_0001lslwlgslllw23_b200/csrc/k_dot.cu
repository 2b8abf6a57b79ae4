// k_dot.cu -- the `dot` edge op (reading R5; Table 2's V->E count 11 needs it):
// per head o < H the message is sum_{d<D} A[o*D+d] * B[o*D+d] (SDDMM-like when C = Edge,
// fused SDDMM+aggregate when C = Dst_V).  Vertex units (TV/WV/BV: one dst row per lane group)
// or edge units (TE/WE/BE: G consecutive CSR positions per lane group, atomics into dst).
//
// L <= 32 lanes split the head's D features (VEC-wide chunks), partial products are summed
// with FFMA and combined by an xor-shuffle butterfly inside the lane group.  The op is
// HBM/L2-bound at 0.43 flop/B (DESIGN.md roofline), so tensor cores cannot raise its roof;
// see DESIGN.md "dot" for the evidence.
#include "k_dispatch.cuh"

namespace ug {

template <int VEC>
__device__ __forceinline__ float dot_partial(const OpArgs &op, int64_t ra, int64_t rb, int o,
                                             int lane, int L) {
    float acc = 0.0f;
    const int d_end = (o + 1) * op.D;
    for (int f = o * op.D + lane * VEC; f < d_end; f += L * VEC) {
        float a[VEC], b[VEC];
        fetch<VEC>(op.A, ra, op_col(op.A, f), a);
        fetch<VEC>(op.B, rb, op_col(op.B, f), b);
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc = __fmaf_rn(a[i], b[i], acc);
    }
    return acc;
}

__device__ __forceinline__ float group_sum(float x, int L, unsigned mask) {
    for (int off = L >> 1; off > 0; off >>= 1) x += __shfl_xor_sync(mask, x, off);
    return x;
}

template <int GOP, int VEC, bool VUNIT>
__global__ void __launch_bounds__(256) k_dot(GraphArgs g, OpArgs op, int L_log2, int G,
                                             int64_t n_groups) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int L = 1 << L_log2;
    const int lane = (int)(t & (L - 1));
    const int64_t grp = t >> L_log2;
    if (grp >= n_groups) return;
    const int wl = threadIdx.x & 31;
    const unsigned mask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (wl & ~(L - 1)));

    if constexpr (VUNIT) {
        const int64_t v_end = min(g.V, (grp + 1) * (int64_t)G);
        for (int64_t v = grp * (int64_t)G; v < v_end; ++v) {
            const int64_t k0 = (int64_t)g.row_ptr[v] - g.rp_base;
            const int64_t k1 = (int64_t)g.row_ptr[v + 1] - g.rp_base;
            for (int o = 0; o < op.H; ++o) {
                float acc = g_init<GOP>();
                for (int64_t k = k0; k < k1; ++k) {
                    const int64_t src = g.col[k];
                    const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                    const float m = group_sum(
                        dot_partial<VEC>(op, op_row(op.A.type, src, v, e), op_row(op.B.type, src, v, e), o, lane, L),
                        L, mask);
                    if constexpr (GOP == UG_GATHER_ASSIGN) {
                        if (lane == 0) op.C[e * op.c_ld + o] = m;
                    } else {
                        acc = g_combine<GOP>(acc, m);
                    }
                }
                if constexpr (GOP != UG_GATHER_ASSIGN) {
                    if (lane == 0) op.C[v * op.c_ld + o] = g_finalize<GOP>(acc, k1 - k0);
                }
            }
        }
    } else {
        const int64_t k0 = grp * (int64_t)G;
        const int64_t k1 = min(g.E, k0 + G);
        for (int o = 0; o < op.H; ++o) {
            float acc = g_init<GOP>();
            int64_t cur = -1;
            for (int64_t k = k0; k < k1; ++k) {
                const int64_t src = g.col[k];
                const int64_t v = (int64_t)g.dst[k] - g.r0;
                const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                const float m = group_sum(
                    dot_partial<VEC>(op, op_row(op.A.type, src, v, e), op_row(op.B.type, src, v, e), o, lane, L),
                    L, mask);
                if constexpr (GOP == UG_GATHER_ASSIGN) {
                    if (lane == 0) op.C[e * op.c_ld + o] = m;
                } else {
                    if (v != cur) {
                        if (cur >= 0 && lane == 0) {
                            float a1[1] = {acc};
                            atomic_flush<GOP, 1>(op.C + cur * op.c_ld + o, a1, 1);
                        }
                        cur = v;
                        acc = g_init<GOP>();
                    }
                    acc = g_combine<GOP>(acc, m);
                }
            }
            if constexpr (GOP != UG_GATHER_ASSIGN) {
                if (cur >= 0 && lane == 0) {
                    float a1[1] = {acc};
                    atomic_flush<GOP, 1>(op.C + cur * op.c_ld + o, a1, 1);
                }
            }
        }
    }
}

cudaError_t launch_dot(bool vertex_units, int gather, const GraphArgs &g, const OpArgs &op,
                       const LaunchCfg &c, cudaStream_t s) {
    const int L = c.L > 32 ? 32 : c.L;
    const int64_t n_groups = cdiv(vertex_units ? g.V : g.E, c.G);
    const int64_t threads = n_groups * (int64_t)L;
    if (threads == 0) return cudaSuccess;
    const int64_t grid = cdiv(threads, c.block);
    const int L_log2 = ilog2(L);
    if (vertex_units) {
        UG_DISPATCH_VEC(c.vec, VEC,
            UG_DISPATCH_GOP(gather, GOP,
                k_dot<GOP, VEC, true><<<(unsigned)grid, c.block, 0, s>>>(g, op, L_log2, c.G, n_groups)));
    } else {
        UG_DISPATCH_VEC(c.vec, VEC,
            UG_DISPATCH_GOP(gather, GOP,
                k_dot<GOP, VEC, false><<<(unsigned)grid, c.block, 0, s>>>(g, op, L_log2, c.G, n_groups)));
    }
    return cudaGetLastError();
}

}  // namespace ug
