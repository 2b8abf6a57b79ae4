// k_vertex.cu -- vertex-parallel owner-computes template: Thread-Vertex and Warp-Vertex
// (Fig. 6(b),(d)) with V-grouping G and feature
// tiling T (Fig. 6(f)).
//
// Canonical form: a unit is one destination row; L lanes share the
// unit's features (TV: L = T threads, WV: L = 32 T); lane l owns the VEC-wide feature
// chunks l, l + L, l + 2L, ... (Fig. 6(f): f = f10*32*T + f11*32 + f2).  A lane group
// processes G consecutive rows.  Rows are owned: no atomics, mean / zero-degree handled in
// registers (pass 2 of PAPER.md:405 inserts no atomics here).  With ftile > 0 the feature
// axis is first cut into column tiles ordered tile-major over the grid, so the rows being
// gathered concurrently touch one ftile-wide column slab of the operands (L2 residency).
// With C = Edge (message creation) the same traversal writes each in-edge's message.
#include "k_dispatch.cuh"

namespace ug {

template <int KE, int GOP, int VEC>
__global__ void __launch_bounds__(256) k_vertex(GraphArgs g, OpArgs op, int L_log2, int G,
                                                int ftile, int64_t n_groups, int n_tiles) {
    constexpr int R = (8 / VEC) > 0 ? (8 / VEC) : 1;   // register chunks per lane (8 floats)
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int L = 1 << L_log2;
    const int lane = (int)(t & (L - 1));
    const int64_t grp = t >> L_log2;
    if (grp >= n_groups * n_tiles) return;
    const int tile = (int)(grp / n_groups);
    const int64_t ugp = grp - (int64_t)tile * n_groups;
    const int f_lo = tile * ftile;
    const int f_hi = min(op.W, f_lo + ftile);
    const int stride = L * VEC;
    const int64_t v_end = min(g.V, (ugp + 1) * (int64_t)G);

    for (int64_t v = ugp * (int64_t)G; v < v_end; ++v) {
        const int64_t k0 = (int64_t)g.row_ptr[v] - g.rp_base;
        const int64_t k1 = (int64_t)g.row_ptr[v + 1] - g.rp_base;
        for (int fb = f_lo + lane * VEC; fb < f_hi; fb += stride * R) {
            int64_t ca[R], cb[R];
#pragma unroll
            for (int j = 0; j < R; ++j) {
                const int f = fb + j * stride;
                ca[j] = op_col(op.A, f);
                cb[j] = op_col(op.B, f);
            }
            if constexpr (GOP == UG_GATHER_ASSIGN) {
                for (int64_t k = k0; k < k1; ++k) {
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
                            st_vec_n<VEC>(op.C + e * op.c_ld + f, m, op.W - f);
                        }
                    }
                }
            } else {
                float acc[R][VEC];
#pragma unroll
                for (int j = 0; j < R; ++j)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[j][i] = g_init<GOP>();
gather_row<KE, GOP, VEC, R, 4>(g, op, v, k0, k1, 1, ca, cb, fb, stride, f_hi, acc);
                const int64_t deg = k1 - k0;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int f = fb + j * stride;
                    if (f < f_hi) {
                        float out[VEC];
#pragma unroll
                        for (int i = 0; i < VEC; ++i) out[i] = g_finalize<GOP>(acc[j][i], deg);
                        st_vec_n<VEC>(op.C + v * op.c_ld + f, out, op.W - f);
                    }
                }
            }
        }
    }
}

cudaError_t launch_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                          const LaunchCfg &c, cudaStream_t s) {
    const int ft = c.ftile > 0 ? c.ftile : op.W;
    const int n_tiles = (int)cdiv(op.W, ft);
    const int64_t n_groups = cdiv(g.V, c.G);
    const int64_t threads = n_groups * n_tiles * (int64_t)c.L;
    if (threads == 0) return cudaSuccess;
    const int block = c.block;
    const int64_t grid = cdiv(threads, block);
    const int L_log2 = ilog2(c.L);
    UG_DISPATCH_VEC(c.vec, VEC,
        UG_DISPATCH_KE(kedge, KE,
            UG_DISPATCH_GOP(gather, GOP,
                k_vertex<KE, GOP, VEC><<<(unsigned)grid, block, 0, s>>>(g, op, L_log2, c.G, ft,
                                                                        n_groups, n_tiles))));
    return cudaGetLastError();
}

// Edge-lanes warp-vertex ("WV_..._E1", round 2): for narrow features (W / VEC <= 8 chunks) the
// lanes of a warp split a destination row's IN-EDGES instead of its features -- lane l takes
// edges k0 + l, k0 + l + 32, ... and reduces every feature of its messages in registers, then an
// xor butterfly over the 32 lanes combines them (owner computes: one launch, no atomics, no
// init).  A row of in-degree d costs ceil(d / 32) dependent gather steps instead of d / UF, which
// is what bounds small, skewed graphs (C1 / C2) under the feature-lane schedules.
template <int KE, int GOP, int VEC, int NC>
__global__ void __launch_bounds__(256) k_vertex_el(GraphArgs g, OpArgs op, int G) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int64_t v0 = warp * G;
    if (v0 >= g.V) return;                            // whole warps leave together
    const int64_t v_end = min(g.V, v0 + (int64_t)G);
    int64_t ca[NC], cb[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        ca[j] = op_col(op.A, min(j * VEC, op.W - 1));
        cb[j] = op_col(op.B, min(j * VEC, op.W - 1));
    }
    for (int64_t v = v0; v < v_end; ++v) {
        const int64_t k0 = (int64_t)g.row_ptr[v] - g.rp_base;
        const int64_t k1 = (int64_t)g.row_ptr[v + 1] - g.rp_base;
        float acc[NC][VEC];
#pragma unroll
        for (int j = 0; j < NC; ++j)
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[j][i] = g_init<GOP>();
        // two in-edges per lane per step (k and k + 32: independent gathers in flight)
        for (int64_t k = k0 + lane; k < k1; k += 64) {
            const bool two = k + 32 < k1;
            const int64_t kb = two ? k + 32 : k;
            const int64_t src0 = g.col[k], src1 = g.col[kb];
            const int64_t e0 = g.eid ? (int64_t)g.eid[k] : k, e1 = g.eid ? (int64_t)g.eid[kb] : kb;
            const int64_t ra0 = op_row(op.A.type, src0, v, e0), rb0 = op_row(op.B.type, src0, v, e0);
            const int64_t ra1 = op_row(op.A.type, src1, v, e1), rb1 = op_row(op.B.type, src1, v, e1);
#pragma unroll
            for (int j = 0; j < NC; ++j) {
                if (j * VEC < op.W) {
                    float m0[VEC], m1[VEC];
                    message<KE, VEC>(op, ra0, ca[j], rb0, cb[j], m0);
                    message<KE, VEC>(op, ra1, ca[j], rb1, cb[j], m1);
#pragma unroll
                    for (int i = 0; i < VEC; ++i) {
                        acc[j][i] = g_combine<GOP>(acc[j][i], m0[i]);
                        if (two) acc[j][i] = g_combine<GOP>(acc[j][i], m1[i]);
                    }
                }
            }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1)
#pragma unroll
            for (int j = 0; j < NC; ++j)
#pragma unroll
                for (int i = 0; i < VEC; ++i)
                    acc[j][i] = g_combine<GOP>(acc[j][i], __shfl_xor_sync(0xffffffffu, acc[j][i], off));
        const int64_t deg = k1 - k0;
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            if (lane == j && j * VEC < op.W) {        // lane j stores chunk j
                float o[VEC];
#pragma unroll
                for (int i = 0; i < VEC; ++i) o[i] = g_finalize<GOP>(acc[j][i], deg);
                st_out<VEC>(op.C + v * op.c_ld + j * VEC, o, op.W - j * VEC, op.c_vec);
            }
        }
    }
}

cudaError_t launch_vertex_el(int kedge, int gather, const GraphArgs &g, const OpArgs &op, const LaunchCfg &c,
                             cudaStream_t s) {
    const int nc = (int)cdiv(op.W, c.vec);
    const int64_t warps = cdiv(g.V, c.G);
    if (warps == 0) return cudaSuccess;
    const int64_t grid = cdiv(warps * 32, 256);
#define UG_EL(NCV)                                                                                       \
    UG_DISPATCH_KE(kedge, KE,                                                                            \
        UG_DISPATCH_RED(gather, GOP, k_vertex_el<KE, GOP, VEC, NCV><<<(unsigned)grid, 256, 0, s>>>(g, op, c.G)))
    UG_DISPATCH_VEC(c.vec, VEC, {
        switch (nc) {
        case 1: UG_EL(1); break;
        case 2: UG_EL(2); break;
        case 3: case 4: UG_EL(4); break;
        default: UG_EL(8); break;
        }
    });
#undef UG_EL
    return cudaGetLastError();
}

}  // namespace ug
