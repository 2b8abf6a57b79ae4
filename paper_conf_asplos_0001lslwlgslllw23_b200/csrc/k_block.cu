// k_block.cu -- Block-Vertex (BV): the block-level vertex schedule of the north star
// (not in the paper, whose space stops at thread/warp: Table 5).
//
// One CTA owns G consecutive destination rows.  Its NW warps split each row's in-edges
// round-robin (warp w takes positions k0+w, k0+w+NW, ...); the 32 lanes of a warp cover a
// 32*VEC*R-wide feature block in registers.  Per-warp partial reductions meet in shared
// memory and are combined in warp order (deterministic), finalised (mean / zero in-degree)
// and stored by the owner CTA: no atomics, and a hub row of in-degree d costs d/NW
// sequential steps instead of d (degree skew).
#include "k_dispatch.cuh"

namespace ug {

template <int KE, int GOP, int VEC>
__global__ void __launch_bounds__(512) k_bvertex(GraphArgs g, OpArgs op, int G) {
    constexpr int R = (8 / VEC) > 0 ? (8 / VEC) : 1;
    constexpr int CH = 32 * VEC * R;   // features per register block
    extern __shared__ float sm[];      // [NW][CH]
    const int NW = blockDim.x >> 5;
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int64_t v_end = min(g.V, ((int64_t)blockIdx.x + 1) * G);

    for (int64_t v = (int64_t)blockIdx.x * G; v < v_end; ++v) {
        const int64_t k0 = (int64_t)g.row_ptr[v] - g.rp_base;
        const int64_t k1 = (int64_t)g.row_ptr[v + 1] - g.rp_base;
        for (int fb0 = 0; fb0 < op.W; fb0 += CH) {
            int64_t ca[R], cb[R];
#pragma unroll
            for (int j = 0; j < R; ++j) {
                const int f = fb0 + j * 32 * VEC + lane * VEC;
                ca[j] = op_col(op.A, f);
                cb[j] = op_col(op.B, f);
            }
            if constexpr (GOP == UG_GATHER_ASSIGN) {
                for (int64_t k = k0 + warp; k < k1; k += NW) {
                    const int64_t src = g.col[k];
                    const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                    const int64_t ra = op_row(op.A.type, src, v, e);
                    const int64_t rb = op_row(op.B.type, src, v, e);
#pragma unroll
                    for (int j = 0; j < R; ++j) {
                        const int f = fb0 + j * 32 * VEC + lane * VEC;
                        if (f < op.W) {
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
                gather_row<KE, GOP, VEC, R, 2>(g, op, v, k0 + warp, k1, NW, ca, cb, fb0 + lane * VEC, 32 * VEC, op.W, acc);
#pragma unroll
                for (int j = 0; j < R; ++j)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) sm[warp * CH + j * 32 * VEC + lane * VEC + i] = acc[j][i];
                __syncthreads();
                const int64_t deg = k1 - k0;
                for (int idx = threadIdx.x; idx < CH; idx += blockDim.x) {
                    const int f = fb0 + idx;
                    if (f < op.W) {
                        float r = g_init<GOP>();
                        for (int w = 0; w < NW; ++w) r = g_combine<GOP>(r, sm[w * CH + idx]);
                        op.C[v * op.c_ld + f] = g_finalize<GOP>(r, deg);
                    }
                }
                __syncthreads();
            }
        }
    }
}

cudaError_t launch_block_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                                const LaunchCfg &c, cudaStream_t s) {
    const int64_t grid = cdiv(g.V, c.G);
    if (grid == 0) return cudaSuccess;
    const int NW = c.block / 32;
    UG_DISPATCH_VEC(c.vec, VEC,
        UG_DISPATCH_KE(kedge, KE,
            UG_DISPATCH_GOP(gather, GOP, {
                constexpr int R = (8 / VEC) > 0 ? (8 / VEC) : 1;
                const size_t smem = (size_t)NW * 32 * VEC * R * sizeof(float);
                k_bvertex<KE, GOP, VEC><<<(unsigned)grid, c.block, smem, s>>>(g, op, c.G);
            })));
    return cudaGetLastError();
}

}  // namespace ug
