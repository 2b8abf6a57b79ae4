// k_msg_el.cu -- message creation with lanes over EDGES ("SV_Gg_E1" with C = Edge; round 2).
//
// Message creation (gather assign, Table 4 rows 1-5) writes one W-wide row per
// edge.  For narrow messages (W <= 8: GAT's per-head scores, the F = 1 messages of the C5
// correctness matrix) the feature-lane schedules leave most lanes idle and, edge-parallel (TE /
// WE), stream the COO destination array beside col_idx.  Here a warp walks one SV chunk (a row
// segment of <= G in-edges: the destination v is the chunk's row, so no per-edge dst is read and a
// Dst_V operand is loaded once per chunk) and its 32 lanes take 32 consecutive in-edges per step:
// the col_idx loads, the Edge-operand loads and the message stores of a step are each one
// contiguous 32 * W-float range (edge id = CSR position on a dst-sorted graph; otherwise the
// stores scatter through eid).  Every message is formed exactly as the other schedules form it
// (edge_fn, one IEEE rounding), so results are bit-identical.
#include "k_split.cuh"

namespace ug {

template <int KE, int NW>
__global__ void __launch_bounds__(256) k_msg_el(GraphArgs g, OpArgs op, const int4 *__restrict__ chunks,
                                               int64_t n_chunks) {
    const int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (u >= n_chunks) return;
    const int4 ch = chunks[u];
    const int64_t v = ch.x;
    const uint64_t stream = l2_policy_evict_first();
    for (int64_t k = ch.y + lane; k < ch.z; k += 32) {
        const int64_t src = (int64_t)ldg_i32_hint(g.col + k, stream);
        const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
        const int64_t ra = op_row(op.A.type, src, v, e);
        const int64_t rb = op_row(op.B.type, src, v, e);
        float m[NW];
#pragma unroll
        for (int j = 0; j < NW; ++j) {
            if (j < op.W) {
                float t[1];
                message<KE, 1>(op, ra, op_col(op.A, j), rb, op_col(op.B, j), t);
                m[j] = t[0];
            }
        }
        float *cp = op.C + e * op.c_ld;
#pragma unroll
        for (int j = 0; j < NW; ++j)
            if (j < op.W) cp[j] = m[j];
    }
}

// Fast form: A is a full-width Src_V operand, identity edge ids, B absent / Dst_V (hoisted per
// chunk) / Edge -- 32-bit offsets, no per-edge type dispatch (C5 u_add_v: F = H = 1).
template <int KE, int NW, int BM>
__global__ void __launch_bounds__(256) k_msg_el_fast(GraphArgs g, OpArgs op, const int4 *__restrict__ chunks,
                                                    int64_t n_chunks) {
    const int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (u >= n_chunks) return;
    const int4 ch = chunks[u];
    const uint64_t stream = l2_policy_evict_first(), keep = l2_policy_evict_last();
    const uint32_t lda = (uint32_t)op.A.ld, ldb = (uint32_t)op.B.ld, ldc = (uint32_t)op.c_ld;
    float bconst[NW];
    if constexpr (BM == 1) {
#pragma unroll
        for (int j = 0; j < NW; ++j) bconst[j] = j < op.W ? __ldg(op.B.p + (int64_t)ch.x * op.B.ld + op_col(op.B, j)) : 0.0f;
    }
    for (int k = ch.y + lane; k < ch.z; k += 32) {
        const uint32_t src = (uint32_t)ldg_i32_hint(g.col + k, stream);
        const float *ap = op.A.p + src * lda;
        float m[NW];
#pragma unroll
        for (int j = 0; j < NW; ++j) {
            if (j < op.W) {
                float a[1];
                ldg_vec_hint<1>(ap + j, a, keep);
                float b = 0.0f;
                if constexpr (BM == 1) b = bconst[j];
                else if constexpr (BM == 2) b = __ldg(op.B.p + ((uint32_t)k * ldb + (uint32_t)op_col(op.B, j)));
                m[j] = edge_fn<KE>(a[0], b);
            }
        }
        float *cp = op.C + (uint32_t)k * ldc;
#pragma unroll
        for (int j = 0; j < NW; ++j)
            if (j < op.W) cp[j] = m[j];
    }
}

cudaError_t launch_msg_el(int kedge, const GraphArgs &g, const OpArgs &op, const SplitPlan &plan, cudaStream_t s) {
    if (plan.n_chunks == 0) return cudaSuccess;
    const int64_t grid = cdiv(plan.n_chunks * 32, 256);
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const uint64_t lim = 1ull << 32;
    const bool fast = op.A.type == UG_T_SRC_V && op.A.div == 1 && g.eid == nullptr &&
                      (uint64_t)g.V_src * (uint64_t)op.A.ld < lim && (uint64_t)g.E * (uint64_t)op.c_ld < lim &&
                      (kedge == K_COPY || op.B.type == UG_T_DST_V ||
                       (op.B.type == UG_T_EDGE && (uint64_t)g.E * (uint64_t)op.B.ld < lim));
    if (fast) {
        const int bm = kedge == K_COPY ? 0 : (op.B.type == UG_T_DST_V ? 1 : 2);
#define UG_MELF(NWV)                                                                                          \
    UG_DISPATCH_KE(kedge, KE, {                                                                               \
        if constexpr (KE == K_COPY) k_msg_el_fast<KE, NWV, 0><<<(unsigned)grid, 256, 0, s>>>(g, op, chunks, plan.n_chunks); \
        else if (bm == 1) k_msg_el_fast<KE, NWV, 1><<<(unsigned)grid, 256, 0, s>>>(g, op, chunks, plan.n_chunks);          \
        else k_msg_el_fast<KE, NWV, 2><<<(unsigned)grid, 256, 0, s>>>(g, op, chunks, plan.n_chunks);                       \
    })
        if (op.W <= 1) {
            UG_MELF(1);
        } else if (op.W <= 2) {
            UG_MELF(2);
        } else if (op.W <= 4) {
            UG_MELF(4);
        } else {
            UG_MELF(8);
        }
#undef UG_MELF
        return cudaGetLastError();
    }
#define UG_MEL(NWV) UG_DISPATCH_KE(kedge, KE, k_msg_el<KE, NWV><<<(unsigned)grid, 256, 0, s>>>(g, op, chunks, plan.n_chunks))
    if (op.W <= 1) {
        UG_MEL(1);
    } else if (op.W <= 2) {
        UG_MEL(2);
    } else if (op.W <= 4) {
        UG_MEL(4);
    } else {
        UG_MEL(8);
    }
#undef UG_MEL
    return cudaGetLastError();
}

}  // namespace ug
