// k_split_dot.cu -- `dot` (SDDMM, reading R5) under the B200 split-vertex schedule SV.
//
// Same work decomposition as k_split.cu: destination rows cut into <= `group`-edge chunks, the
// feature axis cut into ftile = 32 * VEC column tiles visited tile-major, so the gathered
// X[src] column slab of a tile stays L2-resident (C5, F = 602: 60 MB per 64-column slab).
// The 32 lanes of a warp own the tile's columns; the Dst_V operand's tile is loaded once per
// unit.  For a batch of 32 in-edges every lane forms 32 partial products (its columns x the
// 32 edges), and a 5-step transposed butterfly (31 shuffles per 32 edges instead of 5 per edge)
// leaves lane q holding the tile's partial dot of edge q.  Partials of the tiles of one head
// meet in the output with red.global.add.f32 (output zeroed first):
//   * message creation (C = Edge): C[e][h] += partial(e, tile);
//   * sum / mean aggregation: by linearity sum_e sum_tiles = sum_tiles sum_e, so each unit
//     adds its row's partial sum to C[v][h] (mean divides in the epilogue).
// max / min are not linear in the partials and use k_dot instead.  Summation order across
// tiles is unspecified (tolerance R11; exact in integer mode).
#include "k_dispatch.cuh"

namespace ug {

template <int GOP, int VEC>
__global__ void __launch_bounds__(256) k_split_dot(GraphArgs g, OpArgs op, const int4 *__restrict__ chunks,
                                                   int64_t n_chunks, int n_tiles) {
    constexpr int FT = 32 * VEC;               // columns per tile
    const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;   // warp = unit
    const int lane = threadIdx.x & 31;
    if (w >= n_chunks * n_tiles) return;       // whole warps exit together
    const int tile = (int)(w / n_chunks);
    const int64_t c = w - (int64_t)tile * n_chunks;
    const int f = tile * FT + lane * VEC;
    const bool active = f < op.F;
    const int head = (tile * FT) / op.D;       // the host guarantees D % FT == 0 or H == 1
    const int4 ch = chunks[c];
    const int64_t v = ch.x;
    const int64_t k0 = ch.y, k1 = ch.z;
    const int64_t ca = op_col(op.A, active ? f : 0);
    const int64_t cb = op_col(op.B, active ? f : 0);
    const bool bconst = op.B.type == UG_T_DST_V;
    float bv[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) bv[i] = 0.0f;
    if (bconst && active) fetch<VEC>(op.B, v, cb, bv);
    float rowsum = 0.0f;

    for (int64_t kb = k0; kb < k1; kb += 32) {
        const int n = (int)((k1 - kb) < 32 ? (k1 - kb) : 32);
        float p[32];
#pragma unroll
        for (int q = 0; q < 32; ++q) p[q] = 0.0f;
        if (active) {
            constexpr int QB = VEC == 4 ? 4 : 8;   // gathers in flight per lane
#pragma unroll
            for (int q0 = 0; q0 < 32; q0 += QB) {
                float a[QB][VEC], b[QB][VEC];
#pragma unroll
                for (int q = 0; q < QB; ++q) {
                    const int qq = q0 + q;
                    if (qq < n) {
                        const int64_t k = kb + qq;
                        const int64_t src = g.col[k];
                        const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                        fetch<VEC>(op.A, op_row(op.A.type, src, v, e), ca, a[q]);
                        if (bconst) {
#pragma unroll
                            for (int i = 0; i < VEC; ++i) b[q][i] = bv[i];
                        } else {
                            fetch<VEC>(op.B, op_row(op.B.type, src, v, e), cb, b[q]);
                        }
                    } else {
#pragma unroll
                        for (int i = 0; i < VEC; ++i) a[q][i] = b[q][i] = 0.0f;
                    }
                }
#pragma unroll
                for (int q = 0; q < QB; ++q)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) p[q0 + q] = __fmaf_rn(a[q][i], b[q][i], p[q0 + q]);
            }
        }
        // transposed butterfly: after it, p[0] of lane q is the warp-wide sum of p[q]
#pragma unroll
        for (int s = 16; s >= 1; s >>= 1) {
            const bool upper = (lane & s) != 0;
#pragma unroll
            for (int i = 0; i < s; ++i) {
                const float send = upper ? p[i] : p[i + s];
                const float keep = upper ? p[i + s] : p[i];
                p[i] = keep + __shfl_xor_sync(0xffffffffu, send, s);
            }
        }
        if constexpr (GOP == UG_GATHER_ASSIGN) {
            if (lane < n) {
                const int64_t k = kb + lane;
                const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                atomicAdd(op.C + e * op.c_ld + head, p[0]);
            }
        } else {
            rowsum += lane < n ? p[0] : 0.0f;
        }
    }
    if constexpr (GOP != UG_GATHER_ASSIGN) {
#pragma unroll
        for (int s = 16; s >= 1; s >>= 1) rowsum += __shfl_xor_sync(0xffffffffu, rowsum, s);
        if (lane == 0 && k1 > k0) atomicAdd(op.C + v * op.c_ld + head, rowsum);
    }
}

cudaError_t launch_split_dot(int gather, const GraphArgs &g, const OpArgs &op, const LaunchCfg &c,
                             const SplitPlan &plan, cudaStream_t s, cudaEvent_t ev_begin, cudaEvent_t ev_end) {
    const int ft = 32 * c.vec;
    const int n_tiles = (int)cdiv(op.F, ft);
    const int64_t threads = plan.n_chunks * n_tiles * 32;
    if (ev_begin) cudaEventRecord(ev_begin, s);
    if (threads > 0) {
        const int64_t grid = cdiv(threads, c.block);
        const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
        UG_DISPATCH_VEC(c.vec, VEC, {
            if (gather == UG_GATHER_ASSIGN)
                k_split_dot<UG_GATHER_ASSIGN, VEC><<<(unsigned)grid, c.block, 0, s>>>(g, op, chunks, plan.n_chunks, n_tiles);
            else
                k_split_dot<UG_GATHER_SUM, VEC><<<(unsigned)grid, c.block, 0, s>>>(g, op, chunks, plan.n_chunks, n_tiles);
        });
    }
    if (ev_end) cudaEventRecord(ev_end, s);
    return cudaGetLastError();
}

}  // namespace ug
