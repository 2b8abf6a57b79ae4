// k_arg.cu -- max/min aggregation with arg capture, and its backward scatter.
//
// The paper's operators are inference-only; training a max/min aggregation
// (GraphSAGE-max) needs to know which in-edge supplied each output element.
// k_argext computes C = gather_op over in-edges of edge_op(A, B) (Table 4 rows 6-11, max/min)
// and arg[v][f] = the edge id of the supplying edge.  Tie rule: the FIRST edge id attaining the
// extreme under the total order -0 < +0 (R12).  In-edges of a row are stored in edge-id order
// (stable CSR), so a scan that only replaces on a strictly better value keeps the
// first; rows are cut into SV chunks (k_split.cuh) walked by one L-lane slice each, and split
// rows are merged in chunk order by the last-arriving slice (arrival counter), which preserves
// the rule.  One launch, deterministic.
//
// k_argscatter is the backward: out[row(e)][f / div] += grad[v][f] for every (v, f) whose arg
// is e >= 0, row(e) = src of e (a Src_V operand) or e (an Edge operand).
#include "k_dispatch.cuh"

namespace ug {

template <int GOP>
__device__ __forceinline__ bool strictly_better(float m, float cur) {
    // NaN is absorbing (R12): the first NaN message wins and stays
    if (isnan(cur)) return false;
    if (isnan(m)) return true;
    // before(x, y): x precedes y in the total order -0 < +0
    auto before = [](float x, float y) { return x < y || (x == y && signbit(x) && !signbit(y)); };
    return GOP == UG_GATHER_MAX ? before(cur, m) : before(m, cur);
}

template <int KE, int GOP>
__global__ void __launch_bounds__(256) k_argext(GraphArgs g, OpArgs op, int L_log2, int n_tiles,
                                                const int4 *__restrict__ chunks, int n_chunks,
                                                const int4 *__restrict__ split, const int32_t *__restrict__ slot_row,
                                                float *sval, int32_t *sarg, int64_t sld, int32_t *counters,
                                                int32_t *arg, int64_t ld_arg) {
    constexpr int U = 4;
    const int L = 1 << L_log2;
    const int S = 32 >> L_log2;
    const int lane = threadIdx.x & 31;
    const int slice = lane >> L_log2;
    const int sl = lane & (L - 1);
    const int unit = ((int)blockIdx.x * (int)(blockDim.x >> 5) + (int)(threadIdx.x >> 5)) * S + slice;
    if (unit >= n_chunks * n_tiles) return;
    const int tile = n_tiles == 1 ? 0 : unit / n_chunks;
    const int c = unit - tile * n_chunks;
    const int4 ch = chunks[c];
    const int64_t v = ch.x;
    const int f = tile * L + sl;
    const bool active = f < op.W;
    const int64_t ca = op_col(op.A, active ? f : 0), cb = op_col(op.B, active ? f : 0);
    float best = 0.0f;
    int32_t be = -1;
    if (active) {
        int64_t k = ch.y;
        for (; k + U <= ch.z; k += U) {
            float m[U];
            int32_t e[U];
#pragma unroll
            for (int q = 0; q < U; ++q) {
                const int64_t src = g.col[k + q];
                e[q] = g.eid ? g.eid[k + q] : (int32_t)(k + q);
                float t[1];
                message<KE, 1>(op, op_row(op.A.type, src, v, e[q]), ca, op_row(op.B.type, src, v, e[q]), cb, t);
                m[q] = t[0];
            }
#pragma unroll
            for (int q = 0; q < U; ++q)
                if (be < 0 || strictly_better<GOP>(m[q], best)) { best = m[q]; be = e[q]; }
        }
        for (; k < ch.z; ++k) {
            const int64_t src = g.col[k];
            const int32_t e = g.eid ? g.eid[k] : (int32_t)k;
            float t[1];
            message<KE, 1>(op, op_row(op.A.type, src, v, e), ca, op_row(op.B.type, src, v, e), cb, t);
            if (be < 0 || strictly_better<GOP>(t[0], best)) { best = t[0]; be = e; }
        }
    }
    if (ch.w < 0) {                                   // the row is one chunk
        if (active) {
            op.C[v * op.c_ld + f] = be < 0 ? 0.0f : (isnan(best) ? __uint_as_float(UG_CANONICAL_NAN) : best);
            arg[v * ld_arg + f] = be;
        }
        return;
    }
    if (active) {
        sval[(int64_t)ch.w * sld + f] = best;
        sarg[(int64_t)ch.w * sld + f] = be;
    }
    fence_acq_rel_gpu();
    const unsigned smask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (slice * L));
    __syncwarp(smask);
    const int r = slot_row[ch.w];
    const int4 sp = split[r];
    int last = 0;
    if (sl == 0) last = atomicAdd(counters + (int64_t)r * n_tiles + tile, 1) == sp.z - 1;
    last = __shfl_sync(smask, last, slice * L);
    if (!last) return;
    fence_acq_rel_gpu();
    if (sl == 0) counters[(int64_t)r * n_tiles + tile] = 0;    // re-armed for the next call
    if (!active) return;
    best = 0.0f;
    be = -1;
    for (int i = 0; i < sp.z; ++i) {                              // chunk order = edge-id order
        const int64_t slot = sp.y + i;
        const float m = __ldcg(sval + slot * sld + f);
        const int32_t e = __ldcg(sarg + slot * sld + f);
        if (e >= 0 && (be < 0 || strictly_better<GOP>(m, best))) { best = m; be = e; }
    }
    op.C[v * op.c_ld + f] = be < 0 ? 0.0f : (isnan(best) ? __uint_as_float(UG_CANONICAL_NAN) : best);
    arg[v * ld_arg + f] = be;
}

// out[row(e)][f / div] += grad[v][f]; src_of_eid: src vertex by edge id (NULL: use col, the
// CSR position equals the edge id).
__global__ void k_argscatter(const int32_t *__restrict__ arg, int64_t ld_arg, const float *__restrict__ grad,
                             int64_t ld_grad, int64_t V, int W, int to_src, const int32_t *__restrict__ col,
                             const int32_t *__restrict__ src_of_eid, float *out, int64_t ld_out, int div) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= V * W) return;
    const int64_t v = t / W;
    const int f = (int)(t - v * W);
    const int32_t e = arg[v * ld_arg + f];
    if (e < 0) return;
    const int64_t row = to_src ? (int64_t)(src_of_eid ? src_of_eid[e] : col[e]) : (int64_t)e;
    atomicAdd(out + row * ld_out + f / div, grad[v * ld_grad + f]);
}

cudaError_t launch_argext(int kedge, int gather, const GraphArgs &g, const OpArgs &op, int L, const SplitPlan &plan,
                          const int32_t *slot_row, float *sval, int32_t *sarg, int64_t sld, int32_t *counters,
                          int32_t *arg, int64_t ld_arg, cudaStream_t s) {
    const int n_tiles = (int)cdiv(op.W, L);
    const int S = 32 / L;
    const int64_t grid = cdiv(plan.n_chunks * n_tiles, (int64_t)8 * S);
    if (grid == 0) return cudaSuccess;
    const int L_log2 = ilog2(L);
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const int4 *split = reinterpret_cast<const int4 *>(plan.d_split);
    UG_DISPATCH_KE(kedge, KE, {
        if (gather == UG_GATHER_MAX)
            k_argext<KE, UG_GATHER_MAX><<<(unsigned)grid, 256, 0, s>>>(g, op, L_log2, n_tiles, chunks, (int)plan.n_chunks,
                                                                       split, slot_row, sval, sarg, sld, counters, arg, ld_arg);
        else
            k_argext<KE, UG_GATHER_MIN><<<(unsigned)grid, 256, 0, s>>>(g, op, L_log2, n_tiles, chunks, (int)plan.n_chunks,
                                                                       split, slot_row, sval, sarg, sld, counters, arg, ld_arg);
    });
    return cudaGetLastError();
}

cudaError_t launch_argscatter(const int32_t *arg, int64_t ld_arg, const float *grad, int64_t ld_grad, int64_t V, int W,
                              bool to_src, const int32_t *col, const int32_t *src_of_eid, float *out, int64_t ld_out,
                              int div, cudaStream_t s) {
    const int64_t n = V * W;
    if (n == 0) return cudaSuccess;
    k_argscatter<<<(unsigned)cdiv(n, 256), 256, 0, s>>>(arg, ld_arg, grad, ld_grad, V, W, to_src ? 1 : 0, col, src_of_eid,
                                                        out, ld_out, div);
    return cudaGetLastError();
}

}  // namespace ug
