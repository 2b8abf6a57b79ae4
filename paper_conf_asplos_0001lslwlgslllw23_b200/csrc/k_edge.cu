// k_edge.cu -- edge-parallel template: Thread-Edge and Warp-Edge (Fig. 6(c),(e),(f);
// PAPER.md:327, 348, 350) with E-grouping G and feature tiling T, plus the init (a4) and
// epilogue (a6) kernels that edge-parallel aggregation needs.
//
// A unit is one edge (CSR position k; its dst row comes from the COO dst array).  L lanes
// share the edge's features (TE: L = T, WE: L = 32 T).  A lane group processes G
// consecutive positions; because positions are dst-sorted, runs of equal dst are
// pre-reduced in registers and flushed once per run (reading R17).  Because different
// groups can share a dst row, the flush is atomic (pass 2 of PAPER.md:405):
// red.global.add(.v2/.v4).f32 for sum/mean, the integer-order trick for max/min.
// Message creation (C = Edge) writes each edge's message; no atomics, no init.
#include <algorithm>
#include <limits>

#include "k_dispatch.cuh"

namespace ug {

template <int KE, int GOP, int VEC, bool FAST>
__global__ void __launch_bounds__(256) k_edge(GraphArgs g, OpArgs op, int L_log2, int G,
                                              int ftile, int64_t n_groups, int n_tiles) {
    constexpr int R = (8 / VEC) > 0 ? (8 / VEC) : 1;
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
    const int64_t k0 = ugp * (int64_t)G;
    const int64_t k1 = min(g.E, k0 + G);

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
                const int64_t v = (int64_t)g.dst[k] - g.r0;
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
            int64_t cur = -1;
            auto flush = [&]() {
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int f = fb + j * stride;
                    if (f < f_hi) atomic_flush<GOP, VEC>(op.C + cur * op.c_ld + f, acc[j], op.W - f);
                }
            };
            auto reset = [&]() {
#pragma unroll
                for (int j = 0; j < R; ++j)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[j][i] = g_init<GOP>();
            };
            // U edges' row gathers in flight per lane; fewer when each edge already needs
            // several register chunks (keeps registers, hence occupancy, in check)
            constexpr int U = (R * VEC >= 8) ? 2 : 4;
            // a width-1 B operand (e.g. GCN's scalar edge weight) is loaded once per edge
            const bool bscalar = KE != K_COPY && op.B.div == op.F;
            int64_t k = k0;
            for (; k + U <= k1; k += U) {
                int64_t vq[U], ra[U], rb[U];
                float bs[U];
#pragma unroll
                for (int q = 0; q < U; ++q) {
                    const int64_t src = g.col[k + q];
                    vq[q] = (int64_t)g.dst[k + q] - g.r0;
                    const int64_t e = g.eid ? (int64_t)g.eid[k + q] : k + q;
                    ra[q] = op_row(op.A.type, src, vq[q], e);
                    rb[q] = op_row(op.B.type, src, vq[q], e);
                    if constexpr (KE != K_COPY) bs[q] = bscalar ? __ldg(op.B.p + rb[q] * op.B.ld) : 0.0f;
                }
                float m[U][R][VEC];
#pragma unroll
                for (int q = 0; q < U; ++q)
#pragma unroll
                    for (int j = 0; j < R; ++j) {
                        const int f = fb + j * stride;
                        if (f < f_hi) {
                            if constexpr (FAST && KE != K_COPY) {
                                if (bscalar) {
                                    ldg_vec<VEC>(op.A.p + ((uint32_t)ra[q] * (uint32_t)op.A.ld + (uint32_t)f), m[q][j]);
#pragma unroll
                                    for (int i = 0; i < VEC; ++i) m[q][j][i] = edge_fn<KE>(m[q][j][i], bs[q]);
                                } else {
                                    message_fast<KE, VEC>(op, (uint32_t)ra[q], (uint32_t)f, rb[q], cb[j], m[q][j]);
                                }
                            } else if constexpr (FAST) {
                                message_fast<KE, VEC>(op, (uint32_t)ra[q], (uint32_t)f, rb[q], cb[j], m[q][j]);
                            } else {
                                message<KE, VEC>(op, ra[q], ca[j], rb[q], cb[j], m[q][j]);
                            }
                        }
                    }
#pragma unroll
                for (int q = 0; q < U; ++q) {
                    if (vq[q] != cur) {
                        if (cur >= 0) flush();
                        cur = vq[q];
                        reset();
                    }
#pragma unroll
                    for (int j = 0; j < R; ++j)
#pragma unroll
                        for (int i = 0; i < VEC; ++i) acc[j][i] = g_combine<GOP>(acc[j][i], m[q][j][i]);
                }
            }
            for (; k < k1; ++k) {
                const int64_t src = g.col[k];
                const int64_t v = (int64_t)g.dst[k] - g.r0;
                const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                if (v != cur) {
                    if (cur >= 0) flush();
                    cur = v;
                    reset();
                }
                const int64_t ra = op_row(op.A.type, src, v, e);
                const int64_t rb = op_row(op.B.type, src, v, e);
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int f = fb + j * stride;
                    if (f < f_hi) {
                        float mm[VEC];
                        message<KE, VEC>(op, ra, ca[j], rb, cb[j], mm);
#pragma unroll
                        for (int i = 0; i < VEC; ++i) acc[j][i] = g_combine<GOP>(acc[j][i], mm[i]);
                    }
                }
            }
            if (cur >= 0) {
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int f = fb + j * stride;
                    if (f < f_hi) atomic_flush<GOP, VEC>(op.C + cur * op.c_ld + f, acc[j], op.W - f);
                }
            }
        }
    }
}

cudaError_t launch_edge(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                        const LaunchCfg &c, cudaStream_t s) {
    const int ft = c.ftile > 0 ? c.ftile : op.W;
    const int n_tiles = (int)cdiv(op.W, ft);
    const int64_t n_groups = cdiv(g.E, c.G);
    const int64_t threads = n_groups * n_tiles * (int64_t)c.L;
    if (threads == 0) return cudaSuccess;
    const int64_t grid = cdiv(threads, c.block);
    const int L_log2 = ilog2(c.L);
    const bool fast = op.A.type == UG_T_SRC_V && op.A.div == 1 &&
                      (uint64_t)g.V_src * (uint64_t)op.A.ld < (1ull << 32);
    UG_DISPATCH_VEC(c.vec, VEC,
        UG_DISPATCH_KE(kedge, KE,
            UG_DISPATCH_GOP(gather, GOP, {
                if (fast)
                    k_edge<KE, GOP, VEC, true><<<(unsigned)grid, c.block, 0, s>>>(g, op, L_log2, c.G, ft,
                                                                                  n_groups, n_tiles);
                else
                    k_edge<KE, GOP, VEC, false><<<(unsigned)grid, c.block, 0, s>>>(g, op, L_log2, c.G, ft,
                                                                                   n_groups, n_tiles);
            })));
    return cudaGetLastError();
}

// ---------------------------------------------------------------- a4: output init
// C[v][o] <- identity of the reducer (0 for sum/mean, -inf for max, +inf for min).
__global__ void k_init(float *C, int64_t ld, int64_t rows, int W, float value) {
    const int64_t n = rows * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / W;
        C[r * ld + (i - r * W)] = value;
    }
}

cudaError_t launch_init(int gather, const OpArgs &op, int64_t rows, cudaStream_t s) {
    const float inf = std::numeric_limits<float>::infinity();
    const float val = gather == UG_GATHER_MAX ? -inf : gather == UG_GATHER_MIN ? inf : 0.0f;
    const int64_t n = rows * (int64_t)op.W;
    if (n == 0) return cudaSuccess;
    const int64_t grid = std::min<int64_t>(cdiv(n, 256), 148 * 16);
    k_init<<<(unsigned)grid, 256, 0, s>>>(op.C, op.c_ld, rows, op.W, val);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- a6: epilogue
// mean: C = C / deg (one IEEE division, R8); every reducer: zero-in-degree rows -> 0 (R7).
__global__ void k_epilogue(GraphArgs g, float *C, int64_t ld, int W, int mean) {
    const int64_t n = g.V * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = i / W;
        const int64_t deg = (int64_t)g.row_ptr[v + 1] - g.row_ptr[v];
        float *p = C + v * ld + (i - v * W);
        if (deg == 0) *p = 0.0f;
        else if (mean) *p = __fdiv_rn(*p, (float)deg);
        else if (isnan(*p)) *p = __uint_as_float(UG_CANONICAL_NAN);   // min's 0xFFFFFFFF (R12)
    }
}

cudaError_t launch_epilogue(int gather, const GraphArgs &g, const OpArgs &op, cudaStream_t s) {
    const int64_t n = g.V * (int64_t)op.W;
    if (n == 0) return cudaSuccess;
    const int64_t grid = std::min<int64_t>(cdiv(n, 256), 148 * 16);
    k_epilogue<<<(unsigned)grid, 256, 0, s>>>(g, op.C, op.c_ld, op.W, gather == UG_GATHER_MEAN);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- ug_edge_permute
__global__ void k_permute(const int32_t *__restrict__ eid, const float *__restrict__ in,
                          float *__restrict__ out, int64_t E, int W) {
    const int64_t n = E * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t k = i / W;
        const int64_t c = i - k * W;
        const int64_t e = eid ? (int64_t)eid[k] : k;
        out[i] = __ldg(in + e * W + c);
    }
}

cudaError_t launch_permute(const int32_t *eid, const float *in, float *out, int64_t E, int width,
                           cudaStream_t s) {
    const int64_t n = E * (int64_t)width;
    if (n == 0) return cudaSuccess;
    const int64_t grid = std::min<int64_t>(cdiv(n, 256), 148 * 16);
    k_permute<<<(unsigned)grid, 256, 0, s>>>(eid, in, out, E, width);
    return cudaGetLastError();
}

}  // namespace ug

namespace ug {
// out[i][:] = in[idx[i]][:] (vertex renumbering, ug_rows_gather): one warp per row, lanes
// over the features.
__global__ void k_rows_gather(const float *__restrict__ in, int64_t ld_in, const int32_t *__restrict__ idx,
                              int64_t rows, int width, float *__restrict__ out, int64_t ld_out) {
    const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (w >= rows) return;
    const float *src = in + (int64_t)idx[w] * ld_in;
    float *dst = out + w * ld_out;
    for (int f = lane; f < width; f += 32) dst[f] = __ldg(src + f);
}

cudaError_t launch_rows_gather(const float *in, int64_t ld_in, const int32_t *idx, int64_t rows, int width,
                               float *out, int64_t ld_out, cudaStream_t s) {
    k_rows_gather<<<(unsigned)cdiv(rows * 32, 256), 256, 0, s>>>(in, ld_in, idx, rows, width, out, ld_out);
    return cudaGetLastError();
}
}  // namespace ug
