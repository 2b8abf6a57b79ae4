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

// Reduce N values (N a power of two) over the P lanes of a lane segment (P a power of two <= 32,
// segments aligned in the warp) with gather_op GOP, by a transposed butterfly: at offsets P/2,
// P/4, ... each lane sends half of its remaining values and keeps the other half.  After it,
// lane l of the segment holds in v[0 .. max(N / P, 1)) the totals of values
// (l >> (log2 P - log2 N)) when N <= P, or l * (N / P) + i when N > P (contiguous columns).
// N - 1 + log2 P - log2 N shuffles for N <= P, instead of N log2 P for N separate butterflies.
// Fixed tree: deterministic.  Every lane of the warp must call it.
template <int GOP, int N, int P>
__device__ __forceinline__ void seg_reduce_transposed(float (&v)[N], int lane) {
#pragma unroll
    for (int n = N, o = P / 2; n > 1 && o > 0; n >>= 1, o >>= 1) {
        const bool up = lane & o;
#pragma unroll
        for (int i = 0; i < n / 2; ++i) {
            const float send = up ? v[i] : v[i + n / 2];
            const float keep = up ? v[i + n / 2] : v[i];
            v[i] = g_combine<GOP>(keep, __shfl_xor_sync(0xffffffffu, send, o));
        }
    }
    if constexpr (N < P) {
#pragma unroll
        for (int o = P / N / 2; o > 0; o >>= 1) v[0] = g_combine<GOP>(v[0], __shfl_xor_sync(0xffffffffu, v[0], o));
    }
}

// Edge-lanes vertex schedules ("WV_Gg_T1_E1": P = 32 lanes per row; "TV_Gg_Tp_E1": P = p lanes,
// 32 / p rows per warp; round 2): for narrow features (W / VEC <= 8 chunks) the P lanes of a row
// split its IN-EDGES instead of its features -- lane l takes edges k0 + l, k0 + l + P, ... and
// reduces every feature of its messages in registers; a transposed butterfly over the P lanes
// then combines them (owner computes: one launch, no atomics, no init).  A row of in-degree d
// costs ceil(d / 2P) dependent gather steps instead of d / UF, which is what bounds small, skewed
// graphs (C1 / C2) under the feature-lane schedules; P < 32 packs several light rows per warp
// (fewer waves on graphs with more rows than resident warps, e.g. C2).
// register budget of narrow rows (<= 8 values in <= 2 vectors): capping them at 6 CTAs / SM (40
// registers, spill-free; C2's 19.7 K rows at 16 lanes in 1.4 waves instead of 2.1) measured SLOWER
// on every C1 / C2 case (C2 copy_e_max TV_G1_T16_E1 10.88 -> 11.54 us mean, u_mul_e_sum F = 8
// 12.81 -> 14.41 us; profiles/r2/ab_el_r2fin2.jsonl): uncapped (1), kept as an A/B switch
#ifndef UG_EL_MINB_NARROW
#define UG_EL_MINB_NARROW 1
#endif
template <int KE, int GOP, int VEC, int NC, int P>
__global__ void __launch_bounds__(256, (NC * VEC <= 8 && NC <= 2 && (VEC >= 2 || KE == K_COPY)) ? UG_EL_MINB_NARROW : 1) k_vertex_el(GraphArgs g, OpArgs op, int G) {
    constexpr int N = NC * VEC;                       // values per lane (a power of two)
    constexpr int NOUT = N > P ? N / P : 1;           // totals a lane holds after the reduction
    const int64_t seg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / P;   // row group
    const int lane = threadIdx.x & 31;
    const int sl = lane & (P - 1);                    // lane within the row's segment
    const int64_t warp0 = (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * (32 / P);
    if (warp0 * G >= g.V) return;                     // whole warps leave together
    int64_t ca[NC], cb[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        ca[j] = op_col(op.A, min(j * VEC, op.W - 1));
        cb[j] = op_col(op.B, min(j * VEC, op.W - 1));
    }
    for (int r = 0; r < G; ++r) {
        const int64_t v = seg * G + r;
        if ((warp0 * G + r) >= g.V) break;            // warp-uniform: the warp's first row group
        const bool live = v < g.V;
        const int64_t k0 = live ? (int64_t)g.row_ptr[v] - g.rp_base : 0;
        const int64_t k1 = live ? (int64_t)g.row_ptr[v + 1] - g.rp_base : 0;
        float acc[N];
#pragma unroll
        for (int j = 0; j < N; ++j) acc[j] = g_init<GOP>();
        // two in-edges per lane per step (k and k + P: independent gathers in flight)
        for (int64_t k = k0 + sl; k < k1; k += 2 * P) {
            const bool two = k + P < k1;
            const int64_t kb = two ? k + P : k;
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
                        acc[j * VEC + i] = g_combine<GOP>(acc[j * VEC + i], m0[i]);
                        if (two) acc[j * VEC + i] = g_combine<GOP>(acc[j * VEC + i], m1[i]);
                    }
                }
            }
        }
        seg_reduce_transposed<GOP, N, P>(acc, lane);
        const int64_t deg = k1 - k0;
        if (live) {
            if constexpr (N <= P) {
                constexpr int SH = (P >= 32 ? 5 : P >= 16 ? 4 : P >= 8 ? 3 : P >= 4 ? 2 : P >= 2 ? 1 : 0) -
                                   (N >= 32 ? 5 : N >= 16 ? 4 : N >= 8 ? 3 : N >= 4 ? 2 : N >= 2 ? 1 : 0);
                const int col = sl >> SH;
                if ((sl & ((1 << SH) - 1)) == 0 && col < op.W) op.C[v * op.c_ld + col] = g_finalize<GOP>(acc[0], deg);
            } else {
                const int c0 = sl * NOUT;
#pragma unroll
                for (int i = 0; i < NOUT; ++i)
                    if (c0 + i < op.W) op.C[v * op.c_ld + c0 + i] = g_finalize<GOP>(acc[i], deg);
            }
        }
    }
}

// Segmented edge lanes ("WV_Gg_T1_E1", g in {2, 4, 8}, round 2): the warp's g consecutive rows
// share its 32 lanes -- their in-edges are the consecutive CSR positions [row_ptr[v0],
// row_ptr[v0 + g]), lane l takes positions base + l, base + l + 32, ... and accumulates each
// message into the partial of its row (found from the g + 1 row boundaries, loaded once per warp).
// A hub row no longer serialises over one sub-warp's lanes (TV_G1_T8_E1: ceil(d / 16) steps) and
// light rows no longer leave most of a warp idle (WV_G1_T1_E1).  The g x N partials are combined
// by one transposed butterfly (g N <= 32 values: g N - 1 shuffles), which leaves value j = (row,
// feature) in lanes j * (32 / g N) ...; owner computes, one launch.
template <int KE, int GOP, int VEC, int NC, int G>
__global__ void __launch_bounds__(256) k_vertex_seg(GraphArgs g, OpArgs op) {
    constexpr int N = NC * VEC;                       // values per row (a power of two)
    constexpr int NT = G * N;                         // values per warp, <= 32
    static_assert(NT <= 32, "segmented edge lanes: G * N <= 32");
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int64_t v0 = warp * G;
    if (v0 >= g.V) return;                            // whole warps leave together
    int64_t b[G + 1];                                 // row boundaries (warp-uniform loads)
#pragma unroll
    for (int r = 0; r <= G; ++r) b[r] = (int64_t)g.row_ptr[min(v0 + r, g.V)] - g.rp_base;
    int64_t ca[NC], cb[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        ca[j] = op_col(op.A, min(j * VEC, op.W - 1));
        cb[j] = op_col(op.B, min(j * VEC, op.W - 1));
    }
    float acc[NT];
#pragma unroll
    for (int j = 0; j < NT; ++j) acc[j] = g_init<GOP>();
    auto add_edge = [&](int64_t k) {
        int r = 0;                                    // local row of position k
#pragma unroll
        for (int i = 1; i < G; ++i) r += k >= b[i];
        const int64_t v = v0 + r;
        const int64_t src = g.col[k];
        const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
        const int64_t ra = op_row(op.A.type, src, v, e), rb = op_row(op.B.type, src, v, e);
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            if (j * VEC < op.W) {
                float m[VEC];
                message<KE, VEC>(op, ra, ca[j], rb, cb[j], m);
#pragma unroll
                for (int rr = 0; rr < G; ++rr)
#pragma unroll
                    for (int i = 0; i < VEC; ++i)
                        if (r == rr) acc[rr * N + j * VEC + i] = g_combine<GOP>(acc[rr * N + j * VEC + i], m[i]);
            }
        }
    };
    // two positions per lane per step (independent gathers in flight)
    for (int64_t k = b[0] + lane; k < b[G]; k += 64) {
        add_edge(k);
        if (k + 32 < b[G]) add_edge(k + 32);
    }
    seg_reduce_transposed<GOP, NT, 32>(acc, lane);
    constexpr int SH = 5 - (NT >= 32 ? 5 : NT >= 16 ? 4 : NT >= 8 ? 3 : NT >= 4 ? 2 : NT >= 2 ? 1 : 0);
    const int j = lane >> SH;                         // value index: row j / N, feature j % N
    const int rr = j / N, col = j - rr * N;
    if ((lane & ((1 << SH) - 1)) == 0 && col < op.W && v0 + rr < g.V) {
        int64_t deg = 0;
#pragma unroll
        for (int r = 0; r < G; ++r)
            if (r == rr) deg = b[r + 1] - b[r];
        op.C[(v0 + rr) * op.c_ld + col] = g_finalize<GOP>(acc[0], deg);
    }
}

cudaError_t launch_vertex_el(int kedge, int gather, const GraphArgs &g, const OpArgs &op, const LaunchCfg &c,
                             cudaStream_t s) {
    const int nc = (int)cdiv(op.W, c.vec);
    const int ncp = nc <= 1 ? 1 : nc <= 2 ? 2 : nc <= 4 ? 4 : 8;     // NC instantiated
    if (c.L == 32 && c.G > 1 && (c.G == 2 || c.G == 4 || c.G == 8) && c.G * ncp * c.vec <= 32) {
        // segmented edge lanes: the warp's G rows share its lanes
        const int64_t warps = cdiv(g.V, c.G);
        const int64_t sgrid = cdiv(warps * 32, 256);
#define UG_SEG(NCV, GV)                                                                                   \
        UG_DISPATCH_KE(kedge, KE, UG_DISPATCH_RED(gather, GOP, {                                          \
            if constexpr (GV * NCV * VEC <= 32) k_vertex_seg<KE, GOP, VEC, NCV, GV><<<(unsigned)sgrid, 256, 0, s>>>(g, op); \
        }))
#define UG_SEG_G(NCV)                                                                                     \
        switch (c.G) {                                                                                    \
        case 2: UG_SEG(NCV, 2); break;                                                                    \
        case 4: UG_SEG(NCV, 4); break;                                                                    \
        default: UG_SEG(NCV, 8); break;                                                                   \
        }
        UG_DISPATCH_VEC(c.vec, VEC, {
            switch (ncp) {
            case 1: UG_SEG_G(1); break;
            case 2: UG_SEG_G(2); break;
            case 4: UG_SEG_G(4); break;
            default: UG_SEG_G(8); break;
            }
        });
#undef UG_SEG_G
#undef UG_SEG
        return cudaGetLastError();
    }
    const int64_t segs = cdiv(g.V, c.G);
    if (segs == 0) return cudaSuccess;
    const int64_t grid = cdiv(segs * c.L, 256);
#define UG_EL(NCV, PV)                                                                                    \
    UG_DISPATCH_KE(kedge, KE,                                                                            \
        UG_DISPATCH_RED(gather, GOP,                                                                     \
            k_vertex_el<KE, GOP, VEC, NCV, PV><<<(unsigned)grid, 256, 0, s>>>(g, op, c.G)))
#define UG_EL_P(NCV)                                                                                     \
    switch (c.L) {                                                                                       \
    case 8: UG_EL(NCV, 8); break;                                                                        \
    case 16: UG_EL(NCV, 16); break;                                                                      \
    default: UG_EL(NCV, 32); break;                                                                      \
    }
    UG_DISPATCH_VEC(c.vec, VEC, {
        switch (nc) {
        case 1: UG_EL_P(1); break;
        case 2: UG_EL_P(2); break;
        case 3: case 4: UG_EL_P(4); break;
        default: UG_EL_P(8); break;
        }
    });
#undef UG_EL_P
#undef UG_EL
    return cudaGetLastError();
}

}  // namespace ug
