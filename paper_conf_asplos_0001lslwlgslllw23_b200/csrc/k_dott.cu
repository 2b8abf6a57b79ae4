// k_dott.cu -- `dot` between a Src_V and a Dst_V operand for ANY head width D (SDDMM, config C4
// and the wide C5 rows; reading R5) under SV with column tiles ("SV_G.._F128"): the message of
// edge e and head o is  sum_{d<D} P[src][o*D+d] * Q[dst][o*D+d]  (PAPER.md:113-120 dot ops).
//
// k_dotsv keeps a whole Dst_V head in registers and needs D / (NJ * VEC) to be a power of two
// that fits one warp.  For wide or ragged heads (C5: D = 602) the head is cut into column tiles
// of TW = 32 * VEC features, and the grid is tile-major like the aggregation SV kernel, so the
// gathered rows of P come from one L2-resident V x TW slab at a time (without tiling every edge
// reads a whole 2.4 KB row of a 561 MB matrix: DRAM-bound).  Work unit = (head, tile, chunk of
// <= G in-edges of row v), one warp: each lane holds VEC features of the Dst_V row (loaded once
// per unit) and, per in-edge, forms its FMA partial; eight edges' partials are then reduced
// over the warp by a transposed butterfly (9 shuffles per 8 edges instead of 5 per edge) that
// leaves edge i's tile sum in lanes 4i..4i+3.  One tile per head: the sum is the message and is
// stored directly.  More tiles: each tile stores its partial [tile][E][H], and k_dott_fix adds
// the tiles in tile order (deterministic), giving the message.  Aggregations of dot messages
// (u_dot_v_sum, ...) reduce that message tensor with the SV kernel (ug_op.cpp).
#include "k_split.cuh"

namespace ug {

// Sum over the 32 lanes of v[(lane >> 2) & 7] (transposed butterfly, fixed order).
__device__ __forceinline__ float warp_sum8_transposed(float (&v)[8], int lane) {
    {
        const bool up = lane & 16;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const float send = up ? v[i] : v[i + 4];
            const float keep = up ? v[i + 4] : v[i];
            v[i] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
        }
    }
    {
        const bool up = lane & 8;
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            const float send = up ? v[i] : v[i + 2];
            const float keep = up ? v[i + 2] : v[i];
            v[i] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
        }
    }
    const bool up = lane & 4;
    float r = (up ? v[1] : v[0]) + __shfl_xor_sync(0xffffffffu, up ? v[0] : v[1], 4);
    r += __shfl_xor_sync(0xffffffffu, r, 2);
    r += __shfl_xor_sync(0xffffffffu, r, 1);
    return r;
}

#ifndef UG_DOTT_MINB
#define UG_DOTT_MINB 6
#endif

// O32: every row of P is addressable with a 32-bit element offset (V_src * ld < 2^32): the gather
// address is one IMAD + IMAD.WIDE from the column index, as in the SV aggregation kernel
template <int VEC, bool O32>
__global__ void __launch_bounds__(256, UG_DOTT_MINB) k_dott(GraphArgs g, OpArgs op, bool a_is_src,
                                                            const int4 *__restrict__ chunks, int n_chunks,
                                                            int tiles_per_head, float *__restrict__ out,
                                                            int64_t out_ld, int64_t tile_stride) {
    constexpr int TW = 32 * VEC;
    const int lane = threadIdx.x & 31;
    const int u = (int)(blockIdx.x * 8 + (threadIdx.x >> 5));
    const int ht = u / n_chunks;
    if (ht >= op.H * tiles_per_head) return;
    const int c = u - ht * n_chunks;
    const int o = ht / tiles_per_head, t = ht - o * tiles_per_head;
    const int fo = t * TW + lane * VEC;            // feature inside head o
    const bool active = fo < op.D;
    const int nval = active ? min(VEC, op.D - fo) : 0;   // < VEC only in a single head's ragged tail
    const int f = o * op.D + (active ? fo : 0);   // inactive lanes load (and discard) a valid vector
    const Operand &P = a_is_src ? op.A : op.B;     // gathered per edge (Src_V)
    const Operand &Q = a_is_src ? op.B : op.A;     // hoisted (Dst_V, local row v)
    const int4 ch = chunks[c];
    const int64_t v = ch.x;
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
    float q[VEC];
    if (nval == VEC) ldg_vec<VEC>(Q.p + v * Q.ld + f, q);
    else
#pragma unroll
        for (int i = 0; i < VEC; ++i) q[i] = i < nval ? Q.p[v * Q.ld + f + i] : 0.0f;
    const float *__restrict__ Pb = P.p + f;
    const uint32_t ldp = (uint32_t)P.ld, fo32 = (uint32_t)f;
    float *dst = out + (int64_t)t * tile_stride + o;
    const int k1 = ch.z;
    // a batch: 8 column indices, then 8 row gathers (UG_DOTT_PIPE=1 issues the next batch's before
    // reducing the current one -- measured slower, kept for A/B)
    // UG_DOTT_PF: the next batch's 8 column indices are loaded while this batch's rows are gathered
    // (one dependent L2 round trip per batch instead of two; it won in k_dotsv, r2an)
#ifndef UG_DOTT_PF
#define UG_DOTT_PF 0
#endif
    const int last = k1 - 1;
    uint32_t s_pf[8];
    if constexpr (UG_DOTT_PF) {
        if (ch.y < k1) {                              // (an empty chunk has no col[k1 - 1])
#pragma unroll
            for (int i = 0; i < 8; ++i) s_pf[i] = (uint32_t)ldg_i32_hint(g.col + min(ch.y + i, last), stream);
        }
    }
    // MASK: only a head's last column tile can hold inactive lanes or a ragged tail; full tiles
    // (every lane nval == VEC, warp-uniform) skip the 8 x VEC selects per batch (UG_DOTT_FULL)
    auto load_batch = [&](auto mask_tag, int k, float (&x)[8][VEC]) {
        constexpr bool MASK = decltype(mask_tag)::value;
        uint32_t s[8];
        if constexpr (UG_DOTT_PF) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                s[i] = s_pf[i];
                s_pf[i] = (uint32_t)ldg_i32_hint(g.col + min(k + 8 + i, last), stream);
            }
        } else {
#pragma unroll
            for (int i = 0; i < 8; ++i) s[i] = (uint32_t)ldg_i32_hint(g.col + min(k + i, last), stream);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            // branch-free: every lane loads a full vector from a valid address (an inactive lane
            // its head's first columns; a ragged tail reads into the packed row's padding) and
            // zeroes the elements outside the head by select
            if constexpr (O32) ldg_vec_hint<VEC>(P.p + (s[i] * ldp + fo32), x[i], keep);
            else ldg_vec_hint<VEC>(Pb + s[i] * ldp, x[i], keep);
            if constexpr (MASK) {
#pragma unroll
                for (int j = 0; j < VEC; ++j) x[i][j] = j < nval ? x[i][j] : 0.0f;
            }
        }
    };
    float xa[8][VEC];
    auto reduce_store = [&](int k, const float (&x)[8][VEC]) {
        float p[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            float a = 0.0f;
#pragma unroll
            for (int j = 0; j < VEC; ++j) a = __fmaf_rn(x[i][j], q[j], a);
            p[i] = a;
        }
        const float r = warp_sum8_transposed(p, lane);
        const int i = lane >> 2;
        if ((lane & 3) == 0 && k + i < k1) {
            const int64_t e = g.eid ? (int64_t)g.eid[k + i] : (int64_t)(k + i);
            dst[e * out_ld] = r;
        }
    };
    int k = ch.y;
#ifndef UG_DOTT_PIPE
#define UG_DOTT_PIPE 0
#endif
#ifndef UG_DOTT_FULL
#define UG_DOTT_FULL 1
#endif
    using masked = std::true_type;
    if constexpr (!UG_DOTT_PIPE) {
        // one batch in flight per warp: a second (software-pipelined) batch measured slower at every
        // vector width (registers: 64 at VEC 2, spills at VEC 4; profiles/r2/ab_r2l.jsonl)
        if (UG_DOTT_FULL && __all_sync(0xffffffffu, nval == VEC)) {
            for (; k < k1; k += 8) {
                load_batch(std::false_type{}, k, xa);
                reduce_store(k, xa);
            }
        } else {
            for (; k < k1; k += 8) {
                load_batch(masked{}, k, xa);
                reduce_store(k, xa);
            }
        }
    } else {
        float xb[8][VEC];
        if (k < k1) load_batch(masked{}, k, xa);
        while (k < k1) {
            if (k + 8 < k1) load_batch(masked{}, k + 8, xb);
            reduce_store(k, xa);
            k += 8;
            if (k >= k1) break;
            if (k + 8 < k1) load_batch(masked{}, k + 8, xa);
            reduce_store(k, xb);
            k += 8;
        }
    }
}

// message[e][o] = sum over tiles (in order) of part[t][e][o]
__global__ void k_dott_fix(const float *__restrict__ part, int64_t E, int H, int tiles, int64_t tile_stride,
                           float *__restrict__ C, int64_t c_ld) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= E * H) return;
    const int64_t e = i / H;
    const int o = (int)(i - e * H);
    float s = part[e * H + o];
    for (int t = 1; t < tiles; ++t) s += part[(int64_t)t * tile_stride + e * H + o];
    C[e * c_ld + o] = s;
}

#ifndef UG_DOTT_O32
#define UG_DOTT_O32 1
#endif
int dott_tiles(const OpArgs &op, int vec) { return (int)cdiv(op.D, 32 * vec); }

// Message creation into C (c_ld) -- or, when tiles > 1, partials into `part` ([tiles][E][H]) and
// the tile fix-up into C.
cudaError_t launch_dott(const GraphArgs &g, const OpArgs &op, bool a_is_src, int vec, const SplitPlan &plan,
                        float *C, int64_t c_ld, float *part, cudaStream_t s, cudaEvent_t ev_begin,
                        cudaEvent_t ev_end) {
    const int th = dott_tiles(op, vec);
    const int64_t units = plan.n_chunks * (int64_t)op.H * th;
    if (units == 0) return cudaSuccess;
    if (units >= ((int64_t)1 << 31) - 8) return cudaErrorInvalidValue;
    const int64_t grid = cdiv(units, 8);
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const bool direct = th == 1;
    float *dst = direct ? C : part;
    const int64_t dld = direct ? c_ld : op.H;
    const int64_t tstride = (int64_t)g.E * op.H;
    if (ev_begin) cudaEventRecord(ev_begin, s);
    const Operand &P = a_is_src ? op.A : op.B;
    const bool o32 = (uint64_t)g.V_src * (uint64_t)P.ld < (1ull << 32) && UG_DOTT_O32;
    UG_DISPATCH_VEC(vec, VEC, {
        if (o32)
            k_dott<VEC, true><<<(unsigned)grid, 256, 0, s>>>(g, op, a_is_src, chunks, (int)plan.n_chunks, th, dst,
                                                             dld, tstride);
        else
            k_dott<VEC, false><<<(unsigned)grid, 256, 0, s>>>(g, op, a_is_src, chunks, (int)plan.n_chunks, th, dst,
                                                              dld, tstride);
    });
    if (ev_end) cudaEventRecord(ev_end, s);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess || direct) return err;
    const int64_t n = g.E * op.H;
    k_dott_fix<<<(unsigned)cdiv(n, 256), 256, 0, s>>>(part, g.E, op.H, th, tstride, C, c_ld);
    return cudaGetLastError();
}

}  // namespace ug
