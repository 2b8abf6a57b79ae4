// k_dotsv.cu -- `dot` between a Src_V and a Dst_V operand (u_dot_v / v_dot_u, the SDDMM of
// config C4; reading R5) under the SV schedule: the Dst_V row is loaded ONCE per work unit
// and kept in registers, so each in-edge gathers only the source row (half the L2->SM bytes
// of the edge-unit kernel, which loads both rows per edge).
//
// Work unit = one SV chunk (row v, in-edges [k0, k1), scratch slot; longest first, see
// get_plan).  L lanes serve a unit, in aligned groups of w = D/(NJ*VEC) lanes per head: lane
// (o, l) of head o owns the VEC-wide feature chunks o*D + (j*w + l)*VEC, j < NJ, so every load
// instruction of a group reads w*VEC contiguous floats of the head (one 128-byte line per 8
// lanes at VEC 4).  A head's message is an in-register FFMA chain over the lane's NJ*VEC
// features, then a log2(w)-step xor butterfly inside the group.  UE in-edges are gathered per
// step (16 floats per lane in flight), their column indices loaded first.  Message creation
// (C = Edge) stores one value per (edge, head); reductions keep the running value in the
// group's lanes and finalise owned rows in registers, split rows through the SV scratch and
// k_split_fix (chunk order, deterministic).
#include "k_split.cuh"

namespace ug {

#ifndef UG_DOTSV_MINB
#define UG_DOTSV_MINB 4   // resident CTAs per SM the register budget is sized for
#endif

// O32: every row of P is addressable with a 32-bit element offset (V_src * ld < 2^32): a gather
// address is one IMAD + IMAD.WIDE from the column index instead of 64-bit multiply / LEA pairs
// message creation (u_dot_v, GOP assign) holds no running reduction: with 32-bit gather offsets its
// widest instance fits 5 CTAs / SM spill-free (48 registers) -- C4 u_dot_v F = 128 69.6 -> 63.5 us,
// F = 256 155.7 -> 139.2 us, C3 241.7 -> 225.3 us (profiles/r2/ab_r2t_dotsv_minb.jsonl); the
// reductions keep UG_DOTSV_MINB (their NJ = 4 instance spills 144 B at 5)
#ifndef UG_DOTSV_MINB_MSG
#define UG_DOTSV_MINB_MSG 5
#endif
template <int GOP, int VEC, int NJ, bool O32>
__global__ void __launch_bounds__(256, GOP == UG_GATHER_ASSIGN ? UG_DOTSV_MINB_MSG : UG_DOTSV_MINB) k_dotsv(GraphArgs g, OpArgs op, bool a_is_src, const int4 *__restrict__ chunks,
                                                  int64_t n_chunks, int L_log2, int w_log2,
                                                  float *__restrict__ scratch, int64_t sld) {
    constexpr int UE = NJ * VEC >= 16 ? 1 : 16 / (NJ * VEC);   // in-edges per step
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int L = 1 << L_log2, w = 1 << w_log2;
    const int lane = (int)(t & (L - 1));
    const int64_t u = t >> L_log2;
    if (u >= n_chunks) return;
    const int wl = threadIdx.x & 31;
    const unsigned mask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (wl & ~(L - 1)));
    const int4 ch = chunks[u];
    const int64_t v = ch.x;
    const int o = lane >> w_log2;               // this lane's head
    const bool active = o < op.H;
    const int f0 = active ? o * op.D + (lane & (w - 1)) * VEC : 0;   // chunk j at f0 + j * w * VEC
    const Operand &P = a_is_src ? op.A : op.B;  // gathered per edge (Src_V)
    const Operand &Q = a_is_src ? op.B : op.A;  // hoisted (Dst_V, local row v)
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();

    float q[NJ][VEC];
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
        if (active) ldg_vec<VEC>(Q.p + v * Q.ld + f0 + j * w * VEC, q[j]);
        else
#pragma unroll
            for (int i = 0; i < VEC; ++i) q[j][i] = 0.0f;
    }
    const float *__restrict__ Pb = P.p + f0;
    const int jstride = w * VEC;
    const int64_t ldp = P.ld;
    const uint32_t ldp32 = (uint32_t)P.ld, f032 = (uint32_t)f0;
    // gather of chunk j of source row src
    auto gather = [&](int64_t src, int j, float (&r)[VEC]) {
        if constexpr (O32) ldg_vec_hint<VEC>(P.p + ((uint32_t)src * ldp32 + f032 + (uint32_t)(j * jstride)), r, keep);
        else ldg_vec_hint<VEC>(Pb + src * ldp + j * jstride, r, keep);
    };

    float acc = g_init<GOP>();
    auto edge_msg = [&](const float (&p)[NJ][VEC]) {
        float s = 0.0f;
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
            for (int i = 0; i < VEC; ++i) s = __fmaf_rn(p[j][i], q[j][i], s);
        for (int off = w >> 1; off > 0; off >>= 1) s += __shfl_xor_sync(mask, s, off);
        return s;
    };
    auto emit = [&](int k, float m) {
        if constexpr (GOP == UG_GATHER_ASSIGN) {
            if (active && (lane & (w - 1)) == 0) {
                const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
                op.C[e * op.c_ld + o] = m;
            }
        } else {
            acc = g_combine<GOP>(acc, m);
        }
    };
    int k = ch.y;                               // CSR positions are int32
    const int k1 = ch.z;
    // the next step's column indices are loaded while this step's rows are gathered (UG_DOTSV_PF;
    // r2an: C4 u_dot_v F = 128 79.8 -> 69.6 us, C3 276 -> 244 us, C4 u_dot_v_sum 82 -> 74 us)
#ifndef UG_DOTSV_PF
#define UG_DOTSV_PF 1
#endif
    constexpr bool PF = UG_DOTSV_PF && UE <= 4;
    int32_t s_pf[UE];
    if (PF && k + UE <= k1) {
#pragma unroll
        for (int e = 0; e < UE; ++e) s_pf[e] = ldg_i32_hint(g.col + k + e, stream);
    }
    for (; k + UE <= k1; k += UE) {
        float p[UE][NJ][VEC];
        int64_t s[UE];
#pragma unroll
        for (int e = 0; e < UE; ++e) {
            if (PF) {
                s[e] = s_pf[e];
                s_pf[e] = ldg_i32_hint(g.col + min(k + UE + e, k1 - 1), stream);
            } else {
                s[e] = ldg_i32_hint(g.col + k + e, stream);
            }
        }
#pragma unroll
        for (int e = 0; e < UE; ++e) {
#pragma unroll
            for (int j = 0; j < NJ; ++j) {
                if (active) gather(s[e], j, p[e][j]);
                else
#pragma unroll
                    for (int i = 0; i < VEC; ++i) p[e][j][i] = 0.0f;
            }
        }
#pragma unroll
        for (int e = 0; e < UE; ++e) emit(k + e, edge_msg(p[e]));
    }
    // one edge per step: the next edge's column index is loaded while this one is gathered
    int64_t s_next = k < k1 ? ldg_i32_hint(g.col + k, stream) : 0;
    for (; k < k1; ++k) {
        float p[NJ][VEC];
        const int64_t s = s_next;
        if (k + 1 < k1) s_next = ldg_i32_hint(g.col + k + 1, stream);
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
            if (active) gather(s, j, p[j]);
            else
#pragma unroll
                for (int i = 0; i < VEC; ++i) p[j][i] = 0.0f;
        }
        emit(k, edge_msg(p));
    }
    if constexpr (GOP != UG_GATHER_ASSIGN) {
        if (!active || (lane & (w - 1)) != 0) return;
        if (ch.w < 0) {
            const int64_t deg = (int64_t)k1 - ch.y;         // an owned row is one chunk: its whole in-edge list
            op.C[v * op.c_ld + o] = g_finalize<GOP>(acc, deg);
        } else {
            scratch[(int64_t)ch.w * sld + o] = acc;
        }
    }
}

// NJ * VEC features per lane, one head per lane: D % (NJ * VEC) == 0 and w = D / (NJ * VEC)
// a power of two; L = next power of two >= H * w, at most 32 -- the largest NJ that fits
// (fewer butterfly steps per edge: measured on C4 F=128, 8 lanes x 16 features 98 us against
// 32 lanes x 4 features 167 us).  Returns NJ, or 0 when the op does not fit (the caller then
// uses the generic dot kernel).
#ifndef UG_DOTSV_O32
#define UG_DOTSV_O32 1
#endif
int dotsv_nj(const OpArgs &op, int vec, int *L, int *w) {
    for (int nj : {4, 2, 1}) {
        const int per = nj * vec;
        if (op.D % per) continue;
        const int ww = op.D / per;
        if (ww & (ww - 1)) continue;
        const int64_t lanes = (int64_t)op.H * ww;
        if (lanes > 32) continue;
        int l = 1;
        while (l < lanes) l <<= 1;
        *L = l;
        *w = ww;
        return nj;
    }
    return 0;
}

cudaError_t launch_dotsv(int gather, const GraphArgs &g, const OpArgs &op, bool a_is_src, int vec, int block,
                         const SplitPlan &plan, float *scratch, cudaStream_t s, cudaEvent_t ev_begin,
                         cudaEvent_t ev_end) {
    int L = 0, w = 0;
    const int nj = dotsv_nj(op, vec, &L, &w);
    if (nj == 0) return cudaErrorInvalidValue;
    const int64_t threads = plan.n_chunks * (int64_t)L;
    if (threads == 0) return cudaSuccess;
    const int64_t grid = cdiv(threads, block);
    const int64_t sld = cdiv(op.W, 4) * 4;
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    if (ev_begin) cudaEventRecord(ev_begin, s);
    const Operand &P = a_is_src ? op.A : op.B;
    const bool o32 = (uint64_t)g.V_src * (uint64_t)P.ld < (1ull << 32) && UG_DOTSV_O32;
#define UG_DOTSV(NJV)                                                                                     \
    do {                                                                                                  \
        if (o32)                                                                                          \
            k_dotsv<GOP, VEC, NJV, true><<<(unsigned)grid, block, 0, s>>>(g, op, a_is_src, chunks,       \
                                                                          plan.n_chunks, ilog2(L),        \
                                                                          ilog2(w), scratch, sld);        \
        else                                                                                              \
            k_dotsv<GOP, VEC, NJV, false><<<(unsigned)grid, block, 0, s>>>(g, op, a_is_src, chunks,      \
                                                                           plan.n_chunks, ilog2(L),       \
                                                                           ilog2(w), scratch, sld);       \
    } while (0)
    UG_DISPATCH_VEC(vec, VEC,
        UG_DISPATCH_GOP(gather, GOP, {
            switch (nj) {
            case 1: UG_DOTSV(1); break;
            case 2: UG_DOTSV(2); break;
            default: UG_DOTSV(4); break;
            }
        }));
#undef UG_DOTSV
    if (ev_end) cudaEventRecord(ev_end, s);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess || gather == UG_GATHER_ASSIGN || plan.n_split_rows == 0) return err;
    const int64_t fgrid = cdiv(plan.n_split_rows * (int64_t)op.W, 256);
    const int4 *split = reinterpret_cast<const int4 *>(plan.d_split);
    UG_DISPATCH_RED(gather, GOP,
        k_split_fix<GOP, 1><<<(unsigned)fgrid, 256, 0, s>>>(g, op, split, plan.n_split_rows, scratch, sld));
    return cudaGetLastError();
}

}  // namespace ug
