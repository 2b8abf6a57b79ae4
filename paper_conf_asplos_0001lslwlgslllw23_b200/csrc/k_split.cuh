// k_split.cuh -- Split-Vertex (SV), the B200 schedule for wide, skewed aggregations
// (C3/C5).  It composes the paper's two knobs with two B200 facts: a
// 126 MB L2 and 148 SMs that all want equal work.
//
//  * Row splitting (load balance): every destination row is cut into chunks of at most
//    `group` in-edges (a hub of in-degree 4.9e4 becomes ~24 chunks).  A chunk is one work
//    unit; rows with one chunk are owned and finalised in registers; the partial results
//    of split rows go to a scratch slot and a fix-up kernel combines them in chunk order
//    (deterministic; no atomics, no init pass).
//  * Column tiles, tile-major (locality): the feature axis is cut into ftile-wide tiles and
//    the grid is ordered tile-major, so at any time the gathered rows touch one
//    V x ftile slab of X (C5, ftile 64: 60 MB) which stays L2-resident while the next
//    slab streams in; each X element then comes from DRAM about once per tile pass
//    instead of once per in-edge.
//  * L = ftile / VEC lanes per unit (one VEC-wide feature chunk per lane), the in-edge loop
//    unrolled 4x so each lane keeps 4 independent row gathers in flight.
#pragma once
#include <type_traits>
#include "k_dispatch.cuh"

namespace ug {

// Inner in-edge loop of the SV fast path.  BM: 0 no B operand, 1 B is Dst_V (constant over
// the row: loaded once), 2 / 3 B is an Edge tensor (row = CSR position) with per-head broadcast
// / full width, 4 / 5 B is Src_V with broadcast / full width, 6 / 7 B is a per-edge scalar stored
// contiguously (GCN's edge weight; 7 = the same loop at 8 CTAs / SM).  All offsets are 32-bit (the
// host checks rows * ld < 2^32).  The last, partial group of UF edges is predicated (its
// missing slots re-read the row's last edge, an L1 hit, and are not combined), so short rows
// never fall into a serial one-edge-at-a-time tail.  
template <int KE, int GOP, int VEC, int BM, bool IDX = false>
__device__ __forceinline__ void split_fast_loop(const GraphArgs &g, const OpArgs &op, int64_t v, int64_t k,
                                                const int64_t k1, int f, int64_t cb, float (&acc)[VEC],
                                                const int32_t *sidx = nullptr, int64_t kbase = 0) {
    // row gathers in flight per lane: 16 (measured +3 % over 8 on C5 at VEC 2), 8 for float4 rows;
    // half that when a B operand is loaded per edge (register budget of 40 for 6 CTAs / SM)
#ifndef UG_BM2_UF
#define UG_BM2_UF (VEC == 4 ? 4 : 8)
#endif
#ifndef UG_BM6_UF
#define UG_BM6_UF UG_BM2_UF
#endif
#ifndef UG_BM7_UF
#define UG_BM7_UF UG_BM6_UF
#endif
    constexpr int UF = BM == 0 || BM == 1 ? (VEC == 4 ? 8 : 16)
                     : (BM == 7 && KE != K_DIV) ? UG_BM7_UF
                     : (BM == 6 && KE != K_DIV) ? UG_BM6_UF
                     : (BM == 2 && KE != K_DIV) ? UG_BM2_UF : (VEC == 4 ? 4 : 8) / (KE == K_DIV ? 2 : 1);
    const float *__restrict__ Ab = op.A.p;          // warp-uniform base
    const uint64_t keep = l2_policy_evict_last();     // this tile's X column slab
    const uint64_t stream = l2_policy_evict_first();  // col_idx / edge tensors: read once per pass
    const uint32_t lda = (uint32_t)op.A.ld, fo = (uint32_t)f;
    // BM 6: a per-edge scalar stored contiguously (ld 1, column 0) -- the weight of position k is
    // B.p[k], addressed like col_idx (one pointer, immediate offsets; no per-edge IMAD / offset
    // registers)
    const uint32_t ldb = BM >= 6 ? 1u : (uint32_t)op.B.ld, cbo = BM >= 6 ? 0u : (uint32_t)cb;
    constexpr bool bfull = BM == 3 || BM == 5;
    float bconst[VEC];
    if constexpr (BM == 1) fetch<VEC>(op.B, v, cb, bconst);
    const int64_t kl = k1 - 1;
    // PF: the next group's column indices are loaded while this group's rows are gathered, so a
    // group costs one dependent L2 round trip (row) instead of two (col_idx, then row).  Off: it
    // measured slower here (r2an: C3 u_mul_e_sum 285 -> 293 us, C5 21.0 -> 24.3 ms; copy with
    // 6-7 CTAs / SM to make room 215 -> 244 us) -- unlike k_dotsv / k_dotattn_heads, where it wins
#ifndef UG_PF_BM2
#define UG_PF_BM2 0
#endif
#ifndef UG_PF_BM0
#define UG_PF_BM0 0
#endif
    constexpr bool PF = VEC == 4 && ((BM == 2 && UG_PF_BM2) || ((BM == 0 || BM == 1) && UG_PF_BM0));
    uint32_t s_pf[UF];
    if constexpr (PF) {
        if (k + UF <= k1) {                          // (empty rows: col[k1 - 1] may not exist)
#pragma unroll
            for (int q = 0; q < UF; ++q) s_pf[q] = (uint32_t)ldg_i32_hint(g.col + k + q, stream);
        }
    }
    auto group = [&](auto pred_tag, auto n_tag) {
        constexpr bool PRED = decltype(pred_tag)::value;
        constexpr int UF = decltype(n_tag)::value;
        uint32_t s[UF];
        if constexpr (PF && !PRED) {
#pragma unroll
            for (int q = 0; q < UF; ++q) {
                s[q] = s_pf[q];
                s_pf[q] = (uint32_t)ldg_i32_hint(g.col + min(k + UF + q, kl), stream);
            }
        } else if constexpr (IDX) {
            // column indices staged in this warp's shared-memory window (UG_SV_IDX_STAGE)
#pragma unroll
            for (int q = 0; q < UF; ++q) s[q] = (uint32_t)sidx[(PRED ? min(k + q, kl) : k + q) - kbase];
        } else {
#pragma unroll
            for (int q = 0; q < UF; ++q) s[q] = (uint32_t)ldg_i32_hint(g.col + (PRED ? min(k + q, kl) : k + q), stream);
        }
        float m[UF][VEC];
#pragma unroll
        for (int q = 0; q < UF; ++q) ldg_vec_hint<VEC>(Ab + (s[q] * lda + fo), m[q], keep);
#ifndef UG_MUL_FMA
#define UG_MUL_FMA 1
#endif
        // UG_MUL_FMA: a per-edge scalar weight folded into the sum by FMA (the message x * w is then
        // rounded together with the add, not on its own -- inside R11's 1e-5 * sum|terms| bound,
        // exact in integer mode).  On with the contiguous-weight loops: C5 u_mul_e_sum 19.19 ->
        // 18.71 ms, C3 F = 128 256.3 -> 254.2 us (profiles/r2/ab_s2_r2l.jsonl; r2 with BM 2 it lost)
        constexpr bool FMA_W = UG_MUL_FMA && BM >= 6 && KE == K_MUL && (GOP == UG_GATHER_SUM || GOP == UG_GATHER_MEAN);
        if constexpr (FMA_W) {
            float wq[UF];
#pragma unroll
            for (int q = 0; q < UF; ++q)
                wq[q] = BM >= 6 ? __ldg(op.B.p + (PRED ? min(k + q, kl) : k + q))
                                : __ldg(op.B.p + ((uint32_t)(PRED ? min(k + q, kl) : k + q) * ldb + cbo));
#pragma unroll
            for (int q = 0; q < UF; ++q) {
                const bool ok = !PRED || k + q < k1;
#pragma unroll
                for (int i = 0; i < VEC; ++i) acc[i] = ok ? __fmaf_rn(m[q][i], wq[q], acc[i]) : acc[i];
            }
            return;
        }
        if constexpr (BM != 0) {
#pragma unroll
            for (int q = 0; q < UF; ++q) {
                float b[VEC];
                if constexpr (BM == 1) {
#pragma unroll
                    for (int i = 0; i < VEC; ++i) b[i] = bconst[i];
                } else {
                    const uint32_t row = (BM == 2 || BM == 3 || BM >= 6) ? (uint32_t)(PRED ? min(k + q, kl) : k + q) : s[q];
                    // BM 6: 64-bit position arithmetic, so B.p + k becomes one pointer with
                    // immediate offsets (as for col_idx) instead of a 32-bit IMAD per edge
                    const float *bp = BM >= 6 ? op.B.p + (PRED ? min(k + q, kl) : k + q) : op.B.p + (row * ldb + cbo);
                    if constexpr (bfull) {
                        ldg_vec_hint<VEC>(bp, b, BM == 3 ? stream : keep);
                    } else {
#ifdef UG_EXPERIMENT_NO_WEIGHT_LOAD
                        // timing experiment only (wrong results): the per-edge weight load removed
                        const float x = 1.0f + (float)(row & 1) * (float)(uintptr_t)bp * 0.0f;
#else
                        const float x = __ldg(bp);
#endif
#pragma unroll
                        for (int i = 0; i < VEC; ++i) b[i] = x;
                    }
                }
#pragma unroll
                for (int i = 0; i < VEC; ++i) m[q][i] = edge_fn<KE>(m[q][i], b[i]);
            }
        }
#pragma unroll
        for (int q = 0; q < UF; ++q) {
            const bool ok = !PRED || k + q < k1;
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[i] = ok ? g_combine<GOP>(acc[i], m[q][i]) : acc[i];
        }
    };
    for (; k + UF <= k1; k += UF) group(std::false_type{}, std::integral_constant<int, UF>{});
    // the last, partial group: predicated half-groups (fewer registers), not a serial tail.
    // UG_SV_TAIL_FULL: a remainder of more than UF / 2 edges takes ONE predicated full-size group
    // (one dependent round trip instead of two for short rows; A/B switch)
    constexpr int UH = UF / 2 > 0 ? UF / 2 : 1;
#ifndef UG_SV_TAIL_FULL
#define UG_SV_TAIL_FULL 0
#endif
    if constexpr (UG_SV_TAIL_FULL && UF > 1) {
        if (k1 - k > UH) {
            group(std::true_type{}, std::integral_constant<int, UF>{});
            k = k1;
        }
    }
    for (; k < k1; k += UH) group(std::true_type{}, std::integral_constant<int, UH>{});
}

// Message creation (gather ASSIGN, C = Edge) on the fast path: the unit's in-edges are the
// CSR positions [k, k1) (= edge ids), so each edge's message row is stored contiguously across
// the unit's lanes; the Src_V row is gathered per edge, a Dst_V B operand is loaded once per
// unit (BM 1), Edge / Src_V B operands per edge.  UF edges per step (loads first, then stores).
template <int KE, int VEC, int BM>
__device__ __forceinline__ void split_fast_assign(const GraphArgs &g, const OpArgs &op, int64_t v, int64_t k,
                                                  const int64_t k1, int f, int64_t cb) {
#ifndef UG_ASSIGN_UF
#define UG_ASSIGN_UF 4
#endif
    constexpr int UF = UG_ASSIGN_UF;
    const float *__restrict__ Ab = op.A.p;
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
    const uint32_t lda = (uint32_t)op.A.ld, fo = (uint32_t)f;
    const uint32_t ldb = BM >= 6 ? 1u : (uint32_t)op.B.ld, cbo = BM >= 6 ? 0u : (uint32_t)cb;
    constexpr bool bfull = BM == 3 || BM == 5;
    const int nout = op.W - f;
    const bool full_vec = nout >= VEC && op.c_vec >= VEC;
    float bconst[VEC];
    if constexpr (BM == 1) fetch<VEC>(op.B, v, cb, bconst);
    auto one = [&](int64_t kk, uint32_t sq, float (&m)[VEC]) {
        ldg_vec_hint<VEC>(Ab + (sq * lda + fo), m, keep);
        if constexpr (BM != 0) {
            float b[VEC];
            if constexpr (BM == 1) {
#pragma unroll
                for (int i = 0; i < VEC; ++i) b[i] = bconst[i];
            } else {
                const uint32_t row = (BM == 2 || BM == 3 || BM >= 6) ? (uint32_t)kk : sq;
                const float *bp = op.B.p + (row * ldb + cbo);
                if constexpr (bfull) {
                    ldg_vec_hint<VEC>(bp, b, BM == 3 ? stream : keep);
                } else {
                    const float x = __ldg(bp);
#pragma unroll
                    for (int i = 0; i < VEC; ++i) b[i] = x;
                }
            }
#pragma unroll
            for (int i = 0; i < VEC; ++i) m[i] = edge_fn<KE>(m[i], b[i]);
        }
    };
    // UG_ASSIGN_UNSWITCH: the loop unswitched on the (unit-invariant) store form, so full-vector
    // stores carry no ragged-tail branches (36 -> 14 SASS instructions per edge) -- measured SLOWER
    // (C4 u_add_v F = 128 157.7 -> 161.8 us, C3 F = 32 135.7 -> 143.3 us; profiles/r2/ab_r2u_assign.jsonl):
    // message creation is bound by its write stream, not issue.  Off; kept as an A/B switch
#ifndef UG_ASSIGN_UNSWITCH
#define UG_ASSIGN_UNSWITCH 0
#endif
    auto run = [&](auto fv_tag) {
        constexpr bool FV = decltype(fv_tag)::value;
        auto store = [&](int64_t kk, const float (&m)[VEC]) {
            float *cp = op.C + kk * op.c_ld + f;
            if constexpr (FV) {
                st_vec_hint<VEC>(cp, m, stream);
            } else {
                if (full_vec) st_vec_hint<VEC>(cp, m, stream);
                else st_out<VEC>(cp, m, nout, op.c_vec);
            }
        };
        for (; k + UF <= k1; k += UF) {
            uint32_t sq[UF];
#pragma unroll
            for (int q = 0; q < UF; ++q) sq[q] = (uint32_t)ldg_i32_hint(g.col + k + q, stream);
            float m[UF][VEC];
#pragma unroll
            for (int q = 0; q < UF; ++q) one(k + q, sq[q], m[q]);
#pragma unroll
            for (int q = 0; q < UF; ++q) store(k + q, m[q]);
        }
        for (; k < k1; ++k) {
            float m[VEC];
            one(k, (uint32_t)ldg_i32_hint(g.col + k, stream), m);
            store(k, m);
        }
    };
    if (UG_ASSIGN_UNSWITCH && full_vec) run(std::true_type{});
    else run(std::false_type{});
}

// BM = 2 (per-edge scalar B, e.g. u_mul_e_sum): 6 CTAs / SM (40 registers, spill-free) for sum /
// mean, measured 305 -> 291 us on C3 F = 128 and 82 -> 76 us at F = 32 (scripts/gpu_bm2.sh);
// max / min and div keep 5 (48 registers: at 40 they spill 30-80 bytes per thread)
#ifndef UG_BM2_MINB
#define UG_BM2_MINB 5
#endif
#ifndef UG_BM2_SUM_MINB
#define UG_BM2_SUM_MINB 6
#endif
// BM = 6 (a per-edge scalar stored contiguously): its addressing frees the per-edge offset registers
#ifndef UG_BM6_SUM_MINB
#define UG_BM6_SUM_MINB 6
#endif
// BM = 7: the BM 6 loop at 8 CTAs / SM (32 registers) for sum / mean on short-chunk graphs with
// many waves -- C3 u_mul_e_sum F = 128 268.5 -> 252.2 us, C4 92.4 -> 86.3 us, but C5 (long chunks)
// 19.5 -> 21.3 ms and C2 (one wave) 13.6 -> 15.6 us (profiles/r2/ab_s2_r2i.jsonl); chosen at launch
#ifndef UG_BM7_MINB
#define UG_BM7_MINB 8
#endif
#ifndef UG_BM0_MINB
#define UG_BM0_MINB 8
#endif

// Column-index staging (UG_SV_IDX_STAGE, the north star's "TMA or shared-memory staging of CSR
// column-index tiles"; an A/B switch): when a whole warp serves one unit (L = 32), the unit's
// col_idx[k0, k1) is copied into a per-warp shared-memory window of UG_IDX_WIN indices before the
// gathers -- 1: by cp.async (LDGSTS, 4 bytes per lane), 2: by one 1-D bulk TMA copy
// (cp.async.bulk ... mbarrier::complete_tx, issued by lane 0; the window starts at the aligned-down
// 16-byte boundary, and the graph's col_idx allocation is padded so the rounded-up tail is in
// bounds) -- and the in-edge loop reads its indices from shared memory.
#ifndef UG_SV_IDX_STAGE
#define UG_SV_IDX_STAGE 0
#endif
#define UG_IDX_WIN 512
struct IdxStage {
    int32_t *buf;        // this warp's window: UG_IDX_WIN + 4 indices, 16-byte aligned
    uint32_t bar;        // its mbarrier (method 2)
    uint32_t phase;
};

template <int KE, int GOP, int VEC, int BM>
__device__ __forceinline__ void split_loop_staged(const GraphArgs &g, const OpArgs &op, int64_t v, int64_t k0,
                                                  const int64_t k1, int f, int64_t cb, float (&acc)[VEC],
                                                  IdxStage &st) {
    const int lane = threadIdx.x & 31;
    for (int64_t kw = k0; kw < k1; kw += UG_IDX_WIN) {
        const int64_t ke = min(k1, kw + (int64_t)UG_IDX_WIN);
        int64_t kbase = kw;
        if constexpr (UG_SV_IDX_STAGE == 1) {
            const uint32_t dst = (uint32_t)__cvta_generic_to_shared(st.buf);
            for (int64_t i = kw + lane; i < ke; i += 32)
                asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst + (uint32_t)(i - kw) * 4u),
                             "l"(g.col + i) : "memory");
            asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
        } else {
            const int64_t a0 = kw & ~(int64_t)3;           // 16-byte aligned start (col is 256-B aligned)
            kbase = a0;
            if (lane == 0) {
                const uint32_t bytes = (uint32_t)(((ke - a0) * 4 + 15) & ~(int64_t)15);
                const uint32_t dst = (uint32_t)__cvta_generic_to_shared(st.buf);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(st.bar), "r"(bytes)
                             : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(dst), "l"(g.col + a0), "r"(bytes), "r"(st.bar) : "memory");
            }
            asm volatile(
                "{\n\t.reg .pred p;\n\t"
                "WAIT_%=:\n\t"
                "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                "@!p bra WAIT_%=;\n\t}" ::"r"(st.bar), "r"(st.phase) : "memory");
            st.phase ^= 1u;
        }
        __syncwarp();
        split_fast_loop<KE, GOP, VEC, BM, true>(g, op, v, kw, ke, f, cb, acc, st.buf, kbase);
        __syncwarp();                                      // the window is refilled next
    }
}

// One work unit (a chunk of <= G in-edges of one row, one VEC-wide column chunk per lane).
// BM < 0: generic addressing (any operand types, eid); BM >= 0: the fast path with the B
// operand's addressing mode fixed at compile time (see split_fast_loop).
template <int KE, int GOP, int VEC, int BM>
__device__ __forceinline__ void split_unit(const GraphArgs &g, const OpArgs &op, const int4 ch, const int f,
                                           float *__restrict__ scratch, const int64_t sld, IdxStage *st = nullptr,
                                           const bool store = true) {
    constexpr bool FAST = BM >= 0;
    constexpr int U = 4;                       // independent row gathers in flight per lane
    const int64_t v = ch.x;
    const int64_t k1 = ch.z;
    const int64_t ca = op_col(op.A, f);
    const int64_t cb = op_col(op.B, f);

    if constexpr (GOP == UG_GATHER_ASSIGN && FAST) {
        split_fast_assign<KE, VEC, BM>(g, op, v, ch.y, k1, f, cb);
    } else if constexpr (GOP == UG_GATHER_ASSIGN) {
        for (int64_t k = ch.y; k < k1; ++k) {
            const int64_t src = g.col[k];
            const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
            float m[VEC];
            message<KE, VEC>(op, op_row(op.A.type, src, v, e), ca, op_row(op.B.type, src, v, e), cb, m);
            st_out<VEC>(op.C + e * op.c_ld + f, m, op.W - f, op.c_vec);
        }
    } else {
        float acc[VEC];
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = g_init<GOP>();
        int64_t k = ch.y;
        if constexpr (FAST) {
            // A is a full-width Src_V operand smaller than 4 GiB and edge ids are CSR positions:
            // the row address is one IMAD + IMAD.WIDE from the (warp-uniform, L1-broadcast)
            // column index, so each in-edge costs ~6 instructions per lane.  The B operand's
            // addressing mode BM is a template parameter (a Dst_V operand is loaded once).
            if (UG_SV_IDX_STAGE && st) split_loop_staged<KE, GOP, VEC, BM>(g, op, v, k, k1, f, cb, acc, *st);
            else split_fast_loop<KE, GOP, VEC, BM>(g, op, v, k, k1, f, cb, acc);
            k = k1;
        } else {
            for (; k + U <= k1; k += U) {
                float m[U][VEC];
#pragma unroll
                for (int q = 0; q < U; ++q) {
                    const int64_t src = g.col[k + q];
                    const int64_t e = g.eid ? (int64_t)g.eid[k + q] : k + q;
                    message<KE, VEC>(op, op_row(op.A.type, src, v, e), ca, op_row(op.B.type, src, v, e), cb, m[q]);
                }
#pragma unroll
                for (int q = 0; q < U; ++q)
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[i] = g_combine<GOP>(acc[i], m[q][i]);
            }
        }
        for (; k < k1; ++k) {
            const int64_t src = g.col[k];
            const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
            float m[VEC];
            message<KE, VEC>(op, op_row(op.A.type, src, v, e), ca, op_row(op.B.type, src, v, e), cb, m);
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[i] = g_combine<GOP>(acc[i], m[i]);
        }
        // outputs are written once: evict_first keeps them from displacing the X slab in L2
        const uint64_t wpol = l2_policy_evict_first();
        if (!store) return;
        if (ch.w < 0) {
            // sum needs no degree (an empty row's accumulator is already +0)
            const int64_t deg = GOP == UG_GATHER_SUM ? 1 : (int64_t)g.row_ptr[v + 1] - g.row_ptr[v];
            float out[VEC];
#pragma unroll
            for (int i = 0; i < VEC; ++i) out[i] = g_finalize<GOP>(acc[i], deg);
            if (f + VEC <= op.W && op.c_vec >= VEC) st_vec_hint<VEC>(op.C + v * op.c_ld + f, out, wpol);
            else st_out<VEC>(op.C + v * op.c_ld + f, out, op.W - f, op.c_vec);
        } else {
            st_vec_hint<VEC>(scratch + (int64_t)ch.w * sld + f, acc, wpol);
        }
    }
}

// unit -> column tile (units are tile-major): no division for one tile, 32-bit below 2^31
__device__ __forceinline__ int unit_tile(int64_t u, int64_t n_chunks, int n_tiles) {
    if (n_tiles == 1) return 0;
    return u < INT32_MAX ? (int)((uint32_t)u / (uint32_t)n_chunks) : (int)(u / n_chunks);
}

// Single-launch merge of a split row: every chunk of the row has stored its partial; the unit
// that arrives last (per row and column tile) combines the partials in chunk order -- the order
// k_split_fix uses, so results are identical -- and re-arms the counter for the next call on
// this stream.  Called by every lane of a unit whose chunk belongs to a split row.
template <int GOP, int VEC>
__device__ __forceinline__ void split_merge(const GraphArgs &g, const OpArgs &op, const int4 *__restrict__ chunks,
                                            const int64_t n_chunks, const int L_log2, const int ftile,
                                            const int n_tiles, const float *__restrict__ scratch, const int64_t sld,
                                            const int4 *__restrict__ split, const int32_t *__restrict__ slot_row,
                                            int32_t *__restrict__ counters) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int L = 1 << L_log2;
    const int lane = (int)(t & (L - 1));
    const int64_t u = t >> L_log2;
    const int tile = unit_tile(u, n_chunks, n_tiles);
    const int f = tile * ftile + lane * VEC;
    int4 ch;   // re-read (volatile: not kept live from the traversal)
    asm volatile("ld.global.cg.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(ch.x), "=r"(ch.y), "=r"(ch.z), "=r"(ch.w) : "l"(chunks + (u - (int64_t)tile * n_chunks)));
    if (ch.w < 0) return;                         // an owned row: finished in the traversal
    fence_acq_rel_gpu();
    const int wl = threadIdx.x & 31;
    const unsigned umask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (wl & ~(L - 1)));
    __syncwarp(umask);
    const int r = slot_row[ch.w];
    const int4 sp = split[r];
    int last = 0;
    if (lane == 0) last = atomicAdd(counters + (int64_t)r * n_tiles + tile, 1) == sp.z - 1;
    last = __shfl_sync(umask, last, wl & ~(L - 1));
    if (!last) return;
    fence_acq_rel_gpu();
    if (lane == 0) counters[(int64_t)r * n_tiles + tile] = 0;
    if (f >= op.W || lane * VEC >= ftile) return;
    float acc[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = g_init<GOP>();
    for (int c = 0; c < sp.z; ++c) {
        const float *pp = scratch + (int64_t)(sp.y + c) * sld + f;
        float p[VEC];
        if constexpr (VEC == 4) {
            const float4 x = __ldcg(reinterpret_cast<const float4 *>(pp));
            p[0] = x.x; p[1] = x.y; p[2] = x.z; p[3] = x.w;
        } else if constexpr (VEC == 2) {
            const float2 x = __ldcg(reinterpret_cast<const float2 *>(pp));
            p[0] = x.x; p[1] = x.y;
        } else {
            p[0] = __ldcg(pp);
        }
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = g_combine<GOP>(acc[i], p[i]);
    }
    const int64_t v = sp.x;
    const int64_t deg = (int64_t)g.row_ptr[v + 1] - g.row_ptr[v];
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = g_finalize<GOP>(acc[i], deg);
    st_out<VEC>(op.C + v * op.c_ld + f, acc, op.W - f, op.c_vec);
}

template <int KE, int GOP, int VEC, int BM, bool MERGE>
#ifndef UG_ASSIGN_MINB
#define UG_ASSIGN_MINB 6
#endif
__global__ void __launch_bounds__(256, (UG_ASSIGN_MINB > 0 && GOP == UG_GATHER_ASSIGN) ? UG_ASSIGN_MINB : (BM == 0) ? UG_BM0_MINB : (BM == 7) ? UG_BM7_MINB : (BM == 6 && (GOP == UG_GATHER_SUM || GOP == UG_GATHER_MEAN) && KE != K_DIV) ? UG_BM6_SUM_MINB : ((BM == 2 || BM == 6) ? ((GOP == UG_GATHER_SUM || GOP == UG_GATHER_MEAN) && KE != K_DIV ? UG_BM2_SUM_MINB : UG_BM2_MINB) : (BM > 0 ? (VEC == 4 ? 5 : 6) : 4))) k_split(GraphArgs g, OpArgs op, const int4 *__restrict__ chunks,
                                               int64_t n_chunks, int L_log2, int ftile, int n_tiles,
                                               float *__restrict__ scratch, int64_t sld,
                                               const int4 *__restrict__ split, const int32_t *__restrict__ slot_row,
                                               int32_t *__restrict__ counters) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = (int)(t & ((1 << L_log2) - 1));
    const int64_t u = t >> L_log2;
    if (u >= n_chunks * n_tiles) return;          // whole units only: a unit's L lanes leave together
    const int tile = unit_tile(u, n_chunks, n_tiles);
    const int f = tile * ftile + lane * VEC;
    const bool lane_ok = lane * VEC < ftile;       // false only for the idle lanes of a non-pow2 tile
    if constexpr (!MERGE) {
        // split rows (if any) are combined by k_split_fix, a second launch
        if constexpr (UG_SV_IDX_STAGE != 0 && (BM == 0 || BM >= 6) && VEC == 4) {
            if (L_log2 == 5) {                             // one unit per warp: stage its col_idx
                __shared__ __align__(128) int32_t s_idx[8][UG_IDX_WIN + 4];
                __shared__ __align__(8) uint64_t s_bar[8];
                const int w = threadIdx.x >> 5;
                IdxStage st{s_idx[w], (uint32_t)__cvta_generic_to_shared(&s_bar[w]), 0u};
                if constexpr (UG_SV_IDX_STAGE == 2) {
                    if ((threadIdx.x & 31) == 0) {
                        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(st.bar) : "memory");
                        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
                    }
                    __syncwarp();
                }
                // every lane of the warp takes part in the staging; the idle lanes of a ragged last
                // tile gather the tile's first columns (valid addresses) and store nothing
                const bool act = f < op.W && lane_ok;
                split_unit<KE, GOP, VEC, BM>(g, op, chunks[u - (int64_t)tile * n_chunks], act ? f : tile * ftile,
                                             scratch, sld, &st, act);
                return;
            }
        }
        if (f >= op.W || !lane_ok) return;
        split_unit<KE, GOP, VEC, BM>(g, op, chunks[u - (int64_t)tile * n_chunks], f, scratch, sld);
    } else {
        // single-launch merge of split rows: the last-arriving chunk of a row combines them.  A
        // separate instance (launch-bound small graphs): the merge needs every lane of the unit
        // and re-derives its indices after the in-edge loop.
        if (f < op.W && lane_ok) split_unit<KE, GOP, VEC, BM>(g, op, chunks[u - (int64_t)tile * n_chunks], f, scratch, sld);
        split_merge<GOP, VEC>(g, op, chunks, n_chunks, L_log2, ftile, n_tiles, scratch, sld, split, slot_row,
                              counters);
    }
}

// Fix-up of split rows: combine the row's partials in chunk order, finalise, store.
template <int GOP, int VEC>
__global__ void k_split_fix(GraphArgs g, OpArgs op, const int4 *__restrict__ split, int64_t n_split,
                            const float *__restrict__ scratch, int64_t sld) {
    const int64_t per_row = cdiv(op.W, VEC);
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= n_split * per_row) return;
    const int64_t r = t / per_row;
    const int f = (int)(t - r * per_row) * VEC;
    const int4 sp = split[r];
    float acc[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = g_init<GOP>();
    for (int s = 0; s < sp.z; ++s) {
        float p[VEC];
        ldg_vec<VEC>(scratch + (int64_t)(sp.y + s) * sld + f, p);
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = g_combine<GOP>(acc[i], p[i]);
    }
    const int64_t v = sp.x;
    const int64_t deg = (int64_t)g.row_ptr[v + 1] - g.row_ptr[v];
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = g_finalize<GOP>(acc[i], deg);
    st_out<VEC>(op.C + v * op.c_ld + f, acc, op.W - f, op.c_vec);
}

#ifndef UG_SV_BM6
#define UG_SV_BM6 1
#endif
#ifndef UG_SV_BM7
#define UG_SV_BM7 1
#endif
// Launch of one edge_op's SV instances (explicitly instantiated per KE in k_split*.cu).
template <int KE>
cudaError_t launch_split_ke(int gather, const GraphArgs &g, const OpArgs &op, const LaunchCfg &c,
                            const SplitPlan &plan, float *scratch, cudaStream_t s, cudaEvent_t ev_begin,
                            cudaEvent_t ev_end, int32_t *counters) {
    int L = 1;
    while (L * c.vec < c.ftile) L <<= 1;        // lanes past ftile / vec (a non-power-of-two tile) idle
    const int n_tiles = (int)cdiv(op.W, c.ftile);
    const int64_t threads = plan.n_chunks * n_tiles * (int64_t)L;
    if (threads == 0) return cudaSuccess;
    const int64_t grid = cdiv(threads, c.block);
    const int L_log2 = ilog2(L);
    const int64_t sld = cdiv(op.W, 4) * 4;
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const int4 *split_p = reinterpret_cast<const int4 *>(plan.d_split);
    if (plan.n_split_rows == 0 || gather == UG_GATHER_ASSIGN) counters = nullptr;
    if (ev_begin) cudaEventRecord(ev_begin, s);
    // fast path: full-width Src_V A operand, identity edge ids, and every operand row
    // addressable with 32-bit element offsets (rows * ld < 2^32)
    const uint64_t lim = 1ull << 32;
    bool fast = op.A.type == UG_T_SRC_V && op.A.div == 1 && g.eid == nullptr &&
                (uint64_t)g.V_src * (uint64_t)op.A.ld < lim;
    if (KE != K_COPY) {
        const uint64_t brows = op.B.type == UG_T_EDGE ? (uint64_t)g.E : (uint64_t)g.V_src;
        fast = fast && brows * (uint64_t)op.B.ld < lim;
    }
    const int bfl = op.B.div == 1 ? 1 : 0;
    const int bm = !fast ? -1 : KE == K_COPY ? 0
                 : op.B.type == UG_T_DST_V ? 1
                 : op.B.type == UG_T_EDGE ? (op.B.div == op.W && op.B.ld == 1 && UG_SV_BM6 ? 6 : 2 + bfl) : 4 + bfl;
    // occupancy instance of BM 6 (see UG_BM7_MINB): short chunks (< 32 in-edges on average) and a
    // grid of at least four waves at 8 CTAs / SM
    const bool short_chunks = plan.n_chunks > 0 && g.E < 32 * plan.n_chunks;
    const int bm_launch = (bm == 6 && UG_SV_BM7 && short_chunks && threads >= (int64_t)4 * 148 * 2048) ? 7 : bm;
#define UG_SV_LAUNCH(BMV)                                                                                    \
    do {                                                                                                     \
        if constexpr (GOP != UG_GATHER_ASSIGN) {                                                             \
            if (counters) {                                                                                  \
                k_split<KE, GOP, VEC, BMV, true><<<(unsigned)grid, c.block, 0, s>>>(                         \
                    g, op, chunks, plan.n_chunks, L_log2, c.ftile, n_tiles, scratch, sld, split_p,           \
                    plan.d_slot_row, counters);                                                              \
                break;                                                                                       \
            }                                                                                                \
        }                                                                                                    \
        k_split<KE, GOP, VEC, BMV, false><<<(unsigned)grid, c.block, 0, s>>>(                                \
            g, op, chunks, plan.n_chunks, L_log2, c.ftile, n_tiles, scratch, sld, split_p, plan.d_slot_row,   \
            nullptr);                                                                                        \
    } while (0)
    UG_DISPATCH_VEC(c.vec, VEC,
        UG_DISPATCH_GOP(gather, GOP, {
            if constexpr (KE == K_COPY) {
                if (bm == 0) UG_SV_LAUNCH(0); else UG_SV_LAUNCH(-1);
            } else {
                switch (bm_launch) {
                case 1: UG_SV_LAUNCH(1); break;
                case 2: UG_SV_LAUNCH(2); break;
                case 3: UG_SV_LAUNCH(3); break;
                case 4: UG_SV_LAUNCH(4); break;
                case 5: UG_SV_LAUNCH(5); break;
                case 6: UG_SV_LAUNCH(6); break;
                case 7:
                    if constexpr ((GOP == UG_GATHER_SUM || GOP == UG_GATHER_MEAN) && KE != K_DIV) UG_SV_LAUNCH(7);
                    else UG_SV_LAUNCH(6);
                    break;
                default: UG_SV_LAUNCH(-1); break;
                }
            }
        }));
#undef UG_SV_LAUNCH
    if (ev_end) cudaEventRecord(ev_end, s);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess || gather == UG_GATHER_ASSIGN || plan.n_split_rows == 0 || counters) return err;
    const int64_t per_row = cdiv(op.W, c.vec);
    const int64_t fgrid = cdiv(plan.n_split_rows * per_row, 256);
    const int4 *split = reinterpret_cast<const int4 *>(plan.d_split);
    UG_DISPATCH_VEC(c.vec, VEC,
        UG_DISPATCH_RED(gather, GOP,
            k_split_fix<GOP, VEC><<<(unsigned)fgrid, 256, 0, s>>>(g, op, split, plan.n_split_rows,
                                                                  scratch, sld)));
    return cudaGetLastError();
}

#define UG_SV_INSTANTIATE(KE)                                                                            \
    template cudaError_t launch_split_ke<KE>(int, const GraphArgs &, const OpArgs &, const LaunchCfg &, \
                                             const SplitPlan &, float *, cudaStream_t, cudaEvent_t,     \
                                             cudaEvent_t, int32_t *);

}  // namespace ug
