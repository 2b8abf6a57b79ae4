// k_svg.cuh -- SV with TMA row gathers (schedule flag UG_SCHED_TMA, "_M1"): the Split-Vertex
// schedule (k_split.cuh) with the source-row gathers moved off the register file.
//
// The aggregation loop of Fig. 5 gathers one row of X per in-edge.  In the
// register-resident SV kernel every gather in flight costs registers, so a second operand per
// edge (GCN's edge weight, u_mul_e_sum; "heavier in access and computation")
// halves the gathers in flight and the kernel turns latency-bound.  Here:
//
//  * One warp walks a sequence of work units (column tile x row chunk of <= G in-edges, the SV
//    plan, longest first), u = w, w + S, ... over the S resident warps (persistent grid).
//  * Lane 0 issues `cp.async.bulk.tensor.2d...tile::gather4`: FOUR source rows x one
//    TW-float column tile (box {TW, 1}) land in a shared-memory stage, completion counted on
//    that stage's mbarrier (expect_tx).  D stages per warp form a ring, so D x 4 row gathers
//    are in flight per warp with no register cost; issue runs exactly D groups ahead of
//    consumption and flows across unit boundaries (short rows do not drain the pipeline).
//  * All 32 lanes wait on the stage barrier, read their VEC = TW / 32 features of each row
//    (conflict-free LDS.128 / .64), apply edge_op with the B operand (Dst_V: loaded once per
//    unit; Edge: per edge, warp-uniform for a scalar weight) and reduce in registers.
//  * Owned rows are finalised in registers (mean / zero rows); split rows write partials to
//    their scratch slot and k_split_fix combines them in chunk order (deterministic).
//
// Requirements (checked on the host, ug_op.cpp): A is a full-width Src_V operand with
// 16-byte aligned base and row stride (the pack stage provides it), identity edge ids, and
// B (if any) is Dst_V or a per-edge broadcast Edge tensor.
#pragma once
#include <cuda.h>

#include "k_dispatch.cuh"

namespace ug {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
        "r"(parity)
        : "memory");
}

// Four rows r0..r3 of the column tile starting at c0 -> 4 x TW floats at dst (one TMA op).
__device__ __forceinline__ void tma_gather4(uint32_t dst, const CUtensorMap *tm, uint32_t bar, int c0, int r0, int r1,
                                            int r2, int r3, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;" ::"r"(dst),
        "l"(reinterpret_cast<uint64_t>(tm)), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(bar), "l"(pol)
        : "memory");
}

template <int VEC>
__device__ __forceinline__ void lds_vec(const float *p, float (&r)[VEC]) {
    if constexpr (VEC == 4) {
        const float4 t = *reinterpret_cast<const float4 *>(p);
        r[0] = t.x; r[1] = t.y; r[2] = t.z; r[3] = t.w;
    } else if constexpr (VEC == 2) {
        const float2 t = *reinterpret_cast<const float2 *>(p);
        r[0] = t.x; r[1] = t.y;
    } else {
        r[0] = *p;
    }
}

// cp.async (LDGSTS): `bytes` (<= 16) of src into dst, the rest of the 4 * VEC bytes zero-filled.
template <int VEC>
__device__ __forceinline__ void cp_async_vec(uint32_t dst, const float *src, int bytes, uint64_t pol) {
    if constexpr (VEC == 4) {
        asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(dst), "l"(src),
                     "r"(bytes), "l"(pol) : "memory");
    } else if constexpr (VEC == 2) {
        asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2, %3;" ::"r"(dst), "l"(src),
                     "r"(bytes), "l"(pol) : "memory");
    } else {
        asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2, %3;" ::"r"(dst), "l"(src),
                     "r"(bytes), "l"(pol) : "memory");
    }
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

#ifndef UG_SVG_WARPS
#define UG_SVG_WARPS 4
#endif
// Ring per warp: D stages of R = 8 rows (two gather4 / eight cp.async per lane) of TW floats,
// about UG_SVG_RING_KB KB per warp (TW = 128: D = 3, 24 rows in flight; 16 warps per SM).
#ifndef UG_SVG_RING_KB
#define UG_SVG_RING_KB 12
#endif
constexpr int SVG_R = 8;
template <int VEC>
struct SvgDepth {
    static constexpr int D0 = (UG_SVG_RING_KB * 1024) / (SVG_R * 32 * VEC * 4);
    static constexpr int D = D0 < 2 ? 2 : D0;
};

template <int MODE, int VEC>
constexpr size_t svg_smem_bytes() {
    return (size_t)UG_SVG_WARPS * SvgDepth<VEC>::D * (SVG_R * (32 * VEC) + 32) * sizeof(float) +
           (size_t)UG_SVG_WARPS * SvgDepth<VEC>::D * sizeof(uint64_t);
}

// Work-unit cursor over u = t * n_chunks + c, u = w0, w0 + S, ... (32-bit, no division).
struct SvgCursor {
    int c, t;
    __device__ __forceinline__ void init(int w0, int n_chunks) {
        c = w0;
        t = 0;
        while (c >= n_chunks) { c -= n_chunks; ++t; }
    }
    __device__ __forceinline__ void next(int S, int n_chunks) {
        c += S;
        while (c >= n_chunks) { c -= n_chunks; ++t; }
    }
};

// BM: 0 no B operand, 1 B is Dst_V (loaded once per unit), 2 B is an Edge tensor broadcast per
// head (width H or 1: a per-edge scalar for each lane's VEC features).
template <int MODE, int KE, int GOP, int VEC, int BM>
__global__ void __launch_bounds__(UG_SVG_WARPS * 32) k_svg(const __grid_constant__ CUtensorMap tmA, GraphArgs g,
                                                           OpArgs op, const int4 *__restrict__ chunks, int n_chunks,
                                                           int n_tiles, float *__restrict__ scratch, int64_t sld) {
    constexpr int TW = 32 * VEC;                  // columns per unit (one warp)
    constexpr int R = SVG_R;
    constexpr int D = SvgDepth<VEC>::D;
    constexpr uint32_t STAGE = R * TW + 32;       // floats per stage: R rows + edge weights (128-B aligned)
    extern __shared__ __align__(128) float svg_smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float *ring = svg_smem + (size_t)warp * D * STAGE;
    uint64_t *bars = reinterpret_cast<uint64_t *>(svg_smem + (size_t)UG_SVG_WARPS * D * STAGE) + warp * D;
    const uint32_t ring_s = smem_u32(ring), bar_s = smem_u32(bars);
    if constexpr (MODE == 0) {
        if (lane == 0) {
            for (int i = 0; i < D; ++i) mbar_init(bar_s + 8 * i, 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncwarp();
    }
    const int S = gridDim.x * UG_SVG_WARPS;
    const int w0 = blockIdx.x * UG_SVG_WARPS + warp;
    const uint64_t keep = l2_policy_evict_last();     // the column slab of X being swept
    const uint64_t stream = l2_policy_evict_first();  // col_idx, edge weights, outputs
    const uint32_t ldb = (uint32_t)op.B.ld, lda = (uint32_t)op.A.ld;
    const bool wscalar = BM == 2 && op.B.div == op.F;  // one weight per edge: staged with the rows

    // ---------------------------------------------------------------- issue side
    SvgCursor ic;
    ic.init(w0, n_chunks);
    int ik = 0, ik1 = 0;
    // advance to the next unit with edges (issue side); false when the warp's units are exhausted
    auto issue_unit = [&](bool first) {
        if (!first) ic.next(S, n_chunks);
        while (ic.t < n_tiles) {
            const int4 ch = chunks[ic.c];
            if (ch.z > ch.y) { ik = ch.y; ik1 = ch.z; return; }
            ic.next(S, n_chunks);
        }
    };
    issue_unit(true);
    int nx[R];                  // the next stage's R source ids (uniform loads, L1)
    auto load_ids = [&]() {
        if (ic.t >= n_tiles) return;
        const int last = ik1 - 1;
#pragma unroll
        for (int r = 0; r < R; ++r) nx[r] = ldg_i32_hint(g.col + min(ik + r, last), stream);
    };
    load_ids();
    uint32_t ji = 0;            // stages issued
    auto issue = [&]() {
        if (ic.t < n_tiles) {
            const uint32_t s = ji % D;
            const uint32_t dst = ring_s + s * STAGE * 4;
            const int c0 = ic.t * TW;
            if constexpr (MODE == 0) {
                if (lane == 0) {
                    mbar_expect_tx(bar_s + 8 * s, R * TW * 4);
                    tma_gather4(dst, &tmA, bar_s + 8 * s, c0, nx[0], nx[1], nx[2], nx[3], keep);
                    tma_gather4(dst + 4 * TW * 4, &tmA, bar_s + 8 * s, c0, nx[4], nx[5], nx[6], nx[7], keep);
                }
            } else {
                const int f = c0 + lane * VEC;
                const int nb = max(0, min(VEC, op.F - f)) * 4;      // bytes of this lane's chunk in the row
                const float *base = op.A.p + (nb ? f : 0);
#pragma unroll
                for (int r = 0; r < R; ++r)
                    cp_async_vec<VEC>(dst + (r * TW + lane * VEC) * 4, base + (uint32_t)nx[r] * lda, nb, keep);
            }
            if (wscalar && lane < R) {
                const int e = min(ik + lane, ik1 - 1);
                asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst + (R * TW + lane) * 4),
                             "l"(op.B.p + (uint32_t)e * ldb) : "memory");
            }
            ++ji;
            ik += R;
            if (ik >= ik1) issue_unit(false);
            load_ids();
        }
        cp_async_commit();      // (possibly empty) group: keeps wait_group's count per stage
    };
#pragma unroll 1
    for (int i = 0; i < D; ++i) issue();

    // ---------------------------------------------------------------- consume side (all lanes)
    SvgCursor cc;
    cc.init(w0, n_chunks);
    int ck = 0, ck1 = 0, cv = 0, cslot = -1, cf = 0;
    uint32_t colb = 0;          // BM 2: this lane's column of the per-head Edge operand
    float acc[VEC], bconst[VEC];
    auto finish_unit = [&]() {
        if (cf >= op.W) return;
        if (cslot < 0) {
            const int64_t deg = GOP == UG_GATHER_SUM ? 1 : (int64_t)g.row_ptr[cv + 1] - g.row_ptr[cv];
            float out[VEC];
#pragma unroll
            for (int i = 0; i < VEC; ++i) out[i] = g_finalize<GOP>(acc[i], deg);
            float *cp = op.C + (int64_t)cv * op.c_ld + cf;
            if (cf + VEC <= op.W && op.c_vec >= VEC) st_vec_hint<VEC>(cp, out, stream);
            else st_out<VEC>(cp, out, op.W - cf, op.c_vec);
        } else {
            st_vec_hint<VEC>(scratch + (int64_t)cslot * sld + cf, acc, stream);
        }
    };
    // advance to the next unit with edges; empty units (zero in-degree rows) are finished here
    auto cons_unit = [&](bool first) {
        if (!first) cc.next(S, n_chunks);
        while (cc.t < n_tiles) {
            const int4 ch = chunks[cc.c];
            cv = ch.x; ck = ch.y; ck1 = ch.z; cslot = ch.w;
            cf = cc.t * TW + lane * VEC;
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[i] = g_init<GOP>();
            if constexpr (BM == 2) colb = (uint32_t)op_col(op.B, min(cf, op.F - 1));
            if constexpr (BM == 1) {
                // scalar loads: B's rows need not be aligned to the kernel's vector width
                const float *bp = op.B.p + (int64_t)cv * op.B.ld;
#pragma unroll
                for (int i = 0; i < VEC; ++i)
                    bconst[i] = cf + i < op.W ? __ldg(bp + op_col(op.B, cf + i)) : 1.0f;
            }
            if (ck1 > ck) return;
            finish_unit();
            cc.next(S, n_chunks);
        }
    };
    cons_unit(true);
    uint32_t jc = 0;
#pragma unroll 1
    while (cc.t < n_tiles) {
        const int nv = min(R, ck1 - ck);
        float b[R];
        if constexpr (BM == 2) {
            if (!wscalar) {     // per-head weights: this lane's head, per edge
#pragma unroll
                for (int r = 0; r < R; ++r) b[r] = r < nv ? __ldg(op.B.p + ((uint32_t)(ck + r) * ldb + colb)) : 0.0f;
            }
        }
        const uint32_t s = jc % D;
        if constexpr (MODE == 0) mbar_wait(bar_s + 8 * s, (jc / D) & 1);
        cp_async_wait<D - 1>();
        const float *st = ring + s * STAGE;
        if constexpr (BM == 2) {
            if (wscalar) {
                __syncwarp();   // lanes 0..R-1 copied the weights
                const float4 w0v = *reinterpret_cast<const float4 *>(st + R * TW);
                const float4 w1v = *reinterpret_cast<const float4 *>(st + R * TW + 4);
                b[0] = w0v.x; b[1] = w0v.y; b[2] = w0v.z; b[3] = w0v.w;
                b[4] = w1v.x; b[5] = w1v.y; b[6] = w1v.z; b[7] = w1v.w;
            }
        }
        st += lane * VEC;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            if (r < nv) {
                float x[VEC];
                lds_vec<VEC>(st + r * TW, x);
#pragma unroll
                for (int i = 0; i < VEC; ++i) {
                    float m = x[i];
                    if constexpr (BM == 1) m = edge_fn<KE>(x[i], bconst[i]);
                    else if constexpr (BM == 2) m = edge_fn<KE>(x[i], b[r]);
                    acc[i] = g_combine<GOP>(acc[i], m);
                }
            }
        }
        __syncwarp();          // every lane has read stage s: it may be refilled
        issue();
        ++jc;
        ck += R;
        if (ck >= ck1) {
            finish_unit();
            cons_unit(false);
        }
    }
    cp_async_wait<0>();
}

}  // namespace ug
