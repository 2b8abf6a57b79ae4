// k_dotattn.cu -- the dot-product attention chain as ONE traversal (ug_dot_attention, SURVEY 8(f)
// f3: FusedMM-style SDDMM + edge softmax + SpMM, built from the paper's operators
// u_dot_v -> softmax -> u_mul_e_sum, PAPER.md:224 / Table 2):
//     s_e = scale * <q[v]_h, k[u]_h>,   a_e = softmax over v's in-edges,   out[v]_h = sum_e a_e val[u]_h.
//
// Work unit = (head h, SV chunk of <= G in-edges of row v), one warp; lanes own VEC-wide feature
// chunks of the head (NJK chunks of the Dk key features, NJV of the Dv value features).  Per
// batch of 8 in-edges: the lanes' FMA partials of the 8 scores are reduced by the transposed
// butterfly of k_dott (9 shuffles), the 8 scores are broadcast (8 shuffles), and an online
// softmax (running max, one rescale per batch, scores in the log2 domain -> ex2.approx) folds
// the 8 value rows into the running sum.  The score and value rows of an edge are gathered once
// and never written back: the E x H score and attention tensors of the unfused chain are not
// materialised (attn is optional).  Owned rows finish in registers; split rows (hubs) store
// (max, denominator, partial sum) per chunk and k_dotattn_fix merges them in chunk order
// (deterministic).  With attn requested, the raw log2 scores are stored during the traversal and
// k_dotattn_attn normalises them with each row's final (max, denominator).
#include <cstdlib>

#include "k_split.cuh"

namespace ug {

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// Sum over the 32 lanes of v[(lane >> 2) & 7] (transposed butterfly, fixed order; as k_dott).
__device__ __forceinline__ float da_sum8(float (&v)[8], int lane) {
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



// column-index prefetch (the next batch's col_idx loads overlap this batch's row gathers), per
// kernel form -- r2an: packed heads C3 H = 4 D = 16 289 -> 269 us, C4 H = 8 199 -> 190 us; one warp
// per head C4 H = 1 D = 128 203 -> 209 us, so off there
#ifndef UG_DAH_PF
#define UG_DAH_PF 1
#endif
#ifndef UG_DAW_PF
#define UG_DAW_PF 0
#endif

#ifndef UG_DAW_MINB
#define UG_DAW_MINB (VEC == 4 && NJK + NJV > 4 ? 3 : 4)   // resident CTAs per SM (r2ae: 4 beats 3 by 9-11 %)
#endif

template <int VEC, int NJK, int NJV>
__global__ void __launch_bounds__(256, UG_DAW_MINB) k_dotattn(GraphArgs g, DotAttnArgs a, const int4 *__restrict__ chunks,
                                                    int n_chunks, float *__restrict__ scratch, int64_t sld) {
    const int lane = threadIdx.x & 31;
    const int u = (int)(blockIdx.x * 8 + (threadIdx.x >> 5));
    const int h = u / n_chunks;
    if (h >= a.H) return;
    const int4 ch = chunks[u - h * n_chunks];
    const int64_t v = ch.x;
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
    // this lane's key / value feature chunks: j-th at lane * VEC + j * 32 * VEC inside the head
    float q[NJK][VEC];
#pragma unroll
    for (int j = 0; j < NJK; ++j) {
        const int f = lane * VEC + j * 32 * VEC;
        if (f < a.Dk) {
            ldg_vec<VEC>(a.q + v * a.ld_q + h * a.Dk + f, q[j]);
#pragma unroll
            for (int i = 0; i < VEC; ++i) q[j][i] *= a.scale_log2;     // scores in the log2 domain
        } else {
#pragma unroll
            for (int i = 0; i < VEC; ++i) q[j][i] = 0.0f;
        }
    }
    const float *kb = a.k + h * a.Dk + lane * VEC;
    const float *vb = a.val + h * a.Dv + lane * VEC;
    const uint32_t ldk = (uint32_t)a.ld_k, ldv = (uint32_t)a.ld_val;
    float m = -CUDART_INF_F, den = 0.0f;
    float acc[NJV][VEC];
#pragma unroll
    for (int j = 0; j < NJV; ++j)
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[j][i] = 0.0f;
    const int k1 = ch.z;
    const int last = k1 - 1;
    // the next batch's column indices are loaded while this batch is gathered (UG_DAW_PF)
    uint32_t s_pf[8];
    if (UG_DAW_PF && ch.y < k1) {
#pragma unroll
        for (int i = 0; i < 8; ++i) s_pf[i] = (uint32_t)ldg_i32_hint(g.col + min(ch.y + i, last), stream);
    }
    for (int k0 = ch.y; k0 < k1; k0 += 8) {
        uint32_t s[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (UG_DAW_PF) {
                s[i] = s_pf[i];
                s_pf[i] = (uint32_t)ldg_i32_hint(g.col + min(k0 + 8 + i, last), stream);
            } else {
                s[i] = (uint32_t)ldg_i32_hint(g.col + min(k0 + i, last), stream);
            }
        }
        float p[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            float t = 0.0f;
#pragma unroll
            for (int j = 0; j < NJK; ++j) {
                if (lane * VEC + j * 32 * VEC < a.Dk) {
                    float x[VEC];
                    ldg_vec_hint<VEC>(kb + s[i] * ldk + j * 32 * VEC, x, keep);
#pragma unroll
                    for (int c = 0; c < VEC; ++c) t = __fmaf_rn(x[c], q[j][c], t);
                }
            }
            p[i] = t;
        }
        const float r = da_sum8(p, lane);                   // log2 score of edge k0 + (lane >> 2)
        const int me = lane >> 2;
        if (a.attn && (lane & 3) == 0 && k0 + me < k1) {
            const int64_t e = g.eid ? (int64_t)g.eid[k0 + me] : (int64_t)(k0 + me);
            a.attn[e * a.ld_attn + h] = r;                  // normalised by k_dotattn_attn
        }
        float sc[8];
        float mb = -CUDART_INF_F;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            sc[i] = __shfl_sync(0xffffffffu, r, 4 * i);
            if (k0 + i >= k1) sc[i] = -CUDART_INF_F;
            mb = fmaxf(mb, sc[i]);
        }
        const float mn = fmaxf(m, mb);
        const float corr = fast_exp2(m - mn);               // 0 on the first batch (m = -inf)
        den *= corr;
#pragma unroll
        for (int j = 0; j < NJV; ++j)
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc[j][c] *= corr;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const float pe = fast_exp2(sc[i] - mn);           // 0 for the batch's missing edges
            den += pe;
#pragma unroll
            for (int j = 0; j < NJV; ++j) {
                if (lane * VEC + j * 32 * VEC < a.Dv) {
                    float x[VEC];
                    ldg_vec_hint<VEC>(vb + s[i] * ldv + j * 32 * VEC, x, keep);
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc[j][c] = __fmaf_rn(pe, x[c], acc[j][c]);
                }
            }
        }
        m = mn;
    }
    if (ch.w < 0) {
        // an owned row: its whole in-edge list (zero in-degree -> 0, R7)
#pragma unroll
        for (int j = 0; j < NJV; ++j) {
            const int f = lane * VEC + j * 32 * VEC;
            if (f < a.Dv) {
                float o[VEC];
#pragma unroll
                for (int c = 0; c < VEC; ++c) o[c] = den > 0.0f ? __fdiv_rn(acc[j][c], den) : 0.0f;
                st_vec<VEC>(a.out + v * a.ld_out + h * a.Dv + f, o);
            }
        }
        if (a.mden && lane == 0) {
            a.mden[(v * a.H + h) * 2] = m;
            a.mden[(v * a.H + h) * 2 + 1] = den;
        }
    } else {
        float *sp = scratch + ((int64_t)ch.w * a.H + h) * sld;
        if (lane == 0) { sp[0] = m; sp[1] = den; }
#pragma unroll
        for (int j = 0; j < NJV; ++j) {
            const int f = lane * VEC + j * 32 * VEC;
            if (f < a.Dv) st_vec<VEC>(sp + 4 + f, acc[j]);
        }
    }
}

// Packed heads (Dk = Dv = D, w = D / VEC a power of two <= 16): one unit = one SV chunk with a
// group of 32 / w heads (all H when H * w <= 32), L = min(32, pow2(H * w)) lanes, lane = h * w + i
// of the group owning features h*D + i*VEC; units are group-major (the groups' K / V column
// slabs are walked one after another, as the SV column tiles).  A
// head's score is reduced over its w lanes by a log2(w)-step xor butterfly that leaves it in all
// of them, so every lane runs the online softmax of its own head -- no idle lanes for small
// heads (C2: D = 8, w = 2) and no broadcast.  UE in-edges per step.
#ifndef UG_DAH_MINB
#define UG_DAH_MINB 4   // resident CTAs per SM the register budget is sized for
#endif

// float / float2 slices fit 5 CTAs / SM spill-free (48 registers); float4 slices spill there
#ifndef UG_DAH_MINB_NARROW
#define UG_DAH_MINB_NARROW UG_DAH_MINB
#endif
template <int VEC, int UE>
__global__ void __launch_bounds__(256, VEC <= 2 ? UG_DAH_MINB_NARROW : UG_DAH_MINB) k_dotattn_heads(GraphArgs g, DotAttnArgs a, const int4 *__restrict__ chunks,
                                                       int n_chunks, int n_units, int L_log2, int w_log2,
                                                       float *__restrict__ scratch, int64_t sld) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int L = 1 << L_log2, w = 1 << w_log2;
    const int lane = (int)(t & (L - 1));
    const int64_t ut = t >> L_log2;
    if (ut >= n_units) return;                    // whole units: a unit's lanes leave together
    const int grp = n_units == n_chunks ? 0 : (int)ut / n_chunks;   // head group (0: all heads fit one unit)
    const int u = (int)ut - grp * n_chunks;
    const int wl = threadIdx.x & 31;
    const unsigned umask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (wl & ~(L - 1)));
    const int h = ((grp << L_log2) + lane) >> w_log2, i = lane & (w - 1);
    const bool active = h < a.H;
    const int hh = active ? h : 0;
    const int f = hh * a.Dk + i * VEC;            // Dk == Dv
    const int4 ch = chunks[u];
    const int64_t v = ch.x;
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
    float q[VEC];
    ldg_vec<VEC>(a.q + v * a.ld_q + f, q);
#pragma unroll
    for (int c = 0; c < VEC; ++c) q[c] = active ? q[c] * a.scale_log2 : 0.0f;
    const float *kb = a.k + f, *vb = a.val + f;
    const uint32_t ldk = (uint32_t)a.ld_k, ldv = (uint32_t)a.ld_val;
    float m = -CUDART_INF_F, den = 0.0f, acc[VEC];
#pragma unroll
    for (int c = 0; c < VEC; ++c) acc[c] = 0.0f;
    const int k1 = ch.z;
    const int last = k1 - 1;
    uint32_t s_pf[UE];
    if (UG_DAH_PF && ch.y < k1) {
#pragma unroll
        for (int e = 0; e < UE; ++e) s_pf[e] = (uint32_t)ldg_i32_hint(g.col + min(ch.y + e, last), stream);
    }
    for (int k0 = ch.y; k0 < k1; k0 += UE) {
        uint32_t sidx[UE];
#pragma unroll
        for (int e = 0; e < UE; ++e) {
            if (UG_DAH_PF) {
                sidx[e] = s_pf[e];
                s_pf[e] = (uint32_t)ldg_i32_hint(g.col + min(k0 + UE + e, last), stream);
            } else {
                sidx[e] = (uint32_t)ldg_i32_hint(g.col + min(k0 + e, last), stream);
            }
        }
        float kx[UE][VEC], vx[UE][VEC];
#pragma unroll
        for (int e = 0; e < UE; ++e) {
            ldg_vec_hint<VEC>(kb + sidx[e] * ldk, kx[e], keep);
            ldg_vec_hint<VEC>(vb + sidx[e] * ldv, vx[e], keep);
        }
        float sc[UE];
        float mb = -CUDART_INF_F;
#pragma unroll
        for (int e = 0; e < UE; ++e) {
            float p = 0.0f;
#pragma unroll
            for (int c = 0; c < VEC; ++c) p = __fmaf_rn(kx[e][c], q[c], p);
            for (int off = w >> 1; off > 0; off >>= 1) p += __shfl_xor_sync(umask, p, off);
            sc[e] = k0 + e < k1 ? p : -CUDART_INF_F;
            if (a.attn && active && i == 0 && k0 + e < k1) {
                const int64_t eid = g.eid ? (int64_t)g.eid[k0 + e] : (int64_t)(k0 + e);
                a.attn[eid * a.ld_attn + h] = p;          // log2 score, normalised by k_dotattn_attn
            }
            mb = fmaxf(mb, sc[e]);
        }
        const float mn = fmaxf(m, mb);
        const float corr = fast_exp2(m - mn);
        den *= corr;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc[c] *= corr;
#pragma unroll
        for (int e = 0; e < UE; ++e) {
            const float pe = fast_exp2(sc[e] - mn);
            den += pe;
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc[c] = __fmaf_rn(pe, vx[e][c], acc[c]);
        }
        m = mn;
    }
    if (!active) return;
    if (ch.w < 0) {
        float o[VEC];
#pragma unroll
        for (int c = 0; c < VEC; ++c) o[c] = den > 0.0f ? __fdiv_rn(acc[c], den) : 0.0f;
        st_vec<VEC>(a.out + v * a.ld_out + f, o);
        if (a.mden && i == 0) {
            a.mden[(v * a.H + h) * 2] = m;
            a.mden[(v * a.H + h) * 2 + 1] = den;
        }
    } else {
        float *sp = scratch + ((int64_t)ch.w * a.H + h) * sld;
        if (i == 0) { sp[0] = m; sp[1] = den; }
        st_vec<VEC>(sp + 4 + i * VEC, acc);
    }
}

// Split rows: merge the chunks' (max, denominator, partial sum) in chunk order.
__global__ void k_dotattn_fix(DotAttnArgs a, const int4 *__restrict__ split, int64_t n_split,
                              const float *__restrict__ scratch, int64_t sld) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t per = (int64_t)a.H * (a.Dv + 1);     // (head, feature) pairs + one (max, den) slot per head
    if (t >= n_split * per) return;
    const int64_t r = t / per;
    const int rem = (int)(t - r * per);
    const int h = rem / (a.Dv + 1), f = rem - h * (a.Dv + 1);
    const int4 sp = split[r];
    float M = -CUDART_INF_F;
    for (int c = 0; c < sp.z; ++c) M = fmaxf(M, scratch[((int64_t)(sp.y + c) * a.H + h) * sld]);
    float den = 0.0f, acc = 0.0f;
    for (int c = 0; c < sp.z; ++c) {
        const float *p = scratch + ((int64_t)(sp.y + c) * a.H + h) * sld;
        const float w = fast_exp2(p[0] - M);
        den = __fmaf_rn(p[1], w, den);
        if (f < a.Dv) acc = __fmaf_rn(p[4 + f], w, acc);
    }
    const int64_t v = sp.x;
    if (f < a.Dv) a.out[v * a.ld_out + h * a.Dv + f] = den > 0.0f ? __fdiv_rn(acc, den) : 0.0f;
    else if (a.mden) {
        a.mden[(v * a.H + h) * 2] = M;
        a.mden[(v * a.H + h) * 2 + 1] = den;
    }
}

// attn[e][h] = 2^(s_e - max_v) / den_v over CSR positions (row of position k: dst[k] - r0).
__global__ void k_dotattn_attn(GraphArgs g, DotAttnArgs a) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= g.E * a.H) return;
    const int64_t k = t / a.H;
    const int h = (int)(t - k * a.H);
    const int64_t v = (int64_t)g.dst[k] - g.r0;
    const int64_t e = g.eid ? (int64_t)g.eid[k] : k;
    float *p = a.attn + e * a.ld_attn + h;
    const float M = a.mden[(v * a.H + h) * 2], den = a.mden[(v * a.H + h) * 2 + 1];
    *p = __fdiv_rn(fast_exp2(*p - M), den);
}

// Widest VEC (4, 2, 1) dividing Dk and Dv with every row aligned; NJ = chunks per lane (<= 4).
int dotattn_vec(const DotAttnArgs &a) {
    for (int v : {4, 2, 1}) {
        const bool ok = a.Dk % v == 0 && a.Dv % v == 0 && a.ld_q % v == 0 && a.ld_k % v == 0 && a.ld_val % v == 0 &&
                        a.ld_out % v == 0 && (uintptr_t)a.q % (4 * v) == 0 && (uintptr_t)a.k % (4 * v) == 0 &&
                        (uintptr_t)a.val % (4 * v) == 0 && (uintptr_t)a.out % (4 * v) == 0;
        if (ok && cdiv(a.Dk, 32 * v) <= 4 && cdiv(a.Dv, 32 * v) <= 4) return v;
    }
    return 0;
}

cudaError_t launch_dotattn_wide(const GraphArgs &g, const DotAttnArgs &a, int vec, int njk, int njv,
                                const SplitPlan &plan, float *scratch, int64_t sld, cudaStream_t s);
cudaError_t launch_dotattn_tail(const GraphArgs &g, const DotAttnArgs &a, const SplitPlan &plan, float *scratch,
                                int64_t sld, cudaStream_t s);

cudaError_t launch_dotattn(const GraphArgs &g, const DotAttnArgs &a, int vec, const SplitPlan &plan,
                           float *scratch, int64_t sld, cudaStream_t s) {
    const int64_t units = plan.n_chunks * (int64_t)a.H;
    if (units == 0) return cudaSuccess;
    cudaError_t err = cudaSuccess;
    const int wl = a.Dk / vec;
    static const bool force_wide = std::getenv("UG_DOTATTN_WIDE") != nullptr;   // A/B switches
    static const int pack_wl = std::getenv("UG_DOTATTN_PACK_WL") ? std::atoi(std::getenv("UG_DOTATTN_PACK_WL")) : 16;
    // packed heads when a head spans <= 16 lanes (<= 4 butterfly steps per edge; r2ag: C4 H = 1,
    // D = 64 152 -> 133 us, H = 2 D = 64 281 -> 234 us at 16 vs 8); wider heads reduce 8 edges at
    // once by the transposed butterfly (C4 H = 1, D = 128: 303 -> 226 us; H = 8: packed 236 us vs
    // 1,288 us; profiles/r2/ab_r2t.log)
    if (!force_wide && a.Dk == a.Dv && a.Dk % vec == 0 && (wl & (wl - 1)) == 0 && wl <= pack_wl) {
        // packed heads: one unit per (head group, chunk) (k_dotattn_heads)
        int L = 1;
        while (L < a.H * wl && L < 32) L <<= 1;
        const int64_t n_units = plan.n_chunks * cdiv((int64_t)a.H * wl, L);
        if (n_units * L >= (1ll << 31)) return cudaErrorInvalidValue;
        const int64_t grid = cdiv(n_units * L, 256);
        const int4 *ch = reinterpret_cast<const int4 *>(plan.d_chunk);
        UG_DISPATCH_VEC(vec, VEC,
            k_dotattn_heads<VEC, 4><<<(unsigned)grid, 256, 0, s>>>(g, a, ch, (int)plan.n_chunks, (int)n_units,
                                                                   ilog2(L), ilog2(wl), scratch, sld));
    } else {
        // one warp per head: the narrowest vector that still gives every lane a chunk (D = 64:
        // float2 x 32 lanes rather than float4 x 16 lanes with half the warp idle)
        int vw = vec;
        while (vw > 1 && (a.Dk < 32 * vw || a.Dv < 32 * vw) && cdiv(a.Dk, 16 * vw) <= 4 && cdiv(a.Dv, 16 * vw) <= 4)
            vw >>= 1;
        err = launch_dotattn_wide(g, a, vw, (int)cdiv(a.Dk, 32 * vw), (int)cdiv(a.Dv, 32 * vw), plan, scratch, sld, s);
    }
    if (err == cudaSuccess) err = cudaGetLastError();
    if (err != cudaSuccess) return err;
    return launch_dotattn_tail(g, a, plan, scratch, sld, s);
}

// one warp per (head, chunk): heads wider than 32 lanes or not a power-of-two number of lanes
cudaError_t launch_dotattn_wide(const GraphArgs &g, const DotAttnArgs &a, int vec, int njk, int njv,
                                const SplitPlan &plan, float *scratch, int64_t sld, cudaStream_t s) {
    const int64_t units = plan.n_chunks * (int64_t)a.H;
    const int64_t grid = cdiv(units, 8);
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const int nc = (int)plan.n_chunks;
#define UG_DA(V_, K_, W_) k_dotattn<V_, K_, W_><<<(unsigned)grid, 256, 0, s>>>(g, a, chunks, nc, scratch, sld)
#define UG_DA_V(V_, K_)                 \
    switch (njv) {                      \
    case 1: UG_DA(V_, K_, 1); break;    \
    case 2: UG_DA(V_, K_, 2); break;    \
    case 3: UG_DA(V_, K_, 3); break;    \
    default: UG_DA(V_, K_, 4); break;   \
    }
#define UG_DA_K(V_)                     \
    switch (njk) {                      \
    case 1: UG_DA_V(V_, 1); break;      \
    case 2: UG_DA_V(V_, 2); break;      \
    case 3: UG_DA_V(V_, 3); break;      \
    default: UG_DA_V(V_, 4); break;     \
    }
    switch (vec) {
    case 4: UG_DA_K(4); break;
    case 2: UG_DA_K(2); break;
    default: UG_DA_K(1); break;
    }
#undef UG_DA_K
#undef UG_DA_V
#undef UG_DA
    return cudaGetLastError();
}

// split-row merge and optional attention normalisation (both kernel forms)
cudaError_t launch_dotattn_tail(const GraphArgs &g, const DotAttnArgs &a, const SplitPlan &plan, float *scratch,
                                int64_t sld, cudaStream_t s) {
    cudaError_t err = cudaSuccess;
    if (plan.n_split_rows > 0) {
        const int64_t n = plan.n_split_rows * (int64_t)a.H * (a.Dv + 1);
        k_dotattn_fix<<<(unsigned)cdiv(n, 256), 256, 0, s>>>(a, reinterpret_cast<const int4 *>(plan.d_split),
                                                           plan.n_split_rows, scratch, sld);
        if ((err = cudaGetLastError()) != cudaSuccess) return err;
    }
    if (a.attn && g.E > 0) {
        k_dotattn_attn<<<(unsigned)cdiv(g.E * (int64_t)a.H, 256), 256, 0, s>>>(g, a);
        err = cudaGetLastError();
    }
    return err;
}

}  // namespace ug
