// k_gat.cu -- the GAT attention chain as ONE traversal.
//
// PAPER.md:224 describes GAT's graph operators: a message creation el_u + er_v that yields the
// edge scores, then an aggregation-sum that multiplies each source feature by its edge weight.
// Between them GAT applies LeakyReLU and an edge softmax over each destination's in-edges,
// which under the unified abstraction costs four more operators (copy_e_max, e_sub_v,
// copy_e_sum, e_div_v) plus two elementwise passes: six launches and five [E][H] round
// trips through HBM.  Here one owner-computes traversal per destination row does it all:
//
//   one pass, online softmax: s(e,h) = LeakyReLU(el[u][h] + er[v][h]) (never stored);
//       m = running max, den = sum exp(s - m), acc(f) = sum exp(s - m) z[u][f], both rescaled
//       by exp(m_old - m_new) when the max grows (once per group of U edges)
//   out[v][f] = acc(f) / den(h(f))                      (zero in-degree -> 0, R7)
//   (only if attn != NULL) a second walk writes attn[e][h] = exp(s - m) / den
//
// The walk reads 4 B of el per edge and head (an L2-resident [V][H] table) next to the
// u_mul_e_sum gather of z.  Layout (the SV plan of k_split.cu): rows are cut into chunks of at
// most G in-edges; L lanes (VEC features each) cover a column tile of L*VEC features and one
// such slice walks one chunk, S = 32 / L slices per warp, tile-major unit order, U row
// gathers in flight per lane with the next group's column indices prefetched.  A chunk of a
// split row (a hub: degree skew) publishes its (max, den, acc) state; the
// slice that completes the row's last chunk (arrival counter) merges the states in chunk order
// and finalises the row.  Deterministic, one launch, no atomics on the data.
#include "k_dispatch.cuh"

namespace ug {

__device__ __forceinline__ float lrelu(float x, float slope) { return x >= 0.0f ? x : __fmul_rn(slope, x); }

// Scores are carried in the log2 domain, t = s * log2(e), so every exponential is one
// ex2.approx (rel. error ~2^-22): exp(s - m) = exp2(t - t_max).  The extra rounding of the
// scaling perturbs exp(s - m) by ~|s - m| * 2^-24 relative -- far inside the 1e-5 bound.
#define UG_LOG2E 1.4426950408889634f
__device__ __forceinline__ float score2(float el, float er, float slope) {
    return __fmul_rn(lrelu(__fadd_rn(el, er), slope), UG_LOG2E);
}
__device__ __forceinline__ float ex2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// Online-softmax state of one edge slice: running max m, den = sum exp(s - m) and
// acc[i] = sum exp(s - m) z[u][f + i].
template <int VEC>
struct SoftState {
    float m, den, acc[VEC];
    __device__ __forceinline__ void init() {
        m = -CUDART_INF_F;
        den = 0.0f;
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = 0.0f;
    }
    // merge another state (associative up to rounding): rescale both to the larger max
    __device__ __forceinline__ void merge(float m2, float d2, const float (&a2)[VEC]) {
        const float M = fmaxf(m, m2);
        if (M == -CUDART_INF_F) return;
        const float c1 = ex2(__fsub_rn(m, M)), c2 = ex2(__fsub_rn(m2, M));
        den = fmaf(den, c1, d2 * c2);
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = fmaf(acc[i], c1, a2[i] * c2);
        m = M;
    }
};

// One pass over a chunk's edges k0 .. k1 (contiguous CSR positions): U row gathers in flight
// per lane, the next group's column indices prefetched while the current group computes, and
// the running max updated once per group of U edges (one rescale per group).
// O32: el and z rows addressable with 32-bit element offsets (V_src * ld < 2^32, checked on the
// host): one IMAD + IMAD.WIDE per gather instead of a 64-bit multiply and LEA pair
template <int VEC, int U, bool O32 = false>
__device__ __forceinline__ void gat_walk(const GraphArgs &g, const GatArgs &a, int k0, int k1, int h, int f,
                                         bool active, float erv, SoftState<VEC> &st) {
    // padding slots read row 0 (cache-hot) and are masked by t = -inf: no branches
    const float *zb = a.z + (active ? f : 0);
    const float *eb = a.el + h;
#ifndef UG_GAT_HINTS
#define UG_GAT_HINTS 0   // L2 evict hints on the walk's loads: +24 registers, r2aj/r2ak: slower at every budget
#endif
#if UG_GAT_HINTS
    const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
#define UG_GAT_COL(k) ldg_i32_hint(g.col + (k), stream)
#else
#define UG_GAT_COL(k) __ldg(g.col + (k))
#endif
    int32_t nxt[U];
#pragma unroll
    for (int q = 0; q < U; ++q) nxt[q] = k0 + q < k1 ? UG_GAT_COL(k0 + q) : -1;
    for (int k = k0; k < k1; k += U) {
        int32_t cur[U];
#pragma unroll
        for (int q = 0; q < U; ++q) {
            cur[q] = nxt[q];
            nxt[q] = k + U + q < k1 ? UG_GAT_COL(k + U + q) : -1;
        }
        float t[U], zr[U][VEC];
#pragma unroll
        for (int q = 0; q < U; ++q) {
            const uint32_t u = cur[q] < 0 ? 0u : (uint32_t)cur[q];
#if UG_GAT_HINTS
            float tt[1];
            ldg_vec_hint<1>(eb + (int64_t)u * a.ld_el, tt, keep);
            t[q] = tt[0];
            ldg_vec_hint<VEC>(zb + (int64_t)u * a.ld_z, zr[q], keep);
#else
            if constexpr (O32) {
                t[q] = __ldg(a.el + (u * (uint32_t)a.ld_el + (uint32_t)h));
                ldg_vec<VEC>(a.z + (u * (uint32_t)a.ld_z + (uint32_t)(active ? f : 0)), zr[q]);
            } else {
                t[q] = __ldg(eb + (int64_t)u * a.ld_el);
                ldg_vec<VEC>(zb + (int64_t)u * a.ld_z, zr[q]);
            }
#endif
        }
#undef UG_GAT_COL
        float mn = st.m;
#pragma unroll
        for (int q = 0; q < U; ++q) {
            t[q] = cur[q] < 0 ? -CUDART_INF_F : score2(t[q], erv, a.slope);
            mn = fmaxf(mn, t[q]);
        }
        const float c = ex2(__fsub_rn(st.m, mn));     // 0 on the first group (m = -inf)
        st.den *= c;
#pragma unroll
        for (int i = 0; i < VEC; ++i) st.acc[i] *= c;
#pragma unroll
        for (int q = 0; q < U; ++q) {
            const float p = ex2(__fsub_rn(t[q], mn));    // 0 for padding slots (t = -inf)
            st.den += p;
#pragma unroll
            for (int i = 0; i < VEC; ++i) st.acc[i] = fmaf(p, zr[q][i], st.acc[i]);
        }
        st.m = mn;
    }
}

// Attention output of edges k0 + j, k0 + j + nh, ... < k1 of row v: the nh lanes of a head
// split the edges, 4 independent loads in flight per lane.
__device__ __forceinline__ void gat_attn(const GraphArgs &g, const GatArgs &a, int64_t k0, int64_t k1, int h,
                                         float erv, float m, float den, int j, int nh) {
    constexpr int U = 4;
    for (int64_t k = k0 + j; k < k1; k += (int64_t)U * nh) {
        int64_t e[U];
        float t[U];
#pragma unroll
        for (int q = 0; q < U; ++q) {
            const int64_t kk = k + (int64_t)q * nh;
            const int64_t kc = kk < k1 ? kk : k;
            const int64_t u = g.col[kc];
            e[q] = kk < k1 ? (g.eid ? (int64_t)g.eid[kc] : kc) : -1;
            t[q] = __ldg(a.el + u * a.ld_el + h);
        }
#pragma unroll
        for (int q = 0; q < U; ++q)
            if (e[q] >= 0)
                a.attn[e[q] * a.ld_attn + h] = __fdiv_rn(ex2(__fsub_rn(score2(t[q], erv, a.slope), m)), den);
    }
}

template <int VEC>
__device__ __forceinline__ void gat_store(const GatArgs &a, int64_t v, int f, const SoftState<VEC> &st, bool empty) {
    float o[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) o[i] = empty ? 0.0f : __fdiv_rn(st.acc[i], st.den);
    st_vec<VEC>(a.out + v * a.ld_out + f, o);
}

// One slice (L lanes) per (row chunk, column tile), S = 32 / L slices per warp, tile-major
// unit order.  Chunks of rows longer than the chunk size write their (max, den, acc) state to
// scratch; the slice that completes a row's last chunk (per-row arrival counter) merges the
// states in chunk order -- deterministic, one launch, no atomics on the data.
// MB = resident CTAs per SM the register budget is sized for: 6 (40 registers) for float4 slices of
// large graphs, 1 (no cap, 48) otherwise -- r2al: C4 H = 8 F = 128 148.8 -> 128.3 us, C3 H = 4
// F = 64 224 -> 190 us, but C2 14.7 -> 15.7 us, hence by grid size
template <int VEC, int U, bool ATTN, int MB, bool O32>
__global__ void __launch_bounds__(256, MB) k_gat(GraphArgs g, GatArgs a, int L_log2, int n_tiles,
                                             const int4 *__restrict__ chunks, int64_t n_chunks,
                                             const int4 *__restrict__ split, const int32_t *__restrict__ slot_row,
                                             float *sacc, float *sst, int64_t sld, int64_t nfc,
                                             int32_t *counters) {
    const int L = 1 << L_log2;
    const int S = 32 >> L_log2;
    const int lane = threadIdx.x & 31;
    const int slice = lane >> L_log2;
    const int sl = lane & (L - 1);
    // the host guarantees n_chunks * n_tiles < 2^31
    const int unit = ((int)blockIdx.x * (int)(blockDim.x >> 5) + (int)(threadIdx.x >> 5)) * S + slice;
    if (unit >= (int)n_chunks * n_tiles) return;
    const int tile = n_tiles == 1 ? 0 : unit / (int)n_chunks;
    const int c = unit - tile * (int)n_chunks;
    const int4 ch = chunks[c];
    const int64_t v = ch.x;
    const int f = tile * L * VEC + sl * VEC;
    const bool active = f < a.F;
    const int h = active ? (a.D == 1 ? f : f / a.D) : 0;
    const float erv = __ldg(a.er + v * a.ld_er + h);
    SoftState<VEC> st;
    st.init();
    gat_walk<VEC, U, O32>(g, a, ch.y, ch.z, h, f, active, erv, st);
    if (ch.w < 0) {                                   // the row is one chunk: finalise here
        if (active) gat_store<VEC>(a, v, f, st, ch.z == ch.y);
        if constexpr (ATTN) {
            if (active) gat_attn(g, a, ch.y, ch.z, h, erv, st.m, st.den, (f - h * a.D) / VEC, (a.D + VEC - 1) / VEC);
        }
        return;
    }
    // split row: publish this chunk's state, then count arrivals
    const int64_t fc = f / VEC;
    if (active) {
        st_vec<VEC>(sacc + (int64_t)ch.w * sld + f, st.acc);
        sst[((int64_t)ch.w * 2) * nfc + fc] = st.m;
        sst[((int64_t)ch.w * 2 + 1) * nfc + fc] = st.den;
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
    st.init();
    for (int i = 0; i < sp.z; ++i) {
        const int64_t slot = sp.y + i;
        float a2[VEC];
#pragma unroll
        for (int j = 0; j < VEC; ++j) a2[j] = active ? __ldcg(sacc + slot * sld + f + j) : 0.0f;
        const float m2 = active ? __ldcg(sst + (slot * 2) * nfc + fc) : -CUDART_INF_F;
        const float d2 = active ? __ldcg(sst + (slot * 2 + 1) * nfc + fc) : 0.0f;
        st.merge(m2, d2, a2);
    }
    if (active) gat_store<VEC>(a, v, f, st, false);
    if constexpr (ATTN) {
        if (active) {
            const int64_t r0 = (int64_t)g.row_ptr[v] - g.rp_base, r1 = (int64_t)g.row_ptr[v + 1] - g.rp_base;
            gat_attn(g, a, r0, r1, h, erv, st.m, st.den, (f - h * a.D) / VEC, (a.D + VEC - 1) / VEC);
        }
    }
}

#ifndef UG_GAT_O32
#define UG_GAT_O32 1
#endif
cudaError_t launch_gat(const GraphArgs &g, const GatArgs &a, int vec, int L, const SplitPlan &plan,
                       const int32_t *slot_row, float *sacc, float *sst, int64_t sld, int64_t nfc,
                       int32_t *counters, cudaStream_t s) {
    const int n_tiles = (int)cdiv(a.F, (int64_t)L * vec);
    constexpr int block = 256;
    const int S = 32 / L;
    const int64_t grid = cdiv(plan.n_chunks * n_tiles, (int64_t)(block / 32) * S);
    if (grid == 0) return cudaSuccess;
    const int L_log2 = ilog2(L);
    const int4 *chunks = reinterpret_cast<const int4 *>(plan.d_chunk);
    const int4 *split = reinterpret_cast<const int4 *>(plan.d_split);
    const bool big = grid >= 4096;
    const bool o32 = UG_GAT_O32 && (uint64_t)g.V_src * (uint64_t)a.ld_z < (1ull << 32) &&
                     (uint64_t)g.V_src * (uint64_t)a.ld_el < (1ull << 32);
#define UG_GAT_LAUNCH(ATTN_, MB_)                                                                               \
    do {                                                                                                        \
        if (o32)                                                                                                \
            k_gat<VEC, (VEC == 4 ? 4 : 8), ATTN_, MB_, true><<<(unsigned)grid, block, 0, s>>>(                 \
                g, a, L_log2, n_tiles, chunks, plan.n_chunks, split, slot_row, sacc, sst, sld, nfc, counters);  \
        else                                                                                                    \
            k_gat<VEC, (VEC == 4 ? 4 : 8), ATTN_, MB_, false><<<(unsigned)grid, block, 0, s>>>(                \
                g, a, L_log2, n_tiles, chunks, plan.n_chunks, split, slot_row, sacc, sst, sld, nfc, counters);  \
    } while (0)
    // 32-bit offsets only in the uncapped instance: at 6 CTAs / SM they spill 56 B and lose 6-12 %
    // (C4 H = 8 F = 128 127.3 -> 137.4 us), uncapped they win (C2 H = 8 14.67 -> 13.66 us;
    // profiles/r2/ab_r2gat.jsonl)
    const bool o32_small = o32;
    UG_DISPATCH_VEC(vec, VEC, {
        if constexpr (VEC == 4) {
            const bool o32 = o32_small && !big;
            if (a.attn) { if (big) UG_GAT_LAUNCH(true, 6); else UG_GAT_LAUNCH(true, 1); }
            else { if (big) UG_GAT_LAUNCH(false, 6); else UG_GAT_LAUNCH(false, 1); }
        } else {
            if (a.attn) UG_GAT_LAUNCH(true, 1);
            else UG_GAT_LAUNCH(false, 1);
        }
    });
#undef UG_GAT_LAUNCH
    return cudaGetLastError();
}

}  // namespace ug
