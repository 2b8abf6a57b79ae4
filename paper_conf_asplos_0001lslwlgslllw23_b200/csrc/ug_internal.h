// ug_internal.h -- runtime <-> kernel interface of libugraph (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <map>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include "ug.h"

namespace ug {

// Operand as the kernels see it (PAPER.md:232 type_idx_dict + head broadcast, R6).
struct Operand {
    const float *p;   // base pointer (already offset for views where needed)
    int32_t type;     // UG_T_*
    int32_t div;      // F / width: 1 = full width, D = per-head broadcast, F = scalar
    int64_t ld;       // row stride (elements)
};

// CSR view as the kernels see it.  Positions k are LOCAL: k in [0, E).
struct GraphArgs {
    const int32_t *row_ptr;  // row_ptr[v] - rp_base = first local position of local row v
    const int32_t *col;      // col[k]  = global src id of local position k
    const int32_t *eid;      // eid[k]  = edge id of position k (NULL = identity)
    const int32_t *dst;      // dst[k]  = GLOBAL dst row of position k (edge-parallel schedules)
    int64_t V;               // local rows
    int64_t E;               // local edges
    int64_t rp_base;         // row_ptr[r0] of a view (0 for a base graph)
    int64_t r0;              // first global row of a view (0 for a base graph)
    int64_t V_src;           // size of the source-vertex id space (Src_V operand rows)
};

struct OpArgs {
    Operand A, B;
    float *C;
    int64_t c_ld;
    int32_t c_type;   // UG_T_DST_V (aggregate) or UG_T_EDGE (message creation)
    int32_t F;        // feature width
    int32_t W;        // message / output width (F, or H for dot)
    int32_t H, D;     // heads, D = F / H
    int32_t c_vec;    // widest aligned vector store into C (may be < the load width under SV)
};

// Normalised edge ops inside the kernels (copy_rhs is rewritten as copy_lhs on B).
enum KEdge { K_COPY = 0, K_ADD = 1, K_SUB = 2, K_MUL = 3, K_DIV = 4 };

struct LaunchCfg {
    int strategy;     // UG_TV ... UG_SV
    int L;            // lanes per unit (power of two)
    int G;            // units per lane group (or chunk size for SV)
    int block;        // CTA size
    int ftile;        // column tile width (multiple of vec), 0 = whole width
    int vec;          // 1, 2, 4
    bool pack;        // UG_SCHED_PACK: stage A into 128-byte-aligned rows first (SV only)
    bool edgelanes;   // WV aggregation with lanes over a row's in-edges (k_vertex_el)
    bool dott;        // SV dot with column tiles (k_dott): any head width, tile-major partials
    int staged;       // SV aggregation with shared-memory row staging (k_svg): 0 off,
                      // 1 UG_SCHED_TMA (TMA gather4), 2 UG_SCHED_ASYNC (cp.async / LDGSTS)
};

// Split-row plan for UG_SV (built once per (graph, chunk size), cached on the graph).
struct SplitPlan {
    int64_t n_chunks = 0;       // work units per column tile
    int64_t n_split_rows = 0;   // rows cut into >1 chunk
    int64_t n_split_chunks = 0; // chunks belonging to split rows (scratch slots)
    int32_t *d_chunk = nullptr;   // [n_chunks] x 4 int32: row, k0, k1, scratch slot (-1 = owner)
    int32_t *d_split = nullptr;   // [n_split_rows] x 4 int32: row, first slot, n slots, 0
    int32_t *d_slot_row = nullptr; // [n_split_chunks]: index into d_split of the slot's row
};

// Kernel launchers (kernels/*.cu).  All return cudaGetLastError().
cudaError_t launch_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                          const LaunchCfg &c, cudaStream_t s);
cudaError_t launch_msg_el(int kedge, const GraphArgs &g, const OpArgs &op, const SplitPlan &plan, cudaStream_t s);
cudaError_t launch_vertex_el(int kedge, int gather, const GraphArgs &g, const OpArgs &op, const LaunchCfg &c,
                             cudaStream_t s);
cudaError_t launch_edge(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                        const LaunchCfg &c, cudaStream_t s);
cudaError_t launch_block_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                                const LaunchCfg &c, cudaStream_t s);
cudaError_t launch_split_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                                const LaunchCfg &c, const SplitPlan &plan, float *scratch,
                                cudaStream_t s, cudaEvent_t ev_begin = nullptr, cudaEvent_t ev_end = nullptr,
                                int32_t *counters = nullptr);
// SV with shared-memory row staging (k_svg.cu): mode 0 TMA gather4, 1 cp.async; bm = B addressing
// mode (0 none, 1 Dst_V, 2 Edge broadcast).
bool svg_supported(const OpArgs &op, int vec, int mode);
cudaError_t launch_split_staged(int mode, int kedge, int gather, const GraphArgs &g, const OpArgs &op, int vec,
                                int bm, const SplitPlan &plan, float *scratch, cudaStream_t s, cudaEvent_t ev_begin,
                                cudaEvent_t ev_end);
// dot between a Src_V and a Dst_V operand for any head width (k_dott.cu)
int dott_tiles(const OpArgs &op, int vec);
cudaError_t launch_dott(const GraphArgs &g, const OpArgs &op, bool a_is_src, int vec, const SplitPlan &plan,
                        float *C, int64_t c_ld, float *part, cudaStream_t s, cudaEvent_t ev_begin,
                        cudaEvent_t ev_end);
cudaError_t launch_dot(bool vertex_units, int gather, const GraphArgs &g, const OpArgs &op,
                       const LaunchCfg &c, cudaStream_t s);
// dot between a Src_V and a Dst_V operand under SV (k_dotsv.cu): Dst_V row hoisted per unit.
int dotsv_nj(const OpArgs &op, int vec, int *L, int *w);
cudaError_t launch_dotsv(int gather, const GraphArgs &g, const OpArgs &op, bool a_is_src, int vec, int block,
                         const SplitPlan &plan, float *scratch, cudaStream_t s, cudaEvent_t ev_begin,
                         cudaEvent_t ev_end);
cudaError_t launch_init(int gather, const OpArgs &op, int64_t rows, cudaStream_t s);
cudaError_t launch_epilogue(int gather, const GraphArgs &g, const OpArgs &op, cudaStream_t s);
// Fused GAT attention chain (ug_gat_attention, k_gat.cu).
struct GatArgs {
    const float *el, *er, *z;   // [V_src][H], [V][H] (local rows), [V_src][F]
    int64_t ld_el, ld_er, ld_z;
    float *out, *attn;          // [V][F] (local rows); attn [E][H] by edge id or NULL
    int64_t ld_out, ld_attn;
    int32_t F, H, D;
    float slope;
};
cudaError_t launch_gat(const GraphArgs &g, const GatArgs &a, int vec, int L, const SplitPlan &plan,
                       const int32_t *slot_row, float *sacc, float *sst, int64_t sld, int64_t nfc,
                       int32_t *counters, cudaStream_t s);
// Fused dot-product attention chain (ug_dot_attention, k_dotattn.cu).
struct DotAttnArgs {
    const float *q, *k, *val;      // q: Dst_V [V][H*Dk] (local rows), k / val: Src_V [V_src][H*Dk / H*Dv]
    int64_t ld_q, ld_k, ld_val;
    float *out, *attn;             // out [V][H*Dv] (local rows); attn [E][H] by edge id or NULL
    int64_t ld_out, ld_attn;
    float *mden;                   // [V][H][2] final (max, denominator) per row and head (attn only)
    int32_t H, Dk, Dv;
    float scale_log2;              // scale * log2(e)
};
int dotattn_vec(const DotAttnArgs &a);
cudaError_t launch_dotattn(const GraphArgs &g, const DotAttnArgs &a, int vec, const SplitPlan &plan,
                           float *scratch, int64_t sld, cudaStream_t s);
cudaError_t launch_argext(int kedge, int gather, const GraphArgs &g, const OpArgs &op, int L, const SplitPlan &plan,
                          const int32_t *slot_row, float *sval, int32_t *sarg, int64_t sld, int32_t *counters,
                          int32_t *arg, int64_t ld_arg, cudaStream_t s);
cudaError_t launch_argscatter(const int32_t *arg, int64_t ld_arg, const float *grad, int64_t ld_grad, int64_t V, int W,
                              bool to_src, const int32_t *col, const int32_t *src_of_eid, float *out, int64_t ld_out,
                              int div, cudaStream_t s);
cudaError_t launch_permute(const int32_t *eid, const float *in, float *out, int64_t E, int width,
                           cudaStream_t s);

}  // namespace ug

// The opaque graph of the C ABI.
struct ug_graph {
    int64_t V = 0, E = 0;       // local rows / edges
    int64_t V_total = 0;        // vertex-id space (src ids < V_total)
    int64_t r0 = 0;             // first global row (views)
    int64_t e0 = 0;             // first global CSR position (views) == row_ptr[r0]
    bool host_only = false;
    bool is_view = false;
    bool eid_identity = true;
    const ug_graph *parent = nullptr;

    // Host CSR.  Base graphs own the vectors; views point into the parent's arrays.
    std::vector<int32_t> h_row_ptr_v, h_col_v, h_eid_v, h_dst_v;
    const int32_t *h_row_ptr = nullptr;   // global row_ptr values at local rows 0..V
    const int32_t *h_col = nullptr;       // at local position 0
    const int32_t *h_eid = nullptr;       // NULL when identity

    // Device CSR (same offsets as the host pointers).
    int32_t *d_row_ptr = nullptr, *d_col = nullptr, *d_eid = nullptr, *d_dst = nullptr;

    // Allocation bookkeeping.
    bool has_alloc = false;
    ug_allocator alloc{};
    std::vector<void *> owned;
    int device = 0;

    // Table 7 statistics.
    double mean_deg = 0.0, std_nnz = 0.0;
    int64_t max_deg = 0;

    // UG_SV plans keyed by chunk size.
    mutable std::mutex mu;
    mutable std::map<int, ug::SplitPlan> plans;
    // arrival counters of single-launch split-row merges (k_split, k_gat, k_argext), one buffer per
    // (stream, chunk size, column tiles): n_split_rows x n_tiles int32, zeroed once; every call
    // leaves them zero again, and calls on one stream are ordered, so no two calls share them
    mutable std::map<std::tuple<void *, int, int>, int32_t *> stream_counters;
    // src vertex by edge id (device), built on first use when eid is not the identity
    mutable int32_t *d_src_of_eid = nullptr;
    mutable std::vector<void *> plan_allocs;
};
