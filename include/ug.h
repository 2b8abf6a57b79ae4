/*
 * ug.h -- C ABI of libugraph: the unified GNN graph operator of uGrapher
 * (Zhou et al., ASPLOS'23; text at PAPER.md) re-designed for B200 (sm_100a).
 *
 * One call computes, for every destination vertex dst, every in-edge e = (src -> dst) and
 * every feature f (Fig. 5, lines 14-19):
 *     tmp = edge_op(A[a_idx][f], B[b_idx][f]);   C[c_idx][f] = gather_op(C[c_idx][f], tmp)
 * where a_idx/b_idx/c_idx follow the operand's tensor type (type_idx_dict):
 * Src_V -> src, Dst_V -> dst, Edge -> edge id.  The op set is Table 4
 * plus `dot` (R5): all 160 DGL graph operators of Table 2.
 *
 * Conventions (all entry points):
 *   - No exceptions cross this boundary; every function returns a ug_status.
 *   - Feature tensors are fp32, row-major, row stride `ld` (elements, ld >= width).
 *     Vertex ids and CSR arrays are int32.  Edge id = position in the COO given to
 *     ug_graph_create (R9).  E < 2^31.
 *   - Pointers marked "device" must be CUDA device (or managed) memory of the current
 *     device; "host" pointers are plain host memory.  `stream` is a cudaStream_t (NULL =
 *     legacy default stream).
 *   - The library never keeps a caller pointer after a call returns (graphs copy their
 *     input).  The caller owns A, B, C.
 *   - ug_op_run is asynchronous (no host synchronisation) and re-entrant across streams;
 *     graphs are immutable after creation.  Per-call scratch is stream-ordered
 *     (cudaMallocAsync on the call's stream).  The single-launch merges of split rows
 *     (ug_op_run under SV for small operators, ug_gat_attention, ug_op_run_arg) count chunk
 *     arrivals in a per-(graph, stream) counter buffer that every call leaves zeroed: calls on
 *     different streams never share one.  Restriction: a CUDA graph captured on stream S
 *     embeds S's counters, so two replays of it -- or a replay and an eager call on S -- must
 *     not run concurrently.
 *   - The first call of a graph with a given SV chunk size builds and uploads its plan (and
 *     counters) synchronously, in relaxed stream-capture mode: that first call may itself be
 *     inside a CUDA-graph capture.
 */
#ifndef UG_H_
#define UG_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    UG_OK = 0,
    UG_ERR_INVALID_ARG = 1,         /* NULL pointer, negative size, bad enum value        */
    UG_ERR_UNSUPPORTED_OP = 2,      /* op/type combination outside the supported op set  */
    UG_ERR_SHAPE = 3,               /* operand width not F or H, H does not divide F, ...   */
    UG_ERR_INDEX_RANGE = 4,         /* vertex id outside [0, V) at graph creation           */
    UG_ERR_ALIGNMENT = 5,           /* forced vector width incompatible with ld / pointer   */
    UG_ERR_OOM = 6,                 /* allocation failed                                    */
    UG_ERR_CUDA = 7,                /* a CUDA call failed; see ug_last_error()              */
    UG_ERR_UNSUPPORTED_SCHEDULE = 8 /* schedule parameters outside the implemented space    */
} ug_status;

/* edge_op list of Fig. 5 ("copy_lns/rns" read as copy_lhs/copy_rhs) + dot (R5). */
typedef enum {
    UG_EDGE_COPY_LHS = 0, UG_EDGE_COPY_RHS = 1, UG_EDGE_ADD = 2, UG_EDGE_SUB = 3,
    UG_EDGE_MUL = 4, UG_EDGE_DIV = 5, UG_EDGE_DOT = 6
} ug_edge_op;

/* gather_op list of Fig. 5.  The paper's copy_rhs used as a gather is an
 * assignment onto edges (message creation, Table 4 rows 1-5; reading R3). */
typedef enum {
    UG_GATHER_ASSIGN = 0, UG_GATHER_SUM = 1, UG_GATHER_MAX = 2, UG_GATHER_MIN = 3,
    UG_GATHER_MEAN = 4
} ug_gather_op;

/* tensor_type_list / type_idx_dict. */
typedef enum { UG_T_NULL = 0, UG_T_SRC_V = 1, UG_T_DST_V = 2, UG_T_EDGE = 3 } ug_ttype;

/* One operand.  data: device fp32; rows implied by type (V for Src_V/Dst_V, E for Edge);
 * width in {F, H} (H: per-head value broadcast over the head's D = F/H features, R6);
 * ld >= width, in elements.  The output C of a dot op has width H. */
typedef struct {
    void *data;
    int32_t type;   /* ug_ttype */
    int32_t width;
    int64_t ld;
} ug_tensor;

/* op_info of PAPER.md:385-386: [edge_op, gather_op, A, A_Type, B, B_Type, C, C_Type]
 * plus the feature width F and head count H (H | F; H = 1 for scalar broadcasts). */
typedef struct {
    int32_t edge_op;    /* ug_edge_op   */
    int32_t gather_op;  /* ug_gather_op */
    ug_tensor A, B, C;
    int32_t feat;       /* F */
    int32_t heads;      /* H */
} ug_op_info;

/* parallel_strategy of PAPER.md:387-388 and Fig. 6; BV/BE are block-level extensions
 * (north star).  Notation of Table 9: TE_G1_T16 = {UG_TE, 1, 16}. */
typedef enum {
    UG_SCHED_AUTO = 0,
    UG_TV = 1,      /* thread-vertex: T threads share one dst row's features, owner computes   */
    UG_TE = 2,      /* thread-edge:   T threads share one edge's features, atomics into dst    */
    UG_WV = 3,      /* warp-vertex:   T warps per dst row                                       */
    UG_WE = 4,      /* warp-edge:     T warps per edge                                          */
    UG_BV = 5,      /* block-vertex:  one CTA per G rows, its warps split each row's edges     */
    UG_BE = 6,      /* block-edge:    one CTA per G x warps edges, contiguous, segmented reduce */
    UG_SV = 7       /* split-vertex (B200): rows cut into <= `group` edge chunks (scheduled
                       longest first), column tiles of `ftile` features in tile-major order
                       (L2-resident), partials of split rows fixed up in chunk order.  For
                       `dot` between one Src_V and one Dst_V operand the Dst_V row is held in
                       registers per chunk (ftile unused); message creation stores each edge's
                       row contiguously (dst-sorted graphs)                                     */
} ug_strategy;

typedef struct {
    int32_t strategy;       /* ug_strategy                                                      */
    int32_t group;          /* G: units per thread/warp group (V/E grouping);
                               UG_SV: max edges per row chunk                                    */
    int32_t tile;           /* T: feature tiling: threads (TV/TE) or warps (WV/WE)
                               sharing one unit's features; with UG_SCHED_EDGELANES the lanes that
                               share one row's in-edges (TV: 8 or 16; WV: 1 warp)                */
    int32_t block_threads;  /* CTA size (0 -> 256)                                              */
    int32_t ftile;          /* column-tile width for L2 blocking, tile-major grid order; 0 = off.
                               UG_SV: a multiple of vec with ftile / vec <= 32 lanes (rounded up
                               to a power of two, the extra lanes idle); UG_SV dot between a Src_V
                               and a Dst_V operand: 32 / 64 / 128 selects the column-tiled kernel */
    int32_t vec;            /* feature vector width 1/2/4; 0 -> widest the layout allows        */
    int32_t flags;          /* UG_SCHED_PACK | UG_SCHED_TMA | UG_SCHED_ASYNC | UG_SCHED_EDGELANES.  UG_SCHED_PACK (SV only): first stage a full-width Src_V operand whose
                               rows are not 128-byte aligned into an aligned scratch copy, so each
                               column slab occupies whole L2 lines and rows take 16-byte loads   */
} ug_schedule;

#define UG_SCHED_PACK 1
#define UG_SCHED_TMA  2   /* SV aggregation only ("_M1"): source rows are gathered four at a time
                             by TMA (cp.async.bulk.tensor tile::gather4, issued by one lane per
                             warp) into a per-warp ring of shared-memory stages completed on
                             mbarriers, instead of into registers                                */
#define UG_SCHED_EDGELANES 8  /* WV / TV aggregation with W / vec <= 8 ("_E1"): the lanes of a row
                                 (WV_Gg_T1_E1: a warp; TV_Gg_Tt_E1, t in {8, 16}: t lanes, 32 / t
                                 rows per warp) take its in-edges round-robin and reduce all its
                                 features in registers, then combine by a transposed butterfly --
                                 one launch, owner computes; for narrow features on small, skewed
                                 graphs, where feature lanes leave most lanes idle.  SV message
                                 creation ("SV_Gg_E1", W <= 8): one warp per chunk, lanes over
                                 its consecutive in-edges                                       */
#define UG_SCHED_ASYNC 4  /* SV aggregation only ("_A1"): the same ring filled by cp.async
                             (LDGSTS, each lane its own features of the group's four rows).
                             Both staged forms: ftile = 32 * vec columns (128 / 64 / 32), a
                             full-width Src_V A (rows not aligned for the copy width are packed
                             first), identity edge ids, B absent, Dst_V, or a per-head / scalar
                             Edge tensor; otherwise UG_ERR_UNSUPPORTED_SCHEDULE.  Measured
                             against the register SV kernel in profiles/r2_staged_ab.md         */

/* Optional allocator for graph-owned device arrays (e.g. torch's caching allocator).
 * NULL -> cudaMallocAsync / cudaFreeAsync on the given stream. */
typedef struct {
    void *(*alloc)(size_t bytes, void *ctx, void *stream);
    void (*free)(void *ptr, void *ctx, void *stream);
    void *ctx;
} ug_allocator;

typedef struct ug_graph ug_graph;

/* Graph creation flags. */
#define UG_GRAPH_HOST_ONLY 1   /* build and keep the CSR on the host only (no CUDA calls):
                                  for host-side partitioning, stats, selection and tests  */

/*
 * ug_graph_create -- COO -> in-CSR keyed by destination (get_inedges).
 *   num_vertices V >= 0, num_edges E in [0, 2^31); src[E], dst[E] int32 vertex ids.
 *   on_device: 1 if src/dst are device pointers, 0 if host.
 *   Builds row_ptr[V+1], col_idx[E] = src sorted stably by dst (edge-id order inside a
 *   row, R10), eid[E] (omitted when the COO is already dst-sorted), dst_of[E] (COO row array
 *   for edge-parallel schedules) and the Table 7 statistics.  Validates ids
 *   (UG_ERR_INDEX_RANGE).  May synchronise `stream`.  *out owns copies of everything.
 */
ug_status ug_graph_create(int64_t num_vertices, int64_t num_edges,
                          const int32_t *src, const int32_t *dst, int on_device, int flags,
                          const ug_allocator *alloc, void *stream, ug_graph **out);

/* CSR input: row_ptr[V+1] (non-decreasing, row_ptr[0] = 0, row_ptr[V] = E), col_idx[E] = src,
 * eid[E] = COO edge id of CSR position k (NULL = identity).  Host or device per on_device. */
ug_status ug_graph_create_csr(int64_t num_vertices, int64_t num_edges, const int32_t *row_ptr,
                              const int32_t *col_idx, const int32_t *eid, int on_device, int flags,
                              const ug_allocator *alloc, void *stream, ug_graph **out);

/* Frees a graph or a view.  A parent must outlive its views.  Synchronises the device first
 * (cudaDeviceSynchronize), so kernels still reading the graph on any stream finish before its
 * memory is released. */
ug_status ug_graph_destroy(ug_graph *g);

/* Table 7 graph features: V (dst rows), E, mean in-degree,
 * std_nnz = population std of in-degree (R15), max in-degree.  Any out pointer may be NULL. */
ug_status ug_graph_stats(const ug_graph *g, int64_t *V, int64_t *E, double *mean_deg,
                         double *std_nnz, int64_t *max_deg);

/* Copy the host CSR (row_ptr[V+1], col_idx[E], eid[E]) into caller buffers (any may be NULL). */
ug_status ug_graph_csr(const ug_graph *g, int32_t *row_ptr, int32_t *col_idx, int32_t *eid);

/* Edge-balanced destination-row partition (R21): row_splits[k] = smallest row r with
 * row_ptr[r] >= ceil(k E / parts), row_splits[0] = 0, row_splits[parts] = V. */
ug_status ug_graph_partition(const ug_graph *g, int32_t parts, int64_t *row_splits);

/*
 * ug_graph_view_rows -- zero-copy view of destination rows [r0, r1) for sharding.
 *   Inside a view: Src_V operands are indexed by GLOBAL vertex id (pass the full,
 *   all-gathered X); Dst_V operands and C of type Dst_V by LOCAL row v - r0 (pass
 *   X_full + r0*ld and the local output shard); Edge operands and C of type Edge by LOCAL
 *   edge position k - row_ptr[r0].  Requires eid = identity (dst-sorted COO); otherwise
 *   UG_ERR_INVALID_ARG (permute edge tensors once with ug_edge_permute).
 */
ug_status ug_graph_view_rows(const ug_graph *g, int64_t r0, int64_t r1, ug_graph **view);

/*
 * ug_graph_reorder -- vertex renumbering for locality (node renumbering as
 * orthogonal preprocessing).  Host only.  Writes perm[new_id] = old_id
 * (host int32 [V]) for a whole square graph (not a view):
 *   UG_ORDER_DEGREE: descending total (in + out) degree, ties by id;
 *   UG_ORDER_RCM:    reverse Cuthill-McKee on the symmetrised graph;
 *   UG_ORDER_COMMUNITY: Rabbit-style community order (label propagation on the symmetrised
 *                    graph, vertices grouped by community, descending degree inside).
 * The caller renumbers its COO (src' = inv[src], dst' = inv[dst], edge ids unchanged),
 * builds a new graph and gathers vertex tensors with ug_rows_gather(X, perm) -- results then
 * come back in the new numbering (gather them with the inverse permutation).
 */
#define UG_ORDER_DEGREE 1
#define UG_ORDER_RCM 2
#define UG_ORDER_COMMUNITY 3
ug_status ug_graph_reorder(const ug_graph *g, int32_t method, int32_t *perm);

/* out[i][0..width) = in[idx[i]][0..width) for i < rows (device pointers, row strides ld_in /
 * ld_out >= width; idx device int32).  Asynchronous on `stream`. */
ug_status ug_rows_gather(const float *in, int64_t ld_in, const int32_t *idx, int64_t rows, int32_t width,
                         float *out, int64_t ld_out, void *stream);

/* Validate op_info against the supported op set and shapes without running (host only). */
ug_status ug_op_validate(const ug_graph *g, const ug_op_info *op);

/*
 * ug_schedule_select -- automatic choice of parallel_info when it is absent.
 * Keyed by (op class, F, mean degree, degree CV, V) over a table measured on B200
 * (selector_table.json, loaded at first use or via ug_selector_load).  Host only, < 10 us.
 */
ug_status ug_schedule_select(const ug_graph *g, const ug_op_info *op, ug_schedule *out);

/* Replace the selector table with the JSON file at `path` (format in DESIGN.md). */
ug_status ug_selector_load(const char *path);

/* Replace the learned selector model (tier 2 of ug_schedule_select) with the
 * tree file at `path` (text format written by scripts/train_selector.py; default:
 * selector_model.txt next to libugraph.so, or $UG_SELECTOR_MODEL).  "" unloads the model. */
ug_status ug_selector_load_model(const char *path);

/*
 * ug_op_run -- one unified-operator call (the paper's uGrapher(Graph_Tensor, op_info,
 * parallel_info)).  sched NULL or strategy UG_SCHED_AUTO -> ug_schedule_select.
 * Writes every element of C's logical [rows x width] block (rows with zero in-degree get
 * 0, R7).  Enqueues 1-3 kernels on `stream` (init / main / epilogue as the schedule needs);
 * never synchronises.  Requires a device graph (not UG_GRAPH_HOST_ONLY).
 */
ug_status ug_op_run(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched,
                    void *stream);

/* Measurement hook: exactly ug_op_run, and additionally records the caller's cudaEvent_t
 * `ev_begin` / `ev_end` on `stream` immediately before / after the operator's MAIN kernel
 * (the traversal a5, excluding init / epilogue / fix-up launches), so a caller can time the
 * dominant kernel alone with CUDA events.  Either event may be NULL. */
ug_status ug_op_run_events(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched,
                           void *stream, void *ev_begin, void *ev_end);

/* Number of kernel launches ug_op_run would enqueue for (op, sched) (after AUTO). */
ug_status ug_op_launch_count(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched,
                             int32_t *launches);

/* out[k][:] = in[eid[k]][:] for k < E: edge tensor from COO edge-id order to CSR order
 * (device pointers, width columns, dense rows).  Identity copy when eid is identity. */
ug_status ug_edge_permute(const ug_graph *g, const float *in, float *out, int32_t width,
                          void *stream);

/*
 * ug_gat_attention -- the GAT attention chain fused into ONE traversal.
 * PAPER.md:224 lists GAT's graph operators: a message creation el_u + er_v (edge scores) and
 * an aggregation-sum weighting each source feature by its edge weight; GAT's edge softmax
 * between them (LeakyReLU, copy_e_max, e_sub_v + exp, copy_e_sum, e_div_v under the unified
 * abstraction) is folded in.  For every destination v, head h < H and feature f = h*D + d
 * (D = F / H), over v's in-edges e = (u -> v):
 *     s(e,h)  = LeakyReLU(el[u][h] + er[v][h]) = s >= 0 ? s : slope * s
 *     a(e,h)  = exp(s(e,h) - max_e' s(e',h)) / sum_e' exp(s(e',h) - max_e' s(e',h))
 *     out[v][f] = sum_e a(e,h) * z[u][f]
 *   el  [V_src][H] (ld_el), er [V][H] (ld_er), z [V_src][F] (ld_z): device fp32 inputs
 *       (in a view: el, z by global src id; er by local row, as Src_V / Dst_V operands).
 *   out [V][F] (ld_out): device fp32, every row written; zero in-degree rows -> 0 (R7).
 *   attn: NULL, or device fp32 [E][H] (ld_attn) receiving a(e,h) at row = edge id (R9).
 *   Accuracy: within 1e-5 * sum_e a(e,h) |z[u][f]| of the fp64 definition (oracle.gat);
 *   attention within 1e-5 relative.  Deterministic (chunk-order merge).  One kernel launch on
 *   `stream` (re-entrancy and capture: see the conventions at the top).
 *   Errors: UG_ERR_INVALID_ARG (NULL graph / data, host-only graph), UG_ERR_SHAPE (H <= 0,
 *   H does not divide F, ld < width), UG_ERR_OOM, UG_ERR_CUDA.
 */
ug_status ug_gat_attention(const ug_graph *g, const float *el, int64_t ld_el, const float *er,
                           int64_t ld_er, const float *z, int64_t ld_z, int32_t F, int32_t H,
                           float slope, float *out, int64_t ld_out, float *attn, int64_t ld_attn,
                           void *stream);

/* Fused dot-product attention chain (the FusedMM-style SDDMM + SpMM of
 * PAPER.md:588 built from the paper's operators -- u_dot_v message creation (Table 2 dot ops,
 * R5), an edge softmax over each destination's in-edges, and the u_mul_e_sum aggregation, the
 * operator chain of PAPER.md:224 with a dot score) in ONE traversal:
 *     s_e = scale * sum_{d<Dk} q[v][h*Dk+d] * k[u][h*Dk+d]      (e = u -> v, head h < H)
 *     a_e = exp(s_e - max) / sum exp(... )  over the in-edges of v
 *     out[v][h*Dv+j] = sum_e a_e * val[u][h*Dv+j]                 (0 for zero in-degree, R7)
 *   q   [V][H*Dk] device, Dst_V rows (a view's local rows), row stride ld_q
 *   k   [V_total][H*Dk], val [V_total][H*Dv] device, Src_V rows (global ids)
 *   out [V][H*Dv] device (written); attn [E][H] device by edge id (written) or NULL.
 *   Needs Dk and Dv <= 128 * vec where vec (4 / 2 / 1) divides both and every row's alignment;
 *   else UG_ERR_SHAPE.  fp32 in / out; scores in the log2 domain with ex2.approx (R25).
 *   Per-call scratch on `stream` (cudaMallocAsync): re-entrant across streams.  Asynchronous. */
ug_status ug_dot_attention(const ug_graph *g, const float *q, int64_t ld_q, const float *k, int64_t ld_k,
                           const float *val, int64_t ld_val, int32_t H, int32_t Dk, int32_t Dv, float scale,
                           float *out, int64_t ld_out, float *attn, int64_t ld_attn, void *stream);

/*
 * ug_op_run_arg -- a max/min aggregation with arg capture (training of
 * GraphSAGE-max style layers: the paper itself is inference-only).
 * Computes C exactly as ug_op_run would (bit-identical values) for op_info with gather
 * max/min, C of type Dst_V and an elementwise edge_op (not dot), and writes
 *     arg[v][f] = the edge id (R9; the local CSR position inside a view) of the in-edge whose
 *                 message supplied C[v][f]: the FIRST edge id attaining the extreme under the
 *                 total order -0 < +0 (R12); -1 for zero in-degree rows (C = 0, R7).
 *   arg: device int32 [V][F], row stride ld_arg >= F.  One kernel launch; deterministic.
 *   Errors: as ug_op_run; UG_ERR_UNSUPPORTED_OP for sum/mean/assign or dot.
 */
ug_status ug_op_run_arg(const ug_graph *g, const ug_op_info *op, int32_t *arg, int64_t ld_arg,
                        void *stream);

/*
 * ug_arg_scatter -- backward of a max/min aggregation through its arg capture:
 *     for every v, f with e = arg[v][f] >= 0:  out[row(e)][f / (W / out_width)] += grad[v][f]
 *   row(e) = src vertex of edge e (target_type UG_T_SRC_V: d/dA of copy_u_max) or e itself
 *   (UG_T_EDGE: d/dA of copy_e_max).  out is ACCUMULATED into (zero it first); fp32 atomics,
 *   so sums of several contributions to one element are order-dependent within rounding.
 *   arg [V][W] (ld_arg), grad [V][W] (ld_grad), out [rows][out_width] (ld_out): device.
 *   Errors: UG_ERR_INVALID_ARG, UG_ERR_UNSUPPORTED_OP (other target types), UG_ERR_SHAPE.
 */
ug_status ug_arg_scatter(const ug_graph *g, const int32_t *arg, int64_t ld_arg, int32_t W,
                         const float *grad, int64_t ld_grad, int32_t target_type, float *out,
                         int64_t ld_out, int32_t out_width, void *stream);

/* Schedule <-> text, Table 9 notation ("TE_G1_T16", "SV_G2048_F64"). */
ug_status ug_schedule_parse(const char *text, ug_schedule *out);
ug_status ug_schedule_format(const ug_schedule *s, char *buf, size_t len);

const char *ug_status_string(ug_status s);
const char *ug_last_error(void);   /* thread-local detail of the last failing call */
const char *ug_version(void);

/* Per-call scratch (split-row partials, the pack of a misaligned A operand, k_dott partials) is
 * allocated with cudaMallocAsync on the call's stream from the device's default memory pool --
 * outside any framework allocator (e.g. torch's caching allocator).  The pool keeps up to 4 GiB
 * reserved between calls; this returns everything unused to the driver (synchronises the device). */
ug_status ug_scratch_trim(void);

#ifdef __cplusplus
}
#endif
#endif /* UG_H_ */
