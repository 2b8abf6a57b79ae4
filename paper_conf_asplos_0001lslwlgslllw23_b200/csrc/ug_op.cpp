// ug_op.cpp -- the unified operator entry point (uGrapher(Graph_Tensor, op_info,
// parallel_info)): validation against the op set (Table 4,
// PAPER.md:291-307; Table 2), lowering (the paper's two code-generation
// passes, done as template selection), schedule resolution and launch.
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "ug_internal.h"
#include "ug_runtime.h"

namespace ug {

static thread_local std::string g_last_error;

ug_status set_error(ug_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

static int pow2ceil(int64_t x) {
    int p = 1;
    while (p < x && p < (1 << 30)) p <<= 1;
    return p;
}

static bool is_pow2(int x) { return x > 0 && (x & (x - 1)) == 0; }

// ------------------------------------------------------------------------- lowering
ug_status lower(const ug_graph *g, const ug_op_info *op, Lowered *out) {
    if (!g || !op || !out) return set_error(UG_ERR_INVALID_ARG, "NULL graph / op_info");
    const int eo = op->edge_op, go = op->gather_op;
    if (eo < UG_EDGE_COPY_LHS || eo > UG_EDGE_DOT) return set_error(UG_ERR_INVALID_ARG, "edge_op out of range");
    if (go < UG_GATHER_ASSIGN || go > UG_GATHER_MEAN) return set_error(UG_ERR_INVALID_ARG, "gather_op out of range");
    const int F = op->feat, H = op->heads;
    if (F <= 0 || H <= 0 || F % H != 0) return set_error(UG_ERR_SHAPE, "need F > 0, H > 0 and H | F");
    const ug_tensor &C = op->C;
    if (C.type != UG_T_DST_V && C.type != UG_T_EDGE)
        return set_error(UG_ERR_UNSUPPORTED_OP, "C must be a Dst_V (aggregation) or Edge (message creation) tensor");
    const bool to_edges = C.type == UG_T_EDGE;
    if (to_edges != (go == UG_GATHER_ASSIGN))
        return set_error(UG_ERR_UNSUPPORTED_OP,
                         "gather assign writes edges; sum/max/min/mean reduce into Dst_V (Table 4)");
    const bool dot = eo == UG_EDGE_DOT;
    const int W = dot ? H : F;
    if (C.width != W) return set_error(UG_ERR_SHAPE, "C width must be F (or H for dot)");
    if (C.ld < C.width) return set_error(UG_ERR_SHAPE, "C: ld < width");
    // NULL data is legal only for a tensor with zero rows (e.g. Edge tensors of an empty graph).
    auto rows_of = [g](int32_t type) -> int64_t { return type == UG_T_EDGE ? g->E : (type == UG_T_SRC_V ? g->V_total : g->V); };
    if (!C.data && rows_of(C.type) > 0) return set_error(UG_ERR_INVALID_ARG, "C data is NULL");

    // Pass 1: copy ops use one operand; copy_rhs is copy_lhs on B.
    const ug_tensor *opa = nullptr, *opb = nullptr;
    if (eo == UG_EDGE_COPY_LHS) opa = &op->A;
    else if (eo == UG_EDGE_COPY_RHS) opa = &op->B;
    else { opa = &op->A; opb = &op->B; }
    Operand oa{nullptr, UG_T_NULL, 1, 0}, ob{nullptr, UG_T_NULL, 1, 0};
    const ug_tensor *used[2] = {opa, opb};
    Operand *dst_ops[2] = {&oa, &ob};
    for (int i = 0; i < 2; ++i) {
        const ug_tensor *t = used[i];
        if (!t) continue;
        if (t->type != UG_T_SRC_V && t->type != UG_T_DST_V && t->type != UG_T_EDGE)
            return set_error(UG_ERR_UNSUPPORTED_OP, "an operand the edge_op reads has type NULL");
        if (!t->data && rows_of(t->type) > 0) return set_error(UG_ERR_INVALID_ARG, "operand data is NULL");
        if (!(t->width == F || t->width == H || t->width == 1))
            return set_error(UG_ERR_SHAPE, "operand width must be F, H or 1");
        if (t->ld < t->width) return set_error(UG_ERR_SHAPE, "operand ld < width");
        dst_ops[i]->p = (const float *)t->data;
        dst_ops[i]->type = t->type;
        dst_ops[i]->div = F / t->width;
        dst_ops[i]->ld = t->ld;
    }
    if (!opb) ob = oa;   // unused; keep valid pointers for the address arithmetic

    Lowered lw{};
    lw.dot = dot;
    lw.gather = go;
    lw.to_edges = to_edges;
    lw.kedge = dot ? -1
             : (eo <= UG_EDGE_COPY_RHS ? K_COPY
                : eo == UG_EDGE_ADD ? K_ADD : eo == UG_EDGE_SUB ? K_SUB : eo == UG_EDGE_MUL ? K_MUL : K_DIV);
    lw.args.A = oa;
    lw.args.B = ob;
    lw.args.C = (float *)C.data;
    lw.args.c_ld = C.ld;
    lw.args.c_type = C.type;
    lw.args.F = F;
    lw.args.W = W;
    lw.args.H = H;
    lw.args.D = F / H;
    lw.op_class = dot ? (to_edges ? 2 : 3) : (to_edges ? 0 : 1);
    // aggregation subclasses for the selector: two-operand sums (4) and max/min (5)
    if (lw.op_class == 1 && (go == UG_GATHER_MAX || go == UG_GATHER_MIN)) lw.op_class = 5;
    else if (lw.op_class == 1 && opb) lw.op_class = 4;

    // Widest legal feature vector (R22 in DESIGN.md), per tensor: a full-width operand row must
    // be aligned and either F % vec == 0 or padded (ld >= round_up(F, vec)); a broadcast operand
    // must keep a vec chunk inside one head; C stores must be aligned (dot: D % vec == 0).
    const int span = dot ? lw.args.D : F;
    auto operand_vec = [&](const ug_tensor *t, const Operand &o) {
        if (!t) return 4;
        for (int v : {4, 2}) {
            const bool ok = o.div == 1 ? (o.ld % v == 0) && ((uintptr_t)o.p % (4 * v) == 0) &&
                                             (span % v == 0 || o.ld >= ((F + v - 1) / v) * v)
                                       : (o.div % v == 0 || o.div == F);   // a scalar (width 1) broadcasts over every chunk
            if (ok) return v;
        }
        return 1;
    };
    lw.a_vec = operand_vec(opa, oa);
    lw.b_vec = operand_vec(opb, ob);
    lw.c_vec = 1;
    for (int v : {4, 2}) {
        const bool ok = dot ? (lw.args.D % v == 0) : (C.ld % v == 0) && ((uintptr_t)C.data % (4 * v) == 0);
        if (ok) { lw.c_vec = v; break; }
    }
    lw.max_vec = std::min(std::min(lw.a_vec, lw.b_vec), lw.c_vec);
    lw.args.c_vec = dot ? 1 : lw.c_vec;
    lw.pack_ok = !dot && opa && oa.type == UG_T_SRC_V && oa.div == 1 && (oa.ld * 4) % 128 != 0;
    *out = lw;
    return UG_OK;
}

// ------------------------------------------------------------------------- resolution

// dot under SV with one Src_V and one Dst_V full-width operand (u_dot_v / v_dot_u): k_dotsv,
// which keeps the Dst_V row in registers per work unit.  Other dot ops under SV use k_dot.
static bool dotsv_ok(const Lowered &lw, const LaunchCfg &c, bool *a_is_src = nullptr, int *L = nullptr) {
    if (!lw.dot || c.strategy != UG_SV) return false;
    const Operand &A = lw.args.A, &B = lw.args.B;
    if (A.div != 1 || B.div != 1) return false;
    const bool as = A.type == UG_T_SRC_V && B.type == UG_T_DST_V;
    const bool bs = A.type == UG_T_DST_V && B.type == UG_T_SRC_V;
    int l = 0, w = 0;
    if ((!as && !bs) || dotsv_nj(lw.args, c.vec, &l, &w) == 0) return false;
    if (a_is_src) *a_is_src = as;
    if (L) *L = l;
    return true;
}

ug_status resolve(const ug_graph *g, const Lowered &lw, const ug_schedule &s, LaunchCfg *cfg) {
    (void)g;
    LaunchCfg c{};
    c.strategy = s.strategy;
    if (c.strategy < UG_TV || c.strategy > UG_SV)
        return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "strategy out of range");
    // SV stores through any C alignment (st_out), so its vector width is bounded by the operands
    // only; with UG_SCHED_PACK the staged copy of A is 16-byte aligned (a_vec = 4).
    c.pack = c.strategy == UG_SV && (s.flags & UG_SCHED_PACK) && lw.pack_ok;
    if ((s.flags & UG_SCHED_EDGELANES) && c.strategy == UG_SV) {
        // message creation with lanes over edges (k_msg_el): SV chunks, narrow messages
        if (!lw.to_edges || lw.dot || lw.args.W > 8)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "SV _E1: message creation of an elementwise message, W <= 8");
        c.edgelanes = true;
        c.vec = 1;
        c.G = s.group > 0 ? s.group : 1024;
        c.L = 32;
        c.block = 256;
        *cfg = c;
        return UG_OK;
    }
    if (s.flags & UG_SCHED_EDGELANES) {
        // lanes over a row's in-edges (k_vertex_el): WV aggregation of an elementwise message, narrow W
        if ((c.strategy != UG_WV && c.strategy != UG_TV) || lw.dot || lw.to_edges)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "_E1: WV / TV aggregation (or SV message creation) of an elementwise message only");
        // lanes per row: WV a whole warp (T must be 1); TV T in {8, 16} lanes, 32 / T rows per warp
        const int T = s.tile > 0 ? s.tile : (c.strategy == UG_WV ? 1 : 0);
        if (c.strategy == UG_WV ? T != 1 : (T != 8 && T != 16))
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "_E1: WV takes T1, TV takes T8 or T16 lanes per row");
        c.vec = s.vec ? s.vec : lw.max_vec;
        if (c.vec > lw.max_vec) return set_error(UG_ERR_ALIGNMENT, "forced vec wider than the operand layout allows");
        if ((lw.args.W + c.vec - 1) / c.vec > 8)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "_E1: at most 8 feature vectors per row (W <= 8 * vec)");
        c.edgelanes = true;
        c.G = s.group > 0 ? s.group : 1;
        c.L = c.strategy == UG_WV ? 32 : T;
        c.block = 256;
        *cfg = c;
        return UG_OK;
    }
    c.staged = (s.flags & UG_SCHED_TMA) ? 1 : ((s.flags & UG_SCHED_ASYNC) ? 2 : 0);
    if (c.staged) {
        // shared-memory row staging (k_svg): SV aggregation only; a misaligned A is packed first
        if (c.strategy != UG_SV || lw.dot || lw.to_edges)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "staged SV (_M1 / _A1): SV aggregation of an elementwise message only");
        const Operand &A = lw.args.A;
        if (A.type != UG_T_SRC_V || A.div != 1)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "staged SV (_M1 / _A1): A must be a full-width Src_V operand");
        const int ft = s.ftile > 0 ? s.ftile : (lw.args.W >= 128 ? 128 : (lw.args.W >= 64 ? 64 : 32));
        if (ft != 32 && ft != 64 && ft != 128)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "staged SV (_M1 / _A1): ftile must be 32, 64 or 128");
        c.ftile = ft;
        c.vec = ft / 32;
        if (s.vec && s.vec != c.vec)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "staged SV (_M1 / _A1): vec is ftile / 32");
        const int need = c.staged == 1 ? 4 : c.vec;     // TMA rows: 16-byte aligned; cp.async: the copy width
        if ((uintptr_t)A.p % (4 * need) != 0 || A.ld % need != 0) {
            if (!lw.pack_ok) return set_error(UG_ERR_ALIGNMENT, "staged SV: A rows are not aligned for the copy width");
            c.pack = true;
        }
        c.G = s.group > 0 ? s.group : 2048;
        c.L = 32;
        c.block = 32 * 4;
        *cfg = c;
        return UG_OK;
    }
    const bool dott_pair = lw.dot && lw.args.A.div == 1 && lw.args.B.div == 1 &&
                           ((lw.args.A.type == UG_T_SRC_V && lw.args.B.type == UG_T_DST_V) ||
                            (lw.args.A.type == UG_T_DST_V && lw.args.B.type == UG_T_SRC_V));
    if (c.strategy == UG_SV && dott_pair && (s.ftile == 32 || s.ftile == 64 || s.ftile == 128)) {
        // k_dott: column tiles of 32 * vec features of each head, any D (ftile = the widest tile);
        // other ftile values, and dot ops that are not (Src_V, Dst_V) pairs, keep the untiled SV
        // dot kernels (k_dotsv / k_dot), which ignore ftile
        const Operand &A = lw.args.A, &B = lw.args.B;
        const bool as = A.type == UG_T_SRC_V && B.type == UG_T_DST_V;
        const Operand &P = as ? A : B, &Q = as ? B : A;
        auto fits = [&](const Operand &o, int v) { return (uintptr_t)o.p % (4 * v) == 0 && o.ld % v == 0; };
        const bool same = P.p == Q.p && P.ld == Q.ld;          // u_dot_v of one matrix with itself
        c.pack = false;
        int v = s.ftile / 32;
        // widest v <= ftile / 32 with D % v == 0 (one head: any D) and Q's rows aligned for v (P is
        // packed into 128-byte rows when its own rows are not; a Q that is the same matrix
        // follows it).  A ragged head tail (D % v != 0) is gathered as a full vector and masked,
        // so P's rows must reach round_up(D, v) -- packing guarantees it; Q, loaded once per
        // unit, reads its tail element by element.
        for (; v > 1; v >>= 1)
            if ((lw.args.D % v == 0 || lw.args.H == 1) && (fits(Q, v) || same)) break;
        if (v > 1 && (!fits(P, v) || (lw.args.D % v != 0 && P.ld < (lw.args.D + v - 1) / v * v))) c.pack = true;
        if (s.vec && s.vec != v) return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "SV dot: vec follows ftile and the layout");
        c.dott = true;
        c.vec = v;
        c.ftile = 32 * v;
        c.G = s.group > 0 ? s.group : 256;
        c.L = 32;
        *cfg = c;
        return UG_OK;
    }
    const int sv_vec = std::min(c.pack ? 4 : lw.a_vec, lw.b_vec);
    const int allowed = (c.strategy == UG_SV && !lw.dot) ? sv_vec : lw.max_vec;
    c.vec = s.vec ? s.vec : allowed;
    if (!(c.vec == 1 || c.vec == 2 || c.vec == 4)) return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "vec must be 1, 2 or 4");
    if (c.vec > allowed) return set_error(UG_ERR_ALIGNMENT, "forced vec wider than the operand layout allows");
    c.G = s.group > 0 ? s.group : (c.strategy == UG_SV ? 2048 : 1);
    const int T = s.tile > 0 ? s.tile : 1;
    if (!is_pow2(T)) return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "tile T must be a power of two");
    c.block = s.block_threads > 0 ? s.block_threads : 256;
    const int max_block = (c.strategy == UG_BV) ? 512 : 256;
    if (c.block % 32 || c.block > max_block)
        return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "block_threads must be a multiple of 32 and <= 256 (512 for BV)");
    // Lanes: lanes beyond the feature chunks of one unit would have no work; they are not
    // launched (clamp rule).
    const int span = lw.dot ? lw.args.D : lw.args.W;
    const int need = pow2ceil((span + c.vec - 1) / c.vec);
    switch (c.strategy) {
    case UG_TV: case UG_TE: c.L = T; break;
    case UG_WV: case UG_WE: c.L = 32 * T; break;
    default: c.L = 32; break;
    }
    c.L = std::max(1, std::min(c.L, need));
    if (lw.dot) c.L = std::min(c.L, 32);
    c.ftile = s.ftile;
    if (c.ftile < 0 || c.ftile % c.vec) return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "ftile must be a multiple of vec");
    if (c.strategy == UG_SV && !lw.dot) {
        if (c.ftile == 0) c.ftile = std::min(32, need) * c.vec;
        // lanes per unit: ftile / vec rounded up to a power of two (lanes past ftile idle), so a
        // column tile need not be a power-of-two width (e.g. F120: 30 float4 lanes of 32)
        const int L = pow2ceil(c.ftile / c.vec);
        if (c.ftile / c.vec > 32)
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "SV needs ftile / vec <= 32");
        c.L = L;
    }
    if (c.strategy == UG_BE) c.L = std::min(32, need);
    if (c.strategy == UG_SV && lw.dot) {
        int L = 0;
        if (dotsv_ok(lw, c, nullptr, &L)) c.L = L;   // k_dotsv: SV chunks of G in-edges
        else c.G = 1;                                 // other dot ops: one row per lane group (k_dot)
    }
    *cfg = c;
    return UG_OK;
}

static GraphArgs graph_args(const ug_graph *g) {
    GraphArgs a;
    a.row_ptr = g->d_row_ptr;
    a.col = g->d_col;
    a.eid = g->d_eid;
    a.dst = g->d_dst;
    a.V = g->V;
    a.E = g->E;
    a.rp_base = g->e0;
    a.r0 = g->r0;
    a.V_src = g->V_total;
    return a;
}

// Restores this thread's stream-capture mode on scope exit.
struct RelaxedCapture {
    cudaStreamCaptureMode prev = cudaStreamCaptureModeRelaxed;
    RelaxedCapture() { cudaThreadExchangeStreamCaptureMode(&prev); }
    ~RelaxedCapture() { cudaThreadExchangeStreamCaptureMode(&prev); }
};

// Split-row plan for UG_SV (cached per chunk size; uploaded synchronously on first use).  The
// one-time upload (cudaMalloc + cudaMemcpy, not stream work) runs in relaxed capture mode, so
// the first call on a graph may itself be inside a CUDA-graph capture.
static ug_status get_plan(const ug_graph *g, int G, const SplitPlan **out) {
    std::lock_guard<std::mutex> lock(g->mu);
    auto it = g->plans.find(G);
    if (it != g->plans.end()) { *out = &it->second; return UG_OK; }
    RelaxedCapture relaxed;
    std::vector<int32_t> chunks, split, slot_row;
    int64_t slot = 0;
    for (int64_t v = 0; v < g->V; ++v) {
        const int64_t k0 = (int64_t)g->h_row_ptr[v] - g->e0, k1 = (int64_t)g->h_row_ptr[v + 1] - g->e0;
        const int64_t n = std::max<int64_t>(1, (k1 - k0 + G - 1) / G);
        if (n == 1) {
            chunks.insert(chunks.end(), {(int32_t)v, (int32_t)k0, (int32_t)k1, -1});
        } else {
            split.insert(split.end(), {(int32_t)v, (int32_t)slot, (int32_t)n, 0});
            for (int64_t i = 0; i < n; ++i) {
                const int64_t a = k0 + i * G, b = std::min(k1, a + G);
                slot_row.push_back((int32_t)(split.size() / 4 - 1));
                chunks.insert(chunks.end(), {(int32_t)v, (int32_t)a, (int32_t)b, (int32_t)slot++});
            }
        }
    }
    // Longest chunks first (stable): the lane groups sharing a warp then walk equally long
    // in-edge lists (no lanes idling while the warp's longest row finishes -- with CV ~1.8 the
    // longest of 4 rows is far above their mean), and the longest units start first (LPT
    // balance over the SMs).  Kernels address partials by scratch slot, never by chunk
    // position, so the order is free.  UG_SV_ORDER=row keeps row order (A/B measurements).
    const char *order = std::getenv("UG_SV_ORDER");
    if (!(order && std::string(order) == "row")) {
        const size_t nc = chunks.size() / 4;
        std::vector<int32_t> idx(nc);
        for (size_t i = 0; i < nc; ++i) idx[i] = (int32_t)i;
        std::stable_sort(idx.begin(), idx.end(), [&](int32_t a, int32_t b) {
            return chunks[4 * a + 2] - chunks[4 * a + 1] > chunks[4 * b + 2] - chunks[4 * b + 1];
        });
        std::vector<int32_t> sorted(chunks.size());
        for (size_t i = 0; i < nc; ++i)
            for (int j = 0; j < 4; ++j) sorted[4 * i + j] = chunks[4 * (size_t)idx[i] + j];
        chunks.swap(sorted);
    }
    SplitPlan p;
    p.n_chunks = (int64_t)chunks.size() / 4;
    p.n_split_rows = (int64_t)split.size() / 4;
    p.n_split_chunks = slot;
    void *dc = nullptr, *ds = nullptr, *dr = nullptr;
    if (cudaMalloc(&dc, std::max<size_t>(16, chunks.size() * 4)) != cudaSuccess ||
        cudaMalloc(&ds, std::max<size_t>(16, split.size() * 4)) != cudaSuccess ||
        cudaMalloc(&dr, std::max<size_t>(16, slot_row.size() * 4)) != cudaSuccess)
        return set_error(UG_ERR_OOM, "SV plan allocation failed");
    g->plan_allocs.push_back(dc);
    g->plan_allocs.push_back(ds);
    g->plan_allocs.push_back(dr);
    if ((!chunks.empty() && cudaMemcpy(dc, chunks.data(), chunks.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) ||
        (!split.empty() && cudaMemcpy(ds, split.data(), split.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) ||
        (!slot_row.empty() && cudaMemcpy(dr, slot_row.data(), slot_row.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess))
        return set_error(UG_ERR_CUDA, "SV plan upload failed");
    p.d_chunk = (int32_t *)dc;
    p.d_split = (int32_t *)ds;
    p.d_slot_row = (int32_t *)dr;
    auto res = g->plans.emplace(G, p);
    *out = &res.first->second;
    return UG_OK;
}

// Arrival counters of the single-launch split-row merges for calls on `stream` (see ug_graph::
// stream_counters).  Allocated and zeroed once per (stream, chunk size, column tiles), in relaxed
// capture mode like the plans; calls on one stream are ordered, and each call re-arms the counters
// it used, so concurrent calls on different streams never share a counter.
static ug_status get_counters(const ug_graph *g, void *stream, int G, int n_tiles, int64_t n_split_rows,
                              int32_t **out) {
    std::lock_guard<std::mutex> lock(g->mu);
    const auto key = std::make_tuple(stream, G, n_tiles);
    auto it = g->stream_counters.find(key);
    if (it != g->stream_counters.end()) { *out = it->second; return UG_OK; }
    RelaxedCapture relaxed;
    void *d = nullptr;
    const size_t bytes = std::max<size_t>(16, (size_t)n_split_rows * (size_t)n_tiles * 4);
    if (cudaMalloc(&d, bytes) != cudaSuccess) return set_error(UG_ERR_OOM, "counter allocation failed");
    g->plan_allocs.push_back(d);
    if (cudaMemset(d, 0, bytes) != cudaSuccess) return set_error(UG_ERR_CUDA, "counter init failed");
    g->stream_counters.emplace(key, (int32_t *)d);
    *out = (int32_t *)d;
    return UG_OK;
}

// Operators small enough to be launch-bound (per-edge feature work below ~2^26 elements) merge
// split rows inside the traversal launch (k_split<..., MERGE>).
static bool sv_merge_ok(const ug_graph *g, const Lowered &lw) {
    return (double)g->E * (double)lw.args.W < 67108864.0;
}

static int launches_for(const ug_graph *g, const Lowered &lw, const LaunchCfg &c, int64_t n_split_rows) {
    if (c.dott) {
        const int msg = 1 + (dott_tiles(lw.args, c.vec) > 1 ? 1 : 0);
        return lw.to_edges ? msg : msg + (n_split_rows > 0 ? 2 : 1);
    }
    const bool edge_units = c.strategy == UG_TE || c.strategy == UG_WE || c.strategy == UG_BE;
    if (lw.to_edges) return 1;
    if (edge_units) return lw.gather == UG_GATHER_SUM ? 2 : 3;
    if (c.strategy == UG_SV && !lw.dot && !c.staged && sv_merge_ok(g, lw)) return 1;   // merged in the launch
    if (c.strategy == UG_SV && (!lw.dot || dotsv_ok(lw, c))) return n_split_rows > 0 ? 2 : 1;
    return 1;
}

// Per-call scratch (split-row partials, the pack of a misaligned A, k_dott partials) comes from
// the device's default memory pool through cudaMallocAsync on the call's stream -- outside
// torch's caching allocator.  The pool keeps up to UG_SCRATCH_RETAIN bytes (4 GiB: the C5 pack
// plus k_dott's partials) reserved between calls so that steady-state calls do not go back to
// the driver; ug_scratch_trim() returns the rest.  Thread-safe (the mutex-free static init).
#ifndef UG_SCRATCH_RETAIN
#define UG_SCRATCH_RETAIN (4ull << 30)
#endif
static void ensure_pool_retains() {
    static const bool done = [] {
        int dev = 0;
        cudaMemPool_t pool;
        if (cudaGetDevice(&dev) == cudaSuccess && cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t thr = UG_SCRATCH_RETAIN;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        }
        return true;
    }();
    (void)done;
}

}  // namespace ug

using namespace ug;

extern "C" ug_status ug_op_validate(const ug_graph *g, const ug_op_info *op) {
    Lowered lw;
    return lower(g, op, &lw);
}

static ug_status prepare(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched, Lowered *lw,
                         LaunchCfg *cfg) {
    ug_status st = lower(g, op, lw);
    if (st != UG_OK) return st;
    ug_schedule s{};
    if (sched && sched->strategy != UG_SCHED_AUTO) s = *sched;
    else if ((st = select_schedule(g, *lw, &s)) != UG_OK) return st;
    return resolve(g, *lw, s, cfg);
}

extern "C" ug_status ug_op_launch_count(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched,
                                        int32_t *launches) {
    Lowered lw;
    LaunchCfg c;
    if (!launches) return set_error(UG_ERR_INVALID_ARG, "NULL out");
    ug_status st = prepare(g, op, sched, &lw, &c);
    if (st != UG_OK) return st;
    int64_t nsr = 0;
    if (c.strategy == UG_SV && (!lw.dot || dotsv_ok(lw, c) || c.dott) && !lw.to_edges) {
        // count split rows on the host without touching the device
        for (int64_t v = 0; v < g->V; ++v)
            if ((int64_t)g->h_row_ptr[v + 1] - g->h_row_ptr[v] > c.G) ++nsr;
    }
    *launches = launches_for(g, lw, c, nsr);
    return UG_OK;
}

static ug_status run(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched, void *stream,
                     cudaEvent_t ev_begin, cudaEvent_t ev_end) {
    Lowered lw;
    LaunchCfg c;
    ug_status st = prepare(g, op, sched, &lw, &c);
    if (st != UG_OK) return st;
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_op_run needs a device graph (not UG_GRAPH_HOST_ONLY)");
    cudaStream_t s = (cudaStream_t)stream;
    const GraphArgs ga = graph_args(g);
    const bool edge_units = c.strategy == UG_TE || c.strategy == UG_WE || c.strategy == UG_BE;
    cudaError_t err = cudaSuccess;
    const bool agg = !lw.to_edges;
    if (edge_units && agg) {
        err = launch_init(lw.gather, lw.args, g->V, s);
        if (err == cudaSuccess) {
            LaunchCfg ce = c;
            if (c.strategy == UG_BE) ce.L = std::min(c.L, 32);
            if (ev_begin) cudaEventRecord(ev_begin, s);
            err = lw.dot ? launch_dot(false, lw.gather, ga, lw.args, ce, s)
                         : launch_edge(lw.kedge, lw.gather, ga, lw.args, ce, s);
            if (ev_end) cudaEventRecord(ev_end, s);
        }
        if (err == cudaSuccess && lw.gather != UG_GATHER_SUM) err = launch_epilogue(lw.gather, ga, lw.args, s);
    } else if (c.dott) {
        // dot messages by column tiles (k_dott); an aggregation reduces them with SV afterwards
        const SplitPlan *plan = nullptr;
        if ((st = get_plan(g, c.G, &plan)) != UG_OK) return st;
        OpArgs args = lw.args;
        const bool a_src = args.A.type == UG_T_SRC_V;
        Operand &P = a_src ? args.A : args.B;
        Operand &Q = a_src ? args.B : args.A;
        float *packed = nullptr, *part = nullptr, *msg = nullptr;
        ensure_pool_retains();
        auto release = [&]() {
            if (part) cudaFreeAsync(part, s);
            if (msg) cudaFreeAsync(msg, s);
            if (packed) cudaFreeAsync(packed, s);
        };
        if (c.pack) {
            const int64_t ldp = (int64_t)(lw.args.F + 31) / 32 * 32;
            if (cudaMallocAsync((void **)&packed, sizeof(float) * (size_t)(g->V_total * ldp), s) != cudaSuccess)
                return set_error(UG_ERR_OOM, "SV dot pack allocation failed");
            if (cudaMemcpy2DAsync(packed, sizeof(float) * ldp, P.p, sizeof(float) * P.ld, sizeof(float) * lw.args.F,
                                  (size_t)g->V_total, cudaMemcpyDeviceToDevice, s) != cudaSuccess) {
                release();
                return set_error(UG_ERR_CUDA, "SV dot pack copy failed");
            }
            if (Q.p == P.p && Q.ld == P.ld) { Q.p = packed; Q.ld = ldp; }
            P.p = packed;
            P.ld = ldp;
        }
        if ((uint64_t)g->V_total * (uint64_t)P.ld >= (1ull << 32)) {
            release();
            return set_error(UG_ERR_UNSUPPORTED_SCHEDULE, "SV dot: Src_V operand above 2^32 elements");
        }
        const int th = dott_tiles(args, c.vec);
        const int64_t EH = g->E * (int64_t)lw.args.H;
        if (th > 1 && EH > 0 &&
            cudaMallocAsync((void **)&part, sizeof(float) * (size_t)(th * EH), s) != cudaSuccess) {
            release();
            return set_error(UG_ERR_OOM, "SV dot partial allocation failed");
        }
        float *dst = lw.args.C;
        int64_t dld = lw.args.c_ld;
        if (agg) {
            if (EH > 0 && cudaMallocAsync((void **)&msg, sizeof(float) * (size_t)EH, s) != cudaSuccess) {
                release();
                return set_error(UG_ERR_OOM, "SV dot message allocation failed");
            }
            dst = msg;
            dld = lw.args.H;
        }
        err = launch_dott(ga, args, a_src, c.vec, *plan, dst, dld, part, s, ev_begin, ev_end);
        if (err == cudaSuccess && agg) {
            // reduce the messages into Dst_V: copy_e_<gather> over the same chunks
            ug_op_info red{};
            red.edge_op = UG_EDGE_COPY_LHS;
            red.gather_op = lw.gather;
            red.A = ug_tensor{msg, UG_T_EDGE, lw.args.H, lw.args.H};
            red.B = ug_tensor{nullptr, UG_T_NULL, 0, 0};
            red.C = ug_tensor{lw.args.C, UG_T_DST_V, lw.args.H, lw.args.c_ld};
            red.feat = lw.args.H;
            red.heads = lw.args.H;
            ug_schedule rs{};
            rs.strategy = UG_SV;
            rs.group = c.G;
            st = run(g, &red, &rs, stream, nullptr, nullptr);
            release();
            return st;
        }
        release();
    } else if (bool a_src = false; dotsv_ok(lw, c, &a_src)) {
        const SplitPlan *plan = nullptr;
        if ((st = get_plan(g, c.G, &plan)) != UG_OK) return st;
        float *scratch = nullptr;
        const int64_t sld = (lw.args.W + 3) / 4 * 4;
        if (agg && plan->n_split_chunks > 0) {
            ensure_pool_retains();
            err = cudaMallocAsync((void **)&scratch, sizeof(float) * (size_t)(plan->n_split_chunks * sld), s);
            if (err != cudaSuccess) return set_error(UG_ERR_OOM, "SV scratch allocation failed");
        }
        err = launch_dotsv(lw.gather, ga, lw.args, a_src, c.vec, c.block, *plan, scratch, s, ev_begin, ev_end);
        if (scratch) cudaFreeAsync(scratch, s);
    } else if (lw.dot) {
        if (ev_begin) cudaEventRecord(ev_begin, s);
        err = launch_dot(!edge_units, lw.gather, ga, lw.args, c, s);
        if (ev_end) cudaEventRecord(ev_end, s);
    } else if (edge_units) {
        if (ev_begin) cudaEventRecord(ev_begin, s);
        err = launch_edge(lw.kedge, lw.gather, ga, lw.args, c, s);
        if (ev_end) cudaEventRecord(ev_end, s);
    } else if (c.strategy == UG_TV || c.strategy == UG_WV) {
        if (ev_begin) cudaEventRecord(ev_begin, s);
        err = c.edgelanes ? launch_vertex_el(lw.kedge, lw.gather, ga, lw.args, c, s)
                          : launch_vertex(lw.kedge, lw.gather, ga, lw.args, c, s);
        if (ev_end) cudaEventRecord(ev_end, s);
    } else if (c.strategy == UG_BV) {
        if (ev_begin) cudaEventRecord(ev_begin, s);
        err = launch_block_vertex(lw.kedge, lw.gather, ga, lw.args, c, s);
        if (ev_end) cudaEventRecord(ev_end, s);
    } else if (c.edgelanes) {          // UG_SV message creation, lanes over edges
        const SplitPlan *plan = nullptr;
        if ((st = get_plan(g, c.G, &plan)) != UG_OK) return st;
        if (ev_begin) cudaEventRecord(ev_begin, s);
        err = launch_msg_el(lw.kedge, ga, lw.args, *plan, s);
        if (ev_end) cudaEventRecord(ev_end, s);
    } else {  // UG_SV
        const SplitPlan *plan = nullptr;
        if ((st = get_plan(g, c.G, &plan)) != UG_OK) return st;
        float *scratch = nullptr, *packed = nullptr;
        const int64_t sld = (lw.args.W + 3) / 4 * 4;
        OpArgs args = lw.args;
        if (c.pack) {
            // stage A into rows of round_up(F, 32) floats (128-byte aligned): one 2-D copy
            ensure_pool_retains();
            const int64_t ldp = (int64_t)(lw.args.F + 31) / 32 * 32;
            err = cudaMallocAsync((void **)&packed, sizeof(float) * (size_t)(g->V_total * ldp), s);
            if (err != cudaSuccess) return set_error(UG_ERR_OOM, "SV pack allocation failed");
            err = cudaMemcpy2DAsync(packed, sizeof(float) * ldp, args.A.p, sizeof(float) * args.A.ld,
                                    sizeof(float) * lw.args.F, (size_t)g->V_total, cudaMemcpyDeviceToDevice, s);
            if (err != cudaSuccess) { cudaFreeAsync(packed, s); return set_error(UG_ERR_CUDA, "SV pack copy failed"); }
            args.A.p = packed;
            args.A.ld = ldp;
        }
        if (agg && plan->n_split_chunks > 0) {
            ensure_pool_retains();
            err = cudaMallocAsync((void **)&scratch, sizeof(float) * (size_t)(plan->n_split_chunks * sld), s);
            if (err != cudaSuccess) {
                if (packed) cudaFreeAsync(packed, s);
                return set_error(UG_ERR_OOM, "SV scratch allocation failed");
            }
        }
        if (c.staged) {
            // B addressing mode of k_svg: none, Dst_V (any width), or a per-head / scalar Edge tensor
            int bm = -1;
            if (lw.kedge == K_COPY) bm = 0;
            else if (args.B.type == UG_T_DST_V) bm = 1;
            else if (args.B.type == UG_T_EDGE && args.B.div > 1 && (uint64_t)g->E * (uint64_t)args.B.ld < (1ull << 32)) bm = 2;
            const int mode = c.staged - 1;
            if (bm < 0 || g->d_eid != nullptr || (uint64_t)g->V_total * (uint64_t)args.A.ld >= (1ull << 32) ||
                !svg_supported(args, c.vec, mode)) {
                if (scratch) cudaFreeAsync(scratch, s);
                if (packed) cudaFreeAsync(packed, s);
                return set_error(UG_ERR_UNSUPPORTED_SCHEDULE,
                                 "staged SV: needs identity edge ids, an aligned A below 2^32 elements and B absent, "
                                 "Dst_V or a per-head Edge tensor");
            }
            err = launch_split_staged(mode, lw.kedge, lw.gather, ga, args, c.vec, bm, *plan, scratch, s, ev_begin,
                                      ev_end);
        } else {
            // single-launch merge of split rows for launch-bound (small) operators; large ones keep
            // the hot instance without the merge tail and fix split rows in a second launch (< 1 %)
            int32_t *counters = nullptr;
            if (agg && plan->n_split_rows > 0 && sv_merge_ok(g, lw)) {
                const int n_tiles = (int)((lw.args.W + c.ftile - 1) / c.ftile);
                if ((st = get_counters(g, stream, c.G, n_tiles, plan->n_split_rows, &counters)) != UG_OK) {
                    if (scratch) cudaFreeAsync(scratch, s);
                    if (packed) cudaFreeAsync(packed, s);
                    return st;
                }
            }
            err = launch_split_vertex(lw.kedge, lw.gather, ga, args, c, *plan, scratch, s, ev_begin, ev_end,
                                      counters);
        }
        if (scratch) cudaFreeAsync(scratch, s);
        if (packed) cudaFreeAsync(packed, s);
    }
    if (err != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("kernel launch: ") + cudaGetErrorString(err));
    return UG_OK;
}

// One NVTX range per operator call (per-op ranges for nsys / ncu --nvtx); NVTX v3 is
// header-only and costs a branch when no tool is attached.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

extern "C" ug_status ug_op_run(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched, void *stream) {
    NvtxRange r("ug_op_run");
    return run(g, op, sched, stream, nullptr, nullptr);
}

extern "C" ug_status ug_op_run_events(const ug_graph *g, const ug_op_info *op, const ug_schedule *sched,
                                      void *stream, void *ev_begin, void *ev_end) {
    NvtxRange r("ug_op_run");
    return run(g, op, sched, stream, (cudaEvent_t)ev_begin, (cudaEvent_t)ev_end);
}

extern "C" ug_status ug_edge_permute(const ug_graph *g, const float *in, float *out, int32_t width, void *stream) {
    if (!g || !in || !out || width <= 0) return set_error(UG_ERR_INVALID_ARG, "ug_edge_permute: bad arguments");
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_edge_permute needs a device graph");
    cudaError_t e = launch_permute(g->d_eid, in, out, g->E, width, (cudaStream_t)stream);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, cudaGetErrorString(e));
    return UG_OK;
}

// ------------------------------------------------------------------------- text form
static const char *kStrat[] = {"AUTO", "TV", "TE", "WV", "WE", "BV", "BE", "SV"};

extern "C" ug_status ug_schedule_parse(const char *text, ug_schedule *out) {
    if (!text || !out) return set_error(UG_ERR_INVALID_ARG, "ug_schedule_parse: NULL");
    ug_schedule s{};
    std::string t(text);
    size_t pos = t.find('_');
    std::string head = t.substr(0, pos);
    int strat = -1;
    for (int i = 0; i < 8; ++i)
        if (head == kStrat[i]) strat = i;
    if (strat < 0) return set_error(UG_ERR_INVALID_ARG, "unknown strategy '" + head + "'");
    s.strategy = strat;
    while (pos != std::string::npos) {
        size_t nxt = t.find('_', pos + 1);
        std::string tok = t.substr(pos + 1, nxt == std::string::npos ? std::string::npos : nxt - pos - 1);
        if (tok.size() < 2) return set_error(UG_ERR_INVALID_ARG, "bad schedule token '" + tok + "'");
        char *end = nullptr;
        long val = std::strtol(tok.c_str() + 1, &end, 10);
        if (*end != '\0' || val < 0) return set_error(UG_ERR_INVALID_ARG, "bad schedule token '" + tok + "'");
        switch (tok[0]) {
        case 'G': s.group = (int32_t)val; break;
        case 'T': s.tile = (int32_t)val; break;
        case 'B': s.block_threads = (int32_t)val; break;
        case 'F': s.ftile = (int32_t)val; break;
        case 'V': s.vec = (int32_t)val; break;
        case 'P': s.flags = val ? (s.flags | UG_SCHED_PACK) : (s.flags & ~UG_SCHED_PACK); break;
        case 'M': s.flags = val ? (s.flags | UG_SCHED_TMA) : (s.flags & ~UG_SCHED_TMA); break;
        case 'A': s.flags = val ? (s.flags | UG_SCHED_ASYNC) : (s.flags & ~UG_SCHED_ASYNC); break;
        case 'E': s.flags = val ? (s.flags | UG_SCHED_EDGELANES) : (s.flags & ~UG_SCHED_EDGELANES); break;
        default: return set_error(UG_ERR_INVALID_ARG, "bad schedule token '" + tok + "'");
        }
        pos = nxt;
    }
    *out = s;
    return UG_OK;
}

extern "C" ug_status ug_schedule_format(const ug_schedule *s, char *buf, size_t len) {
    if (!s || !buf || s->strategy < 0 || s->strategy > 7) return set_error(UG_ERR_INVALID_ARG, "ug_schedule_format: bad args");
    std::string r = kStrat[s->strategy];
    if (s->strategy != UG_SCHED_AUTO) {
        r += "_G" + std::to_string(s->group > 0 ? s->group : (s->strategy == UG_SV ? 2048 : 1));
        if (s->strategy != UG_SV && s->strategy != UG_BV && s->strategy != UG_BE)
            r += "_T" + std::to_string(s->tile > 0 ? s->tile : 1);
        if (s->ftile) r += "_F" + std::to_string(s->ftile);
        if (s->block_threads) r += "_B" + std::to_string(s->block_threads);
        if (s->vec) r += "_V" + std::to_string(s->vec);
        if (s->flags & UG_SCHED_PACK) r += "_P1";
        if (s->flags & UG_SCHED_TMA) r += "_M1";
        if (s->flags & UG_SCHED_ASYNC) r += "_A1";
        if (s->flags & UG_SCHED_EDGELANES) r += "_E1";
    }
    std::snprintf(buf, len, "%s", r.c_str());
    return UG_OK;
}

extern "C" const char *ug_status_string(ug_status s) {
    switch (s) {
    case UG_OK: return "UG_OK";
    case UG_ERR_INVALID_ARG: return "UG_ERR_INVALID_ARG";
    case UG_ERR_UNSUPPORTED_OP: return "UG_ERR_UNSUPPORTED_OP";
    case UG_ERR_SHAPE: return "UG_ERR_SHAPE";
    case UG_ERR_INDEX_RANGE: return "UG_ERR_INDEX_RANGE";
    case UG_ERR_ALIGNMENT: return "UG_ERR_ALIGNMENT";
    case UG_ERR_OOM: return "UG_ERR_OOM";
    case UG_ERR_CUDA: return "UG_ERR_CUDA";
    case UG_ERR_UNSUPPORTED_SCHEDULE: return "UG_ERR_UNSUPPORTED_SCHEDULE";
    }
    return "UG_ERR_UNKNOWN";
}

extern "C" const char *ug_last_error(void) { return g_last_error.c_str(); }

extern "C" const char *ug_version(void) { return "ugraph-b200 0.2 (sm_100a)"; }

extern "C" ug_status ug_scratch_trim(void) {
    int dev = 0;
    cudaMemPool_t pool;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetDefaultMemPool(&pool, dev) != cudaSuccess)
        return set_error(UG_ERR_CUDA, "ug_scratch_trim: no device pool");
    if (cudaDeviceSynchronize() != cudaSuccess || cudaMemPoolTrimTo(pool, 0) != cudaSuccess)
        return set_error(UG_ERR_CUDA, "ug_scratch_trim: trim failed");
    return UG_OK;
}

// ------------------------------------------------------------------------- fused GAT chain
namespace ug {
static bool aligned(const void *p, int64_t ld, int vec) {
    return ((uintptr_t)p % (4 * vec)) == 0 && ld % vec == 0;
}
}  // namespace ug

extern "C" ug_status ug_gat_attention(const ug_graph *g, const float *el, int64_t ld_el, const float *er,
                                      int64_t ld_er, const float *z, int64_t ld_z, int32_t F, int32_t H,
                                      float slope, float *out, int64_t ld_out, float *attn, int64_t ld_attn,
                                      void *stream) {
    using namespace ug;
    if (!g) return set_error(UG_ERR_INVALID_ARG, "ug_gat_attention: NULL graph");
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_gat_attention needs a device graph");
    if (F <= 0 || H <= 0 || F % H != 0) return set_error(UG_ERR_SHAPE, "ug_gat_attention: need F > 0, H > 0, H | F");
    if (ld_el < H || ld_er < H || ld_z < F || ld_out < F || (attn && ld_attn < H))
        return set_error(UG_ERR_SHAPE, "ug_gat_attention: ld < width");
    if (g->V > 0 && (!er || !out)) return set_error(UG_ERR_INVALID_ARG, "ug_gat_attention: NULL er / out");
    if (g->E > 0 && (!el || !z)) return set_error(UG_ERR_INVALID_ARG, "ug_gat_attention: NULL el / z");
    if (g->V == 0) return UG_OK;
    const int D = F / H;
    int vec = 4;
    while (vec > 1 && (D % vec != 0 || !aligned(z, ld_z, vec) || !aligned(out, ld_out, vec))) vec >>= 1;
    int L = 1;
    while (L < 32 && (int64_t)L * vec < F) L <<= 1;
    const int n_tiles = (F + L * vec - 1) / (L * vec);
    // rows are cut into chunks of <= G in-edges (the SV plan): latency of the longest chunk
    // vs. merge overhead; UG_GAT_CHUNK overrides (experiments)
    int G = 32;
    if (const char *ev = std::getenv("UG_GAT_CHUNK")) G = std::max(1, std::atoi(ev));
    const SplitPlan *plan = nullptr;
    ug_status st = get_plan(g, G, &plan);
    if (st != UG_OK) return st;
    if (plan->n_chunks * n_tiles >= (int64_t)1 << 31)
        return set_error(UG_ERR_SHAPE, "ug_gat_attention: more than 2^31 (chunk, tile) units");
    GatArgs a;
    a.el = el; a.er = er; a.z = z;
    a.ld_el = ld_el; a.ld_er = ld_er; a.ld_z = ld_z;
    a.out = out; a.attn = attn; a.ld_out = ld_out; a.ld_attn = ld_attn;
    a.F = F; a.H = H; a.D = D; a.slope = slope;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t sld = (F + 3) / 4 * 4, nfc = (F + vec - 1) / vec;
    // split-row partials (per call, stream-ordered) and this stream's arrival counters
    float *scratch = nullptr;
    int32_t *counters = nullptr;
    if (plan->n_split_chunks > 0) {
        if ((st = get_counters(g, stream, G, n_tiles, plan->n_split_rows, &counters)) != UG_OK) return st;
        ensure_pool_retains();
        const size_t part = sizeof(float) * (size_t)plan->n_split_chunks * (size_t)(sld + 2 * nfc);
        if (cudaMallocAsync((void **)&scratch, part, s) != cudaSuccess)
            return set_error(UG_ERR_OOM, "ug_gat_attention: scratch allocation failed");
    }
    float *sst = scratch ? scratch + plan->n_split_chunks * sld : nullptr;
    cudaError_t e = launch_gat(graph_args(g), a, vec, L, *plan, plan->d_slot_row, scratch, sst, sld, nfc,
                               counters, s);
    if (scratch) cudaFreeAsync(scratch, s);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("ug_gat_attention: ") + cudaGetErrorString(e));
    return UG_OK;
}

// ------------------------------------------------------------------------- fused dot attention (f3)
extern "C" ug_status ug_dot_attention(const ug_graph *g, const float *q, int64_t ld_q, const float *k, int64_t ld_k,
                                      const float *val, int64_t ld_val, int32_t H, int32_t Dk, int32_t Dv,
                                      float scale, float *out, int64_t ld_out, float *attn, int64_t ld_attn,
                                      void *stream) {
    using namespace ug;
    if (!g) return set_error(UG_ERR_INVALID_ARG, "ug_dot_attention: NULL graph");
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_dot_attention needs a device graph");
    if (H <= 0 || Dk <= 0 || Dv <= 0) return set_error(UG_ERR_SHAPE, "ug_dot_attention: need H, Dk, Dv > 0");
    if (ld_q < (int64_t)H * Dk || ld_k < (int64_t)H * Dk || ld_val < (int64_t)H * Dv || ld_out < (int64_t)H * Dv ||
        (attn && ld_attn < H))
        return set_error(UG_ERR_SHAPE, "ug_dot_attention: ld < width");
    if (g->V > 0 && (!q || !out)) return set_error(UG_ERR_INVALID_ARG, "ug_dot_attention: NULL q / out");
    if (g->E > 0 && (!k || !val)) return set_error(UG_ERR_INVALID_ARG, "ug_dot_attention: NULL k / val");
    if (g->V == 0) return UG_OK;
    DotAttnArgs a;
    a.q = q; a.k = k; a.val = val;
    a.ld_q = ld_q; a.ld_k = ld_k; a.ld_val = ld_val;
    a.out = out; a.attn = attn; a.ld_out = ld_out; a.ld_attn = ld_attn;
    a.mden = nullptr;
    a.H = H; a.Dk = Dk; a.Dv = Dv;
    a.scale_log2 = scale * 1.4426950408889634f;
    const int vec = dotattn_vec(a);
    if (vec == 0) return set_error(UG_ERR_SHAPE, "ug_dot_attention: Dk and Dv must be <= 128 * vec (vec 4 / 2 / 1)");
    if ((uint64_t)g->V_total * (uint64_t)std::max(ld_k, ld_val) >= (1ull << 32))
        return set_error(UG_ERR_SHAPE, "ug_dot_attention: k / val above 2^32 elements");
    int G = 32;     // as the GAT traversal: split latency of the longest chunk vs merge cost
    if (const char *ev = std::getenv("UG_DOTATTN_CHUNK")) G = std::max(1, std::atoi(ev));
    const SplitPlan *plan = nullptr;
    ug_status st = get_plan(g, G, &plan);
    if (st != UG_OK) return st;
    if (plan->n_chunks * (int64_t)H >= ((int64_t)1 << 31) - 8)
        return set_error(UG_ERR_SHAPE, "ug_dot_attention: more than 2^31 (chunk, head) units");
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t sld = ((int64_t)Dv + 4 + 3) / 4 * 4;
    const size_t part = sizeof(float) * (size_t)plan->n_split_chunks * (size_t)H * (size_t)sld;
    const size_t md = attn ? sizeof(float) * (size_t)g->V * (size_t)H * 2 : 0;
    float *scratch = nullptr;
    if (part + md > 0) {
        ensure_pool_retains();
        if (cudaMallocAsync((void **)&scratch, part + md, s) != cudaSuccess)
            return set_error(UG_ERR_OOM, "ug_dot_attention: scratch allocation failed");
        if (attn) a.mden = reinterpret_cast<float *>(reinterpret_cast<char *>(scratch) + part);
    }
    cudaError_t e = launch_dotattn(graph_args(g), a, vec, *plan, scratch, sld, s);
    if (scratch) cudaFreeAsync(scratch, s);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("ug_dot_attention: ") + cudaGetErrorString(e));
    return UG_OK;
}

// ------------------------------------------------------------------------- arg capture (f2)
extern "C" ug_status ug_op_run_arg(const ug_graph *g, const ug_op_info *op, int32_t *arg, int64_t ld_arg,
                                   void *stream) {
    using namespace ug;
    Lowered lw;
    ug_status st = lower(g, op, &lw);
    if (st != UG_OK) return st;
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_op_run_arg needs a device graph");
    if (lw.to_edges || lw.dot || (lw.gather != UG_GATHER_MAX && lw.gather != UG_GATHER_MIN))
        return set_error(UG_ERR_UNSUPPORTED_OP, "ug_op_run_arg: max/min aggregation of an elementwise message only");
    if (!arg && g->V > 0) return set_error(UG_ERR_INVALID_ARG, "ug_op_run_arg: NULL arg");
    if (ld_arg < lw.args.W) return set_error(UG_ERR_SHAPE, "ug_op_run_arg: ld_arg < F");
    if (g->V == 0) return UG_OK;
    const int W = lw.args.W;
    int L = 1;
    while (L < 32 && L < W) L <<= 1;
    const int n_tiles = (W + L - 1) / L;
    const int G = 32;
    const SplitPlan *plan = nullptr;
    if ((st = get_plan(g, G, &plan)) != UG_OK) return st;
    if (plan->n_chunks * n_tiles >= (int64_t)1 << 31)
        return set_error(UG_ERR_SHAPE, "ug_op_run_arg: more than 2^31 (chunk, tile) units");
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t sld = (W + 3) / 4 * 4;
    float *scratch = nullptr;
    int32_t *counters = nullptr;
    if (plan->n_split_chunks > 0) {
        // partial values + partial args (per call, stream-ordered); this stream's arrival counters
        if ((st = get_counters(g, stream, G, n_tiles, plan->n_split_rows, &counters)) != UG_OK) return st;
        ensure_pool_retains();
        if (cudaMallocAsync((void **)&scratch, (size_t)plan->n_split_chunks * sld * 8, s) != cudaSuccess)
            return set_error(UG_ERR_OOM, "ug_op_run_arg: scratch allocation failed");
    }
    int32_t *sarg = scratch ? reinterpret_cast<int32_t *>(scratch + plan->n_split_chunks * sld) : nullptr;
    cudaError_t e = launch_argext(lw.kedge, lw.gather, graph_args(g), lw.args, L, *plan, plan->d_slot_row, scratch,
                                  sarg, sld, counters, arg, ld_arg, s);
    if (scratch) cudaFreeAsync(scratch, s);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("ug_op_run_arg: ") + cudaGetErrorString(e));
    return UG_OK;
}

extern "C" ug_status ug_arg_scatter(const ug_graph *g, const int32_t *arg, int64_t ld_arg, int32_t W,
                                    const float *grad, int64_t ld_grad, int32_t target_type, float *out,
                                    int64_t ld_out, int32_t out_width, void *stream) {
    using namespace ug;
    if (!g) return set_error(UG_ERR_INVALID_ARG, "ug_arg_scatter: NULL graph");
    if (g->host_only) return set_error(UG_ERR_INVALID_ARG, "ug_arg_scatter needs a device graph");
    if (target_type != UG_T_SRC_V && target_type != UG_T_EDGE)
        return set_error(UG_ERR_UNSUPPORTED_OP, "ug_arg_scatter: target must be a Src_V or Edge tensor");
    if (W <= 0 || out_width <= 0 || W % out_width != 0 || ld_arg < W || ld_grad < W || ld_out < out_width)
        return set_error(UG_ERR_SHAPE, "ug_arg_scatter: need out_width | W and ld >= width");
    if (g->V == 0) return UG_OK;
    if (!arg || !grad || !out) return set_error(UG_ERR_INVALID_ARG, "ug_arg_scatter: NULL data");
    const int32_t *src_of_eid = nullptr;
    if (target_type == UG_T_SRC_V && g->d_eid) {
        std::lock_guard<std::mutex> lock(g->mu);
        if (!g->d_src_of_eid) {
            std::vector<int32_t> h(g->E);
            for (int64_t k = 0; k < g->E; ++k) h[g->h_eid[k]] = g->h_col[k];
            void *d = nullptr;
            if (cudaMalloc(&d, std::max<size_t>(16, h.size() * 4)) != cudaSuccess)
                return set_error(UG_ERR_OOM, "ug_arg_scatter: allocation failed");
            g->plan_allocs.push_back(d);
            if (!h.empty() && cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess)
                return set_error(UG_ERR_CUDA, "ug_arg_scatter: upload failed");
            g->d_src_of_eid = (int32_t *)d;
        }
        src_of_eid = g->d_src_of_eid;
    }
    cudaError_t e = launch_argscatter(arg, ld_arg, grad, ld_grad, g->V, W, target_type == UG_T_SRC_V, g->d_col,
                                      src_of_eid, out, ld_out, W / out_width, (cudaStream_t)stream);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("ug_arg_scatter: ") + cudaGetErrorString(e));
    return UG_OK;
}
