// ug_reorder.cpp -- vertex renumbering for locality (node
// renumbering such as Rabbit order is orthogonal preprocessing, Fig. 19 evaluates it).
//
// The unified operator gathers one source row per in-edge, so the cache footprint of a run
// of destination rows is the set of their sources.  Renumbering vertices so that neighbours
// get nearby ids turns those gathers into reuse of recently touched L2 lines (and of the SV
// schedule's column slab).  Two host-side orders:
//   UG_ORDER_DEGREE -- descending total degree (in + out), ties by id: hot rows contiguous;
//   UG_ORDER_RCM    -- reverse Cuthill-McKee on the symmetrised graph: BFS from a minimum-
//                      degree vertex of each component, neighbours visited in ascending
//                      degree, the whole order reversed (bandwidth reduction; good for
//                      mesh-like graphs, weak on small-world graphs whose BFS levels explode);
//   UG_ORDER_COMMUNITY -- community order in the spirit of Rabbit order (the renumbering of
//                      PAPER.md:566 / Fig. 19): communities found by label propagation on the
//                      symmetrised graph (10 sweeps, vertices in a fixed pseudo-random order,
//                      each adopting the most frequent neighbour label, ties to the smaller
//                      label), then vertices grouped by community (communities by first
//                      appearance), descending degree inside a community.
// Plain C++ (one thread), O(E log d); the permutation is returned to the caller, who
// renumbers the COO and gathers the vertex tensors with ug_rows_gather.
#include <cuda_runtime.h>

#include <algorithm>
#include <numeric>
#include <vector>

#include "ug_internal.h"
#include "ug_runtime.h"

namespace ug {
cudaError_t launch_rows_gather(const float *in, int64_t ld_in, const int32_t *idx, int64_t rows, int width,
                               float *out, int64_t ld_out, cudaStream_t s);
}

extern "C" ug_status ug_graph_reorder(const ug_graph *g, int32_t method, int32_t *perm) {
    using namespace ug;
    if (!g || !perm) return set_error(UG_ERR_INVALID_ARG, "ug_graph_reorder: NULL argument");
    if (g->is_view || g->V != g->V_total)
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_reorder: needs a whole square graph (not a view)");
    if (method != UG_ORDER_DEGREE && method != UG_ORDER_RCM && method != UG_ORDER_COMMUNITY)
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_reorder: unknown method");
    const int64_t V = g->V, E = g->E;
    // symmetrised adjacency: in-neighbours from the CSR, out-neighbours by a counting sort
    std::vector<int64_t> deg(V, 0);
    for (int64_t v = 0; v < V; ++v) deg[v] += (int64_t)g->h_row_ptr[v + 1] - g->h_row_ptr[v];
    for (int64_t k = 0; k < E; ++k) deg[g->h_col[k]] += 1;
    std::vector<int32_t> order(V);
    std::iota(order.begin(), order.end(), 0);
    if (method == UG_ORDER_DEGREE) {
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return deg[a] > deg[b]; });
        std::copy(order.begin(), order.end(), perm);
        return UG_OK;
    }
    std::vector<int64_t> ptr(V + 1, 0);
    for (int64_t v = 0; v < V; ++v) ptr[v + 1] = ptr[v] + deg[v];
    std::vector<int32_t> adj(ptr[V]);
    std::vector<int64_t> fill(ptr.begin(), ptr.end() - 1);
    for (int64_t v = 0; v < V; ++v)
        for (int64_t k = (int64_t)g->h_row_ptr[v] - g->e0; k < (int64_t)g->h_row_ptr[v + 1] - g->e0; ++k) {
            const int32_t u = g->h_col[k];
            adj[fill[v]++] = u;
            adj[fill[u]++] = (int32_t)v;
        }
    if (method == UG_ORDER_COMMUNITY) {
        std::vector<int32_t> label(V), visit(V);
        std::iota(label.begin(), label.end(), 0);
        std::iota(visit.begin(), visit.end(), 0);
        uint64_t x = 0x9E3779B97F4A7C15ull;                // fixed seed: deterministic order
        for (int64_t i = V - 1; i > 0; --i) {
            x ^= x << 13; x ^= x >> 7; x ^= x << 17;
            std::swap(visit[i], visit[(int64_t)(x % (uint64_t)(i + 1))]);
        }
        std::vector<int32_t> nl;
        for (int sweep = 0; sweep < 10; ++sweep) {
            int64_t changed = 0;
            for (int32_t v : visit) {
                if (ptr[v] == ptr[v + 1]) continue;
                nl.assign(adj.begin() + ptr[v], adj.begin() + ptr[v + 1]);
                for (int32_t &u : nl) u = label[u];
                std::sort(nl.begin(), nl.end());
                int32_t best = label[v];
                int64_t best_n = 0;
                for (size_t i = 0; i < nl.size();) {
                    size_t j = i;
                    while (j < nl.size() && nl[j] == nl[i]) ++j;
                    if ((int64_t)(j - i) > best_n) { best_n = (int64_t)(j - i); best = nl[i]; }
                    i = j;
                }
                if (best != label[v]) { label[v] = best; ++changed; }
            }
            if (changed * 1000 < V) break;                   // < 0.1 % of labels moved
        }
        // communities in order of first appearance (by vertex id), degree-descending inside
        std::vector<int64_t> rank(V, -1);
        int64_t nc = 0;
        for (int64_t v = 0; v < V; ++v)
            if (rank[label[v]] < 0) rank[label[v]] = nc++;
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
            const int64_t ra = rank[label[a]], rb = rank[label[b]];
            return ra != rb ? ra < rb : deg[a] > deg[b];
        });
        std::copy(order.begin(), order.end(), perm);
        return UG_OK;
    }
    // start vertices: ascending degree (peripheral-ish), ties by id
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return deg[a] < deg[b]; });
    std::vector<char> seen(V, 0);
    std::vector<int32_t> res;
    res.reserve(V);
    std::vector<int32_t> nb;
    for (int32_t s0 : order) {
        if (seen[s0]) continue;
        seen[s0] = 1;
        size_t head = res.size();
        res.push_back(s0);
        while (head < res.size()) {
            const int32_t u = res[head++];
            nb.clear();
            for (int64_t k = ptr[u]; k < ptr[u + 1]; ++k)
                if (!seen[adj[k]]) {
                    seen[adj[k]] = 1;
                    nb.push_back(adj[k]);
                }
            std::stable_sort(nb.begin(), nb.end(), [&](int32_t a, int32_t b) { return deg[a] < deg[b]; });
            res.insert(res.end(), nb.begin(), nb.end());
        }
    }
    std::reverse(res.begin(), res.end());
    std::copy(res.begin(), res.end(), perm);
    return UG_OK;
}

extern "C" ug_status ug_rows_gather(const float *in, int64_t ld_in, const int32_t *idx, int64_t rows, int32_t width,
                                    float *out, int64_t ld_out, void *stream) {
    using namespace ug;
    if (rows < 0 || width <= 0 || ld_in < width || ld_out < width)
        return set_error(UG_ERR_SHAPE, "ug_rows_gather: bad shape");
    if (rows == 0) return UG_OK;
    if (!in || !idx || !out) return set_error(UG_ERR_INVALID_ARG, "ug_rows_gather: NULL argument");
    cudaError_t e = launch_rows_gather(in, ld_in, idx, rows, width, out, ld_out, (cudaStream_t)stream);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("ug_rows_gather: ") + cudaGetErrorString(e));
    return UG_OK;
}
