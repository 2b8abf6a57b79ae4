// ug_graph.cpp -- graph object of libugraph: COO/CSR ingest (step a1), statistics
// (Table 7), edge-balanced partition and zero-copy row views (north
// star (4)).  Host-side C++; device arrays through the caller's allocator or
// cudaMallocAsync.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>
#include <string>

#include "ug_internal.h"
#include "ug_runtime.h"

using ug::set_error;

namespace {

void *dev_alloc(ug_graph *g, size_t bytes, cudaStream_t s) {
    if (bytes == 0) bytes = 4;
    void *p = nullptr;
    if (g->has_alloc) {
        p = g->alloc.alloc(bytes, g->alloc.ctx, s);
    } else if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) {
        p = nullptr;
    }
    if (p) g->owned.push_back(p);
    return p;
}

// Host CSR -> device arrays; stats.  g->h_* vectors must be filled.
ug_status finish_graph(ug_graph *g, const ug_allocator *alloc, cudaStream_t s) {
    g->h_row_ptr = g->h_row_ptr_v.data();
    g->h_col = g->h_col_v.data();
    g->h_eid = g->eid_identity ? nullptr : g->h_eid_v.data();
    // Table 7 stats: mean in-degree, population std of in-degree (R15), max.
    const int64_t V = g->V;
    double s1 = 0.0;
    int64_t mx = 0;
    const double mean = V > 0 ? (double)g->E / (double)V : 0.0;
    for (int64_t v = 0; v < V; ++v) {
        const int64_t d = (int64_t)g->h_row_ptr[v + 1] - g->h_row_ptr[v];
        s1 += ((double)d - mean) * ((double)d - mean);
        mx = std::max(mx, d);
    }
    g->mean_deg = mean;
    g->std_nnz = V > 0 ? std::sqrt(s1 / (double)V) : 0.0;
    g->max_deg = mx;
    if (g->host_only) return UG_OK;

    if (alloc) {
        g->has_alloc = true;
        g->alloc = *alloc;
    }
    if (cudaGetDevice(&g->device) != cudaSuccess) return set_error(UG_ERR_CUDA, "cudaGetDevice failed");
    const size_t rp = sizeof(int32_t) * (size_t)(V + 1), ne = sizeof(int32_t) * (size_t)g->E;
    g->d_row_ptr = (int32_t *)dev_alloc(g, rp, s);
    g->d_col = (int32_t *)dev_alloc(g, ne + 64, s);   // +64 B: a 16-byte-rounded bulk copy of the tail stays in bounds
    g->d_dst = (int32_t *)dev_alloc(g, ne, s);
    if (!g->eid_identity) g->d_eid = (int32_t *)dev_alloc(g, ne, s);
    if (!g->d_row_ptr || !g->d_col || !g->d_dst || (!g->eid_identity && !g->d_eid))
        return set_error(UG_ERR_OOM, "device allocation of the CSR failed");
    cudaError_t e = cudaMemcpyAsync(g->d_row_ptr, g->h_row_ptr, rp, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && ne) e = cudaMemcpyAsync(g->d_col, g->h_col, ne, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && ne) e = cudaMemcpyAsync(g->d_dst, g->h_dst_v.data(), ne, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && ne && !g->eid_identity)
        e = cudaMemcpyAsync(g->d_eid, g->h_eid_v.data(), ne, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return set_error(UG_ERR_CUDA, std::string("graph upload: ") + cudaGetErrorString(e));
    return UG_OK;
}

template <typename T>
bool fetch_input(std::vector<T> &out, const T *p, int64_t n, int on_device) {
    out.resize((size_t)n);
    if (n == 0) return true;
    if (on_device) return cudaMemcpy(out.data(), p, sizeof(T) * (size_t)n, cudaMemcpyDeviceToHost) == cudaSuccess;
    std::memcpy(out.data(), p, sizeof(T) * (size_t)n);
    return true;
}

}  // namespace

extern "C" ug_status ug_graph_create(int64_t V, int64_t E, const int32_t *src, const int32_t *dst,
                                     int on_device, int flags, const ug_allocator *alloc, void *stream,
                                     ug_graph **out) {
    if (!out || V < 0 || E < 0 || E >= (int64_t(1) << 31) || V >= (int64_t(1) << 31) ||
        (E > 0 && (!src || !dst)))
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_create: bad arguments");
    *out = nullptr;
    ug_graph *g = new (std::nothrow) ug_graph();
    if (!g) return UG_ERR_OOM;
    g->V = V;
    g->V_total = V;
    g->E = E;
    g->host_only = (flags & UG_GRAPH_HOST_ONLY) != 0;
    std::vector<int32_t> hs, hd;
    if (!fetch_input(hs, src, E, on_device) || !fetch_input(hd, dst, E, on_device)) {
        delete g;
        return set_error(UG_ERR_CUDA, "ug_graph_create: copying COO from device failed");
    }
    bool sorted = true;
    for (int64_t e = 0; e < E; ++e) {
        if (hs[e] < 0 || hs[e] >= V || hd[e] < 0 || hd[e] >= V) {
            delete g;
            return set_error(UG_ERR_INDEX_RANGE, "ug_graph_create: vertex id out of range at edge " + std::to_string(e));
        }
        if (e > 0 && hd[e] < hd[e - 1]) sorted = false;
    }
    // Stable counting sort by dst (edge-id order inside a row, R10): row_ptr by an
    // exclusive scan of the in-degree histogram.
    g->h_row_ptr_v.assign((size_t)V + 1, 0);
    for (int64_t e = 0; e < E; ++e) g->h_row_ptr_v[hd[e] + 1]++;
    for (int64_t v = 0; v < V; ++v) g->h_row_ptr_v[v + 1] += g->h_row_ptr_v[v];
    g->eid_identity = sorted;
    if (sorted) {
        g->h_col_v = std::move(hs);
        g->h_dst_v = std::move(hd);
    } else {
        g->h_col_v.resize((size_t)E);
        g->h_dst_v.resize((size_t)E);
        g->h_eid_v.resize((size_t)E);
        std::vector<int32_t> fill(g->h_row_ptr_v.begin(), g->h_row_ptr_v.end() - 1);
        for (int64_t e = 0; e < E; ++e) {
            const int32_t k = fill[hd[e]]++;
            g->h_col_v[k] = hs[e];
            g->h_dst_v[k] = hd[e];
            g->h_eid_v[k] = (int32_t)e;
        }
    }
    ug_status st = finish_graph(g, alloc, (cudaStream_t)stream);
    if (st != UG_OK) {
        ug_graph_destroy(g);
        return st;
    }
    *out = g;
    return UG_OK;
}

extern "C" ug_status ug_graph_create_csr(int64_t V, int64_t E, const int32_t *row_ptr, const int32_t *col_idx,
                                         const int32_t *eid, int on_device, int flags,
                                         const ug_allocator *alloc, void *stream, ug_graph **out) {
    if (!out || V < 0 || E < 0 || E >= (int64_t(1) << 31) || !row_ptr || (E > 0 && !col_idx))
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_create_csr: bad arguments");
    *out = nullptr;
    ug_graph *g = new (std::nothrow) ug_graph();
    if (!g) return UG_ERR_OOM;
    g->V = V;
    g->V_total = V;
    g->E = E;
    g->host_only = (flags & UG_GRAPH_HOST_ONLY) != 0;
    if (!fetch_input(g->h_row_ptr_v, row_ptr, V + 1, on_device) || !fetch_input(g->h_col_v, col_idx, E, on_device) ||
        (eid && !fetch_input(g->h_eid_v, eid, E, on_device))) {
        delete g;
        return set_error(UG_ERR_CUDA, "ug_graph_create_csr: copying CSR from device failed");
    }
    if (g->h_row_ptr_v[0] != 0 || g->h_row_ptr_v[V] != E) {
        delete g;
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_create_csr: row_ptr[0] != 0 or row_ptr[V] != E");
    }
    g->h_dst_v.resize((size_t)E);
    for (int64_t v = 0; v < V; ++v) {
        if (g->h_row_ptr_v[v + 1] < g->h_row_ptr_v[v]) {
            delete g;
            return set_error(UG_ERR_INVALID_ARG, "ug_graph_create_csr: row_ptr decreases");
        }
        for (int64_t k = g->h_row_ptr_v[v]; k < g->h_row_ptr_v[v + 1]; ++k) g->h_dst_v[k] = (int32_t)v;
    }
    g->eid_identity = true;
    for (int64_t k = 0; k < E; ++k) {
        if (g->h_col_v[k] < 0 || g->h_col_v[k] >= V) {
            delete g;
            return set_error(UG_ERR_INDEX_RANGE, "ug_graph_create_csr: col_idx out of range");
        }
        if (eid) {
            if (g->h_eid_v[k] < 0 || g->h_eid_v[k] >= E) {
                delete g;
                return set_error(UG_ERR_INDEX_RANGE, "ug_graph_create_csr: eid out of range");
            }
            if (g->h_eid_v[k] != k) g->eid_identity = false;
        }
    }
    if (g->eid_identity) g->h_eid_v.clear();
    ug_status st = finish_graph(g, alloc, (cudaStream_t)stream);
    if (st != UG_OK) {
        ug_graph_destroy(g);
        return st;
    }
    *out = g;
    return UG_OK;
}

extern "C" ug_status ug_graph_destroy(ug_graph *g) {
    if (!g) return UG_ERR_INVALID_ARG;
    if (!g->host_only) {
        // kernels on any stream (torch's non-blocking streams included) may still read the CSR or
        // the plans: wait for the device before the memory can be handed to another allocation
        cudaDeviceSynchronize();
        for (void *p : g->owned) {
            if (g->has_alloc) g->alloc.free(p, g->alloc.ctx, nullptr);
            else cudaFree(p);
        }
        for (void *p : g->plan_allocs) cudaFree(p);
    }
    delete g;
    return UG_OK;
}

extern "C" ug_status ug_graph_stats(const ug_graph *g, int64_t *V, int64_t *E, double *mean_deg,
                                    double *std_nnz, int64_t *max_deg) {
    if (!g) return set_error(UG_ERR_INVALID_ARG, "ug_graph_stats: NULL graph");
    if (V) *V = g->V;
    if (E) *E = g->E;
    if (mean_deg) *mean_deg = g->mean_deg;
    if (std_nnz) *std_nnz = g->std_nnz;
    if (max_deg) *max_deg = g->max_deg;
    return UG_OK;
}

extern "C" ug_status ug_graph_csr(const ug_graph *g, int32_t *row_ptr, int32_t *col_idx, int32_t *eid) {
    if (!g) return set_error(UG_ERR_INVALID_ARG, "ug_graph_csr: NULL graph");
    const int64_t base = g->e0;
    if (row_ptr)
        for (int64_t v = 0; v <= g->V; ++v) row_ptr[v] = (int32_t)(g->h_row_ptr[v] - base);
    if (col_idx && g->E) std::memcpy(col_idx, g->h_col, sizeof(int32_t) * (size_t)g->E);
    if (eid) {
        for (int64_t k = 0; k < g->E; ++k) eid[k] = g->h_eid ? g->h_eid[k] : (int32_t)k;
    }
    return UG_OK;
}

extern "C" ug_status ug_graph_partition(const ug_graph *g, int32_t parts, int64_t *splits) {
    if (!g || parts < 1 || !splits) return set_error(UG_ERR_INVALID_ARG, "ug_graph_partition: bad arguments");
    // r_k = smallest row with row_ptr[r] - base >= ceil(k E / P): binary search (R21).
    const int64_t E = g->E, V = g->V, base = g->e0;
    const int32_t *rp = g->h_row_ptr;
    splits[0] = 0;
    for (int32_t k = 1; k < parts; ++k) {
        const int64_t target = (E * k + parts - 1) / parts;
        int64_t lo = 0, hi = V;   // answer in [0, V]
        while (lo < hi) {
            const int64_t mid = (lo + hi) / 2;
            if ((int64_t)rp[mid] - base >= target) hi = mid;
            else lo = mid + 1;
        }
        splits[k] = lo;
    }
    splits[parts] = V;
    return UG_OK;
}

extern "C" ug_status ug_graph_view_rows(const ug_graph *g, int64_t r0, int64_t r1, ug_graph **view) {
    if (!g || !view || r0 < 0 || r1 < r0 || r1 > g->V)
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_view_rows: bad range");
    if (!g->eid_identity)
        return set_error(UG_ERR_INVALID_ARG, "ug_graph_view_rows: graph is not dst-sorted (permute edge tensors)");
    ug_graph *w = new (std::nothrow) ug_graph();
    if (!w) return UG_ERR_OOM;
    w->is_view = true;
    w->parent = g;
    w->host_only = g->host_only;
    w->V_total = g->V_total;
    w->r0 = g->r0 + r0;
    w->V = r1 - r0;
    const int64_t k0 = (int64_t)g->h_row_ptr[r0] - g->e0;       // local position in g
    const int64_t k1 = (int64_t)g->h_row_ptr[r1] - g->e0;
    w->E = k1 - k0;
    w->e0 = g->h_row_ptr[r0];
    w->eid_identity = true;
    w->h_row_ptr = g->h_row_ptr + r0;
    w->h_col = g->h_col + k0;
    w->h_eid = nullptr;
    if (!g->host_only) {
        w->d_row_ptr = g->d_row_ptr + r0;
        w->d_col = g->d_col + k0;
        w->d_dst = g->d_dst + k0;
        w->device = g->device;
    }
    double s1 = 0.0;
    int64_t mx = 0;
    const double mean = w->V > 0 ? (double)w->E / (double)w->V : 0.0;
    for (int64_t v = 0; v < w->V; ++v) {
        const int64_t d = (int64_t)w->h_row_ptr[v + 1] - w->h_row_ptr[v];
        s1 += ((double)d - mean) * ((double)d - mean);
        mx = std::max(mx, d);
    }
    w->mean_deg = mean;
    w->std_nnz = w->V > 0 ? std::sqrt(s1 / (double)w->V) : 0.0;
    w->max_deg = mx;
    *view = w;
    return UG_OK;
}
