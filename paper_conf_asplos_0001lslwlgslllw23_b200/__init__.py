"""ugraph-b200: the unified GNN graph operator of uGrapher (ASPLOS'23) on B200 (sm_100a).

Thin Python binding over the C ABI in include/ug.h (libugraph.so).  Everything here is
argument marshalling: torch supplies device memory and the current stream; every step of
the operator runs in the library's CUDA kernels.  There is no CPU fallback.

    g = Graph(V, src, dst)                         # ug_graph_create (COO -> in-CSR)
    op_run(g, "mul", "sum", A=X, a_type="u", B=w, b_type="e", C=Y, c_type="v")
                                                   # uGrapher(graph, op_info, parallel_info)
    schedule_select(g, ...)                        # parallel_info when absent
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _ffi
from ._ffi import (EDGE_OPS, GATHER_OPS, STRATEGIES, TTYPES, UgError, UgOpInfo, UgSchedule,
                   UgTensor, check, lib)

__all__ = ["Graph", "op_run", "prepare", "PreparedOp", "schedule_select", "launch_count", "parse_schedule",
           "format_schedule", "validate", "edge_permute", "selector_load", "selector_load_model", "gat_attention", "dot_attention", "op_run_arg", "arg_scatter", "reorder", "rows_gather", "Renumbered", "UgError", "scratch_trim",
           "version"]


def version():
    return lib.ug_version().decode()


def scratch_trim():
    """Return the per-call scratch the library's memory pool keeps reserved (ug_scratch_trim)."""
    check(lib.ug_scratch_trim(), "ug_scratch_trim")


_raw_stream = None


def _current_stream(stream):
    """cudaStream_t for a call: `stream` if given, else torch's current stream on the current
    device (the raw handle getter: ~0.3 us instead of ~3 us for a torch.cuda.Stream object,
    which matters for the C1/C2 ops whose device time is ~10 us; scripts/probe_host.py)."""
    global _raw_stream
    if stream is not None:
        return int(stream)
    if _raw_stream is None:
        import torch
        if torch.cuda.is_available():
            get = getattr(torch._C, "_cuda_getCurrentRawStream", None)
            cur = torch.cuda.current_device
            _raw_stream = ((lambda: get(cur())) if get is not None
                           else (lambda: torch.cuda.current_stream().cuda_stream))
        else:
            _raw_stream = lambda: 0  # noqa: E731  (host-only graphs; ug_op_run then rejects the call)
    return _raw_stream()


def _int32_buffer(x):
    """(pointer, on_device, keepalive) for an int32 array (numpy or torch, host or CUDA)."""
    try:
        import torch
        if isinstance(x, torch.Tensor):
            if x.dtype != torch.int32:
                raise TypeError("index tensors must be int32")
            x = x.contiguous()
            return x.data_ptr(), int(x.is_cuda), x
    except ImportError:
        pass
    a = np.ascontiguousarray(x, dtype=np.int32)
    return a.ctypes.data, 0, a


class Graph:
    """A destination-keyed CSR graph owned by libugraph (ug_graph)."""

    def __init__(self, num_vertices, src=None, dst=None, *, host_only=False, stream=None, _handle=None,
                 _parent=None):
        self._parent = _parent
        self._dims_cache = None
        self._host_only = bool(host_only) if _parent is None else _parent._host_only
        self._device = None
        if not self._host_only:
            import torch
            self._device = _parent._device if _parent is not None else torch.cuda.current_device()
        if _handle is not None:
            self._h = _handle
            return
        sp, sdev, ka = _int32_buffer(src)
        dp, ddev, kb = _int32_buffer(dst)
        if sdev != ddev:
            raise ValueError("src and dst must both be host or both device arrays")
        E = int(ka.shape[0])
        h = ctypes.c_void_p()
        flags = _ffi.UG_GRAPH_HOST_ONLY if host_only else 0
        st = lib.ug_graph_create(int(num_vertices), E, sp, dp, sdev, flags, None,
                                 None if host_only else _current_stream(stream), ctypes.byref(h))
        check(st, "ug_graph_create")
        self._h = h

    @classmethod
    def from_csr(cls, num_vertices, row_ptr, col_idx, eid=None, *, host_only=False, stream=None):
        rp, rdev, ka = _int32_buffer(row_ptr)
        cp, cdev, kb = _int32_buffer(col_idx)
        ep, kc = (None, None)
        if eid is not None:
            ep, _, kc = _int32_buffer(eid)
        h = ctypes.c_void_p()
        flags = _ffi.UG_GRAPH_HOST_ONLY if host_only else 0
        st = lib.ug_graph_create_csr(int(num_vertices), int(kb.shape[0]), rp, cp, ep, rdev, flags, None,
                                     None if host_only else _current_stream(stream), ctypes.byref(h))
        check(st, "ug_graph_create_csr")
        return cls(num_vertices, host_only=host_only, _handle=h)

    @property
    def handle(self):
        return self._h

    def __del__(self, _destroy=lib.ug_graph_destroy):   # bound at import: safe at interpreter exit
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            _destroy(h)
            self._h = None

    def stats(self):
        V, E, mx = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        mean, std = ctypes.c_double(), ctypes.c_double()
        check(lib.ug_graph_stats(self._h, ctypes.byref(V), ctypes.byref(E), ctypes.byref(mean),
                                 ctypes.byref(std), ctypes.byref(mx)), "ug_graph_stats")
        return {"V": V.value, "E": E.value, "mean_deg": mean.value, "std_nnz": std.value,
                "max_deg": mx.value}

    def dims(self):
        """(rows of a Src_V operand, rows of a Dst_V operand / aggregation output, rows of an Edge
        operand / message output): (V_total, V, E) -- for a view, V and E are its local rows and
        edges while Src_V operands still span the parent's vertex-id space."""
        if self._dims_cache is None:
            st = self.stats()
            vsrc = self._parent.dims()[0] if self._parent is not None else st["V"]
            self._dims_cache = (vsrc, st["V"], st["E"])
        return self._dims_cache

    @property
    def num_rows(self):
        return self.stats()["V"]

    @property
    def num_edges(self):
        return self.stats()["E"]

    def csr(self):
        s = self.stats()
        rp = np.zeros(s["V"] + 1, np.int32)
        col = np.zeros(max(s["E"], 1), np.int32)
        eid = np.zeros(max(s["E"], 1), np.int32)
        check(lib.ug_graph_csr(self._h, rp.ctypes.data, col.ctypes.data, eid.ctypes.data), "ug_graph_csr")
        return rp, col[:s["E"]], eid[:s["E"]]

    def row_ptr(self):
        """Host row_ptr[V+1] only (local positions for a view)."""
        rp = np.zeros(self.stats()["V"] + 1, np.int32)
        check(lib.ug_graph_csr(self._h, rp.ctypes.data, None, None), "ug_graph_csr")
        return rp

    def partition(self, parts):
        out = np.zeros(parts + 1, np.int64)
        check(lib.ug_graph_partition(self._h, int(parts), out.ctypes.data), "ug_graph_partition")
        return out

    def view_rows(self, r0, r1):
        h = ctypes.c_void_p()
        check(lib.ug_graph_view_rows(self._h, int(r0), int(r1), ctypes.byref(h)), "ug_graph_view_rows")
        return Graph(0, _handle=h, _parent=self)


def _tensor(x, ttype, graph=None):
    """ug_tensor for one operand.  The C ABI has no row count, so the rows each tensor type
    implies (Src_V: V_total, Dst_V: V, Edge: E, Graph.dims) are checked here, with the device and
    the row stride: a short, overlapping or off-device tensor would otherwise be read or written
    out of bounds by the kernels."""
    if x is None:
        return UgTensor(None, TTYPES[None], 0, 0)
    import torch
    if not isinstance(x, torch.Tensor):
        raise TypeError("operands must be torch tensors on the CUDA device")
    if x.dtype != torch.float32:
        raise TypeError("operands must be float32")
    if x.dim() == 1:
        x = x.view(-1, 1)
    if x.dim() != 2 or (x.shape[1] > 1 and x.stride(1) != 1):
        raise ValueError("operands must be 2-D with unit column stride")
    if x.shape[0] > 1 and x.stride(0) < x.shape[1]:
        raise ValueError("operand rows overlap (row stride < width, e.g. an expand()ed tensor)")
    if graph is not None:
        if graph._device is not None and (not x.is_cuda or x.device.index != graph._device):
            raise ValueError(f"operands must live on the graph's device cuda:{graph._device}")
        if ttype in TTYPES and ttype is not None:
            vsrc, v, e = graph.dims()
            need = {"u": vsrc, "v": v, "e": e}[ttype]
            if x.shape[0] < need:
                raise ValueError(f"a {ttype!r} operand needs {need} rows, got {x.shape[0]}")
    ld = x.stride(0) if x.shape[0] > 1 else x.shape[1]
    return UgTensor(x.data_ptr(), TTYPES[ttype], x.shape[1], max(ld, x.shape[1]))


def _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph=None):
    if F is None:
        ref = A if A is not None else B
        F = ref.shape[1] if ref.dim() == 2 else 1
        if edge_op == "dot" and C is not None and H is None:
            H = C.shape[1] if C.dim() == 2 else 1
    if H is None:
        H = 1
    return UgOpInfo(EDGE_OPS[edge_op], GATHER_OPS[gather_op], _tensor(A, a_type, graph), _tensor(B, b_type, graph),
                    _tensor(C, c_type, graph), int(F), int(H))


def parse_schedule(text):
    s = UgSchedule()
    check(lib.ug_schedule_parse(text.encode(), ctypes.byref(s)), f"ug_schedule_parse({text})")
    return s


def format_schedule(s):
    buf = ctypes.create_string_buffer(64)
    check(lib.ug_schedule_format(ctypes.byref(s), buf, 64), "ug_schedule_format")
    return buf.value.decode()


_sched_cache = {}


def _sched(schedule):
    if schedule is None:
        return None
    if isinstance(schedule, UgSchedule):
        return ctypes.byref(schedule)
    s = _sched_cache.get(schedule)
    if s is None:
        s = parse_schedule(schedule)
        if len(_sched_cache) < 4096:
            _sched_cache[schedule] = s
    return ctypes.byref(s)


def op_run(graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None, c_type="v",
           F=None, H=None, schedule=None, stream=None):
    """One unified-operator call (uGrapher(Graph_Tensor, op_info, parallel_info)).

    A, B, C: CUDA float32 tensors [rows, width] (row stride may exceed width); types are
    "u" (Src_V), "v" (Dst_V), "e" (Edge) or None.  C is written in place.  schedule: None
    (automatic) or Table 9 notation such as "TE_G1_T16" / "SV_G2048_F64".
    Asynchronous on `stream` (default: torch's current stream).
    """
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
    check(lib.ug_op_run(graph.handle, ctypes.byref(info), _sched(schedule), _current_stream(stream)),
          "ug_op_run")
    return C


def op_run_events(graph, edge_op, gather_op, ev_begin, ev_end, A=None, a_type=None, B=None, b_type=None,
                  C=None, c_type="v", F=None, H=None, schedule=None, stream=None):
    """op_run that also records torch.cuda.Event pair (ev_begin, ev_end) around the main kernel
    (measurement hook, ug_op_run_events).  The events must have been recorded once before."""
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
    check(lib.ug_op_run_events(graph.handle, ctypes.byref(info), _sched(schedule), _current_stream(stream),
                               ctypes.c_void_p(ev_begin.cuda_event), ctypes.c_void_p(ev_end.cuda_event)),
          "ug_op_run_events")
    return C


class PreparedOp:
    """An op_run call with its op_info / parallel_info marshalled once (serving loops, CUDA-graph
    capture).  The tensors' storage must stay alive and in place; call it like op_run."""

    def __init__(self, graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None,
                 c_type="v", F=None, H=None, schedule=None):
        self.info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
        check(lib.ug_op_validate(graph.handle, ctypes.byref(self.info)), "ug_op_validate")
        if schedule is None:
            self.sched = UgSchedule()
            check(lib.ug_schedule_select(graph.handle, ctypes.byref(self.info), ctypes.byref(self.sched)),
                  "ug_schedule_select")
        elif isinstance(schedule, UgSchedule):
            self.sched = schedule
        else:
            self.sched = parse_schedule(schedule)
        self.schedule = format_schedule(self.sched)
        self._keep = (graph, A, B, C)
        self._h = graph.handle
        self._iref = ctypes.byref(self.info)
        self._sref = ctypes.byref(self.sched)

    def __call__(self, stream=None):
        st = lib.ug_op_run(self._h, self._iref, self._sref, _current_stream(stream))
        if st != _ffi.UG_OK:
            raise UgError(st, "ug_op_run")


def prepare(graph, edge_op, gather_op, **kw):
    """PreparedOp factory: same arguments as op_run (schedule=None resolves AUTO once)."""
    return PreparedOp(graph, edge_op, gather_op, **kw)


def validate(graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None, c_type="v",
             F=None, H=None):
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
    check(lib.ug_op_validate(graph.handle, ctypes.byref(info)), "ug_op_validate")


def schedule_select(graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None,
                    c_type="v", F=None, H=None):
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
    s = UgSchedule()
    check(lib.ug_schedule_select(graph.handle, ctypes.byref(info), ctypes.byref(s)), "ug_schedule_select")
    return format_schedule(s)


def launch_count(graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None, c_type="v",
                 F=None, H=None, schedule=None):
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, c_type, F, H, graph)
    n = ctypes.c_int32()
    check(lib.ug_op_launch_count(graph.handle, ctypes.byref(info), _sched(schedule), ctypes.byref(n)),
          "ug_op_launch_count")
    return n.value


def edge_permute(graph, inp, out, stream=None):
    check(lib.ug_edge_permute(graph.handle, inp.data_ptr(), out.data_ptr(), inp.shape[1],
                              _current_stream(stream)), "ug_edge_permute")
    return out


def selector_load(path):
    check(lib.ug_selector_load(str(path).encode()), "ug_selector_load")


def selector_load_model(path):
    """Load the learned selector trees (ug_selector_load_model); "" unloads them."""
    check(lib.ug_selector_load_model(str(path).encode()), "ug_selector_load_model")


def _mat(x, name):
    import torch
    if not isinstance(x, torch.Tensor) or x.dtype != torch.float32 or not x.is_cuda:
        raise TypeError(f"{name} must be a float32 CUDA tensor")
    if x.dim() == 1:
        x = x.view(-1, 1)
    if x.dim() != 2 or (x.shape[1] > 1 and x.stride(1) != 1):
        raise ValueError(f"{name} must be 2-D with unit column stride")
    return x.data_ptr(), max(x.stride(0), x.shape[1])


def gat_attention(graph, el, er, z, heads, slope=0.2, out=None, attn=None, stream=None):
    """GAT attention chain in ONE traversal (ug_gat_attention):
    out[v] = sum over in-edges e=(u->v) of softmax_e(LeakyReLU(el[u] + er[v])) per head * z[u].
    el, er: [V, H]; z: [V, F] (H | F).  Returns out [V, F] (and fills attn [E, H] if given)."""
    import torch
    H = int(heads)
    F = int(z.shape[1])
    V = er.shape[0]
    if out is None:
        out = torch.empty(V, F, device=z.device, dtype=torch.float32)
    pel, lel = _mat(el, "el")
    per, ler = _mat(er, "er")
    pz, lz = _mat(z, "z")
    po, lo = _mat(out, "out")
    pa, la = (None, 0) if attn is None else _mat(attn, "attn")
    check(lib.ug_gat_attention(graph.handle, pel, lel, per, ler, pz, lz, F, H, float(slope), po, lo, pa, la,
                               _current_stream(stream)), "ug_gat_attention")
    return out


def dot_attention(graph, q, k, val, heads, scale=None, out=None, attn=None, stream=None):
    """Dot-product attention chain in ONE traversal (ug_dot_attention, the
    FusedMM-style SDDMM + SpMM of PAPER.md:588 from the operators of PAPER.md:224):
    out[v] = sum over in-edges e=(u->v) of softmax_e(scale * <q[v], k[u]>) per head * val[u].
    q: [V, H*Dk] (Dst_V rows), k: [V_total, H*Dk], val: [V_total, H*Dv] (Src_V rows); scale
    defaults to 1/sqrt(Dk).  Returns out [V, H*Dv] (and fills attn [E, H] if given)."""
    import torch
    H = int(heads)
    Dk = int(q.shape[1]) // H
    Dv = int(val.shape[1]) // H
    if Dk * H != q.shape[1] or Dv * H != val.shape[1] or k.shape[1] != q.shape[1]:
        raise ValueError("q / k widths must be H*Dk, val H*Dv")
    vsrc, V, E = graph.dims()
    if q.shape[0] < V or k.shape[0] < vsrc or val.shape[0] < vsrc:
        raise ValueError("q needs one row per destination vertex, k / val one per source id")
    if out is None:
        out = torch.empty(V, H * Dv, device=val.device, dtype=torch.float32)
    if scale is None:
        scale = 1.0 / float(Dk) ** 0.5
    pq, lq = _mat(q, "q")
    pk, lk = _mat(k, "k")
    pv, lv = _mat(val, "val")
    po, lo = _mat(out, "out")
    pa, la = (None, 0) if attn is None else _mat(attn, "attn")
    if attn is not None and attn.shape[0] < E:
        raise ValueError("attn needs one row per edge")
    check(lib.ug_dot_attention(graph.handle, pq, lq, pk, lk, pv, lv, H, Dk, Dv, float(scale), po, lo, pa, la,
                               _current_stream(stream)), "ug_dot_attention")
    return out


def op_run_arg(graph, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, C=None, F=None, H=None,
               arg=None, stream=None):
    """max/min aggregation with arg capture (ug_op_run_arg): fills C [V, F] as
    op_run would and returns arg [V, F] int32 = the supplying edge id (first on ties, -1 for
    zero in-degree rows)."""
    import torch
    info = _op_info(edge_op, gather_op, A, a_type, B, b_type, C, "v", F, H, graph)
    if arg is None:
        arg = torch.empty(C.shape[0], C.shape[1], dtype=torch.int32, device=C.device)
    if arg.dtype != torch.int32 or arg.dim() != 2 or arg.stride(1) != 1:
        raise TypeError("arg must be a 2-D int32 tensor with unit column stride")
    if not arg.is_cuda or arg.device != C.device or arg.shape[0] < C.shape[0] or arg.shape[1] < C.shape[1]:
        raise ValueError("arg must be an int32 CUDA tensor on C's device with at least C's shape")
    check(lib.ug_op_run_arg(graph.handle, ctypes.byref(info), arg.data_ptr(), max(arg.stride(0), arg.shape[1]),
                            _current_stream(stream)), "ug_op_run_arg")
    return arg


def arg_scatter(graph, arg, grad, target_type, out, stream=None):
    """out[row(e)][f / (W / out_width)] += grad[v][f] for e = arg[v][f] >= 0 (ug_arg_scatter);
    target_type "u" (row = src of e) or "e" (row = e)."""
    import torch
    if not isinstance(arg, torch.Tensor) or arg.dtype != torch.int32 or not arg.is_cuda or arg.dim() != 2 \
            or arg.stride(1) != 1:
        raise TypeError("arg must be a 2-D int32 CUDA tensor with unit column stride (from op_run_arg)")
    if arg.shape[0] < graph.dims()[1] or grad.shape[0] < graph.dims()[1] or grad.shape[1] != arg.shape[1]:
        raise ValueError("arg / grad need one row per destination vertex and equal widths")
    rows_out = graph.dims()[0] if target_type == "u" else graph.dims()[2]
    if out.shape[0] < rows_out:
        raise ValueError(f"out needs {rows_out} rows")
    W = int(arg.shape[1])
    pg, lg = _mat(grad, "grad")
    po, lo = _mat(out, "out")
    check(lib.ug_arg_scatter(graph.handle, arg.data_ptr(), max(arg.stride(0), W), W, pg, lg, TTYPES[target_type],
                             po, lo, int(out.shape[1] if out.dim() == 2 else 1), _current_stream(stream)),
          "ug_arg_scatter")
    return out


ORDERS = {"degree": 1, "rcm": 2, "community": 3}


def reorder(graph, method="rcm"):
    """perm[new_id] = old_id (ug_graph_reorder: "degree", "rcm" or "community")."""
    V = graph.stats()["V"]
    perm = np.zeros(max(V, 1), np.int32)
    check(lib.ug_graph_reorder(graph.handle, ORDERS[method], perm.ctypes.data), "ug_graph_reorder")
    return perm[:V]


def rows_gather(X, idx, out=None, stream=None):
    """out[i] = X[idx[i]] on the device (ug_rows_gather); idx: int32 CUDA tensor."""
    import torch
    if out is None:
        out = torch.empty(idx.shape[0], X.shape[1], device=X.device, dtype=X.dtype)
    px, lx = _mat(X, "X")
    po, lo = _mat(out, "out")
    if idx.dtype != torch.int32 or not idx.is_cuda:
        raise TypeError("idx must be an int32 CUDA tensor")
    check(lib.ug_rows_gather(px, lx, idx.data_ptr(), int(idx.shape[0]), int(X.shape[1]), po, lo,
                             _current_stream(stream)), "ug_rows_gather")
    return out


class Renumbered:
    """A graph renumbered for locality: `graph` is built on the new vertex ids from the COO
    re-sorted by new destination, so its EDGE IDS ARE NEW TOO (the new CSR positions).
    to_new(X) / to_old(Y) move vertex tensors between numberings; edges_to_new(W) moves an
    edge tensor given in the original edge-id order into the new order (before a call), and
    edges_to_old(M) moves an edge output (message creation, GAT attention) back (after)."""

    def __init__(self, num_vertices, src, dst, method="rcm"):
        import torch
        src = np.ascontiguousarray(src, np.int32)
        dst = np.ascontiguousarray(dst, np.int32)
        base = Graph(num_vertices, src, dst, host_only=True)
        self.perm = reorder(base, method)
        self.inv = np.empty_like(self.perm)
        self.inv[self.perm] = np.arange(len(self.perm), dtype=np.int32)
        nsrc, ndst = self.inv[src], self.inv[dst]
        order = np.argsort(ndst, kind="stable")          # dst-sorted: identity edge positions
        self.edge_order = order.astype(np.int32)         # new CSR position -> original edge id
        self.graph = Graph(num_vertices, nsrc[order], ndst[order])
        self._perm_d = torch.from_numpy(self.perm).cuda()
        self._inv_d = torch.from_numpy(self.inv).cuda()
        self._eord_d = torch.from_numpy(self.edge_order).cuda()
        inv_e = np.empty_like(self.edge_order)
        inv_e[self.edge_order] = np.arange(len(self.edge_order), dtype=np.int32)
        self._einv_d = torch.from_numpy(inv_e).cuda()       # original edge id -> new position

    def to_new(self, X):
        return rows_gather(X, self._perm_d)

    def to_old(self, Y):
        return rows_gather(Y, self._inv_d)

    def edges_to_new(self, W):
        """Edge tensor in original edge-id order -> the renumbered graph's edge order."""
        return rows_gather(W, self._eord_d)

    def edges_to_old(self, M):
        """Edge tensor in the renumbered graph's edge order -> original edge-id order."""
        return rows_gather(M, self._einv_d)
