"""Backward of the sum / mean aggregations through the same unified operator (SURVEY 8(f) f2:
out-edge operators, "transposed aggregation for grad of copy_u_sum").

The paper is inference-only; training needs get_outedges, i.e.
the reversed graph.  Every backward step is again a graph operator of the 160-op set:
  * d/dX of copy_u_sum(X)         = copy_u_sum over the reversed graph of dY
  * d/dX of copy_u_mean(X)        = u_div_e_sum over the reversed graph of (dY, deg_e), deg_e =
    the in-degree of edge e's destination (one IEEE division per message, in the kernel)
  * d/dX of u_mul_e_sum(X, w)     = u_mul_e_sum over the reversed graph of (dY, w)
    (the reversed graph is built from the same COO with src / dst swapped, so edge ids -- and
    hence the rows of w -- are unchanged)
  * d/dw of u_mul_e_sum(X, w)     = u_dot_v message creation over the forward graph:
    dw[e, h] = sum_{d in head h} X[src(e)][d] * dY[dst(e)][d]
  * d/dX of copy_u_max / copy_u_min(X) and d/dE of copy_e_max / copy_e_min(E): the forward
    records which in-edge supplied every output element (ug_op_run_arg; first edge id on
    ties) and the backward scatters dY to that edge's source row (or to the edge itself)
    with ug_arg_scatter
"""
from __future__ import annotations

import numpy as np
import torch

from . import Graph, arg_scatter, op_run, op_run_arg


class GraphPair:
    """A graph and its reverse (out-edge CSR), sharing edge ids."""

    def __init__(self, num_vertices, src, dst):
        self.V = int(num_vertices)
        src = np.ascontiguousarray(src, dtype=np.int32)
        dst = np.ascontiguousarray(dst, dtype=np.int32)
        self.fwd = Graph(self.V, src, dst)
        self.rev = Graph(self.V, dst, src)
        deg = np.bincount(dst, minlength=self.V).astype(np.float32)
        self.in_deg = torch.from_numpy(deg)
        self._deg_e_host = torch.from_numpy(deg[dst].reshape(-1, 1).copy())   # graph structure, once
        self._deg_e = {}

    def deg_e(self, device):
        """[E, 1]: in-degree of each edge's destination (edge-id order), the mean backward's divisor."""
        if device not in self._deg_e:
            self._deg_e[device] = self._deg_e_host.to(device)
        return self._deg_e[device]


def _agg(graph, edge_op, gather_op, X, w=None, F=None, H=1):
    F = F or X.shape[1]
    Y = torch.empty(X.shape[0] if graph is None else graph.stats()["V"], F, device=X.device)
    op_run(graph, edge_op, gather_op, A=X.contiguous(), a_type="u", B=None if w is None else w.contiguous(),
           b_type=None if w is None else "e", C=Y, c_type="v", F=F, H=H)
    return Y


class _CopyUReduce(torch.autograd.Function):
    @staticmethod
    def forward(ctx, gp, X, mean):
        ctx.gp, ctx.mean = gp, mean
        return _agg(gp.fwd, "copy_lhs", "mean" if mean else "sum", X)

    @staticmethod
    def backward(ctx, dY):
        gp = ctx.gp
        g = dY.contiguous()
        if ctx.mean:
            # dX[u] = sum over out-edges e = (u -> v) of dY[v] / deg(v): u_div_e_sum on the reverse
            return None, _agg(gp.rev, "div", "sum", g, gp.deg_e(g.device)), None
        return None, _agg(gp.rev, "copy_lhs", "sum", g), None


class _UMulESum(torch.autograd.Function):
    @staticmethod
    def forward(ctx, gp, X, w):
        ctx.gp = gp
        ctx.save_for_backward(X, w)
        H = w.shape[1]
        return _agg(gp.fwd, "mul", "sum", X, w, H=H)

    @staticmethod
    def backward(ctx, dY):
        gp = ctx.gp
        X, w = ctx.saved_tensors
        dY = dY.contiguous()
        H = w.shape[1]
        dX = dw = None
        if ctx.needs_input_grad[1]:
            dX = _agg(gp.rev, "mul", "sum", dY, w, H=H)
        if ctx.needs_input_grad[2]:
            dw = torch.empty(w.shape[0], H, device=w.device)
            op_run(gp.fwd, "dot", "assign", A=X.contiguous(), a_type="u", B=dY, b_type="v", C=dw, c_type="e",
                   F=X.shape[1], H=H)
        return None, dX, dw


def copy_u_sum(gp: GraphPair, X):
    return _CopyUReduce.apply(gp, X, False)


def copy_u_mean(gp: GraphPair, X):
    return _CopyUReduce.apply(gp, X, True)


def u_mul_e_sum(gp: GraphPair, X, w):
    """w: [E, H] per-edge (per-head) weights; X: [V, F] with H | F."""
    if w.dim() == 1:
        w = w.view(-1, 1)
    return _UMulESum.apply(gp, X, w)


class _CopyExtreme(torch.autograd.Function):
    @staticmethod
    def forward(ctx, gp, X, a_type, gather):
        F = X.shape[1]
        Y = torch.empty(gp.V, F, device=X.device)
        arg = op_run_arg(gp.fwd, "copy_lhs", gather, A=X.contiguous(), a_type=a_type, C=Y, F=F)
        ctx.gp, ctx.a_type, ctx.rows = gp, a_type, X.shape[0]
        ctx.save_for_backward(arg)
        return Y

    @staticmethod
    def backward(ctx, dY):
        (arg,) = ctx.saved_tensors
        dX = torch.zeros(ctx.rows, dY.shape[1], device=dY.device)
        arg_scatter(ctx.gp.fwd, arg, dY.contiguous(), ctx.a_type, dX)
        return None, dX, None, None


def copy_u_max(gp: GraphPair, X):
    return _CopyExtreme.apply(gp, X, "u", "max")


def copy_u_min(gp: GraphPair, X):
    return _CopyExtreme.apply(gp, X, "u", "min")


def copy_e_max(gp: GraphPair, Ee):
    """Ee: [E, F] edge features in edge-id order."""
    return _CopyExtreme.apply(gp, Ee, "e", "max")


def copy_e_min(gp: GraphPair, Ee):
    return _CopyExtreme.apply(gp, Ee, "e", "min")
