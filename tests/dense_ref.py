"""Dense brute-force formulation of the graph operators (test-only pin for the oracle).

Independent of oracle/ug_oracle.c: no in-edge lists, no loops over edges.  The graph is
held as dense one-hot incidence matrices S[E,V] (src) and T[E,V] (dst); operand rows are
gathered by matrix products (exact: one-hot), aggregation is T^T @ M, i.e. the adjacency
product the north star names ("sum aggregation equals A.X"), mean is D^-1 A X, max/min
are masked dense reductions over the [V, E] mask.  fp64 except where the definition
fixes fp32 (each message rounded once, R11).  Only for tiny graphs (V, E <= a few hundred).
"""
import numpy as np


def incidence(V, src, dst):
    E = len(src)
    S = np.zeros((E, V))
    T = np.zeros((E, V))
    S[np.arange(E), src] = 1.0
    T[np.arange(E), dst] = 1.0
    return S, T


def adjacency(V, src, dst):
    """A[v][u] = multiplicity of edge u->v."""
    S, T = incidence(V, src, dst)
    return T.T @ S


def _rows(X, t, S, T, F):
    if X is None:
        return None
    X = np.asarray(X, dtype=np.float32)
    if X.ndim == 1:
        X = X[:, None]
    if X.shape[1] != F:                    # width H: broadcast each value over D = F/H
        X = np.repeat(X, F // X.shape[1], axis=1)
    X64 = X.astype(np.float64)
    if t == "u":
        return (S @ X64).astype(np.float32)
    if t == "v":
        return (T @ X64).astype(np.float32)
    return X.astype(np.float32)


def messages(V, src, dst, edge_op, A, a_type, B, b_type, F, H):
    S, T = incidence(V, src, dst)
    a = _rows(A, a_type, S, T, F)
    b = _rows(B, b_type, S, T, F)
    if edge_op == "copy_lhs":
        return a
    if edge_op == "copy_rhs":
        return b
    if edge_op == "dot":
        E = len(src)
        p = a.astype(np.float64) * b.astype(np.float64)
        return p.reshape(E, H, F // H).sum(axis=2).astype(np.float32)
    with np.errstate(all="ignore"):
        return {"add": np.add, "sub": np.subtract, "mul": np.multiply,
                "div": np.divide}[edge_op](a, b).astype(np.float32)


def op(V, src, dst, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None,
       c_type="v", F=None, H=1):
    M = messages(V, src, dst, edge_op, A, a_type, B, b_type, F, H)
    if c_type == "e":
        return M
    S, T = incidence(V, src, dst)
    deg = T.sum(axis=0)
    if gather_op in ("sum", "mean"):
        Y = T.T @ M.astype(np.float64)
        if gather_op == "mean":
            Y = np.divide(Y, deg[:, None], out=np.zeros_like(Y), where=deg[:, None] > 0)
        return Y.astype(np.float32)
    mask = T.T > 0                                 # [V, E]
    fill = -np.inf if gather_op == "max" else np.inf
    big = np.where(mask[:, :, None], M[None, :, :].astype(np.float64), fill)
    Y = big.max(axis=1) if gather_op == "max" else big.min(axis=1)
    Y[deg == 0] = 0.0
    return Y.astype(np.float32)
