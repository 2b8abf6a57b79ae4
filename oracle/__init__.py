"""CPU oracle for the unified graph operator -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path
(``paper_conf_asplos_0001lslwlgslllw23_b200``) never imports it, and the two share no code.

The arithmetic lives in ``oracle/ug_oracle.c`` (plain single-threaded C, the edge loop of
PAPER.md Fig. 5 under Table 4); this module is ctypes marshalling only.  Every function
here is pinned by ``tests/test_oracle_*.py`` (dense brute force, golden example,
invariants, integer mode).  Nothing here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ug_oracle.c")
_LIB = os.path.join(_HERE, "libugoracle.so")

# The oracle's own numbering (see ug_oracle.c); public names follow the paper / DGL.
EDGE_OPS = {"copy_lhs": 0, "copy_rhs": 1, "add": 2, "sub": 3, "mul": 4, "div": 5, "dot": 6}
GATHER_OPS = {"assign": 0, "sum": 1, "max": 2, "min": 3, "mean": 4}
TYPES = {None: 0, "u": 1, "v": 2, "e": 3}

_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with the flags SURVEY 8(c) fixes: -O2 -ffp-contract=off, no fast-math."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                               "-shared", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        p = ctypes.c_void_p
        i64 = ctypes.c_int64
        ci = ctypes.c_int
        lib.ugo_op.argtypes = [i64, i64, p, p, ci, ci,
                               p, ci, ci, i64,
                               p, ci, ci, i64,
                               p, ci, i64,
                               ci, ci, p, i64, p, i64]
        lib.ugo_op.restype = ci
        lib.ugo_inedges.argtypes = [i64, i64, p, p, p]
        lib.ugo_inedges.restype = ci
        lib.ugo_stats.argtypes = [i64, i64, p, p, p, p]
        lib.ugo_stats.restype = None
        lib.ugo_partition.argtypes = [i64, p, ci, p]
        lib.ugo_partition.restype = None
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


def _c32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def op(V, src, dst, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None,
       c_type="v", F=None, H=1, rows=None, bound=False):
    """One unified-operator call (Fig. 5, Table 4).

    A, B: 2-D float32 arrays (rows = V or E, width = F or H) or None; *_type in {"u","v","e",None}.
    c_type "v" -> aggregation (result [V, W]); "e" -> message creation (result [E, W]);
    W = F, or H for dot.  rows: optional int64 subset of output rows; the returned array is
    then [len(rows), W] in that order.  bound=True also returns the Q11 tolerance scale.
    """
    lib = _load()
    src = _c32(src)
    dst = _c32(dst)
    E = int(src.shape[0])
    W = H if edge_op == "dot" else F
    nrow_out = V if c_type == "v" else E
    ops = []
    for X in (A, B):
        if X is None:
            ops.append((None, 1, 0))
        else:
            X = np.ascontiguousarray(X, dtype=np.float32)
            if X.ndim == 1:
                X = X.reshape(-1, 1)
            ops.append((X, X.shape[1], X.shape[1]))
    (Aa, aw, ald), (Ba, bw, bld) = ops
    if rows is None:
        C = np.zeros((nrow_out, W), dtype=np.float32)
        rows_a, nrows = None, 0
        nb = nrow_out
    else:
        rows_a = np.ascontiguousarray(rows, dtype=np.int64)
        nrows = int(rows_a.shape[0])
        C = np.zeros((nrow_out, W), dtype=np.float32)  # written at its own row index
        nb = nrows
    bnd = np.zeros((nb, W), dtype=np.float64) if bound else None
    rc = lib.ugo_op(V, E, _ptr(src), _ptr(dst), EDGE_OPS[edge_op], GATHER_OPS[gather_op],
                    _ptr(Aa), TYPES[a_type], aw, ald,
                    _ptr(Ba), TYPES[b_type], bw, bld,
                    _ptr(C), TYPES[c_type], W,
                    int(F), int(H), _ptr(rows_a), nrows, _ptr(bnd), W)
    if rc != 0:
        raise ValueError(f"oracle rejected op ({edge_op},{gather_op},{a_type},{b_type},{c_type}) rc={rc}")
    if rows is not None:
        C = C[rows_a]
    return (C, bnd) if bound else C


def inedges(V, dst):
    """In-edge lists as (row_ptr[V+1], edge_ids[E]) int64, stable by edge id."""
    lib = _load()
    dst = _c32(dst)
    E = int(dst.shape[0])
    row_ptr = np.zeros(V + 1, dtype=np.int64)
    eids = np.zeros(max(E, 1), dtype=np.int64)
    if lib.ugo_inedges(V, E, _ptr(dst), _ptr(row_ptr), _ptr(eids)) != 0:
        raise ValueError("vertex id out of range")
    return row_ptr, eids[:E]


def stats(V, dst):
    """(mean in-degree, std_nnz = population std of in-degree, max in-degree) -- Table 7."""
    lib = _load()
    dst = _c32(dst)
    m = ctypes.c_double()
    s = ctypes.c_double()
    mx = ctypes.c_int64()
    lib.ugo_stats(V, int(dst.shape[0]), _ptr(dst), ctypes.byref(m), ctypes.byref(s), ctypes.byref(mx))
    return m.value, s.value, mx.value


def partition(row_ptr, parts):
    """Edge-balanced dst-row split points r_0..r_P (R21)."""
    lib = _load()
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    V = int(row_ptr.shape[0]) - 1
    out = np.zeros(parts + 1, dtype=np.int64)
    lib.ugo_partition(V, _ptr(row_ptr), int(parts), _ptr(out))
    return out


def gat(V, src, dst, el, er, z, H, slope=0.2, bound=False):
    """GAT attention chain by definition, fp64: edge softmax of
    LeakyReLU(el_u + er_v) per head over each destination's in-edges, then the attention-weighted
    sum of z_u.  el, er: [V, H]; z: [V, F] float32.  Returns (out [V, F], attn [E, H]) as float64,
    plus the tolerance scale sum_e a |z| when bound=True."""
    lib = _load()
    if not hasattr(lib, "_gat_ready"):
        p, i64, ci = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        lib.ugo_gat.argtypes = [i64, i64, p, p, p, i64, p, i64, p, i64, ci, ci, ctypes.c_double, p, p, p]
        lib.ugo_gat.restype = ci
        lib._gat_ready = True
    src = _c32(src)
    dst = _c32(dst)
    E = int(src.shape[0])
    el = np.ascontiguousarray(el, dtype=np.float32).reshape(V, -1)
    er = np.ascontiguousarray(er, dtype=np.float32).reshape(V, -1)
    z = np.ascontiguousarray(z, dtype=np.float32)
    F = int(z.shape[1])
    out = np.zeros((V, F), dtype=np.float64)
    attn = np.zeros((max(E, 1), H), dtype=np.float64)
    bnd = np.zeros((V, F), dtype=np.float64) if bound else None
    rc = lib.ugo_gat(V, E, _ptr(src), _ptr(dst), _ptr(el), el.shape[1], _ptr(er), er.shape[1],
                     _ptr(z), F, F, int(H), float(slope), _ptr(out), _ptr(attn), _ptr(bnd))
    if rc != 0:
        raise ValueError(f"oracle rejected gat (F={F}, H={H}) rc={rc}")
    return (out, attn[:E], bnd) if bound else (out, attn[:E])


def dot_attention(V, src, dst, q, k, val, H, scale=None, bound=False):
    """Dot-product attention chain (FusedMM-style SDDMM + softmax + SpMM, PAPER.md:588
    and :224) by definition, fp64: per head, s_e = scale * <q[dst], k[src]>, softmax over each
    destination's in-edges, out = sum_e a_e val[src].  q: [V, H*Dk], k: [V, H*Dk], val: [V, H*Dv]
    float32; scale defaults to 1/sqrt(Dk).  Returns (out [V, H*Dv], attn [E, H]) float64, plus the
    tolerance scale sum_e a_e |val| when bound=True."""
    lib = _load()
    if not hasattr(lib, "_dotattn_ready"):
        p, i64, ci = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        lib.ugo_dot_attention.argtypes = [i64, i64, p, p, p, i64, p, i64, p, i64, ci, ci, ci, ctypes.c_double,
                                          p, p, p]
        lib.ugo_dot_attention.restype = ci
        lib._dotattn_ready = True
    src = _c32(src)
    dst = _c32(dst)
    E = int(src.shape[0])
    q = np.ascontiguousarray(q, dtype=np.float32)
    k = np.ascontiguousarray(k, dtype=np.float32)
    val = np.ascontiguousarray(val, dtype=np.float32)
    Dk = q.shape[1] // H
    Dv = val.shape[1] // H
    if scale is None:
        scale = 1.0 / np.sqrt(Dk)
    out = np.zeros((V, H * Dv), dtype=np.float64)
    attn = np.zeros((max(E, 1), H), dtype=np.float64)
    bnd = np.zeros((V, H * Dv), dtype=np.float64) if bound else None
    rc = lib.ugo_dot_attention(V, E, _ptr(src), _ptr(dst), _ptr(q), q.shape[1], _ptr(k), k.shape[1],
                               _ptr(val), val.shape[1], int(H), int(Dk), int(Dv), float(scale),
                               _ptr(out), _ptr(attn), _ptr(bnd))
    if rc != 0:
        raise ValueError(f"oracle rejected dot_attention (H={H}) rc={rc}")
    return (out, attn[:E], bnd) if bound else (out, attn[:E])


def op_arg(V, src, dst, edge_op, gather_op, A=None, a_type=None, B=None, b_type=None, F=None, H=1):
    """Max/min aggregation with arg capture: returns (C [V, F] float32,
    arg [V, F] int64 edge ids, -1 for zero in-degree rows); ties keep the first edge id."""
    lib = _load()
    if not hasattr(lib, "_arg_ready"):
        p, i64, ci = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        lib.ugo_op_arg.argtypes = [i64, i64, p, p, ci, ci, p, ci, ci, i64, p, ci, ci, i64, p, i64, ci, ci, p, i64]
        lib.ugo_op_arg.restype = ci
        lib._arg_ready = True
    src = _c32(src)
    dst = _c32(dst)
    E = int(src.shape[0])
    ops = []
    for X in (A, B):
        if X is None:
            ops.append((None, 1, 0))
        else:
            X = np.ascontiguousarray(X, dtype=np.float32)
            if X.ndim == 1:
                X = X.reshape(-1, 1)
            ops.append((X, X.shape[1], X.shape[1]))
    (Aa, aw, ald), (Ba, bw, bld) = ops
    C = np.zeros((V, F), dtype=np.float32)
    arg = np.zeros((V, F), dtype=np.int64)
    rc = lib.ugo_op_arg(V, E, _ptr(src), _ptr(dst), EDGE_OPS[edge_op], GATHER_OPS[gather_op],
                        _ptr(Aa), TYPES[a_type], aw, ald, _ptr(Ba), TYPES[b_type], bw, bld,
                        _ptr(C), F, int(F), int(H), _ptr(arg), F)
    if rc != 0:
        raise ValueError(f"oracle rejected arg op ({edge_op},{gather_op}) rc={rc}")
    return C, arg
