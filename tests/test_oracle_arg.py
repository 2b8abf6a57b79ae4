"""Pins for oracle.op_arg (max/min aggregation with arg capture) -- no GPU.

Pinned by brute force: per (v, f) the candidate set is every edge with dst = v, messages are
formed with numpy in fp32 (one rounding, R11), the extreme is taken under the total order
-0 < +0 (R12) and the expected arg is the SMALLEST edge id attaining it (the tie rule); plus
a hand-worked example and integer-valued inputs full of ties."""
import numpy as np
import pytest

import oracle
import ugdata


def _key(x):
    """Monotone int key of float32 under the total order -0 < +0 (no NaN)."""
    b = np.asarray(x, np.float32).view(np.int32).astype(np.int64)
    return np.where(b < 0, -(b & 0x7FFFFFFF) - 1, b)


def _messages(eo, A, a_t, B, b_t, src, dst):
    E = len(src)
    rows = lambda t: src if t == "u" else (dst if t == "v" else np.arange(E))
    a = A[rows(a_t)]
    if eo == "copy_lhs":
        return a
    b = B[rows(b_t)]
    b = np.broadcast_to(b, a.shape)
    with np.errstate(all="ignore"):
        return {"add": a + b, "sub": a - b, "mul": a * b, "div": a / b}[eo].astype(np.float32)


def _brute(V, src, dst, eo, go, A, a_t, B, b_t, F):
    msg = _messages(eo, A, a_t, B, b_t, src, dst)
    k = _key(msg)
    C = np.zeros((V, F), np.float32)
    arg = -np.ones((V, F), np.int64)
    for v in range(V):
        es = np.nonzero(dst == v)[0]
        if len(es) == 0:
            continue
        kk = k[es]
        best = kk.max(axis=0) if go == "max" else kk.min(axis=0)
        for f in range(F):
            first = es[np.nonzero(kk[:, f] == best[f])[0][0]]    # smallest edge id among ties
            arg[v, f] = first
            C[v, f] = msg[first, f]
    return C, arg


OPS = [("copy_lhs", "u", None), ("copy_lhs", "e", None), ("add", "u", "e"), ("sub", "e", "v"),
       ("mul", "u", "v"), ("div", "v", "u")]


@pytest.mark.parametrize("go", ["max", "min"])
@pytest.mark.parametrize("eo,a_t,b_t", OPS)
@pytest.mark.parametrize("mode", ["float", "int"])
def test_op_arg_bruteforce(eo, a_t, b_t, go, mode):
    for seed in range(4):
        V = 8 + 9 * seed
        E = 4 * V + seed
        F = 3
        src, dst = ugdata.random_multigraph(V, E, seed)
        rows = lambda t: V if t in ("u", "v") else E
        A = ugdata.values(rows(a_t), F, seed, 1, mode=mode, k=2)
        B = None if b_t is None else ugdata.values(rows(b_t), F, seed, 2, mode=mode,
                                                   role="den" if eo == "div" else "num", k=2)
        C, arg = oracle.op_arg(V, src, dst, eo, go, A=A, a_type=a_t, B=B, b_type=b_t, F=F)
        bc, barg = _brute(V, src, dst, eo, go, A, a_t, B, b_t, F)
        np.testing.assert_array_equal(arg, barg)
        np.testing.assert_array_equal(C.view(np.uint32), bc.view(np.uint32))
        # the value half agrees with the (separately pinned) plain max/min aggregation
        ref = oracle.op(V, src, dst, eo, go, A=A, a_type=a_t, B=B, b_type=b_t, c_type="v", F=F)
        np.testing.assert_array_equal(C.view(np.uint32), ref.view(np.uint32))


def test_op_arg_hand_worked():
    """Edges (id: src->dst) 0: 0->2, 1: 1->2, 2: 3->2, 3: 2->0; vertex 1 and 3 have no in-edges.
    X = [2, 5, 9, 5] (one feature): into vertex 2 arrive X[0]=2, X[1]=5, X[3]=5.
    max -> 5 from edge 1 (edge 2 ties, later id); min -> 2 from edge 0; vertex 0 <- edge 3."""
    src = np.array([0, 1, 3, 2], np.int32)
    dst = np.array([2, 2, 2, 0], np.int32)
    X = np.array([[2.0], [5.0], [9.0], [5.0]], np.float32)
    C, arg = oracle.op_arg(4, src, dst, "copy_lhs", "max", A=X, a_type="u", F=1)
    assert arg[:, 0].tolist() == [3, -1, 1, -1] and C[:, 0].tolist() == [9.0, 0.0, 5.0, 0.0]
    C, arg = oracle.op_arg(4, src, dst, "copy_lhs", "min", A=X, a_type="u", F=1)
    assert arg[:, 0].tolist() == [3, -1, 0, -1] and C[:, 0].tolist() == [9.0, 0.0, 2.0, 0.0]


def test_op_arg_signed_zero_order():
    """-0 < +0: max picks the +0 edge even when the -0 edge comes first, min the -0 edge."""
    src = np.array([0, 1], np.int32)
    dst = np.array([2, 2], np.int32)
    X = np.array([[-0.0], [0.0], [1.0]], np.float32)
    _, arg = oracle.op_arg(3, src, dst, "copy_lhs", "max", A=X, a_type="u", F=1)
    assert arg[2, 0] == 1
    _, arg = oracle.op_arg(3, src, dst, "copy_lhs", "min", A=X, a_type="u", F=1)
    assert arg[2, 0] == 0


def test_op_arg_rejects_sum_and_dot():
    src = np.array([0], np.int32)
    dst = np.array([1], np.int32)
    X = np.ones((2, 2), np.float32)
    with pytest.raises(ValueError):
        oracle.op_arg(2, src, dst, "copy_lhs", "sum", A=X, a_type="u", F=2)
    with pytest.raises(ValueError):
        oracle.op_arg(2, src, dst, "dot", "max", A=X, a_type="u", B=X, b_type="v", F=2)
