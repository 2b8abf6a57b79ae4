"""Pins for the CPU oracle (oracle/ug_oracle.c) -- none of these need a GPU.

Each test pins the oracle to something other than itself (the prompt's rule 3):
  * dense brute force (tests/dense_ref.py: one-hot incidence products, masked reductions)
    on tiny random multigraphs for all 160 ops of Table 2;
  * a hand-worked 6-vertex example (tests/golden/six_vertex.json);
  * closed forms / invariants (in-degree, antisymmetry, linearity, relabelling);
  * library special cases (scipy.sparse SpMM, torch.scatter_reduce);
  * integer mode, where every order of summation is exact.
"""
import json
import os

import numpy as np
import pytest

import oracle
import ugdata
from opset import all_ops, message_functions, name, table2_class
import dense_ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "six_vertex.json")


def make_operands(op, V, E, F, H, seed, mode, edge_width=None):
    """Operand arrays for op; Edge operands take width edge_width (F or H)."""
    eo, l, r, g, c = op
    arrs = []
    for i, t in enumerate((l, r)):
        if t is None:
            arrs.append(None)
            continue
        rows = V if t in ("u", "v") else E
        width = F
        if t == "e" and edge_width is not None and eo != "dot":
            width = edge_width
        role = "den" if (eo == "div" and i == 1) else ("edge" if t == "e" else "num")
        arrs.append(ugdata.values(rows, width, seed, 10 + i, mode=mode, role=role, k=4))
    return arrs


def run_both(op, V, src, dst, F, H, A, B):
    eo, l, r, g, c = op
    kw = dict(A=A, a_type=l, B=B, b_type=r, c_type=c, F=F, H=H)
    return oracle.op(V, src, dst, eo, g, **kw), dense_ref.op(V, src, dst, eo, g, **kw)


def assert_close_or_exact(op, got, ref, exact):
    eo, l, r, g, c = op
    assert got.shape == ref.shape
    if exact or (g in ("max", "min", "assign") and eo != "dot"):
        np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))
    else:
        # fp64 accumulation in a different order, then one fp32 rounding: <= 1 ulp apart
        np.testing.assert_allclose(got, ref, rtol=2.0 ** -23, atol=1e-30)


def test_table2_counts():
    """The enumeration reproduces Table 2 exactly: 11/1/20/4/44/80 = 160."""
    ops = all_ops()
    assert len(message_functions()) == 32
    assert len(ops) == 160
    counts = {}
    for op in ops:
        k = table2_class(op)
        counts[k] = counts.get(k, 0) + 1
    assert counts == {("V", "E"): 11, ("E", "E"): 1, ("V&E", "E"): 20,
                      ("E", "V"): 4, ("V", "V"): 44, ("V&E", "V"): 80}
    assert len({name(o) for o in ops}) == 160


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("op", all_ops(), ids=name)
def test_bruteforce_all_ops(op, mode):
    """Oracle == dense brute force for every op on random multigraphs (self-loops,
    duplicate edges, zero-in-degree vertices), scalar (H=1) and per-head (H=2) operands."""
    for seed in range(6):
        V = 5 + 7 * seed
        E = 3 * V + seed
        src, dst = ugdata.random_multigraph(V, E, seed)
        for (F, H, ew) in ((4, 1, None), (4, 2, 2), (6, 1, 1)):
            A, B = make_operands(op, V, E, F, H, 100 * seed + F, mode, ew)
            got, ref = run_both(op, V, src, dst, F, H, A, B)
            assert_close_or_exact(op, got, ref, exact=(mode == "int"))


def test_vertex_operand_broadcast():
    """Width-H vertex operands broadcast over their head's D features (R6)."""
    V, E, F, H = 17, 60, 6, 3
    src, dst = ugdata.random_multigraph(V, E, 3)
    X = ugdata.values(V, F, 1, 1)
    att = ugdata.values(V, H, 1, 2)
    for eo in ("add", "mul", "sub", "div"):
        got, ref = run_both((eo, "u", "v", "sum", "v"), V, src, dst, F, H, X, att)
        np.testing.assert_allclose(got, ref, rtol=2.0 ** -23, atol=1e-30)


def test_golden_six_vertex():
    """Hand-computed literals (no program wrote them)."""
    g = json.load(open(GOLDEN))
    V = g["V"]
    src = np.array(g["src"], np.int32)
    dst = np.array(g["dst"], np.int32)
    tensors = {"X": np.array(g["X"], np.float32), "w": np.array(g["w"], np.float32)[:, None]}
    for case in g["cases"]:
        F = case.get("F", g["F"])
        A = tensors[case["A"]] if case["A"] else None
        B = tensors[case["B"]] if case["B"] else None
        got = oracle.op(V, src, dst, case["edge_op"], case["gather_op"], A=A, a_type=case["a_type"],
                        B=B, b_type=case["b_type"], c_type=case["c_type"], F=F, H=case["H"])
        np.testing.assert_array_equal(got, np.array(case["expect"], np.float32), err_msg=case["name"])


@pytest.fixture(scope="module")
def c2():
    src, dst = ugdata.graph("C2")
    return ugdata.CONFIGS["C2"].V, src, dst


def test_ones_closed_forms(c2):
    """Constant-1 features: sum = in-degree (exact), mean = max = min = 1; 0 on empty rows."""
    V, src, dst = c2
    F = 8
    X = np.ones((V, F), np.float32)
    deg = np.bincount(dst, minlength=V).astype(np.float32)
    s = oracle.op(V, src, dst, "copy_lhs", "sum", X, "u", F=F)
    np.testing.assert_array_equal(s, np.repeat(deg[:, None], F, 1))
    live = (deg > 0).astype(np.float32)[:, None]
    for g in ("mean", "max", "min"):
        np.testing.assert_array_equal(oracle.op(V, src, dst, "copy_lhs", g, X, "u", F=F),
                                      np.repeat(live, F, 1))


def test_antisymmetry_and_symmetry(c2):
    """u_sub_v == -(v_sub_u) and u_add_v == v_add_u, bit-exact (IEEE, R11)."""
    V, src, dst = c2
    X = ugdata.values(V, 16, 7, 1)
    a = oracle.op(V, src, dst, "sub", "assign", X, "u", X, "v", c_type="e", F=16)
    b = oracle.op(V, src, dst, "sub", "assign", X, "v", X, "u", c_type="e", F=16)
    np.testing.assert_array_equal(a, -b)
    a = oracle.op(V, src, dst, "add", "sum", X, "u", X, "v", F=16)
    b = oracle.op(V, src, dst, "add", "sum", X, "v", X, "u", F=16)
    np.testing.assert_array_equal(a, b)


def test_weight_one_is_copy(c2):
    """u_mul_e_sum with w == 1 equals copy_u_sum bit-exactly (same messages, same order)."""
    V, src, dst = c2
    X = ugdata.values(V, 16, 7, 1)
    w = np.ones((len(src), 1), np.float32)
    np.testing.assert_array_equal(oracle.op(V, src, dst, "mul", "sum", X, "u", w, "e", F=16),
                                  oracle.op(V, src, dst, "copy_lhs", "sum", X, "u", F=16))


def test_total_mass_and_ordering(c2):
    """sum_v copy_e_sum = sum_e e; and max >= mean >= min elementwise."""
    V, src, dst = c2
    w = ugdata.values(len(src), 4, 9, 2)
    s = oracle.op(V, src, dst, "copy_lhs", "sum", w, "e", F=4)
    np.testing.assert_allclose(s.astype(np.float64).sum(0), w.astype(np.float64).sum(0), rtol=1e-5)
    X = ugdata.values(V, 8, 9, 3)
    mx = oracle.op(V, src, dst, "copy_lhs", "max", X, "u", F=8)
    mn = oracle.op(V, src, dst, "copy_lhs", "min", X, "u", F=8)
    me = oracle.op(V, src, dst, "copy_lhs", "mean", X, "u", F=8)
    assert (mx >= me).all() and (me >= mn).all()


def test_linearity(c2):
    """sum aggregation is linear: agg(2X + Y) ~= 2 agg(X) + agg(Y)."""
    V, src, dst = c2
    X = ugdata.values(V, 8, 11, 1)
    Y = ugdata.values(V, 8, 11, 2)
    lhs = oracle.op(V, src, dst, "copy_lhs", "sum", (2 * X + Y).astype(np.float32), "u", F=8)
    rhs = 2 * oracle.op(V, src, dst, "copy_lhs", "sum", X, "u", F=8) + oracle.op(V, src, dst, "copy_lhs", "sum", Y, "u", F=8)
    np.testing.assert_allclose(lhs, rhs, atol=1e-4)


def test_relabel_equivariance(c2):
    """Permuting vertex ids permutes the output rows: exact for max/min and integer sums."""
    V, src, dst = c2
    rng = np.random.default_rng(5)
    perm = rng.permutation(V).astype(np.int32)        # new id of old vertex i
    X = ugdata.values(V, 8, 13, 1, mode="int")
    Xp = np.empty_like(X)
    Xp[perm] = X
    for g in ("max", "min", "sum", "mean"):
        a = oracle.op(V, src, dst, "copy_lhs", g, X, "u", F=8)
        b = oracle.op(V, perm[src], perm[dst], "copy_lhs", g, Xp, "u", F=8)
        np.testing.assert_array_equal(b[perm], a)


def test_scipy_spmm(c2):
    """copy_u_sum == CSR SpMM (scipy.sparse, fp64) up to one fp32 rounding."""
    import scipy.sparse as sp
    V, src, dst = c2
    X = ugdata.values(V, 32, 17, 1)
    A = sp.csr_matrix((np.ones(len(src)), (dst, src)), shape=(V, V))
    ref = (A @ X.astype(np.float64)).astype(np.float32)
    np.testing.assert_allclose(oracle.op(V, src, dst, "copy_lhs", "sum", X, "u", F=32), ref,
                               rtol=2.0 ** -23, atol=1e-30)


def test_torch_scatter_reduce(c2):
    """Reducers == torch.scatter_reduce(include_self=False) on a zero-initialised output."""
    import torch
    V, src, dst = c2
    X = ugdata.values(V, 8, 19, 1)
    msg = torch.from_numpy(X)[torch.from_numpy(src).long()]
    idx = torch.from_numpy(dst).long()[:, None].expand(-1, 8)
    for g, tr in (("max", "amax"), ("min", "amin")):
        ref = torch.zeros(V, 8).scatter_reduce(0, idx, msg, tr, include_self=False).numpy()
        np.testing.assert_array_equal(oracle.op(V, src, dst, "copy_lhs", g, X, "u", F=8), ref)
    ref = torch.zeros(V, 8, dtype=torch.float64).scatter_reduce(0, idx, msg.double(), "mean",
                                                                  include_self=False).float().numpy()
    np.testing.assert_allclose(oracle.op(V, src, dst, "copy_lhs", "mean", X, "u", F=8), ref,
                               rtol=2.0 ** -23, atol=1e-30)


def test_message_creation_gather(c2):
    """Message creation == X[src] op X[dst] (bit-exact)."""
    V, src, dst = c2
    X = ugdata.values(V, 8, 23, 1)
    Y = ugdata.values(V, 8, 23, 2, role="den")
    for eo, f in (("add", np.add), ("sub", np.subtract), ("mul", np.multiply), ("div", np.divide)):
        ref = f(X[src], Y[dst]).astype(np.float32)
        np.testing.assert_array_equal(oracle.op(V, src, dst, eo, "assign", X, "u", Y, "v", c_type="e", F=8), ref)


def test_signed_zero_order():
    """max/min use the total order -0 < +0 (R12)."""
    src = np.array([0, 1, 0, 1], np.int32)
    dst = np.array([2, 2, 3, 3], np.int32)
    X = np.array([[-0.0], [0.0], [0.0], [0.0]], np.float32)
    X[1, 0] = 0.0
    mx = oracle.op(4, src, dst, "copy_lhs", "max", X, "u", F=1)
    mn = oracle.op(4, src, dst, "copy_lhs", "min", X, "u", F=1)
    assert not np.signbit(mx[2, 0]) and np.signbit(mn[2, 0])
    # reversed edge order gives the same answer
    mx2 = oracle.op(4, src[::-1].copy(), dst[::-1].copy(), "copy_lhs", "max", X, "u", F=1)
    assert not np.signbit(mx2[2, 0])


def test_rows_subset(c2):
    """Computing a subset of output rows gives exactly those rows of the full result."""
    V, src, dst = c2
    X = ugdata.values(V, 8, 29, 1)
    full = oracle.op(V, src, dst, "copy_lhs", "mean", X, "u", F=8)
    rows = np.array([0, 5, V - 1, 17, 17], np.int64)
    np.testing.assert_array_equal(oracle.op(V, src, dst, "copy_lhs", "mean", X, "u", F=8, rows=rows), full[rows])
    fe = oracle.op(V, src, dst, "mul", "assign", X, "u", X, "v", c_type="e", F=8)
    er = np.array([3, 1, len(src) - 1], np.int64)
    np.testing.assert_array_equal(oracle.op(V, src, dst, "mul", "assign", X, "u", X, "v", c_type="e", F=8, rows=er), fe[er])


def test_bound_scale():
    """The tolerance scale is sum |terms| (sum), that / deg (mean), max |term| (max/min)."""
    src = np.array([0, 1, 2], np.int32)
    dst = np.array([3, 3, 3], np.int32)
    X = np.array([[1.0], [-2.0], [4.0], [0.5]], np.float32)
    _, b = oracle.op(4, src, dst, "copy_lhs", "sum", X, "u", F=1, bound=True)
    assert b[3, 0] == 7.0
    _, b = oracle.op(4, src, dst, "copy_lhs", "mean", X, "u", F=1, bound=True)
    assert b[3, 0] == 7.0 / 3
    _, b = oracle.op(4, src, dst, "copy_lhs", "max", X, "u", F=1, bound=True)
    assert b[3, 0] == 4.0


def test_rejects_outside_opset():
    src = np.array([0], np.int32)
    dst = np.array([1], np.int32)
    X = np.ones((2, 1), np.float32)
    with pytest.raises(ValueError):
        oracle.op(2, src, dst, "copy_lhs", "sum", X, "u", c_type="e", F=1)     # reducer onto edges
    with pytest.raises(ValueError):
        oracle.op(2, src, dst, "copy_lhs", "assign", X, "u", c_type="v", F=1)  # assign onto vertices
    with pytest.raises(ValueError):
        oracle.op(2, src, dst, "copy_lhs", "sum", X, "u", F=3, H=2)            # H does not divide F


def test_inedges_stable():
    src, dst = ugdata.random_multigraph(50, 400, 1)
    row_ptr, eids = oracle.inedges(50, dst)
    np.testing.assert_array_equal(eids, np.argsort(dst, kind="stable"))
    np.testing.assert_array_equal(np.diff(row_ptr), np.bincount(dst, minlength=50))


def test_stats_and_partition():
    src, dst = ugdata.graph("C3")
    V = ugdata.CONFIGS["C3"].V
    deg = np.bincount(dst, minlength=V)
    m, s, mx = oracle.stats(V, dst)
    assert abs(m - deg.mean()) < 1e-12 and abs(s - deg.std()) < 1e-9 and mx == deg.max()
    row_ptr = np.zeros(V + 1, np.int64)
    row_ptr[1:] = np.cumsum(deg)
    E = len(dst)
    for P in (1, 2, 3, 8):
        sp = oracle.partition(row_ptr, P)
        assert sp[0] == 0 and sp[-1] == V and (np.diff(sp) >= 0).all()
        for k in range(1, P):
            tgt = -(-k * E // P)
            r = sp[k]
            assert row_ptr[r] >= tgt and (r == 0 or row_ptr[r - 1] < tgt)


def test_generator_shapes():
    for k, c in ugdata.CONFIGS.items():
        if k == "C5":
            continue
        src, dst = ugdata.graph(k)
        assert len(src) == c.E and src.dtype == np.int32
        assert (np.diff(dst) >= 0).all() and src.max() < c.V and dst.max() < c.V
        s2, d2 = ugdata.graph(k)
        assert (s2 == src).all() and (d2 == dst).all()
