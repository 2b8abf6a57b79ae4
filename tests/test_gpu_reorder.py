"""GPU: an operator on a renumbered graph (ug.Renumbered: ug_graph_reorder + ug_rows_gather)
returns, mapped back, exactly the result on the original numbering -- bit-exact for max and
for integer-valued sums (every order of summation is exact), edge tensors re-ordered with the
edges."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


@pytest.mark.parametrize("method", ["rcm", "degree", "community"])
@pytest.mark.parametrize("graph", ["multigraph", "community"])
def test_renumbered_ops_match_oracle(method, graph):
    if graph == "multigraph":
        V = 600
        src, dst = ugdata.random_multigraph(V, 5000, 4)
    else:
        V = 4000
        src, dst = ugdata.community_graph(V, 40000, 20, 0.9, 5)
    E = len(src)
    rn = ug.Renumbered(V, src, dst, method)
    F = 16
    X = ugdata.values(V, F, 1, 1, mode="int", k=4)
    w = ugdata.values(E, 1, 1, 2, mode="int", role="edge", k=4)
    Xn = rn.to_new(torch.from_numpy(X).cuda())
    wn = rn.edges_to_new(torch.from_numpy(w).cuda())
    for eo, go, B, bt in (("copy_lhs", "sum", None, None), ("copy_lhs", "max", None, None),
                          ("mul", "sum", wn, "e"), ("copy_lhs", "mean", None, None)):
        Yn = torch.empty(V, F, device="cuda")
        ug.op_run(rn.graph, eo, go, A=Xn, a_type="u", B=B, b_type=bt, C=Yn, c_type="v", F=F)
        Y = rn.to_old(Yn).cpu().numpy()
        ref = oracle.op(V, src, dst, eo, go, A=X, a_type="u", B=None if B is None else w, b_type=bt, F=F)
        np.testing.assert_array_equal(Y.view(np.uint32), ref.view(np.uint32))


def test_rows_gather():
    X = torch.randn(100, 37, device="cuda")
    idx = torch.randint(0, 100, (250,), device="cuda", dtype=torch.int32)
    out = ug.rows_gather(X, idx)
    assert torch.equal(out, X[idx.long()])


def test_renumbered_edge_outputs_back_to_old_order():
    """Message creation on the renumbered graph, mapped back with edges_to_old, equals the
    oracle's message rows in the ORIGINAL edge-id order (bit-exact)."""
    V = 600
    src, dst = ugdata.random_multigraph(V, 5000, 8)
    E = len(src)
    rn = ug.Renumbered(V, src, dst, "rcm")
    F = 8
    X = ugdata.values(V, F, 2, 1)
    w = ugdata.values(E, F, 2, 2, role="edge")
    Xn = rn.to_new(torch.from_numpy(X).cuda())
    wn = rn.edges_to_new(torch.from_numpy(w).cuda())
    Mn = torch.empty(E, F, device="cuda")
    ug.op_run(rn.graph, "mul", "assign", A=Xn, a_type="u", B=wn, b_type="e", C=Mn, c_type="e", F=F)
    M = rn.edges_to_old(Mn).cpu().numpy()
    ref = oracle.op(V, src, dst, "mul", "assign", A=X, a_type="u", B=w, b_type="e", c_type="e", F=F)
    np.testing.assert_array_equal(M.view(np.uint32), ref.view(np.uint32))
