"""GPU parity of max/min aggregation with arg capture (ug_op_run_arg) and of its backward
scatter (ug_arg_scatter) -- SURVEY 8(f) f2.  Values and args are compared bit-exactly with
oracle.op_arg (index work and max/min are exact, north star); gradients with the reference
built from the oracle's args (exact in integer mode, fp32 atomics otherwise)."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")
from paper_conf_asplos_0001lslwlgslllw23_b200 import autograd as uga  # noqa: E402

OPS = [("copy_lhs", "u", None), ("copy_lhs", "e", None), ("add", "u", "e"), ("sub", "e", "v"),
       ("mul", "u", "v"), ("div", "v", "u")]


def _graphs():
    out = []
    V = 300
    s, d = ugdata.random_multigraph(V, 2400, 5)            # unsorted COO: eid != identity
    out.append(("multigraph", V, s, d))
    V = 2001                                               # hub of in-degree 2000 + ring: split rows
    s = np.concatenate([np.arange(1, V), np.arange(V)]).astype(np.int32)
    d = np.concatenate([np.zeros(V - 1, np.int32), (np.arange(V) + 1) % V]).astype(np.int32)
    out.append(("hub", V, s, d))
    c = ugdata.CONFIGS["C2"]
    s, d = ugdata.graph("C2")
    out.append(("C2", c.V, s, d))
    return out


GRAPHS = _graphs()


@pytest.mark.parametrize("gname,V,src,dst", GRAPHS, ids=[g[0] for g in GRAPHS])
@pytest.mark.parametrize("eo,a_t,b_t", OPS)
@pytest.mark.parametrize("go", ["max", "min"])
def test_op_run_arg_matches_oracle(gname, V, src, dst, eo, a_t, b_t, go):
    E = len(src)
    g = ug.Graph(V, src, dst)
    for F, mode in ((3, "int"), (40, "float")):
        rows = lambda t: V if t in ("u", "v") else E
        A = ugdata.values(rows(a_t), F, 7, 1, mode=mode, k=2)
        B = None if b_t is None else ugdata.values(rows(b_t), F, 7, 2, mode=mode,
                                                   role="den" if eo == "div" else "num", k=2)
        C = torch.full((V, F), float("nan"), device="cuda")
        Bd = None if B is None else torch.from_numpy(B).cuda()
        arg = ug.op_run_arg(g, eo, go, A=torch.from_numpy(A).cuda(), a_type=a_t, B=Bd, b_type=b_t, C=C, F=F)
        C2 = torch.empty(V, F, device="cuda")
        ug.op_run(g, eo, go, A=torch.from_numpy(A).cuda(), a_type=a_t, B=Bd, b_type=b_t, C=C2, c_type="v", F=F)
        torch.cuda.synchronize()
        rc, rarg = oracle.op_arg(V, src, dst, eo, go, A=A, a_type=a_t, B=B, b_type=b_t, F=F)
        np.testing.assert_array_equal(arg.cpu().numpy(), rarg)
        np.testing.assert_array_equal(C.cpu().numpy().view(np.uint32), rc.view(np.uint32))
        assert torch.equal(C, C2)


def test_arg_rejects_sum():
    V = 10
    s, d = ugdata.random_multigraph(V, 30, 1)
    g = ug.Graph(V, s, d)
    X = torch.randn(V, 4, device="cuda")
    with pytest.raises(ug.UgError, match="UNSUPPORTED_OP"):
        ug.op_run_arg(g, "copy_lhs", "sum", A=X, a_type="u", C=torch.empty(V, 4, device="cuda"), F=4)


@pytest.mark.parametrize("gname,V,src,dst", GRAPHS, ids=[g[0] for g in GRAPHS])
@pytest.mark.parametrize("go", ["max", "min"])
def test_copy_u_extreme_backward(gname, V, src, dst, go):
    """dX[u] = sum of dY[v][f] over (v, f) whose arg edge has source u (integer dY: exact)."""
    F = 8
    gp = uga.GraphPair(V, src, dst)
    X = torch.from_numpy(ugdata.values(V, F, 3, 1, mode="int", k=3)).cuda().requires_grad_(True)
    Y = (uga.copy_u_max if go == "max" else uga.copy_u_min)(gp, X)
    dY = torch.from_numpy(ugdata.values(V, F, 3, 2, mode="int", k=4)).cuda()
    Y.backward(dY)
    _, arg = oracle.op_arg(V, src, dst, "copy_lhs", go, A=X.detach().cpu().numpy(), a_type="u", F=F)
    ref = np.zeros((V, F), np.float64)
    vv, ff = np.nonzero(arg >= 0)
    np.add.at(ref, (src[arg[vv, ff]], ff), dY.cpu().numpy()[vv, ff])
    np.testing.assert_array_equal(X.grad.cpu().numpy(), ref.astype(np.float32))


def test_copy_e_max_backward_matches_torch_scatter_reduce():
    """Float edge features (no ties): the gradient equals torch's scatter_reduce(amax) autograd."""
    V = 400
    src, dst = ugdata.random_multigraph(V, 3000, 9)
    E = len(src)
    gp = uga.GraphPair(V, src, dst)
    Ee = torch.from_numpy(ugdata.values(E, 6, 4, 1)).cuda()
    a = Ee.clone().requires_grad_(True)
    Y = uga.copy_e_max(gp, a)
    dY = torch.randn(V, 6, device="cuda")
    Y.backward(dY)
    b = Ee.clone().requires_grad_(True)
    d = torch.from_numpy(dst).long().cuda()[:, None].expand(E, 6)
    R = torch.zeros(V, 6, device="cuda").scatter_reduce(0, d, b, "amax", include_self=False)
    R.backward(dY)
    assert torch.equal(Y.detach(), R.detach())
    torch.testing.assert_close(a.grad, b.grad, rtol=0, atol=0)
