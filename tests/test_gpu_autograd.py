"""Backward through the unified operator.

Two checks per operator: (1) parity -- the forward and every gradient against the ORACLE
evaluating the backward's defining graph operator (the transposed aggregation over the reversed
graph, u_div_e_sum for the mean, u_dot_v for the edge-weight gradient) within 1e-5 * sum|terms|
(R11); (2) calculus -- the same gradients against torch autograd of a float64 index_add_
reference, which shows those operators ARE the gradients."""
import numpy as np
import pytest
import torch

import oracle
import ugdata
from gpu_util import assert_parity

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")
from paper_conf_asplos_0001lslwlgslllw23_b200 import autograd as uga  # noqa: E402


@pytest.fixture(scope="module", params=["C2", "multigraph"])
def graph(request):
    if request.param == "C2":
        c = ugdata.CONFIGS["C2"]
        src, dst = ugdata.graph("C2")
        V = c.V
    else:   # unsorted COO with self-loops, duplicates and zero-in-degree rows
        V = 500
        src, dst = ugdata.random_multigraph(V, 4000, 11)
    return V, src, dst, uga.GraphPair(V, src, dst)


def ref_agg(V, src, dst, X, w=None, mean=False):
    s = torch.from_numpy(src).long().cuda()
    d = torch.from_numpy(dst).long().cuda()
    m = X[s]
    if w is not None:
        H = w.shape[1]
        m = (m.view(len(s), H, -1) * w[:, :, None]).view(len(s), -1)
    Y = torch.zeros(V, X.shape[1], dtype=X.dtype, device=X.device).index_add(0, d, m)
    if mean:
        deg = torch.bincount(d, minlength=V).to(X.dtype).clamp(min=1)[:, None]
        Y = Y / deg
    return Y


def oracle_check(got, op, V, src, dst, A, a_type, B=None, b_type=None, c_type="v", F=None, H=1, what=""):
    ref, bnd = oracle.op(V, src, dst, op[0], op[1], A=A, a_type=a_type, B=B, b_type=b_type, c_type=c_type,
                         F=F or A.shape[1], H=H, bound=True)
    assert_parity((op[0], a_type, b_type, op[1], c_type), got.detach().cpu().numpy(), ref, bnd, False, what=what)


def check(a, b, rtol=1e-5):
    b = b.float()
    torch.testing.assert_close(a, b, rtol=rtol, atol=rtol * (b.abs().max().item() + 1e-6))


@pytest.mark.parametrize("mean", [False, True])
def test_copy_u_sum_mean_backward(graph, mean):
    V, src, dst, gp = graph
    X = torch.randn(V, 48, device="cuda", requires_grad=True)
    G = torch.randn(V, 48, device="cuda")
    Y = (uga.copy_u_mean if mean else uga.copy_u_sum)(gp, X)
    (Y * G).sum().backward()
    X64 = X.detach().double().requires_grad_(True)
    Yr = ref_agg(V, src, dst, X64, mean=mean)
    (Yr * G.double()).sum().backward()
    check(Y.detach(), Yr.detach())
    check(X.grad, X64.grad)
    Xn, Gn = X.detach().cpu().numpy(), G.cpu().numpy()
    oracle_check(Y, ("copy_lhs", "mean" if mean else "sum"), V, src, dst, Xn, "u", what="forward")
    if mean:
        deg_e = np.bincount(dst, minlength=V).astype(np.float32)[dst].reshape(-1, 1)
        oracle_check(X.grad, ("div", "sum"), V, dst, src, Gn, "u", deg_e, "e", what="mean backward")
    else:
        oracle_check(X.grad, ("copy_lhs", "sum"), V, dst, src, Gn, "u", what="sum backward")


@pytest.mark.parametrize("H", [1, 4])
def test_u_mul_e_sum_backward(graph, H):
    V, src, dst, gp = graph
    E = len(src)
    X = torch.randn(V, 32, device="cuda", requires_grad=True)
    w = (torch.rand(E, H, device="cuda") + 0.5).requires_grad_(True)
    G = torch.randn(V, 32, device="cuda")
    Y = uga.u_mul_e_sum(gp, X, w)
    (Y * G).sum().backward()
    X64 = X.detach().double().requires_grad_(True)
    w64 = w.detach().double().requires_grad_(True)
    Yr = ref_agg(V, src, dst, X64, w64)
    (Yr * G.double()).sum().backward()
    check(Y.detach(), Yr.detach())
    check(X.grad, X64.grad)
    check(w.grad, w64.grad)
    Xn, Gn, wn = X.detach().cpu().numpy(), G.cpu().numpy(), w.detach().cpu().numpy()
    oracle_check(Y, ("mul", "sum"), V, src, dst, Xn, "u", wn, "e", H=H, what="forward")
    oracle_check(X.grad, ("mul", "sum"), V, dst, src, Gn, "u", wn, "e", H=H, what="dX")
    oracle_check(w.grad, ("dot", "assign"), V, src, dst, Xn, "u", Gn, "v", c_type="e", F=32, H=H, what="dw")
