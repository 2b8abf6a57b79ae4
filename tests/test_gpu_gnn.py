"""GNN layers through the DGL-style shim vs a CPU reference built from the
oracle's graph operators and fp64 numpy dense algebra.

Tolerances are derived, not tuned: where the graph operator is the layer's last step (GCN, GAT)
its input is the GPU's own dense result (the same torch call, bit-identical), so the layer is
held to the operator bar itself, 1e-5 * sum|terms| (R11 / R23) plus one rounding of the bias add;
where dense layers follow the aggregation (GIN, GraphSAGE) that bar is propagated through them
with fp32 GEMM rounding bounds ((K + 2) * 2^-24 * |x| |W|) -- `lin_err`."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")
from paper_conf_asplos_0001lslwlgslllw23_b200 import gnn  # noqa: E402


@pytest.fixture(scope="module")
def c2():
    c = ugdata.CONFIGS["C2"]
    src, dst = ugdata.graph("C2")
    return c.V, src, dst, gnn.GraphData(c.V, src, dst)


def mm(a, b):
    return (a.astype(np.float64) @ b.astype(np.float64)).astype(np.float32)


U = 2.0 ** -24        # fp32 unit roundoff


def within(got, ref, bound, what=""):
    got = got.detach().cpu().numpy().astype(np.float64)
    err = np.abs(got - ref)
    bad = ~(err <= bound)
    assert not bad.any(), f"{what}: {bad.sum()} elements beyond the derived bound; max err/bound " \
                          f"{(err / np.maximum(bound, 1e-30)).max():.3g}"


def lin(x, W, b=None):
    """x @ W (+ b) in fp64 -- W as [fin, fout]."""
    y = x.astype(np.float64) @ W.astype(np.float64)
    return y + b.astype(np.float64) if b is not None else y


def lin_err(x_abs, W, err_in, b=None):
    """Error bound of the fp32 GEMM y = x W (+ b) given an input error bound err_in."""
    K = W.shape[0]
    Wa = np.abs(W.astype(np.float64))
    e = err_in @ Wa + (K + 2) * U * (x_abs @ Wa)
    if b is not None:
        e = e + 2 * U * np.abs(b.astype(np.float64))
    return e


def test_switching_table_recognises_builtins(c2):
    assert gnn._message_spec(gnn.fn.u_mul_e("h", "w", "m")) == ("mul", [("h", "u"), ("w", "e")])
    assert gnn._message_spec(gnn.fn.copy_u("h", "m")) == ("copy_lhs", [("h", "u")])
    assert gnn._message_spec(gnn.fn.e_div_v("a", "b", "m")) == ("div", [("a", "e"), ("b", "v")])
    with pytest.raises(AttributeError):
        gnn.fn.u_pow_v


def test_gcn_layer(c2):
    V, src, dst, gd = c2
    torch.manual_seed(0)
    layer = gnn.GCNConv(32, 16).cuda()
    h = torch.randn(V, 32, device="cuda")
    w = gnn.gcn_norm(gd, src, dst)
    with torch.no_grad():
        out = layer(gd, h, w)
        z = (h @ layer.W).cpu().numpy()                  # the layer's own GEMM (same call, same bits)
    ref, bnd = oracle.op(V, src, dst, "mul", "sum", z, "u", w.cpu().numpy(), "e", F=16, bound=True)
    b = layer.b.detach().cpu().numpy().astype(np.float64)
    within(out, ref + b, 1e-5 * bnd + 2 * U * (np.abs(ref) + np.abs(b)), "GCN")


def test_gin_and_sage_layers(c2):
    V, src, dst, gd = c2
    torch.manual_seed(1)
    h = torch.randn(V, 24, device="cuda")
    hn = h.cpu().numpy().astype(np.float64)
    gin = gnn.GINConv(24, 16, eps=0.1).cuda()
    with torch.no_grad():
        out = gin(gd, h)
    agg, bnd = oracle.op(V, src, dst, "copy_lhs", "sum", h.cpu().numpy(), "u", F=24, bound=True)
    x = 1.1 * hn + agg
    ex = 1e-5 * bnd + 3 * U * (1.1 * np.abs(hn) + np.abs(agg))          # aggregation + (1+eps)h + add
    W1, b1 = gin.l1.weight.detach().cpu().numpy().T, gin.l1.bias.detach().cpu().numpy()
    W2, b2 = gin.l2.weight.detach().cpu().numpy().T, gin.l2.bias.detach().cpu().numpy()
    y1 = lin(x, W1, b1)
    e1 = lin_err(np.abs(x), W1, ex, b1)
    r1 = np.maximum(y1, 0)                                               # ReLU: 1-Lipschitz
    ref = lin(r1, W2, b2)
    within(out, ref, lin_err(np.abs(r1) + e1, W2, e1, b2), "GIN")
    for aggr in ("sum", "mean", "max"):
        sage = gnn.SAGEConv(24, 16, aggr).cuda()
        with torch.no_grad():
            out = sage(gd, h)
        a, bnd = oracle.op(V, src, dst, "copy_lhs", aggr, h.cpu().numpy(), "u", F=24, bound=True)
        Ws, bs = sage.self_lin.weight.detach().cpu().numpy().T, sage.self_lin.bias.detach().cpu().numpy()
        Wn = sage.neigh_lin.weight.detach().cpu().numpy().T
        ea = 1e-5 * bnd if aggr != "max" else np.zeros_like(bnd)        # max is exact (R11)
        ys, yn = lin(hn, Ws, bs), lin(a.astype(np.float64), Wn)
        err = (lin_err(np.abs(hn), Ws, np.zeros_like(hn), bs) + lin_err(np.abs(a), Wn, ea)
               + 2 * U * (np.abs(ys) + np.abs(yn)))
        within(out, ys + yn, err, f"SAGE-{aggr}")


@pytest.mark.parametrize("fused", [True, False])
def test_gat_layer(c2, fused):
    """The fused traversal against oracle.gat on the layer's own el / er / z (R23 bound); the
    unfused 6-op chain against the per-op oracle chain (each op's own bound, composed)."""
    V, src, dst, gd = c2
    torch.manual_seed(2)
    H, D = 4, 8
    gat = gnn.GATConv(16, D, H).cuda()
    h = torch.randn(V, 16, device="cuda")
    with torch.no_grad():
        out = gat(gd, h, fused=fused)
        z = h @ gat.W
        zh = z.view(-1, H, D)
        el = (zh * gat.al).sum(-1).cpu().numpy()
        er = (zh * gat.ar).sum(-1).cpu().numpy()
    zn = z.cpu().numpy()
    ref, attn, bnd = oracle.gat(V, src, dst, el, er, zn, H, 0.2, bound=True)
    # fused: the R23 bound.  Unfused: every attention a_e is rounded through exp (<= 2 ulp),
    # e_sub_v / e_div_v (1 ulp each) and a denominator summed in some order over deg(v) positive
    # terms (<= (deg(v) - 1) u relative): a_e carries <= (deg(v) + 8) u relative error, which the
    # final weighted sum passes on as (deg(v) + 8) u * sum_e a_e |z| = (deg(v) + 8) u * bnd.
    deg = np.bincount(dst, minlength=V).astype(np.float64)[:, None]
    tol = 1e-5 * bnd if fused else 1e-5 * bnd + (deg + 8) * U * bnd
    within(out, ref, tol, f"GAT fused={fused}")


@pytest.mark.parametrize("fused", [True, False])
def test_dotgat_layer(c2, fused):
    """Dot-product attention layer: the fused ug_dot_attention traversal and the unfused operator
    chain, both against oracle.dot_attention on the layer's own z (R25 bound; the unfused chain
    adds the rounding of its separately stored scores, exp and denominator, as in test_gat_layer)."""
    V, src, dst, gd = c2
    torch.manual_seed(3)
    H, D = 4, 16
    layer = gnn.DotGATConv(16, D, H).cuda()
    h = torch.randn(V, 16, device="cuda")
    with torch.no_grad():
        out = layer(gd, h, fused=fused)
        z = (h @ layer.W).cpu().numpy()
    ref, attn, bnd = oracle.dot_attention(V, src, dst, z, z, z, H, scale=1.0 / D ** 0.5, bound=True)
    deg = np.bincount(dst, minlength=V).astype(np.float64)[:, None]
    tol = 1e-5 * bnd if fused else 1e-5 * bnd + (deg + 16) * U * bnd
    within(out, ref, tol, f"DotGAT fused={fused}")
