"""GNN layers through the DGL-style shim vs a CPU reference built from the
oracle's graph operators and fp64 numpy dense algebra."""
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


def close(got, ref, rtol=2e-4):
    got = got.detach().cpu().numpy()
    scale = np.abs(ref).max() + 1e-6
    np.testing.assert_allclose(got, ref, rtol=rtol, atol=rtol * scale)


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
    z = mm(h.cpu().numpy(), layer.W.detach().cpu().numpy())
    ref = oracle.op(V, src, dst, "mul", "sum", z, "u", w.cpu().numpy(), "e", F=16) + layer.b.detach().cpu().numpy()
    close(out, ref)


def test_gin_and_sage_layers(c2):
    V, src, dst, gd = c2
    torch.manual_seed(1)
    h = torch.randn(V, 24, device="cuda")
    hn = h.cpu().numpy()
    gin = gnn.GINConv(24, 16, eps=0.1).cuda()
    with torch.no_grad():
        out = gin(gd, h)
    agg = oracle.op(V, src, dst, "copy_lhs", "sum", hn, "u", F=24)
    x = (1.1 * hn.astype(np.float64) + agg).astype(np.float32)
    l1 = np.maximum(mm(x, gin.l1.weight.detach().cpu().numpy().T) + gin.l1.bias.detach().cpu().numpy(), 0)
    ref = mm(l1, gin.l2.weight.detach().cpu().numpy().T) + gin.l2.bias.detach().cpu().numpy()
    close(out, ref)
    for aggr in ("sum", "mean", "max"):
        sage = gnn.SAGEConv(24, 16, aggr).cuda()
        with torch.no_grad():
            out = sage(gd, h)
        a = oracle.op(V, src, dst, "copy_lhs", aggr, hn, "u", F=24)
        ref = (mm(hn, sage.self_lin.weight.detach().cpu().numpy().T) + sage.self_lin.bias.detach().cpu().numpy()
               + mm(a, sage.neigh_lin.weight.detach().cpu().numpy().T))
        close(out, ref)


def test_gat_layer(c2):
    V, src, dst, gd = c2
    torch.manual_seed(2)
    H, D = 4, 8
    gat = gnn.GATConv(16, D, H).cuda()
    h = torch.randn(V, 16, device="cuda")
    with torch.no_grad():
        out = gat(gd, h)
    z = mm(h.cpu().numpy(), gat.W.detach().cpu().numpy())
    zh = z.reshape(V, H, D).astype(np.float64)
    el = (zh * gat.al.detach().cpu().numpy()).sum(-1).astype(np.float32)
    er = (zh * gat.ar.detach().cpu().numpy()).sum(-1).astype(np.float32)
    e = oracle.op(V, src, dst, "add", "assign", el, "u", er, "v", c_type="e", F=H, H=H)
    e = np.where(e > 0, e, 0.2 * e).astype(np.float32)
    emax = oracle.op(V, src, dst, "copy_lhs", "max", e, "e", F=H, H=H)
    es = oracle.op(V, src, dst, "sub", "assign", e, "e", emax, "v", c_type="e", F=H, H=H)
    ex = np.exp(es.astype(np.float64)).astype(np.float32)
    den = oracle.op(V, src, dst, "copy_lhs", "sum", ex, "e", F=H, H=H)
    a = oracle.op(V, src, dst, "div", "assign", ex, "e", den, "v", c_type="e", F=H, H=H)
    ref = oracle.op(V, src, dst, "mul", "sum", z, "u", a, "e", F=H * D, H=H)
    close(out, ref, rtol=5e-4)
