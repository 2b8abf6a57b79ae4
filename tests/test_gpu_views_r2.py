"""Row views (the sharded form's local graphs, ug_graph_view_rows) through the round-2 kernels:
the single-launch SV merge, the edge-lanes schedule, the column-tiled SV dot (k_dott) and the
fused dot attention.  Each shard's output, concatenated in row order, must equal the unsharded
call: bit-exact in integer mode (every partial sum exact); for the attention (exp) within the
R25 bound of the unsharded oracle.  Views index Src_V operands globally, Dst_V / C rows and Edge
rows locally (include/ug.h)."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def _graph():
    V, E = 2000, 16000
    src, dst = ugdata.random_multigraph(V, E, 19, zero_in_frac=0.1)
    hub = np.arange(0, 600, dtype=np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(600, 11, np.int32)]).astype(np.int32)
    order = np.argsort(dst, kind="stable")           # views need a dst-sorted graph
    return V, src[order], dst[order]


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("eo,gop,sch", [("copy_lhs", "sum", "SV_G16"), ("mul", "max", "SV_G8_F32"),
                                        ("copy_lhs", "mean", "WV_G1_T1_E1"), ("mul", "sum", "WV_G2_T1_E1")])
def test_views_aggregation(P, eo, gop, sch):
    V, src, dst = _graph()
    g = ug.Graph(V, src, dst)
    E = len(src)
    F = 16
    X = torch.from_numpy(ugdata.values(V, F, 4, 1, mode="int", k=4)).cuda()
    w = torch.from_numpy(ugdata.values(E, 1, 4, 2, mode="int", role="edge", k=4)).cuda()
    kw = dict(A=X, a_type="u", B=w if eo == "mul" else None, b_type="e" if eo == "mul" else None)
    full = torch.empty(V, F, device="cuda")
    ug.op_run(g, eo, gop, C=full, c_type="v", schedule=sch, **kw)
    sp = g.partition(P)
    rp = g.row_ptr()
    parts = []
    for k in range(P):
        r0, r1 = int(sp[k]), int(sp[k + 1])
        view = g.view_rows(r0, r1)
        kv = dict(kw)
        if eo == "mul":
            kv["B"] = w[int(rp[r0]):int(rp[r1])]
        out = torch.empty(r1 - r0, F, device="cuda")
        ug.op_run(view, eo, gop, C=out, c_type="v", schedule=sch, **kv)
        parts.append(out)
    torch.cuda.synchronize()
    assert torch.equal(torch.cat(parts).view(torch.int32), full.view(torch.int32)), (P, eo, gop, sch)


@pytest.mark.parametrize("P", [2, 3])
def test_views_dott(P):
    V, src, dst = _graph()
    g = ug.Graph(V, src, dst)
    E = len(src)
    F = 300                                              # 3 column tiles of 128 (k_dott partials)
    X = torch.from_numpy(ugdata.values(V, F, 6, 1, mode="int", k=2)).cuda()
    full = torch.empty(E, 1, device="cuda")
    ug.op_run(g, "dot", "assign", A=X, a_type="u", B=X, b_type="v", C=full, c_type="e", F=F, H=1,
              schedule="SV_G64_F128")
    sp = g.partition(P)
    rp = g.row_ptr()
    parts = []
    for k in range(P):
        r0, r1 = int(sp[k]), int(sp[k + 1])
        view = g.view_rows(r0, r1)
        out = torch.empty(int(rp[r1] - rp[r0]), 1, device="cuda")
        ug.op_run(view, "dot", "assign", A=X, a_type="u", B=X[r0:r1], b_type="v", C=out, c_type="e", F=F, H=1,
                  schedule="SV_G64_F128")
        parts.append(out)
    torch.cuda.synchronize()
    assert torch.equal(torch.cat(parts).view(torch.int32), full.view(torch.int32))


@pytest.mark.parametrize("H,D", [(4, 8), (1, 128)])
def test_views_dot_attention(H, D):
    V, src, dst = _graph()
    g = ug.Graph(V, src, dst)
    F = H * D
    q = ugdata.values(V, F, 8, 1)
    k = ugdata.values(V, F, 8, 2)
    val = ugdata.values(V, F, 8, 3)
    qd, kd, vd = (torch.from_numpy(x).cuda() for x in (q, k, val))
    sp = g.partition(3)
    parts = []
    for i in range(3):
        r0, r1 = int(sp[i]), int(sp[i + 1])
        parts.append(ug.dot_attention(g.view_rows(r0, r1), qd[r0:r1], kd, vd, H))
    torch.cuda.synchronize()
    got = torch.cat(parts).cpu().numpy().astype(np.float64)
    ref, _, bnd = oracle.dot_attention(V, src, dst, q, k, val, H, bound=True)
    assert np.all(np.abs(got - ref) <= 1e-5 * bnd)
