"""GPU parity of the column-tiled SV dot kernel (k_dott: "SV_G.._F128" for u_dot_v / v_dot_u)
against the oracle, for ANY head width D = F / H (R5: the message is sum_{d<D} a_d b_d per head).

Message creation and every reducer over dot messages; float mode within 1e-5 * sum_d |a_d b_d|
(Q11 / R14), integer mode bit-exact; widths that give one tile per head (direct store), several
tiles per head (partials + tile fix-up), ragged heads (D = 301, 86, 50, 25) and odd vector widths;
a dst-sorted and an unsorted graph (edge-id indirection); misaligned rows (packing); and the
full-size C4 / C5 configurations on sampled edges.
"""
import numpy as np
import pytest
import torch

import oracle
import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle, to_dev, out_tensor

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")

OPS = [("dot", "u", "v", g, "e" if g == "assign" else "v") for g in ("assign", "sum", "max", "min", "mean")] + \
      [("dot", "v", "u", "assign", "e"), ("dot", "v", "u", "sum", "v")]
SHAPES = [(602, 1), (602, 2), (602, 7), (100, 1), (100, 2), (96, 1), (96, 2), (64, 1), (128, 4), (20, 1), (50, 2)]


def _graph(kind):
    V, E = 300, 2200
    src, dst = ugdata.random_multigraph(V, E, 41, zero_in_frac=0.15)
    hub = np.arange(0, 200, dtype=np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(200, 3, np.int32)]).astype(np.int32)
    if kind == "sorted":
        order = np.argsort(dst, kind="stable")
        src, dst = src[order], dst[order]
    return V, len(src), src, dst, ug.Graph(V, src, dst)


@pytest.fixture(scope="module", params=["sorted", "unsorted"])
def graph(request):
    return _graph(request.param)


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("F,H", SHAPES)
def test_dott_ops(graph, F, H, mode):
    V, E, src, dst, g = graph
    for op in OPS:
        A, B = operand_arrays(op, V, E, F, H, seed=F + H, mode=mode)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        for sch in ("SV_G7_F128", "SV_G64_F64", "SV_G16_F32"):
            got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
            assert_parity(op, got, ref, bound, mode == "int", what=f"{op} {sch} F={F} H={H}")


@pytest.mark.parametrize("layout", [(None, 0), (101, 0), (100, 1), (104, 2)])
def test_dott_layouts(layout):
    V, E, src, dst, g = _graph("sorted")
    ld, off = layout
    F, H = 100, 2
    op = ("dot", "u", "v", "assign", "e")
    A, B = operand_arrays(op, V, E, F, H, seed=3, mode="float")
    ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
    for sch in ("SV_G16_F128", "SV_G16_F64_P1"):
        got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch, ld=ld, offset=off)
        assert_parity(op, got, ref, bound, False, what=f"{sch} ld={ld} off={off}")


def test_dott_same_matrix_packed():
    """u_dot_v with one matrix as both operands (ld 602: packed once, used for both)."""
    V, E, src, dst, g = _graph("sorted")
    F = 602
    X = ugdata.values(V, F, 8, 1)
    Xd = to_dev(X)
    C = out_tensor(("dot", "u", "v", "assign", "e"), V, E, F, 1)
    ug.op_run(g, "dot", "assign", A=Xd, a_type="u", B=Xd, b_type="v", C=C, c_type="e", F=F, H=1,
              schedule="SV_G64_F128")
    torch.cuda.synchronize()
    ref, bnd = oracle.op(V, src, dst, "dot", "assign", A=X, a_type="u", B=X, b_type="v", c_type="e", F=F, H=1,
                         bound=True)
    assert_parity(("dot", "u", "v", "assign", "e"), C.cpu().numpy(), ref, bnd, False, what="same matrix")


@pytest.mark.parametrize("cfg,F,H", [("C4", 128, 1), ("C4", 256, 1), ("C4", 128, 4), ("C3", 128, 1)])
def test_dott_full_size(cfg, F, H):
    c = ugdata.CONFIGS[cfg]
    src, dst = ugdata.graph(cfg)
    V, E = c.V, len(src)
    g = ug.Graph(V, src, dst)
    X = ugdata.values(V, F, 4, 1, mode="int", k=2)
    Xd = to_dev(X)
    op = ("dot", "u", "v", "assign", "e")
    C = out_tensor(op, V, E, F, H)
    ug.op_run(g, "dot", "assign", A=Xd, a_type="u", B=Xd, b_type="v", C=C, c_type="e", F=F, H=H,
              schedule="SV_G256_F128")
    torch.cuda.synchronize()
    rng = np.random.default_rng(3)
    erows = np.unique(np.concatenate([rng.choice(E, 3000, replace=False), [0, E - 1]])).astype(np.int64)
    ref = oracle.op(V, src[erows], dst[erows], "dot", "assign", A=X, a_type="u", B=X, b_type="v", c_type="e",
                    F=F, H=H)
    got = C[torch.from_numpy(erows).cuda()].cpu().numpy()
    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.slow
@pytest.mark.parametrize("gop", ["assign", "sum"])
def test_dott_C5(gop):
    """C5 Reddit-shaped u_dot_v / u_dot_v_sum at F = 602 (5 column tiles per head), float mode,
    sampled edges / rows vs the oracle."""
    c = ugdata.CONFIGS["C5"]
    src, dst = ugdata.graph("C5")
    V, E = c.V, len(src)
    g = ug.Graph(V, src, dst)
    X = ugdata.values(V, 602, 6, 1)
    Xd = to_dev(X)
    cty = "e" if gop == "assign" else "v"
    op = ("dot", "u", "v", gop, cty)
    C = out_tensor(op, V, E, 602, 1)
    ug.op_run(g, "dot", gop, A=Xd, a_type="u", B=Xd, b_type="v", C=C, c_type=cty, F=602, H=1,
              schedule="SV_G512_F128")
    torch.cuda.synchronize()
    rng = np.random.default_rng(9)
    if gop == "assign":
        rows = np.unique(np.concatenate([rng.choice(E, 4000, replace=False), [0, E - 1]])).astype(np.int64)
        ref, bnd = oracle.op(V, src[rows], dst[rows], "dot", gop, A=X, a_type="u", B=X, b_type="v", c_type="e",
                             F=602, H=1, bound=True)
    else:
        deg = np.bincount(dst, minlength=V)
        rows = np.unique(np.concatenate([rng.choice(V, 30, replace=False), [int(np.argmax(deg))]])).astype(np.int64)
        sub = np.nonzero(np.isin(dst, rows))[0]
        ref, bnd = oracle.op(V, src[sub], dst[sub], "dot", gop, A=X, a_type="u", B=X, b_type="v", c_type="v",
                             F=602, H=1, rows=rows, bound=True)
    got = C[torch.from_numpy(rows).cuda()].cpu().numpy()
    assert_parity(op, got, ref, bnd, False, what=f"C5 u_dot_v {gop}")
