"""GPU parity of the staged SV kernel (k_svg: "_M1" TMA gather4, "_A1" cp.async) against the oracle.

Every aggregation whose gathered operand is a full-width Src_V tensor and whose second operand
is absent, Dst_V (full width or per head) or a per-edge Edge tensor (scalar or per head),
under every reducer, in float mode (1e-5 * sum|terms|) and integer mode (bit-exact), at
column widths that exercise every tile width (32 / 64 / 128 columns), ragged last tiles and
W < tile, on a dst-sorted skewed multigraph with a hub row (split into many chunks), zero
in-degree rows and self-loops; plus misaligned layouts (packed first), the full-size C3 / C5
configurations, and the schedules the kernel must reject.
"""
import itertools

import numpy as np
import pytest
import torch

import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle, to_dev, out_tensor
from opset import all_ops, name

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def svg_ops():
    out = []
    for op in all_ops():
        eo, l, r, g, c = op
        if c != "v" or eo == "dot":
            continue
        if eo == "copy_lhs" and l == "u":
            out.append(op)
        elif eo != "copy_lhs" and l == "u" and r in ("v", "e"):
            out.append(op)
    return out


@pytest.fixture(scope="module")
def sorted_graph():
    V, E = 400, 2400
    src, dst = ugdata.random_multigraph(V, E, 91, zero_in_frac=0.15)
    hub = np.arange(0, 300, dtype=np.int32)          # a hub of in-degree >= 300
    src = np.concatenate([src, hub % V]).astype(np.int32)
    dst = np.concatenate([dst, np.full(300, 7, np.int32)]).astype(np.int32)
    order = np.argsort(dst, kind="stable")            # dst-sorted: identity edge ids
    src, dst = src[order], dst[order]
    return V, len(src), src, dst, ug.Graph(V, src, dst)


SCHED = ["SV_G7_M1", "SV_G64_F32_M1", "SV_G16_F64_M1", "SV_G512_F128_M1", "SV_G5_F128_M1",
         "SV_G7_A1", "SV_G64_F32_A1", "SV_G16_F64_A1", "SV_G512_F128_A1", "SV_G5_F128_A1"]


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("op", svg_ops(), ids=name)
def test_svg_all_ops(sorted_graph, op, mode):
    V, E, src, dst, g = sorted_graph
    for (F, H, ew, vw) in ((20, 1, 1, None), (64, 4, 4, None), (100, 1, 1, None), (200, 2, 2, 2)):
        A, B = operand_arrays(op, V, E, F, H, seed=F, mode=mode, edge_width=ew)
        if op[2] == "v" and vw:
            # per-head Dst_V operand (R6 broadcast)
            B = ugdata.values(V, vw, F + 1, 11, mode=mode, role="den" if op[0] == "div" else "num", k=4)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        for sch in SCHED:
            got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
            assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F} H={H}")


@pytest.mark.parametrize("layout", [(None, 0), (101, 0), (100, 1), (104, 4)])
def test_svg_layouts(sorted_graph, layout):
    """Row strides not a multiple of 4 floats / 4-byte-offset bases are packed before TMA."""
    V, E, src, dst, g = sorted_graph
    ld, off = layout
    F = 100
    for op in [("mul", "u", "e", "sum", "v"), ("copy_lhs", "u", None, "max", "v"), ("sub", "u", "v", "mean", "v")]:
        A, B = operand_arrays(op, V, E, F, 1, seed=5, mode="float", edge_width=1)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, 1)
        for sch in ("SV_G16_M1", "SV_G16_F64_M1_P1", "SV_G16_A1", "SV_G16_F64_A1", "SV_G16_F32_A1"):
            got = run_gpu(ug, g, op, A, B, V, E, F, 1, schedule=sch, ld=ld, offset=off)
            assert_parity(op, got, ref, bound, False, what=f"{name(op)} {sch} ld={ld} off={off}")


def test_svg_rejects(sorted_graph):
    V, E, src, dst, g = sorted_graph
    X = torch.randn(V, 64, device="cuda")
    Y = torch.empty(V, 64, device="cuda")
    M = torch.empty(E, 64, device="cuda")
    wfull = torch.randn(E, 64, device="cuda")
    with pytest.raises(ug.UgError):      # message creation
        ug.op_run(g, "add", "assign", A=X, a_type="u", B=X, b_type="v", C=M, c_type="e", schedule="SV_G16_M1")
    with pytest.raises(ug.UgError):      # A is not Src_V
        ug.op_run(g, "copy_lhs", "sum", A=wfull, a_type="e", C=Y, c_type="v", schedule="SV_G16_M1")
    with pytest.raises(ug.UgError):      # full-width Edge B operand
        ug.op_run(g, "mul", "sum", A=X, a_type="u", B=wfull, b_type="e", C=Y, c_type="v", schedule="SV_G16_M1")
    with pytest.raises(ug.UgError):      # ftile not 32 / 64 / 128
        ug.op_run(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v", schedule="SV_G16_F16_M1")
    # a graph whose COO is not dst-sorted (edge ids are not CSR positions)
    g2 = ug.Graph(V, src[::-1].copy(), dst[::-1].copy())
    with pytest.raises(ug.UgError):
        ug.op_run(g2, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v", schedule="SV_G16_M1")
    assert ug.format_schedule(ug.parse_schedule("SV_G512_F128_P1_M1")) == "SV_G512_F128_P1_M1"
    assert ug.format_schedule(ug.parse_schedule("SV_G64_F64_A1")) == "SV_G64_F64_A1"


@pytest.mark.parametrize("cfg, F, sch", [("C3", 128, "SV_G512_F128_M1"), ("C3", 32, "SV_G128_F32_M1"),
                                         ("C4", 128, "SV_G128_F128_M1"), ("C3", 128, "SV_G512_F128_A1"),
                                         ("C3", 32, "SV_G128_F32_A1"), ("C4", 128, "SV_G128_F64_A1")])
def test_svg_full_size_integer_cross_schedule(cfg, F, sch):
    """Integer mode at full size: k_svg == k_split bit-for-bit on EVERY row (u_mul_e_sum, copy_u_sum,
    copy_u_max), and equal to the oracle on a sample of rows plus the hub."""
    import oracle
    c = ugdata.CONFIGS[cfg]
    src, dst = ugdata.graph(cfg)
    V, E = c.V, len(src)
    g = ug.Graph(V, src, dst)
    deg = np.bincount(dst, minlength=V)
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([rng.choice(V, 100, replace=False), [int(np.argmax(deg))]])).astype(np.int64)
    sub = np.nonzero(np.isin(dst, rows))[0]
    X = ugdata.values(V, F, 9, 1, mode="int", k=4)
    w = ugdata.values(E, 1, 9, 2, mode="int", role="edge", k=4)
    Xd, wd = to_dev(X), to_dev(w)
    for op, B, bd in ((("mul", "u", "e", "sum", "v"), w, wd), (("copy_lhs", "u", None, "sum", "v"), None, None),
                      (("copy_lhs", "u", None, "max", "v"), None, None)):
        eo, l, r, gop, cc = op
        outs = []
        for s in (sch, sch.replace("_M1", "").replace("_A1", "")):
            C = out_tensor(op, V, E, F, 1)
            ug.op_run(g, eo, gop, A=Xd, a_type="u", B=bd, b_type=r, C=C, c_type="v", F=F, H=1, schedule=s)
            outs.append(C)
        torch.cuda.synchronize()
        assert torch.equal(outs[0].view(torch.int32), outs[1].view(torch.int32)), (cfg, name(op))
        ref = oracle.op(V, src[sub], dst[sub], eo, gop, A=X, a_type="u", B=(B[sub] if B is not None else None),
                        b_type=r, c_type="v", F=F, H=1, rows=rows)
        got = outs[0][torch.from_numpy(rows).cuda()].cpu().numpy()
        np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.slow
@pytest.mark.parametrize("gop", ["sum", "mean"])
def test_svg_C5(gop):
    """C5 Reddit-shaped, F = 602 (ld 602: packed to 608 first), float mode vs the oracle on sampled
    rows; u_mul_e_sum too (the weighted aggregation)."""
    import oracle
    c = ugdata.CONFIGS["C5"]
    src, dst = ugdata.graph("C5")
    V, E = c.V, len(src)
    g = ug.Graph(V, src, dst)
    deg = np.bincount(dst, minlength=V)
    rng = np.random.default_rng(11)
    rows = np.unique(np.concatenate([rng.choice(V, 40, replace=False), [int(np.argmax(deg))]])).astype(np.int64)
    sub = np.nonzero(np.isin(dst, rows))[0]
    X = ugdata.values(V, 602, 3, 1)
    w = ugdata.values(E, 1, 3, 2, role="edge")
    Xd, wd = to_dev(X), to_dev(w)
    for (op, B, bd), sch in itertools.product(((("copy_lhs", "u", None, gop, "v"), None, None),
                                                (("mul", "u", "e", gop, "v"), w, wd)),
                                               ("SV_G512_F128_P1_M1", "SV_G512_F128_P1_A1")):
        eo, l, r, _, cc = op
        C = out_tensor(op, V, E, 602, 1)
        ug.op_run(g, eo, gop, A=Xd, a_type="u", B=bd, b_type=r, C=C, c_type="v", F=602, H=1, schedule=sch)
        torch.cuda.synchronize()
        ref, bnd = oracle.op(V, src[sub], dst[sub], eo, gop, A=X, a_type="u", B=(B[sub] if B is not None else None),
                             b_type=r, c_type="v", F=602, H=1, rows=rows, bound=True)
        got = C[torch.from_numpy(rows).cuda()].cpu().numpy()
        assert_parity(op, got, ref, bnd, False, what=f"C5 {name(op)} {sch}")
