"""GPU parity: every op x every schedule family through the C ABI vs the CPU oracle.

Bit-exact for copy / elementwise messages and max/min (and for everything in integer mode);
|gpu - oracle| <= 1e-5 * sum|terms| for sum / mean / dot (reading R11, north star).
"""
import numpy as np
import pytest
import torch

import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle
from opset import all_ops, name

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")

# Every schedule family (Fig. 6 + north-star block level + the B200 SV schedule),
# with grouping / tiling / tile-major variants.  Each is exercised on all 160 ops.
SCHEDULES = ["TV_G1_T1", "TV_G3_T4", "WV_G1_T1", "WV_G2_T2_F8", "TE_G1_T4", "TE_G5_T32",
             "WE_G7_T1", "WE_G2_T2_F8", "BV_G1", "BV_G3_B128", "BE_G64", "SV_G7", "SV_G64_F8",
             "TV_G1_T8_V1", "WE_G4_T1_V1", "SV_G16_P1", "SV_G64_F8_P1"]


@pytest.fixture(scope="module")
def small_graph():
    # C1-shaped degree skew, scaled down, NOT dst-sorted: exercises the eid indirection.
    V, E = 300, 1500
    src, dst = ugdata.random_multigraph(V, E, 77, zero_in_frac=0.15)
    hub = np.arange(0, 120, dtype=np.int32)        # one hub row of in-degree >= 120
    src = np.concatenate([src, hub % V])
    dst = np.concatenate([dst, np.full(120, 5, np.int32)])
    g = ug.Graph(V, src, dst)
    return V, len(src), src, dst, g


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("op", all_ops(), ids=name)
def test_all_ops_all_schedules(small_graph, op, mode):
    V, E, src, dst, g = small_graph
    for (F, H, ew) in ((20, 1, 1), (18, 3, 3)):
        A, B = operand_arrays(op, V, E, F, H, seed=F, mode=mode, edge_width=ew)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        for sch in SCHEDULES:
            got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
            assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F}")


@pytest.mark.parametrize("op", [o for o in all_ops() if o[0] in ("copy_lhs", "mul", "dot")], ids=name)
def test_auto_schedule_and_broadcast_vertex(small_graph, op):
    """AUTO schedule; vertex operands of width H (per-head broadcast, R6)."""
    V, E, src, dst, g = small_graph
    F, H = 16, 4
    A, B = operand_arrays(op, V, E, F, H, seed=3, mode="float", vertex_width=None if op[0] == "dot" else H,
                          edge_width=H)
    ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
    got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=None)
    assert_parity(op, got, ref, bound, False, what=name(op))


@pytest.mark.parametrize("layout", [(None, 0), (24, 0), (23, 1), (20, 2)])
@pytest.mark.parametrize("sch", ["WV_G1_T1", "TE_G2_T8", "SV_G16", "SV_G16_P1", "BV_G1", "TV_G1_T4", None])
def test_strided_and_misaligned_layouts(small_graph, layout, sch):
    """Row stride ld > width and 4/8-byte-offset base pointers select narrower vectors."""
    V, E, src, dst, g = small_graph
    ld, off = layout
    F, H = 18, 1
    for op in [("mul", "u", "e", "sum", "v"), ("sub", "v", "u", "assign", "e"), ("copy_lhs", "u", None, "max", "v")]:
        A, B = operand_arrays(op, V, E, F, H, seed=5, mode="float", edge_width=1)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch, ld=ld, offset=off)
        assert_parity(op, got, ref, bound, False, what=f"{name(op)} {sch} ld={ld} off={off}")


def test_padding_untouched(small_graph):
    """C's padding columns (ld > width) are never written."""
    V, E, src, dst, g = small_graph
    X = torch.randn(V, 18, device="cuda")
    buf = torch.full((V, 24), float("nan"), device="cuda")
    C = buf[:, :18]
    for sch in ["WV_G1_T1", "SV_G16", "TE_G4_T8", "BV_G1", "WE_G4_T1_V2", "SV_G4_F4_V2"]:
        ug.op_run(g, "copy_lhs", "mean", A=X, a_type="u", C=C, c_type="v", schedule=sch)
        torch.cuda.synchronize()
        assert torch.isnan(buf[:, 18:]).all(), sch


def test_forced_vec_alignment_error(small_graph):
    V, E, src, dst, g = small_graph
    X = torch.randn(V, 18, device="cuda")
    C = torch.empty(V, 18, device="cuda")
    with pytest.raises(ug.UgError, match="ALIGNMENT"):
        ug.op_run(g, "copy_lhs", "sum", A=X, a_type="u", C=C, c_type="v", schedule="WV_G1_T1_V4")


def test_empty_and_degenerate_graphs():
    for (V, src, dst) in [(5, np.zeros(0, np.int32), np.zeros(0, np.int32)),
                          (1, np.zeros(3, np.int32), np.zeros(3, np.int32)),
                          (4, np.array([3, 3], np.int32), np.array([0, 0], np.int32))]:
        g = ug.Graph(V, src, dst)
        E = len(src)
        for op in [("copy_lhs", "u", None, "sum", "v"), ("copy_lhs", "u", None, "max", "v"),
                   ("add", "u", "v", "mean", "v"), ("mul", "u", "v", "assign", "e"),
                   ("dot", "u", "v", "min", "v")]:
            A, B = operand_arrays(op, V, E, 8, 1, seed=1, mode="int")
            ref, bound = run_oracle(op, V, src, dst, A, B, 8, 1)
            for sch in ["TV_G1_T1", "WV_G1_T1", "TE_G1_T8", "WE_G2_T1", "BV_G1", "BE_G32", "SV_G2"]:
                got = run_gpu(ug, g, op, A, B, V, E, 8, 1, schedule=sch)
                assert_parity(op, got, ref, bound, True, what=f"{name(op)} {sch} V={V} E={E}")


def test_signed_zero_max_min():
    """-0 < +0 in max/min on owner-computes and atomic schedules (R12)."""
    src = np.array([0, 1, 0, 1], np.int32)
    dst = np.array([2, 2, 3, 3], np.int32)
    g = ug.Graph(4, src, dst)
    X = torch.tensor([[-0.0], [0.0], [0.0], [0.0]], device="cuda")
    for sch in ["TV_G1_T1", "WV_G1_T1", "TE_G1_T1", "TE_G4_T1", "BV_G1", "SV_G1", "SV_G8"]:
        mx = torch.empty(4, 1, device="cuda")
        mn = torch.empty(4, 1, device="cuda")
        ug.op_run(g, "copy_lhs", "max", A=X, a_type="u", C=mx, c_type="v", schedule=sch)
        ug.op_run(g, "copy_lhs", "min", A=X, a_type="u", C=mn, c_type="v", schedule=sch)
        torch.cuda.synchronize()
        assert not torch.signbit(mx[2, 0]) and torch.signbit(mn[2, 0]), sch


def test_cross_schedule_bitwise_agreement(small_graph):
    """All schedules agree bit-exactly on exact ops (float mode)."""
    V, E, src, dst, g = small_graph
    for op in [("sub", "u", "e", "max", "v"), ("div", "e", "v", "assign", "e"), ("copy_lhs", "e", None, "min", "v")]:
        A, B = operand_arrays(op, V, E, 16, 2, seed=9, mode="float", edge_width=2)
        outs = [run_gpu(ug, g, op, A, B, V, E, 16, 2, schedule=s) for s in SCHEDULES]
        for o in outs[1:]:
            np.testing.assert_array_equal(o.view(np.uint32), outs[0].view(np.uint32))


def test_torch_third_opinion(small_graph):
    """Test-only library cross-check: torch.scatter_reduce (include_self=False)."""
    V, E, src, dst, g = small_graph
    X = torch.randn(V, 32, device="cuda")
    s = torch.from_numpy(src).long().cuda()
    d = torch.from_numpy(dst).long().cuda()
    idx = d[:, None].expand(-1, 32)
    for gop, red in (("max", "amax"), ("min", "amin"), ("sum", "sum"), ("mean", "mean")):
        C = torch.empty(V, 32, device="cuda")
        ug.op_run(g, "copy_lhs", gop, A=X, a_type="u", C=C, c_type="v")
        ref = torch.zeros(V, 32, device="cuda").scatter_reduce(0, idx, X[s], red, include_self=False)
        torch.testing.assert_close(C, ref, rtol=1e-5, atol=1e-5)


@pytest.mark.parametrize("mode", ["float", "int"])
def test_message_creation_sv_fast_path(mode):
    """Message creation (gather assign, C = Edge) under SV on a dst-sorted graph (edge id = CSR
    position): the fast path with the Src_V row gathered per edge and the B operand by addressing
    mode (none / Dst_V hoisted / Edge / Src_V) -- bit-exact against the oracle for all 32 ops."""
    V, E = 300, 1500
    src, dst = ugdata.random_multigraph(V, E, 78, zero_in_frac=0.15)
    order = np.argsort(dst, kind="stable")
    src, dst = src[order], dst[order]
    g = ug.Graph(V, src, dst)
    ops = [o for o in all_ops() if o[3] == "assign"]
    assert len(ops) == 32
    for op in ops:
        for (F, H, ew) in ((20, 1, 1), (18, 3, 3), (64, 1, 64)):
            A, B = operand_arrays(op, V, E, F, H, seed=F + 1, mode=mode, edge_width=ew)
            ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
            for sch in ("SV_G7", "SV_G64_F8", "SV_G16_P1", "SV_G32_F64"):
                got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
                assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F}")


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("kind", ["sorted", "unsorted"])
def test_sv_non_power_of_two_tiles(mode, kind):
    """SV column tiles whose width is not a power of two lanes (F12 / F24 / F40 at float4: 3, 6, 10
    lanes of a 4 / 8 / 16-lane unit, the rest idle) on every aggregation op: the fast path with
    each B addressing mode (sorted graph, incl. the contiguous edge weight of BM 6) and the generic
    one (unsorted: eid), the single-launch merge of split rows (small operator) included."""
    V, E = 300, 1500
    src, dst = ugdata.random_multigraph(V, E, 79, zero_in_frac=0.15)
    hub = np.arange(0, 140, dtype=np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(140, 11, np.int32)]).astype(np.int32)
    if kind == "sorted":
        order = np.argsort(dst, kind="stable")
        src, dst = src[order], dst[order]
    E = len(src)
    g = ug.Graph(V, src, dst)
    for op in [o for o in all_ops() if o[4] == "v" and o[0] != "dot"]:
        for (F, H, ew) in ((20, 1, 1), (24, 2, 2)):
            A, B = operand_arrays(op, V, E, F, H, seed=F + 5, mode=mode, edge_width=ew)
            ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
            for sch in ("SV_G7_F12", "SV_G64_F24_P1", "SV_G16_F40"):
                got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
                assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F} {kind}")
