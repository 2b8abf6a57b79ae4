"""GPU parity of the edge-lanes vertex schedules ("WV_G1_T1_E1": a warp per row; "WV_Gg_T1_E1": g rows
sharing a warp's lanes (k_vertex_seg); "TV_Gg_Tt_E1": t in {8, 16} lanes per row, 32 / t rows per
warp; k_vertex_el): every
aggregation op (all 32 message functions except dot x 4 reducers) in float mode (1e-5 * sum|terms|)
and integer mode (bit-exact), widths 1..8 feature vectors, on an unsorted skewed multigraph
(edge-id indirection, a hub row wider than the warp, zero in-degree rows)."""
import numpy as np
import pytest

import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle
from opset import all_ops, name

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


@pytest.fixture(scope="module")
def graph():
    V, E = 300, 1500
    src, dst = ugdata.random_multigraph(V, E, 33, zero_in_frac=0.15)
    hub = np.arange(0, 150, dtype=np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(150, 9, np.int32)]).astype(np.int32)
    return V, len(src), src, dst, ug.Graph(V, src, dst)


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("op", [o for o in all_ops() if o[4] == "v" and o[0] != "dot"], ids=name)
def test_edgelanes_all_aggregations(graph, op, mode):
    V, E, src, dst, g = graph
    for (F, H, ew) in ((20, 1, 1), (12, 3, 3), (32, 1, 32), (4, 1, 1), (8, 1, 8)):
        A, B = operand_arrays(op, V, E, F, H, seed=F, mode=mode, edge_width=ew)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        # WV_G{2,4,8}_T1_E1 with G * N <= 32 values: the segmented kernel (k_vertex_seg), else
        # G rows one after another
        for sch in ("WV_G1_T1_E1", "WV_G4_T1_E1", "WV_G2_T1_E1", "WV_G8_T1_E1", "TV_G1_T8_E1", "TV_G3_T16_E1"):
            got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
            assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F} H={H}")


def test_edgelanes_rejects(graph):
    import torch
    V, E, src, dst, g = graph
    X = torch.randn(V, 64, device="cuda")
    Y = torch.empty(V, 64, device="cuda")
    M = torch.empty(E, 8, device="cuda")
    with pytest.raises(ug.UgError):      # 16 float4 chunks > 8
        ug.op_run(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v", schedule="WV_G1_T1_E1")
    with pytest.raises(ug.UgError):      # message creation
        ug.op_run(g, "copy_lhs", "assign", A=X[:, :8], a_type="u", C=M, c_type="e", F=8,
                  schedule="WV_G1_T1_E1")
    for bad in ("TV_G1_T1_E1", "TV_G1_T4_E1", "WV_G1_T2_E1", "BV_G1_E1"):   # lanes per row: WV 32, TV 8 / 16
        with pytest.raises(ug.UgError):
            ug.op_run(g, "copy_lhs", "sum", A=X[:, :8], a_type="u", C=Y[:, :8], c_type="v", F=8,
                      schedule=bad)
    assert ug.format_schedule(ug.parse_schedule("WV_G4_T1_E1")) == "WV_G4_T1_E1"


@pytest.fixture(scope="module")
def sorted_graph(graph):
    V, E, src, dst, _ = graph
    order = np.argsort(dst, kind="stable")
    return V, E, src[order], dst[order], ug.Graph(V, src[order], dst[order])


@pytest.mark.parametrize("kind", ["unsorted", "sorted"])
@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("op", [o for o in all_ops() if o[3] == "assign" and o[0] != "dot"], ids=name)
def test_edgelanes_message_creation(graph, sorted_graph, op, mode, kind):
    """SV message creation with lanes over edges ("SV_G.._E1", k_msg_el): bit-exact messages for
    W = 1, 3 (per-head operands of width 1) and 8 -- on the unsorted graph (generic form, stores
    through eid) and the dst-sorted one (the fast form for Src_V A with none / Dst_V / Edge B)."""
    V, E, src, dst, g = graph if kind == "unsorted" else sorted_graph
    for (F, H, ew) in ((1, 1, 1), (3, 3, 1), (8, 2, 8)):
        A, B = operand_arrays(op, V, E, F, H, seed=F + 7, mode=mode, edge_width=ew)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
        for sch in ("SV_G7_E1", "SV_G1024_E1"):
            got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
            assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F} H={H}")
