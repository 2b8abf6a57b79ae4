"""GPU parity of the SV dot kernel (k_dotsv: u_dot_v / v_dot_u with the Dst_V row held in
registers per work unit) against the CPU oracle, for every gather (message creation and the
four reducers), several (F, H) shapes that the kernel takes (one head per lane, butterfly
over the head's lanes), chunk sizes that split the hub row, float and integer mode.
Integer mode is bit-exact; float mode within 1e-5 * sum|a_d b_d| (reading R11 / R14)."""
import numpy as np
import pytest

import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")

SHAPES = [(16, 1), (64, 1), (128, 1), (256, 1), (128, 4), (64, 8), (32, 2), (8, 1), (24, 3)]
GATHERS = [("assign", "e"), ("sum", "v"), ("max", "v"), ("min", "v"), ("mean", "v")]


@pytest.fixture(scope="module")
def graph():
    V, E = 400, 2400
    src, dst = ugdata.random_multigraph(V, E, 91, zero_in_frac=0.1)
    hub = np.arange(0, 150, dtype=np.int32)          # hub row of in-degree >= 150 (split at G <= 128)
    src = np.concatenate([src, (hub * 7) % V])
    dst = np.concatenate([dst, np.full(150, 9, np.int32)])
    return V, len(src), src, dst, ug.Graph(V, src, dst)


@pytest.mark.parametrize("F,H", SHAPES)
@pytest.mark.parametrize("mode", ["float", "int"])
def test_dotsv_parity(graph, F, H, mode):
    V, E, src, dst, g = graph
    for lhs, rhs in (("u", "v"), ("v", "u")):
        for gop, c in GATHERS:
            op = ("dot", lhs, rhs, gop, c)
            A, B = operand_arrays(op, V, E, F, H, seed=F + H, mode=mode)
            ref, bound = run_oracle(op, V, src, dst, A, B, F, H)
            for sch in ("SV_G4", "SV_G32", "SV_G2048"):
                got = run_gpu(ug, g, op, A, B, V, E, F, H, schedule=sch)
                assert_parity(op, got, ref, bound, mode == "int", what=f"{lhs}_dot_{rhs} {gop} F={F} H={H} {sch}")


def test_dotsv_is_the_kernel_that_runs(graph):
    """Reductions under SV_G4 split the hub row: k_dotsv + the chunk-order fix-up = 2 launches
    (the generic vertex-unit dot kernel would be 1); a shape the kernel does not take (H = 3
    heads of D = 6 features at vec 2: 3 lanes per head) keeps the generic kernel."""
    import torch
    V, E, src, dst, g = graph
    X = torch.zeros(V, 128, device="cuda")
    Y = torch.zeros(V, 1, device="cuda")
    assert ug.launch_count(g, "dot", "sum", A=X, a_type="u", B=X, b_type="v", C=Y, c_type="v",
                           F=128, H=1, schedule="SV_G4") == 2
    X3 = torch.zeros(V, 18, device="cuda")
    Y3 = torch.zeros(V, 3, device="cuda")
    assert ug.launch_count(g, "dot", "sum", A=X3, a_type="u", B=X3, b_type="v", C=Y3, c_type="v",
                           F=18, H=3, schedule="SV_G4") == 1
