"""GPU parity of the SV loops for a contiguous per-edge scalar weight (k_split.cuh BM 6 at 6 CTAs / SM,
BM 7 at 8 CTAs / SM; GCN's u_mul_e_sum with an [E, 1] weight, the product folded into the sum by FMA,
DESIGN.md R11) against the oracle, float mode within 1e-5 * sum|terms| and integer mode bit-exact.

The graph is large and sparse (600 K rows, 1.2 M in-edges, mean in-degree 2, one hub row of 3,000
in-edges) so that the launcher's BM 7 rule fires (chunks of < 32 in-edges on average, a grid of
>= 4 waves at 8 CTAs / SM) while E * W < 2^26 keeps the single-launch merge instance of the split
hub row (last-arriving chunk); max takes BM 6 (BM 7 is sum / mean only)."""
import numpy as np
import pytest

import ugdata
from gpu_util import assert_parity, operand_arrays, run_gpu, run_oracle
from opset import name

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


@pytest.fixture(scope="module")
def big_sparse():
    V, E = 600_000, 1_200_000
    src, dst = ugdata.random_multigraph(V, E, 91, zero_in_frac=0.1)
    hub = (np.arange(3000, dtype=np.int64) * 7919 % V).astype(np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(3000, 12345, np.int32)]).astype(np.int32)
    order = np.argsort(dst, kind="stable")          # dst-sorted: identity edge ids (the fast path)
    src, dst = src[order], dst[order]
    return V, len(src), src, dst, ug.Graph(V, src, dst)


@pytest.mark.parametrize("mode", ["float", "int"])
@pytest.mark.parametrize("gop", ["sum", "mean", "max"])
def test_contiguous_edge_weight_modes(big_sparse, gop, mode):
    V, E, src, dst, g = big_sparse
    op = ("mul", "u", "e", gop, "v")
    for F, sch in ((32, "SV_G128_F32"), (32, "SV_G16_F16"), (8, "SV_G64"), (32, None)):
        A, B = operand_arrays(op, V, E, F, 1, seed=F + 3, mode=mode, edge_width=1)
        assert B.shape == (E, 1)
        ref, bound = run_oracle(op, V, src, dst, A, B, F, 1)
        got = run_gpu(ug, g, op, A, B, V, E, F, 1, schedule=sch)
        assert_parity(op, got, ref, bound, mode == "int", what=f"{name(op)} {sch} F={F}")
