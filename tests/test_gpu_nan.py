"""NaN inputs (R12): a max / min over messages any of which is NaN is the canonical NaN
0x7FFFFFFF on EVERY schedule (owner-computes max.NaN / min.NaN, the atomic integer-order path with
an absorbing NaN code, the SV merge, arg capture) -- bit-exact against the oracle; sums and means
propagate NaN to exactly the rows the oracle does; op_run_arg returns the first NaN in-edge."""
import numpy as np
import pytest
import torch

import oracle
import ugdata
from gpu_util import run_gpu
from opset import all_ops, name

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")

SCHEDULES = ["TV_G1_T1", "WV_G2_T2_F8", "TE_G1_T4", "WE_G7_T1", "BV_G1", "BE_G64", "SV_G7", "SV_G64_F8",
             "SV_G16_P1", None]


def _graph():
    V, E = 200, 1200
    src, dst = ugdata.random_multigraph(V, E, 55, zero_in_frac=0.15)
    hub = np.arange(0, 90, dtype=np.int32)
    src = np.concatenate([src, hub]).astype(np.int32)
    dst = np.concatenate([dst, np.full(90, 4, np.int32)]).astype(np.int32)
    return V, len(src), src, dst


def _nan_inputs(op, V, E, F, seed):
    eo, l, r, g, c = op
    rng = np.random.default_rng(seed)
    out = []
    for i, t in enumerate((l, r)):
        if t is None:
            out.append(None)
            continue
        rows = V if t in ("u", "v") else E
        w = F if t != "e" else 1
        x = ugdata.values(rows, w, seed, 10 + i, role="den" if (eo == "div" and i == 1) else "num")
        x[rng.random(x.shape) < 0.02] = np.nan
        out.append(x)
    return out


@pytest.mark.parametrize("op", [o for o in all_ops() if o[3] in ("max", "min", "sum") and o[0] != "dot"], ids=name)
def test_nan_all_schedules(op):
    V, E, src, dst = _graph()
    g = ug.Graph(V, src, dst)
    F = 12
    A, B = _nan_inputs(op, V, E, F, 7)
    ref = oracle.op(V, src, dst, op[0], op[3], A=A, a_type=op[1], B=B, b_type=op[2], c_type="v", F=F, H=1)
    for sch in SCHEDULES:
        got = run_gpu(ug, g, op, A, B, V, E, F, 1, schedule=sch)
        assert np.array_equal(np.isnan(got), np.isnan(ref)), (name(op), sch)
        if op[3] in ("max", "min"):
            assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (name(op), sch)


@pytest.mark.parametrize("gop", ["max", "min"])
def test_nan_arg_capture(gop):
    V, E, src, dst = _graph()
    g = ug.Graph(V, src, dst)
    F = 8
    X = ugdata.values(V, F, 3, 1)
    X[np.random.default_rng(2).random(X.shape) < 0.03] = np.nan
    C = torch.empty(V, F, device="cuda")
    arg = ug.op_run_arg(g, "copy_lhs", gop, A=torch.from_numpy(X).cuda(), a_type="u", C=C, F=F)
    torch.cuda.synchronize()
    Cr, ar = oracle.op_arg(V, src, dst, "copy_lhs", gop, A=X, a_type="u", F=F)
    np.testing.assert_array_equal(C.cpu().numpy().view(np.uint32), Cr.view(np.uint32))
    np.testing.assert_array_equal(arg.cpu().numpy(), ar)
