"""Shared helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np
import torch

import oracle
import ugdata

TOL = 1e-5   # north star: max error 1e-5 normalised by sum |terms| (reading R11)


def operand_arrays(op, V, E, F, H, seed, mode, vertex_width=None, edge_width=None, dot_width=None):
    """Numpy operands for op: vertex operands width F (or vertex_width), Edge operands width
    F (or edge_width); dot operands width F."""
    eo, l, r, g, c = op
    out = []
    for i, t in enumerate((l, r)):
        if t is None:
            out.append(None)
            continue
        rows = V if t in ("u", "v") else E
        if eo == "dot":
            w = (edge_width or F) if t == "e" else (dot_width or F)
        elif t == "e":
            w = edge_width or F
        else:
            w = vertex_width or F
        role = "den" if (eo == "div" and i == 1) else ("edge" if t == "e" else "num")
        out.append(ugdata.values(rows, w, seed, 10 + i, mode=mode, role=role, k=4))
    return out


def to_dev(x, ld=None, offset=0):
    """numpy [rows, w] -> CUDA float32 tensor view with row stride ld and element offset."""
    if x is None:
        return None
    rows, w = x.shape
    ld = ld or w
    buf = torch.full((rows * ld + offset + 8,), float("nan"), dtype=torch.float32, device="cuda")
    t = buf[offset:offset + rows * ld].view(rows, ld)[:, :w]
    t.copy_(torch.from_numpy(x))
    return t


def out_tensor(op, V, E, F, H, ld=None, offset=0):
    eo, l, r, g, c = op
    W = H if eo == "dot" else F
    rows = V if c == "v" else E
    ld = ld or W
    buf = torch.full((rows * ld + offset + 8,), float("nan"), dtype=torch.float32, device="cuda")
    return buf[offset:offset + rows * ld].view(rows, ld)[:, :W]


def run_gpu(ugm, graph, op, A, B, V, E, F, H, schedule=None, ld=None, offset=0):
    eo, l, r, g, c = op
    Ad = to_dev(A, ld, offset)
    Bd = to_dev(B, ld, offset)
    C = out_tensor(op, V, E, F, H, ld, offset)
    ugm.op_run(graph, eo, g, A=Ad, a_type=l, B=Bd, b_type=r, C=C, c_type=c, F=F, H=H, schedule=schedule)
    torch.cuda.synchronize()
    return C.cpu().numpy()


def run_oracle(op, V, src, dst, A, B, F, H, rows=None):
    eo, l, r, g, c = op
    return oracle.op(V, src, dst, eo, g, A=A, a_type=l, B=B, b_type=r, c_type=c, F=F, H=H,
                     rows=rows, bound=True)


def exact_op(op):
    eo, l, r, g, c = op
    return eo != "dot" and g in ("assign", "max", "min")


def assert_parity(op, got, ref, bound, integer_mode, what=""):
    assert got.shape == ref.shape, (got.shape, ref.shape)
    if integer_mode or exact_op(op):
        bad = np.nonzero(got.view(np.uint32) != ref.view(np.uint32))
        assert bad[0].size == 0, (
            f"{what}: {bad[0].size} elements differ bitwise; first at {bad[0][0]},{bad[1][0]}: "
            f"gpu={got[bad[0][0], bad[1][0]]!r} oracle={ref[bad[0][0], bad[1][0]]!r}")
        return
    err = np.abs(got.astype(np.float64) - ref.astype(np.float64))
    lim = TOL * bound
    bad = np.nonzero(~(err <= lim))
    assert bad[0].size == 0, (
        f"{what}: {bad[0].size} elements out of tolerance; first at {bad[0][0]},{bad[1][0]}: "
        f"gpu={got[bad[0][0], bad[1][0]]!r} oracle={ref[bad[0][0], bad[1][0]]!r} bound={bound[bad[0][0], bad[1][0]]}")
