#!/usr/bin/env python
"""Device time (CUDA events queued behind a spin kernel, median) of one op on one config
under a list of schedules (AUTO first).  Experiments only.

    python scripts/time_ops.py C3 u_mul_e_sum 128 SV_G128_F128 TE_G32_T16
"""
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402

OPS = {  # name -> (edge_op, gather, A type, B type, C type, B width (None = F))
    "copy_u_sum": ("copy_lhs", "sum", "u", None, "v", None),
    "copy_u_mean": ("copy_lhs", "mean", "u", None, "v", None),
    "copy_u_max": ("copy_lhs", "max", "u", None, "v", None),
    "u_mul_e_sum": ("mul", "sum", "u", "e", "v", 1),
    "u_add_v_sum": ("add", "sum", "u", "v", "v", None),
    "u_mul_v_sum": ("mul", "sum", "u", "v", "v", None),
    "u_add_v": ("add", "assign", "u", "v", "e", None),
    "u_dot_v": ("dot", "assign", "u", "v", "e", None),
}


def main():
    cfg, op, F = sys.argv[1], sys.argv[2], int(sys.argv[3])
    scheds = sys.argv[4:]
    eo, go, a, b, c, bw = OPS[op]
    C = ugdata.CONFIGS[cfg]
    src, dst = ugdata.graph(cfg)
    g = ug.Graph(C.V, src, dst)
    E = len(src)
    rows = lambda t: C.V if t in ("u", "v") else E
    A = torch.rand(rows(a), F, device="cuda") - 0.5
    B = (torch.rand(rows(b), bw or F, device="cuda") + 0.5) if b else None
    W = 1 if eo == "dot" else F
    out = torch.empty(C.V if c == "v" else E, W, device="cuda")
    kw = dict(A=A, a_type=a, B=B, b_type=b, C=out, c_type=c, F=F, H=1)
    res = []
    for s in [None] + scheds:
        name = s or "AUTO:" + ug.schedule_select(g, eo, go, **kw)
        try:
            for _ in range(3):
                ug.op_run(g, eo, go, schedule=s, **kw)
            ts = []
            for _ in range(15):
                torch.cuda._sleep(200_000)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                ug.op_run(g, eo, go, schedule=s, **kw)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e3)
            res.append((name, round(statistics.median(ts), 1)))
        except ug.UgError as e:
            res.append((name, str(e)[:60]))
    print(json.dumps({"config": cfg, "op": op, "F": F, "us": res}))


if __name__ == "__main__":
    main()
