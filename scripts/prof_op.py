#!/usr/bin/env python
"""Run one operator on one config a few times (for ncu / compute-sanitizer / quick timing).

    python scripts/prof_op.py --config C3 --op u_mul_e_sum --F 128 --schedule TE_G32_T16 --reps 5
"""
import argparse
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402

OPS = {
    "copy_u_sum": ("copy_lhs", "sum", "u", None, "v"),
    "copy_u_mean": ("copy_lhs", "mean", "u", None, "v"),
    "copy_u_max": ("copy_lhs", "max", "u", None, "v"),
    "u_mul_e_sum": ("mul", "sum", "u", "e", "v"),
    "u_add_v": ("add", "assign", "u", "v", "e"),
    "u_dot_v": ("dot", "assign", "u", "v", "e"),
    "u_dot_v_sum": ("dot", "sum", "u", "v", "v"),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--op", default="copy_u_sum", choices=sorted(OPS))
    ap.add_argument("--F", type=int, default=64)
    ap.add_argument("--schedule", default=None)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--ld", type=int, default=None, help="row stride of the feature tensor (padding)")
    a = ap.parse_args()
    c = ugdata.CONFIGS[a.config]
    src, dst = ugdata.graph(a.config)
    V, E = c.V, len(src)
    g = ug.Graph(V, src, dst)
    eo, go, at, bt, ct = OPS[a.op]
    X = (torch.rand(V, a.ld or a.F, device="cuda") - 0.5)[:, :a.F]
    B = {"e": torch.rand(E, 1, device="cuda") + 0.5, "v": X, "u": X, None: None}[bt]
    W = 1 if eo == "dot" else a.F
    C = torch.empty(V if ct == "v" else E, (a.ld or W) if W > 1 else 1, device="cuda")[:, :W]
    kw = dict(A=X, a_type=at, B=B, b_type=bt, C=C, c_type=ct, F=a.F, H=1)
    sched = a.schedule or ug.schedule_select(g, eo, go, **kw)
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(400_000)
        e0.record()
        ug.op_run(g, eo, go, schedule=sched, **kw)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{a.config} {a.op} F={a.F} ld={a.ld or a.F} {sched}: median {statistics.median(ts) * 1e3:.1f} us")


if __name__ == "__main__":
    main()
