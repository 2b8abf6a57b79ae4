#!/usr/bin/env python
"""A/B timing of schedules on the BASELINE configs: each graph is built once, then every
(op, F, schedule) case is timed (median of --reps CUDA-event timings, each launch queued behind a
spin kernel so the events see device time).  One JSON line per case.

    python scripts/ab_sched.py --cases "C3:u_mul_e_sum:128:SV_G512_F128_P1,SV_G512_F128_M1" ...
"""
import argparse
import json
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
    "u_mul_e_max": ("mul", "max", "u", "e", "v"),
    "u_sub_v_sum": ("sub", "sum", "u", "v", "v"),
    "u_add_v": ("add", "assign", "u", "v", "e"),
    "u_dot_v": ("dot", "assign", "u", "v", "e"),
    "u_dot_v_sum": ("dot", "sum", "u", "v", "v"),
    "copy_e_max": ("copy_lhs", "max", "e", None, "v"),
    "copy_e_sum": ("copy_lhs", "sum", "e", None, "v"),
}


def logical_bytes(V, E, F, op, H=1):
    eo, go, a, b, c = OPS[op]
    B = 4 * (V + 1) + 4 * E
    for t, w in ((a, F), (b, 1 if op.startswith("u_mul_e") else F)):
        if t in ("u", "e"):
            B += 4 * E * w
        elif t == "v":
            B += 4 * V * w
    B += 4 * E * (1 if eo == "dot" else F) if go == "assign" else 4 * V * (1 if eo == "dot" else F)
    return B


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cases", nargs="+", required=True, help="CFG:OP:F:SCHED1,SCHED2,...")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--tag", default="")
    a = ap.parse_args()
    graphs = {}
    for case in a.cases:
        cfg, op, F, scheds = case.split(":")
        F = int(F)
        if cfg not in graphs:
            graphs.clear()
            torch.cuda.empty_cache()
            src, dst = ugdata.graph(cfg)
            graphs[cfg] = (ug.Graph(ugdata.CONFIGS[cfg].V, src, dst), len(src))
        g, E = graphs[cfg]
        V = ugdata.CONFIGS[cfg].V
        eo, go, at, bt, ct = OPS[op]
        X = torch.rand(E if at == "e" else V, F, device="cuda") - 0.5
        B = {"e": torch.rand(E, 1, device="cuda") + 0.5, "v": X, None: None}[bt]
        W = 1 if eo == "dot" else F
        C = torch.empty(V if ct == "v" else E, W, device="cuda")
        kw = dict(A=X, a_type=at, B=B, b_type=bt, C=C, c_type=ct, F=F, H=1)
        by = logical_bytes(V, E, F, op)
        for sched in scheds.split(","):
            s = None if sched == "auto" else sched
            name = sched if s else "auto=" + ug.schedule_select(g, eo, go, **kw)
            try:
                for _ in range(3):
                    ug.op_run(g, eo, go, schedule=s, **kw)
                ts = []
                for _ in range(a.reps):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    torch.cuda._sleep(200_000)
                    e0.record()
                    ug.op_run(g, eo, go, schedule=s, **kw)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                us = statistics.median(ts) * 1e3
                # the event timestamps tick in ~1.02 us steps: the mean over many reps dithers
                # through that quantum and resolves smaller differences than the median
                print(json.dumps({"tag": a.tag, "config": cfg, "op": op, "F": F, "schedule": name,
                                  "us": round(us, 2), "mean_us": round(statistics.fmean(ts) * 1e3, 3),
                                  "gbs": round(by / (us * 1e-6) / 1e9, 1)}), flush=True)
            except Exception as e:  # noqa: BLE001 -- report and continue the sweep
                print(json.dumps({"tag": a.tag, "config": cfg, "op": op, "F": F, "schedule": name,
                                  "error": str(e)[:200]}), flush=True)
        del X, B, C


if __name__ == "__main__":
    main()
