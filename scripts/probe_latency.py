#!/usr/bin/env python
"""Latency floor probe for small graphs (C1 / C2): device time (CUDA events, queued behind a
spin kernel) of an empty torch kernel, and of op_run per schedule with its launch count.

    python scripts/probe_latency.py [--config C1] [--op u_mul_e_sum]
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


def dev_time(fn, reps=30, warm=5):
    ts = []
    for i in range(warm + reps):
        torch.cuda._sleep(300_000)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        if i >= warm:
            ts.append(e0.elapsed_time(e1) * 1e3)
    return round(statistics.median(ts), 2)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C1")
    ap.add_argument("--schedules", nargs="*", default=None)
    args = ap.parse_args()
    x = torch.zeros(1, device="cuda")
    res = {"empty_kernel_us": dev_time(lambda: x.add_(1.0)),
           "two_empty_kernels_us": dev_time(lambda: (x.add_(1.0), x.add_(1.0)))}
    c = ugdata.CONFIGS[args.config]
    src, dst = ugdata.graph(args.config)
    g = ug.Graph(c.V, src, dst)
    E = len(src)
    F = 16
    X = torch.rand(c.V, F, device="cuda")
    w = torch.rand(E, 1, device="cuda")
    Y = torch.empty(c.V, F, device="cuda")
    kw = dict(A=X, a_type="u", B=w, b_type="e", C=Y, c_type="v", F=F, H=1)
    scheds = args.schedules or ["TE_G1_T4", "TE_G1_T8", "WE_G4_T1", "BV_G1_B256", "BV_G1_B128", "SV_G16_F64",
                                "SV_G32_F64", "SV_G128_F64", "WV_G1_T1", "TV_G1_T4"]
    res["auto"] = ug.schedule_select(g, "mul", "sum", **kw)
    rows = []
    for s in [res["auto"]] + scheds:
        try:
            t = dev_time(lambda: ug.op_run(g, "mul", "sum", schedule=s, **kw))
            rows.append({"schedule": s, "us": t, "launches": ug.launch_count(g, "mul", "sum", schedule=s, **kw)})
        except ug.UgError as e:
            rows.append({"schedule": s, "error": str(e)})
    res["u_mul_e_sum"] = rows
    st = g.stats()
    res["graph"] = st
    print(json.dumps(res))


if __name__ == "__main__":
    main()
