#!/usr/bin/env python
"""Locality from vertex renumbering (PAPER.md:566-568 / Fig. 19): copy_u_sum
and u_mul_e_sum on a community graph whose ids were shuffled, before and after
ug_graph_reorder (RCM / degree), device time (CUDA events behind a spin kernel, median), with
the AUTO schedule; plus the one-time cost of computing the order.

    python scripts/reorder_bench.py [--V 2000000] [--E 40000000] [--F 64]
"""
import argparse
import json
import os
import statistics
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402


def dev_ms(fn, reps=10):
    for _ in range(2):
        fn()
    ts = []
    for _ in range(reps):
        torch.cuda._sleep(200_000)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return round(statistics.median(ts), 4)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--V", type=int, default=2_000_000)
    ap.add_argument("--E", type=int, default=40_000_000)
    ap.add_argument("--blocks", type=int, default=4000)
    ap.add_argument("--p-in", type=float, default=0.9)
    ap.add_argument("--F", type=int, default=64)
    args = ap.parse_args()
    V, E, F = args.V, args.E, args.F
    src, dst = ugdata.community_graph(V, E, args.blocks, args.p_in, 11)
    res = {"graph": f"community graph V={V} E={E} blocks={args.blocks} p_in={args.p_in}, ids shuffled", "F": F}
    g = ug.Graph(V, src, dst)
    X = torch.rand(V, F, device="cuda")
    w = torch.rand(E, 1, device="cuda")
    Y = torch.empty(V, F, device="cuda")
    for nm, eo, B, bt in (("copy_u_sum", "copy_lhs", None, None), ("u_mul_e_sum", "mul", w, "e")):
        s = ug.schedule_select(g, eo, "sum", A=X, a_type="u", B=B, b_type=bt, C=Y, c_type="v", F=F)
        res[f"{nm}_original"] = {"schedule": s, "ms": dev_ms(lambda: ug.op_run(g, eo, "sum", A=X, a_type="u", B=B,
                                                                                  b_type=bt, C=Y, c_type="v", F=F))}
    for method in ("community", "rcm", "degree"):
        t0 = time.perf_counter()
        rn = ug.Renumbered(V, src, dst, method)
        t_order = time.perf_counter() - t0
        Xn = rn.to_new(X)
        wn = rn.edges_to_new(w)
        Yn = torch.empty(V, F, device="cuda")
        res[f"{method}_preprocess_s"] = round(t_order, 2)
        res[f"{method}_rows_gather_ms"] = dev_ms(lambda: rn.to_new(X))
        for nm, eo, B, bt in (("copy_u_sum", "copy_lhs", None, None), ("u_mul_e_sum", "mul", wn, "e")):
            s = ug.schedule_select(rn.graph, eo, "sum", A=Xn, a_type="u", B=B, b_type=bt, C=Yn, c_type="v", F=F)
            res[f"{nm}_{method}"] = {"schedule": s, "ms": dev_ms(lambda: ug.op_run(rn.graph, eo, "sum", A=Xn, a_type="u",
                                                                                     B=B, b_type=bt, C=Yn, c_type="v",
                                                                                     F=F))}
        del rn, Xn, wn, Yn
    print(json.dumps(res))


if __name__ == "__main__":
    main()
