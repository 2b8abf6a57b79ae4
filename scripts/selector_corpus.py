#!/usr/bin/env python
"""Training corpus for the learned schedule selector.

The paper trains LightGBM on 128 graphs of the Network Repository with the Table 7 features
(#V, #E, std_nnz, op info).  No dataset is reachable offline, so the corpus is synthetic:
Chung-Lu graphs (ugdata.chung_lu) with log-uniform V and mean degree, lognormal degree skew
sigma in [0.3, 1.6], directed or undirected -- spanning the five configs' ranges.  For every
(graph, op class, F) every candidate schedule of scripts/sweep.py is timed on the B200 (CUDA
events behind a spin kernel, median of 5).  One JSON line per (graph, class, F):
{features..., "times": {schedule: ms}}.

    python scripts/selector_corpus.py --graphs 48 --out gpurun_out/selector_corpus.jsonl
"""
import argparse
import json
import math
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402
from sweep import CLASS_OPS, candidates, time_schedule  # noqa: E402

WIDTHS = (8, 16, 32, 64, 128, 256)


def graph_params(i, seed):
    rng = np.random.default_rng(seed + 7919 * i)
    V = int(math.exp(rng.uniform(math.log(2_000), math.log(400_000))))
    deg = math.exp(rng.uniform(math.log(2.0), math.log(120.0)))
    E = int(min(V * deg, 12_000_000))
    directed = bool(rng.integers(0, 2))
    if not directed and E % 2:
        E -= 1
    sigma = float(rng.uniform(0.3, 1.6))
    return V, E, directed, sigma, int(rng.integers(1, 1 << 30))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", type=int, default=48)
    ap.add_argument("--seed", type=int, default=4242)
    ap.add_argument("--classes", nargs="+", default=["agg", "agg_bin", "agg_ext", "msg", "dot_msg"])
    ap.add_argument("--widths-per-class", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/selector_corpus.jsonl")
    ap.add_argument("--budget-s", type=float, default=2400)
    args = ap.parse_args()
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    out = open(args.out, "a")
    t_start = time.time()
    for i in range(args.graphs):
        if time.time() - t_start > args.budget_s:
            break
        V, E, directed, sigma, gseed = graph_params(i, args.seed)
        src, dst = ugdata.chung_lu(V, E, directed, sigma, 0.5 if directed else sigma, gseed)
        g = ug.Graph(V, src, dst)
        st = g.stats()
        cv = st["std_nnz"] / max(st["mean_deg"], 1e-9)
        rng = np.random.default_rng(gseed)
        for cls in args.classes:
            nm, eo, go, a, b, ct = CLASS_OPS[cls][0]
            for F in sorted(rng.choice(WIDTHS, args.widths_per_class, replace=False).tolist()):
                X = torch.rand(V, F, device="cuda") - 0.5
                w = torch.rand(E, 1, device="cuda") + 0.5
                Cw = 1 if eo == "dot" else F
                C = torch.empty(V if ct == "v" else E, Cw, device="cuda")
                kw = dict(A=X, a_type=a, B=(w if b == "e" else (X if b else None)), b_type=b, C=C, c_type=ct,
                          F=F, H=1)
                times = {}
                for sched in candidates(cls, F, E):
                    ms, err = time_schedule(g, kw, eo, go, sched, 5)
                    if ms is not None:
                        times[sched] = ms
                rec = {"graph": i, "V": V, "E": E, "directed": directed, "sigma": sigma, "mean_deg": st["mean_deg"],
                       "std_nnz": st["std_nnz"], "cv": cv, "max_deg": st["max_deg"], "class": cls, "op": nm, "F": F,
                       "times": times}
                out.write(json.dumps(rec) + "\n")
                out.flush()
                best = min(times, key=times.get)
                print(f"g{i:02d} V={V:7d} E={E:9d} cv={cv:4.2f} {cls:8s} F={F:3d} best {best:18s} "
                      f"{times[best] * 1e3:9.1f} us  ({len(times)} schedules)", flush=True)
                del X, w, C
        del g
        torch.cuda.empty_cache()
    print(f"corpus done in {time.time() - t_start:.0f} s")


if __name__ == "__main__":
    main()
