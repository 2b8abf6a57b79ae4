#!/usr/bin/env python
"""Small driver for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every
schedule family on a tiny skewed graph and on C1, a few ops each, through the C ABI.

    compute-sanitizer --tool memcheck  python scripts/sanitize.py
    compute-sanitizer --tool racecheck python scripts/sanitize.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402

SCHEDS = ["TV_G1_T1", "TV_G3_T4", "WV_G1_T1", "WV_G2_T2_F8", "TE_G1_T4", "TE_G5_T32", "WE_G7_T1",
          "BV_G1", "BV_G3_B128", "BE_G64", "SV_G7", "SV_G64_F8", None]
OPS = [("copy_lhs", "u", None, "sum", "v"), ("mul", "u", "e", "max", "v"), ("sub", "v", "u", "mean", "v"),
       ("div", "u", "e", "assign", "e"), ("dot", "u", "v", "sum", "v"), ("dot", "u", "v", "assign", "e")]


def graphs():
    V = 97
    src, dst = ugdata.random_multigraph(V, 600, 3)
    src = np.concatenate([src, np.arange(80, dtype=np.int32)])
    dst = np.concatenate([dst, np.full(80, 7, np.int32)])
    yield V, src, dst
    c = ugdata.CONFIGS["C1"]
    s, d = ugdata.graph("C1")
    yield c.V, s, d


def main():
    n = 0
    for V, src, dst in graphs():
        E = len(src)
        g = ug.Graph(V, src, dst)
        for F, H in ((18, 3), (20, 1), (16, 1), (24, 3)):   # the last two also take k_dotsv
            X = torch.randn(V, F, device="cuda")
            w = torch.randn(E, H, device="cuda").abs() + 0.5
            for (eo, a, b, go, c) in OPS:
                Bt = {"e": w, "v": X, "u": X, None: None}[b]
                W = H if eo == "dot" else F
                C = torch.empty(V if c == "v" else E, W, device="cuda")
                for s in SCHEDS:
                    ug.op_run(g, eo, go, A=X, a_type=a, B=Bt, b_type=b, C=C, c_type=c, F=F, H=H, schedule=s)
                    n += 1
        torch.cuda.synchronize()
    print(f"sanitize driver: {n} op calls ok")


if __name__ == "__main__":
    main()
