#!/usr/bin/env python
"""Small driver for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every
schedule family on a tiny skewed graph and on C1, a few ops each, through the C ABI -- plus the
kernels with cross-CTA protocols: SV's single-launch split-row merge, the staged SV ring (TMA
gather4 / cp.async + mbarriers), the column-tiled dot (k_dott), the fused GAT and dot-attention
chains (last-arriver / chunk merges) and arg capture + its backward scatter.

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
          "BV_G1", "BV_G3_B128", "BE_G64", "SV_G7", "SV_G64_F8", "SV_G5_F32", None]
STAGED = ["SV_G7_M1", "SV_G7_A1", "SV_G16_F64_M1", "SV_G16_F32_A1"]       # aggregation ops only
DOTT = ["SV_G7_F128", "SV_G16_F32"]                                          # u_dot_v ops only
# dst-sorted graph: the SV fast path (B addressing modes incl. the contiguous edge weight, FMA fold),
# non-power-of-two column tiles, and the edge-lanes kernels (TV sub-warps, segmented WV)
FAST = ["SV_G7", "SV_G64_F8", "SV_G16_F12"]
FAST_EL = ["TV_G1_T8_E1", "TV_G1_T16_E1", "WV_G2_T1_E1", "WV_G4_T1_E1"]
OPS = [("copy_lhs", "u", None, "sum", "v"), ("mul", "u", "e", "max", "v"), ("mul", "u", "e", "sum", "v"),
       ("sub", "v", "u", "mean", "v"),
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
        order = np.argsort(dst, kind="stable")
        gs = ug.Graph(V, src[order], dst[order])      # dst-sorted: the staged SV kernels need identity edge ids
        for F, H in ((18, 3), (20, 1), (16, 1), (24, 3)):   # the last two also take k_dotsv
            X = torch.randn(V, F, device="cuda")
            w = torch.randn(E, H, device="cuda").abs() + 0.5
            for (eo, a, b, go, c) in OPS:
                Bt = {"e": w, "v": X, "u": X, None: None}[b]
                W = H if eo == "dot" else F
                C = torch.empty(V if c == "v" else E, W, device="cuda")
                extra = []
                if eo != "dot" and c == "v" and a == "u" and (b in (None, "v") or (b == "e" and H < F)):
                    extra = STAGED
                if eo == "dot" and a == "u" and b == "v":
                    extra = DOTT
                if eo != "dot" and c == "v" and F != 18:
                    extra = extra + ["WV_G1_T1_E1", "WV_G3_T1_E1"]      # edge-lanes (narrow F)
                fast = []
                if eo != "dot" and c == "v":
                    fast = FAST + (FAST_EL if F != 18 else [])
                for s, gg in [(s, gs if s in STAGED else g) for s in SCHEDS + extra] + [(s, gs) for s in fast]:
                    try:
                        ug.op_run(gg, eo, go, A=X, a_type=a, B=Bt, b_type=b, C=C, c_type=c, F=F, H=H, schedule=s)
                    except ug.UgError as err:
                        raise RuntimeError(f"{eo} {a} {b} {go} {c} F={F} H={H} {s}: {err}") from err
                    n += 1
        # fused chains and arg capture (single-launch merges across CTAs)
        for H, F in ((1, 16), (4, 32)):
            el, er = torch.randn(V, H, device="cuda"), torch.randn(V, H, device="cuda")
            z = torch.randn(V, F, device="cuda")
            att = torch.empty(E, H, device="cuda")
            ug.gat_attention(g, el, er, z, H, 0.2, attn=att)
            ug.dot_attention(g, z, z, z, H, attn=att)
            n += 2
        X = torch.randn(V, 16, device="cuda")
        C = torch.empty(V, 16, device="cuda")
        arg = ug.op_run_arg(g, "copy_lhs", "max", A=X, a_type="u", C=C, F=16)
        gx = torch.zeros(V, 16, device="cuda")
        ug.arg_scatter(g, arg, torch.ones(V, 16, device="cuda"), "u", gx)
        n += 2
        torch.cuda.synchronize()
    print(f"sanitize driver: {n} op calls ok")


if __name__ == "__main__":
    main()
