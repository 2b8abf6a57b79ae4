#!/usr/bin/env python
"""Run one fused traversal a few times (for ncu): ug_gat_attention or ug_dot_attention.

    python scripts/prof_fused.py --config C2 --kind gat --H 8 --F 64 --reps 3
"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--kind", choices=["gat", "dot"], default="gat")
    ap.add_argument("--H", type=int, default=8)
    ap.add_argument("--F", type=int, default=64)
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    c = ugdata.CONFIGS[a.config]
    s, d = ugdata.graph(a.config)
    g = ug.Graph(c.V, s, d)
    z = torch.randn(c.V, a.F, device="cuda")
    out = torch.empty_like(z)
    el, er = torch.randn(c.V, a.H, device="cuda"), torch.randn(c.V, a.H, device="cuda")
    for _ in range(a.reps):
        if a.kind == "gat":
            ug.gat_attention(g, el, er, z, a.H, 0.2, out=out)
        else:
            ug.dot_attention(g, z, z, z, a.H, out=out)
    torch.cuda.synchronize()
    print("ok", a.config, a.kind)


if __name__ == "__main__":
    main()
