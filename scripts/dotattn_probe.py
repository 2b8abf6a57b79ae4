#!/usr/bin/env python
"""Device time of the fused dot-product attention traversal (ug_dot_attention), or with --gat of
the fused GAT traversal (ug_gat_attention), over a grid of (config, heads, feature width) cases,
for register-budget A/Bs of k_dotattn / k_dotattn_heads / k_gat.
One JSON line per case: us = median CUDA-event time of one call (the GPU is kept busy while the
host launches, so it is device time plus the launch gap)."""
import argparse, json, os, sys
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402
from probe_latency import dev_time  # noqa: E402

CASES = [("C2", 8, 64), ("C3", 4, 64), ("C3", 1, 128), ("C4", 8, 128), ("C4", 1, 128), ("C4", 4, 256),
         ("C4", 1, 64), ("C4", 2, 128), ("C3", 2, 128), ("C2", 1, 64)]

ap = argparse.ArgumentParser()
ap.add_argument("--tag", default="")
ap.add_argument("--gat", action="store_true")
args = ap.parse_args()
graphs = {}
for cfg, H, F in CASES:
    c = ugdata.CONFIGS[cfg]
    if cfg not in graphs:
        s, d = ugdata.graph(cfg)
        graphs[cfg] = (ug.Graph(c.V, s, d), len(s))
    g, E = graphs[cfg]
    z = torch.randn(c.V, F, device="cuda")
    o = torch.empty(c.V, F, device="cuda")
    if args.gat:
        el, er = torch.randn(c.V, H, device="cuda"), torch.randn(c.V, H, device="cuda")
        t = dev_time(lambda: ug.gat_attention(g, el, er, z, H, 0.2, out=o))
        by = 4 * (c.V + 1) + 4 * E + 4 * E * H + 4 * c.V * H + 4 * E * F + 4 * c.V * F
    else:
        t = dev_time(lambda: ug.dot_attention(g, z, z, z, H, out=o))
        by = 4 * (c.V + 1) + 4 * E + 4 * c.V * F + 2 * 4 * E * F + 4 * c.V * F
    print(json.dumps({"tag": args.tag, "kind": "gat" if args.gat else "dot", "config": cfg, "H": H, "F": F, "us": t,
                      "gbs": round(by / (t * 1e-6) / 1e9, 1)}), flush=True)
