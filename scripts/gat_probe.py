#!/usr/bin/env python
"""Device time of the fused GAT traversal (ug_gat_attention) and of the fused dot-product
attention traversal (ug_dot_attention) on C1-C4-shaped graphs, and the 6-op GAT chain on C2
(bench.gat_chain_graph)."""
import json, os, statistics, sys
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402
from probe_latency import dev_time  # noqa: E402

out = []
for cfg, H, F in (("C1", 1, 16), ("C2", 8, 64), ("C2", 1, 16), ("C3", 4, 64), ("C4", 8, 128)):
    c = ugdata.CONFIGS[cfg]
    s, d = ugdata.graph(cfg)
    g = ug.Graph(c.V, s, d)
    el, er = torch.randn(c.V, H, device="cuda"), torch.randn(c.V, H, device="cuda")
    z = torch.randn(c.V, F, device="cuda")
    o = torch.empty(c.V, F, device="cuda")
    t = dev_time(lambda: ug.gat_attention(g, el, er, z, H, 0.2, out=o))
    E = len(s)
    by = 4 * (c.V + 1) + 4 * E + 4 * E * H + 4 * c.V * H + 4 * E * F + 4 * c.V * F
    out.append({"config": cfg, "H": H, "F": F, "us": t, "gbs": round(by / (t * 1e-6) / 1e9, 1)})
    # dot attention (q = z, k = z, val = z): gathers k[u] and val[u] rows per edge, q[v] per unit
    t2 = dev_time(lambda: ug.dot_attention(g, z, z, z, H, out=o))
    by2 = 4 * (c.V + 1) + 4 * E + 4 * c.V * F + 2 * 4 * E * F + 4 * c.V * F
    out.append({"config": cfg, "op": "dot_attention", "H": H, "F": F, "us": t2,
                "gbs": round(by2 / (t2 * 1e-6) / 1e9, 1)})
    if cfg == "C2" and H == 8:
        out.append(bench.gat_chain_graph(ug, torch, "cuda", g))
print(json.dumps(out))
