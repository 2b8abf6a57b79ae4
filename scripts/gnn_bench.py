#!/usr/bin/env python
"""End-to-end GNN-layer inference through the DGL-style shim (the paper's
Fig. 13/14 workload shape, on synthetic graphs): per model x config, the
forward latency of a 2-layer model (CUDA events, median of 20 after warm-up), with the share
spent in graph operators vs dense torch ops, next to the same model written with plain torch
index ops (index_add_ / scatter_reduce) as context -- not a comparison system of the paper.

    python scripts/gnn_bench.py --configs C1 C2 C3 --out gpurun_out/gnn_bench.json
"""
import argparse
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_0001lslwlgslllw23_b200 import gnn  # noqa: E402
import ugdata  # noqa: E402

HIDDEN = {"GCN": 16, "GIN": 64, "SAGE": 64, "GAT": 8}   # per-model hidden sizes ("default")


def torch_aggr(h, s, d, V, how):
    out = torch.zeros(V, h.shape[1], device=h.device)
    if how == "sum":
        return out.index_add_(0, d, h[s])
    red = {"mean": "mean", "max": "amax"}[how]
    return out.scatter_reduce(0, d[:, None].expand(-1, h.shape[1]), h[s], red, include_self=False)


def build(model, fin, fout):
    hid = HIDDEN[model.split("_")[0]]
    if model == "GCN":
        return [gnn.GCNConv(fin, hid), gnn.GCNConv(hid, fout)]
    if model == "GIN":
        return [gnn.GINConv(fin, hid), gnn.GINConv(hid, fout)]
    if model.startswith("SAGE"):
        agg = model.split("_")[1]
        return [gnn.SAGEConv(fin, hid, agg), gnn.SAGEConv(hid, fout, agg)]
    return [gnn.GATConv(fin, hid, 8), gnn.GATConv(hid * 8, fout, 1)]


def forward_ug(layers, gd, h, w):
    for i, l in enumerate(layers):
        if isinstance(l, gnn.GCNConv):
            h = l(gd, h, w)
        else:
            h = l(gd, h)
        if i + 1 < len(layers):
            h = torch.relu(h)
    return h


def forward_torch(layers, gd, h, w, s, d):
    V = gd.V
    for i, l in enumerate(layers):
        if isinstance(l, gnn.GCNConv):
            z = h @ l.W
            h = torch.zeros(V, z.shape[1], device=z.device).index_add_(0, d, z[s] * w) + l.b
        elif isinstance(l, gnn.GINConv):
            h = l.l2(torch.relu(l.l1((1 + l.eps) * h + torch_aggr(h, s, d, V, "sum"))))
        elif isinstance(l, gnn.SAGEConv):
            h = l.self_lin(h) + l.neigh_lin(torch_aggr(h, s, d, V, l.agg))
        else:
            H, D = l.H, l.D
            z = h @ l.W
            zh = z.view(-1, H, D)
            el, er = (zh * l.al).sum(-1), (zh * l.ar).sum(-1)
            e = torch.nn.functional.leaky_relu(el[s] + er[d], 0.2)
            emax = torch.zeros(V, H, device=e.device).scatter_reduce(0, d[:, None].expand(-1, H), e, "amax",
                                                                     include_self=False)
            ex = torch.exp(e - emax[d])
            den = torch.zeros(V, H, device=e.device).index_add_(0, d, ex)
            a = ex / den[d]
            h = torch.zeros(V, H * D, device=e.device).index_add_(0, d, (zh[s] * a[:, :, None]).reshape(-1, H * D))
        if i + 1 < len(layers):
            h = torch.relu(h)
    return h


def timeit(f, reps=20):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", nargs="+", default=["C1", "C2", "C3"])
    ap.add_argument("--models", nargs="+", default=["GCN", "GIN", "SAGE_sum", "SAGE_mean", "SAGE_max", "GAT"])
    ap.add_argument("--fin", type=int, default=128)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    res = []
    for cfg in a.configs:
        c = ugdata.CONFIGS[cfg]
        src, dst = ugdata.graph(cfg)
        gd = gnn.GraphData(c.V, src, dst)
        s = torch.from_numpy(src).long().cuda()
        d = torch.from_numpy(dst).long().cuda()
        w = gnn.gcn_norm(gd, src, dst)
        h0 = torch.randn(c.V, a.fin, device="cuda")
        for model in a.models:
            torch.manual_seed(0)
            layers = [l.cuda() for l in build(model, a.fin, 16)]
            with torch.no_grad():
                y1 = forward_ug(layers, gd, h0, w)
                y2 = forward_torch(layers, gd, h0, w, s, d)
                err = float((y1 - y2).abs().max() / (y2.abs().max() + 1e-6))
                t_ug = timeit(lambda: forward_ug(layers, gd, h0, w))
                t_pt = timeit(lambda: forward_torch(layers, gd, h0, w, s, d))
            r = {"config": cfg, "model": model, "ug_ms": round(t_ug, 4), "torch_index_ops_ms": round(t_pt, 4),
                 "speedup": round(t_pt / t_ug, 2), "max_rel_diff": err}
            print(json.dumps(r), flush=True)
            res.append(r)
    if a.out:
        json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
