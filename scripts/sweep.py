#!/usr/bin/env python
"""Schedule sweep on B200: times every candidate schedule of the decoupled space
(§4.2, Table 9 notation) for each op class x config x F with CUDA events, writes one
JSON line per (config, op, F, schedule) and a selector table (`selector_table.json`) holding
the measured best schedule per key -- the B200 analogue of the paper's grid search
 that the selector (ug_schedule_select) reads.

    python scripts/sweep.py --configs C1 C2 C3 C4 C5 --out gpurun_out/sweep.jsonl \
        --table paper_conf_asplos_0001lslwlgslllw23_b200/selector_table.json
"""
import argparse
import itertools
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402

# op class -> representative ops (name, edge_op, gather, A type, B type, C type)
CLASS_OPS = {
    "agg": [("copy_u_sum", "copy_lhs", "sum", "u", None, "v")],
    "agg_bin": [("u_mul_e_sum", "mul", "sum", "u", "e", "v")],
    "agg_ext": [("copy_u_max", "copy_lhs", "max", "u", None, "v")],
    "msg": [("u_add_v", "add", "assign", "u", "v", "e")],
    "dot_msg": [("u_dot_v", "dot", "assign", "u", "v", "e")],
    "dot_agg": [("u_dot_v_sum", "dot", "sum", "u", "v", "v")],
}

# F per config and class (SURVEY 8(d) widths)
WIDTHS = {
    "C1": {"agg": [16], "agg_bin": [16], "agg_ext": [16], "msg": [16], "dot_msg": [16], "dot_agg": [16]},
    "C2": {"agg": [8, 64], "agg_bin": [64], "agg_ext": [8, 64], "msg": [8, 64], "dot_msg": [64], "dot_agg": [64]},
    "C3": {"agg": [32, 64, 128], "agg_bin": [32, 128], "agg_ext": [32, 128], "msg": [32], "dot_msg": [128],
           "dot_agg": [64]},
    "C4": {"agg": [128], "agg_bin": [128], "agg_ext": [128], "msg": [128], "dot_msg": [128, 256], "dot_agg": [128]},
    "C5": {"agg": [602], "agg_bin": [602], "agg_ext": [602], "msg": [1], "dot_msg": [602], "dot_agg": [602]},
}


def candidates(cls, F, E, quick=False):
    c = []
    Ts = [t for t in (1, 2, 4, 8, 16, 32) if t <= max(1, F)]
    if cls in ("agg", "agg_bin", "agg_ext", "dot_agg"):
        c += [f"TV_G{g}_T{t}" for g in (1, 4) for t in Ts]
        c += [f"WV_G{g}_T1" for g in (1, 2, 8)]
        if cls != "dot_agg" and F <= 32:
            c += [f"WV_G{g}_T1_E1" for g in (1, 2, 4)]    # lanes over in-edges (narrow F); g > 1 segmented
            c += [f"TV_G1_T{t}_E1" for t in (8, 16)]       # 32 / t rows per warp, t edge lanes each
        c += [f"TE_G{g}_T{t}" for g in (1, 8, 32) for t in Ts if t >= 4]
        c += [f"WE_G{g}_T1" for g in (4, 32, 128)]
        vec = 4 if F % 4 == 0 else (2 if F % 2 == 0 else 1)
        # edge-parallel with tile-major column tiles (L2 residency of the gathered slab)
        c += [f"TE_G{g}_T{ft // vec}_F{ft}" for g in (8, 32) for ft in (32, 64) if ft < F and ft // vec <= 32]
        c += [f"BV_G{g}_B{b}" for g in (1, 4) for b in (128, 256, 512)]
        c += [f"BE_G{g}" for g in (64, 512)]
        if cls != "dot_agg":
            fts = [f for f in (16, 32, 64, 128) if f <= max(16, 2 * F)]
            c += [f"SV_G{g}_F{f}" for g in (16, 32, 64, 128, 512, 2048) for f in fts]
            c += [f"SV_G{g}_F{f}_P1" for g in (32, 128, 512) for f in (64, 128) if f <= max(16, 2 * F)]
        else:
            c += [f"SV_G{g}" for g in (16, 32, 64, 128, 512, 1024)]
            c += [f"SV_G{g}_F{f}" for g in (64, 256, 512) for f in (64, 128)]     # k_dott messages + SV reduce
    else:
        c += [f"TE_G{g}_T{t}" for g in (1, 2, 4, 8) for t in Ts]
        c += [f"WE_G{g}_T1" for g in (1, 4, 16)]
        c += [f"TV_G1_T{t}" for t in Ts if t >= 4]
        c += [f"WV_G{g}_T1" for g in (1, 4)]
        c += ["BV_G1_B256", "BE_G256"]
        if cls == "dot_msg":
            c += [f"SV_G{g}" for g in (16, 32, 64, 128, 512)]
            c += [f"SV_G{g}_F{f}" for g in (64, 256, 512) for f in (64, 128)]     # k_dott (column tiles)
        else:   # message creation under SV: row chunks x column tiles, Dst_V operand hoisted
            c += [f"SV_G{g}_F{f}" for g in (16, 32, 64) for f in (16, 32, 64) if f <= max(16, F)]
            if F <= 8:
                c += [f"SV_G{g}_E1" for g in (64, 1024)]          # lanes over edges (narrow messages)
    if E > 50_000_000:   # C5: drop the schedules that take seconds (atomic per-element TE at F=602)
        c = [s for s in c if not (s.startswith("TE") and cls.startswith("agg") and "_F" not in s) and not s.startswith("TV")
             and not s.startswith("WV")]
    if quick:
        c = c[::3]
    return c


def time_schedule(g, kw, eo, go, sched, reps):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 * reps)]
    try:
        for _ in range(2):
            ug.op_run(g, eo, go, schedule=sched, **kw)
        torch.cuda.synchronize()
    except ug.UgError as e:
        return None, str(e)
    ts = []
    for i in range(reps):
        torch.cuda._sleep(400_000)      # queue the op behind a spin kernel: device time only,
        ev[2 * i].record()              # no host launch latency inside the events
        ug.op_run(g, eo, go, schedule=sched, **kw)
        ev[2 * i + 1].record()
    torch.cuda.synchronize()
    ts = sorted(ev[2 * i].elapsed_time(ev[2 * i + 1]) for i in range(reps))
    # interquartile mean: the event clock ticks in ~1.02 us steps, so on launch-bound graphs
    # (C1 / C2) the median snaps to a tick; the middle half's mean dithers through it and still
    # ignores outliers (equal to the median for the ms-scale ops)
    q = len(ts) // 4
    mid = ts[q:len(ts) - q] if len(ts) >= 4 else ts
    return statistics.fmean(mid), None


def logical_bytes(V, E, F, H, eo, go, a, b, c, wa, wb):
    B = 4 * (V + 1) + 4 * E
    for t, w in ((a, wa), (b, wb)):
        if t in ("u", "e"):
            B += 4 * E * w
        elif t == "v":
            B += 4 * V * w
    W = H if eo == "dot" else F
    B += 4 * E * W if c == "e" else 4 * V * W
    return B


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", nargs="+", default=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--classes", nargs="+", default=list(CLASS_OPS))
    ap.add_argument("--out", default="gpurun_out/sweep.jsonl")
    ap.add_argument("--table", default=None)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--first-op-only", action="store_true")
    args = ap.parse_args()
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    out = open(args.out, "a")
    best = {}
    for cfg in args.configs:
        c = ugdata.CONFIGS[cfg]
        src, dst = ugdata.graph(cfg)
        V, E = c.V, len(src)
        g = ug.Graph(V, src, dst)
        st = g.stats()
        cv = st["std_nnz"] / max(st["mean_deg"], 1e-9)
        for cls in args.classes:
            ops = CLASS_OPS[cls][:1] if args.first_op_only else CLASS_OPS[cls]
            for F in WIDTHS[cfg][cls]:
                H = 1
                X = torch.rand(V, F, device="cuda") - 0.5
                w = torch.rand(E, 1, device="cuda") + 0.5
                for (nm, eo, go, a, b, ct) in ops:
                    Cw = 1 if eo == "dot" else F
                    C = torch.empty(V if ct == "v" else E, Cw, device="cuda")
                    kw = dict(A=X, a_type=a, B=(w if b == "e" else (X if b else None)), b_type=b, C=C, c_type=ct,
                              F=F, H=H)
                    wb = 1 if b == "e" else F
                    by = logical_bytes(V, E, F, H, eo, go, a, b, ct, F, wb)
                    auto = ug.schedule_select(g, eo, go, **kw)
                    results = []
                    for sched in candidates(cls, F, E, args.quick):
                        ms, err = time_schedule(g, kw, eo, go, sched, args.reps)
                        rec = {"config": cfg, "class": cls, "op": nm, "F": F, "V": V, "E": E,
                               "mean_deg": st["mean_deg"], "cv": cv, "schedule": sched, "ms": ms,
                               "gbs": (by / (ms * 1e-3) / 1e9) if ms else None, "error": err}
                        out.write(json.dumps(rec) + "\n")
                        out.flush()
                        if ms is not None:
                            results.append((ms, sched))
                    results.sort()
                    ams, _ = time_schedule(g, kw, eo, go, auto, args.reps)
                    # the selector's own pick beside the sweep (the Fig. 12 analogue)
                    out.write(json.dumps({"config": cfg, "class": cls, "op": nm, "F": F, "V": V, "E": E,
                                          "mean_deg": st["mean_deg"], "cv": cv, "schedule": auto, "auto": True,
                                          "ms": ams, "best_schedule": results[0][1], "best_ms": results[0][0],
                                          "gbs": (by / (ams * 1e-3) / 1e9) if ams else None, "error": None}) + "\n")
                    print(f"{cfg} {cls:8s} {nm:12s} F={F:4d}  best {results[0][1]:18s} {results[0][0]:9.4f} ms  "
                          f"({by / results[0][0] / 1e6:8.1f} GB/s)  auto {auto:18s} {ams:9.4f} ms  "
                          f"worst {results[-1][1]} {results[-1][0]:.4f} ms", flush=True)
                    key = (cls, cfg, F)
                    if nm == CLASS_OPS[cls][0][0]:
                        best[key] = (results[0][1], V, st["mean_deg"], cv)
                    del C
                del X, w
        del g
        torch.cuda.empty_cache()
    if args.table:
        entries = []
        for (cls, cfg, F), (sched, V, deg, cv) in sorted(best.items(), key=lambda kv: (kv[0][0], kv[0][2])):
            entries.append({"class": cls, "F_lo": F * 0.75, "F_hi": F * 1.34, "deg_lo": deg / 2, "deg_hi": deg * 2,
                            "cv_lo": cv * 0.6, "cv_hi": cv * 1.6, "V_lo": V / 4, "V_hi": V * 4,
                            "schedule": sched, "measured_on": f"{cfg} (B200)"})
        with open(args.table, "w") as f:
            json.dump({"version": 1, "device": torch.cuda.get_device_name(),
                       "generated": time.strftime("%Y-%m-%d %H:%M:%S"),
                       "how": "scripts/sweep.py: median of CUDA-event timings per schedule",
                       "entries": entries}, f, indent=1)
        print("wrote", args.table, len(entries), "entries")


if __name__ == "__main__":
    main()
