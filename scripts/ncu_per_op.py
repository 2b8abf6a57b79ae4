#!/usr/bin/env python
"""ncu DRAM bytes and L2 hit rate per (op, config) of bench.py's per_op_graph set (C1-C4), the
per-kernel evidence SURVEY 8(d) asks for (PAPER.md:511 reports the same metrics).

  on the GPU box:  ncu --metrics <M> --clock-control none -k regex:'^k_' --csv \
                       --log-file gpurun_out/ncu_per_op.csv python scripts/ncu_per_op.py run gpurun_out/ncu_per_op_order.json
  here:            python scripts/ncu_per_op.py parse gpurun_out/ncu_per_op.csv gpurun_out/ncu_per_op_order.json \
                       profiles/r2/ncu_per_op.json

`run` executes every op of bench.SECONDARY once (after one untimed warm-up call outside the
profiled range is impossible under ncu, so each op runs twice and the second call's launches are
kept) and records, in order, how many library kernels each call launches; `parse` maps ncu's
launch list back to the ops by that order.
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

METRICS = ("gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,"
           "lts__t_sectors_srcunit_tex_op_read.sum")


def run(order_path):
    import torch
    import bench
    import paper_conf_asplos_0001lslwlgslllw23_b200 as ug
    import ugdata
    order = []
    graphs = {}
    for (cfg, nm, eo, go, a, b, c, F, H, wa, wb) in bench.SECONDARY:
        if cfg not in graphs:
            s, d = ugdata.graph(cfg)
            graphs[cfg] = (ug.Graph(ugdata.CONFIGS[cfg].V, s, d), len(s))
        g, E = graphs[cfg]
        V = ugdata.CONFIGS[cfg].V
        rows = lambda t: V if t in ("u", "v") else E
        A = torch.rand(rows(a), wa, device="cuda") - 0.5
        B = (torch.rand(rows(b), wb, device="cuda") + 0.5) if b else None
        W = H if eo == "dot" else F
        C = torch.empty(V if c == "v" else E, W, device="cuda")
        kw = dict(A=A, a_type=a, B=B, b_type=b, C=C, c_type=c, F=F, H=H)
        sched = ug.schedule_select(g, eo, go, **kw)
        n = ug.launch_count(g, eo, go, schedule=sched, **kw)
        for _ in range(2):
            ug.op_run(g, eo, go, schedule=sched, **kw)
            torch.cuda.synchronize()
        order.append({"config": cfg, "op": nm, "F": F, "H": H, "schedule": sched, "launches": n})
    json.dump(order, open(order_path, "w"), indent=1)


def parse(csv_path, order_path, out_path):
    lines = open(csv_path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    launches = {}
    for r in csv.DictReader(lines[start:]):
        d = launches.setdefault(int(r["ID"]), {"kernel": r["Kernel Name"].split("(")[0]})
        unit = r.get("Metric Unit", "")
        v = float(r["Metric Value"].replace(",", ""))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1.0,
                 "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "sector": 1, "%": 1}.get(unit, 1)   # time -> us
        d[r["Metric Name"]] = v * scale
    seq = [launches[k] for k in sorted(launches)]
    order = json.load(open(order_path))
    out, i = [], 0
    for o in order:
        n = o["launches"]
        i += n                        # first call (warm-up) of the op
        ks = seq[i:i + n]
        i += n
        dram = sum(k.get("dram__bytes_read.sum", 0) + k.get("dram__bytes_write.sum", 0) for k in ks)
        l2sm = sum(k.get("lts__t_sectors_srcunit_tex_op_read.sum", 0) for k in ks) * 32
        main = max(ks, key=lambda k: k.get("gpu__time_duration.sum", 0))
        out.append({**o, "kernels": [k["kernel"] for k in ks],
                    "ncu_us": round(sum(k.get("gpu__time_duration.sum", 0) for k in ks), 2),
                    "dram_bytes": int(dram), "l2_to_sm_bytes": int(l2sm),
                    "l2_hit_rate_pct_main_kernel": round(main.get("lts__t_sector_hit_rate.pct", 0), 1)})
    json.dump({"how": "ncu --metrics " + METRICS + " --clock-control none, one cold call per op after a warm-up "
                      "call (scripts/ncu_per_op.py)", "ops": out}, open(out_path, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    if sys.argv[1] == "run":
        run(sys.argv[2])
    else:
        parse(sys.argv[2], sys.argv[3], sys.argv[4])
