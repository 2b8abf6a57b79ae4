#!/usr/bin/env python
"""Summarise ncu output for profiles/ (run here, on the CPU host, after gpurun brings the
reports back).

  python scripts/ncu_summary.py launches gpurun_out/launches_r1.csv        # kernel shares
  python scripts/ncu_summary.py full gpurun_out/prof_k_split_r1.ncu-rep     # key metrics
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum",
    "lts__t_sectors_srcunit_tex_op_read.sum",
    "lts__t_sector_hit_rate.pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__throughput.max.pct_of_peak_sustained_elapsed",
    "lts__lts2xbar_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "lts__lts2xbar_cycles_active.max.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_srcunit_tex.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_srcunit_ltcfabric.sum",
    "l1tex__m_xbar2l1tex_read_bytes.sum.pct_of_peak_sustained_elapsed",
    "l1tex__t_bytes.sum",
    "l1tex__t_sector_hit_rate.pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed.sum",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__occupancy_limit_registers",
    "sm__maximum_warps_per_active_cycle_pct",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_lg_throttle",
    "smsp__pcsamp_warps_issue_stalled_wait",
    "smsp__pcsamp_warps_issue_stalled_selected",
]


def launches(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(lines[start:]))
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(")[0]
        unit = r.get("Metric Unit", "ns")
        v = float(r["Metric Value"].replace(",", ""))
        scale = {"ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3}.get(unit, 1e-6)
        tot[name] += v * scale
        cnt[name] += 1
    all_ms = sum(tot.values())
    out = {k: {"launches": cnt[k], "total_ms": round(v, 4), "avg_ms": round(v / cnt[k], 4),
               "share": round(v / all_ms, 4)} for k, v in sorted(tot.items(), key=lambda kv: -kv[1])}
    return out


def full(path):
    txt = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"]).decode()
    rdr = list(csv.reader(io.StringIO(txt)))
    hdr, units = rdr[0], rdr[1]
    res = []
    for row in rdr[2:]:
        d = dict(zip(hdr, row))
        rec = {"kernel": d.get("Kernel Name", "")[:120], "id": d.get("ID")}
        for k in KEYS:
            for h in hdr:
                if h == k:
                    rec[k] = d[h] + (" " + units[hdr.index(h)] if units[hdr.index(h)] else "")
        res.append(rec)
    return res


def traffic(path, key, out="profiles/ncu_traffic.json"):
    """Add the bench kernel's per-launch DRAM / L2->SM bytes (base units) to ncu_traffic.json under
    key CONFIG:OP:F:SCHEDULE (read by bench.py into roofline.traffic / l2_frac / dram_frac)."""
    txt = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv", "--print-units", "base"]).decode()
    rdr = list(csv.reader(io.StringIO(txt)))
    hdr = rdr[0]
    rows = [dict(zip(hdr, r)) for r in rdr[2:]]
    d = max(rows, key=lambda r: float(r.get("gpu__time_duration.sum", "0").replace(",", "") or 0))
    f = lambda k: float(d[k].replace(",", ""))
    ent = {"dram_bytes_per_launch": f("dram__bytes_read.sum") + f("dram__bytes_write.sum"),
           "dram_read": f("dram__bytes_read.sum"), "dram_write": f("dram__bytes_write.sum"),
           "l2_to_sm_bytes": f("lts__t_sectors_srcunit_tex_op_read.sum") * 32,
           "kernel_ms": f("gpu__time_duration.sum") * 1e-6,
           "lts_throughput_pct": f("lts__throughput.avg.pct_of_peak_sustained_elapsed"),
           "lts_hit_rate_pct": f("lts__t_sector_hit_rate.pct"),
           "kernel": d.get("Kernel Name", "")[:100],
           "source": f"{path} (ncu --set full --clock-control none, one launch of the bench kernel)"}
    db = json.load(open(out)) if __import__("os").path.exists(out) else {}
    db[key] = ent
    json.dump(db, open(out, "w"), indent=1)
    return ent


if __name__ == "__main__":
    mode, path = sys.argv[1], sys.argv[2]
    if mode == "traffic":
        print(json.dumps(traffic(path, sys.argv[3]), indent=1))
    else:
        print(json.dumps(launches(path) if mode == "launches" else full(path), indent=1))
