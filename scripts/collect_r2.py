#!/usr/bin/env python
"""Copy one evidence run of scripts/gpu_evidence.sh (gpurun_out/*_<tag>*) into profiles/ and
summarise it (run here, on the CPU host):

    python scripts/collect_r2.py r2fa

bench + reference lines, launch list + kernel shares, the ncu --set full summary of the bench
kernel and its per-launch traffic entry (profiles/ncu_traffic.json, read by bench.py), per-op ncu
(profiles/ncu_per_op.json + table), the gloo N = 2 dry run, the sweep + Fig. 12 table, sanitizer logs."""
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")
R2 = os.path.join(P, "r2")


def last_json(path):
    for line in reversed(open(path).read().splitlines()):
        line = line.strip()
        if line.startswith("{"):
            return json.loads(line)
    raise SystemExit(f"no JSON line in {path}")


def run(*args, out=None):
    r = subprocess.run([sys.executable, *args], cwd=ROOT, capture_output=True, text=True, check=True)
    if out:
        open(out, "w").write(r.stdout)
    return r.stdout


def main(tag):
    g = lambda name: os.path.join(G, name)
    json.dump(last_json(g(f"bench_{tag}.log")), open(os.path.join(R2, "bench_line_r2.json"), "w"))
    json.dump(last_json(g(f"bench_ref_{tag}.log")), open(os.path.join(R2, "bench_reference_line_r2.json"), "w"))
    shutil.copy(g(f"launches_{tag}.csv"), os.path.join(R2, "launches_C5_copy_u_sum_r2.csv"))
    run("scripts/ncu_summary.py", "launches", g(f"launches_{tag}.csv"),
        out=os.path.join(R2, "launches_C5_copy_u_sum_r2.json"))
    rep = g(f"prof_k_split_{tag}.ncu-rep")
    shutil.copy(rep, os.path.join(R2, "k_split_C5_r2.ncu-rep"))
    run("scripts/ncu_summary.py", "full", rep, out=os.path.join(R2, "k_split_C5_r2.json"))
    run("scripts/ncu_summary.py", "traffic", rep, "C5:copy_u_sum:602:SV_G512_F128_P1")
    run("scripts/ncu_per_op.py", "parse", g(f"ncu_per_op_{tag}.csv"), g(f"ncu_per_op_order_{tag}.json"),
        os.path.join(P, "ncu_per_op.json"))
    ops = json.load(open(os.path.join(P, "ncu_per_op.json")))["ops"]
    rows = ["| config | op | F | schedule | kernels | ncu cold µs | DRAM MB | L2→SM MB | L2 hit % (main kernel) |",
            "|---|---|---|---|---|---|---|---|---|"]
    for o in ops:
        rows.append(f"| {o['config']} | {o['op']} | {o['F']} | {o['schedule']} | {', '.join(k.replace('void ', '') for k in o['kernels'])} "
                    f"| {o['ncu_us']} | {o['dram_bytes'] / 1e6:.1f} | {o['l2_to_sm_bytes'] / 1e6:.1f} "
                    f"| {o['l2_hit_rate_pct_main_kernel']} |")
    open(os.path.join(R2, "ncu_per_op.md"), "w").write("\n".join(rows) + "\n")
    shutil.copy(g(f"bench_dry2_{tag}.log"), os.path.join(R2, f"bench_dry2_{tag}.log"))
    if os.path.exists(g(f"sweep_{tag}.jsonl")):
        shutil.copy(g(f"sweep_{tag}.jsonl"), os.path.join(R2, "sweep_r2_auto.jsonl"))
        run("scripts/fig12.py", os.path.join(R2, "sweep_r2_auto.jsonl"), out=os.path.join(R2, "fig12_auto_vs_best.md"))
    # ncu --set full of the kernels changed in the second session (one launch each)
    summ = {}
    for name in ("C3_u_mul_e_sum", "C5_u_dot_v", "C2_copy_e_max"):
        js = g(f"prof_{name}_{tag}.json")          # summarised on the box (scripts/gpu_evidence.sh)
        if os.path.exists(js):
            try:
                summ[name] = json.load(open(js))
            except ValueError:
                pass
    if summ:
        json.dump(summ, open(os.path.join(R2, "ncu_kernels_r2b.json"), "w"), indent=1)
    for tool in ("memcheck", "racecheck", "synccheck"):
        src = g(f"sanitize_{tool}_{tag}.log")
        if not os.path.exists(src):                # compute-sanitizer closed on the pool
            continue
        lines = [l for l in open(src).read().splitlines() if "=========" in l or "sanitize driver" in l]
        open(os.path.join(P, "sanitizer", f"r2_{tool}.log"), "w").write("\n".join(lines[-3:]) + "\n")
    b = json.load(open(os.path.join(R2, "bench_line_r2.json")))
    print(json.dumps({k: b.get(k) for k in ("value", "ms_per_step", "roofline", "clocks")})[:900])


if __name__ == "__main__":
    main(sys.argv[1])
