#!/usr/bin/env python
"""bench.py -- the unified graph operator on B200 (one JSON line on rank 0).

Default workload (BASELINE.json configs[4], the largest single-GPU config and the one the
north-star target is quoted on): C5 Reddit-shaped synthetic graph (232,965 v / 114,615,892 e),
copy_u_sum at F = 602 (GraphSage/GCN-style aggregation, Fig. 4).

A "step" is one full call of the operator (ug_op_run: every kernel it enqueues) over the
whole graph with inputs resident in HBM; N > 1 (torchrun) shards destination rows by edge
count, and a step is the NCCL all-gather of X plus the local op.

  value         effective GB/s = logical algorithmic bytes / device time
  e2e           same metric through the public API with host (pinned) X in and Y out
  roofline      the dominant kernel (main traversal) timed with CUDA events inside the
                timed region, algorithmic bytes / its average duration vs measured HBM peak
  cpu_baseline  the CPU oracle (oracle/, 1 core) on a bounded row sample, same metric
  --impl reference   times the oracle alone (this tier's reference arm)
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "graph-op latency and effective HBM GB/s vs ~8 TB/s, per op×graph, 1/2/4/8 GPU"
OPS = {  # name -> (edge_op, gather_op, A type, B type)
    "copy_u_sum": ("copy_lhs", "sum", "u", None),
    "copy_u_mean": ("copy_lhs", "mean", "u", None),
    "copy_u_max": ("copy_lhs", "max", "u", None),
    "u_mul_e_sum": ("mul", "sum", "u", "e"),
    "u_dot_v": ("dot", "assign", "u", "v"),
}


def logical_bytes(V, E, F, op, H=1):
    """4(V+1) row_ptr + 4E col_idx + 4 E w per u/e operand + 4 V w per v operand
    + output (4 V F for C = v, 4 E w_out for C = e)."""
    eo, go, a, b = OPS[op]
    B = 4 * (V + 1) + 4 * E
    for t, w in ((a, F), (b, 1 if op == "u_mul_e_sum" else F)):
        if t in ("u", "e"):
            B += 4 * E * w
        elif t == "v":
            B += 4 * V * w
    B += 4 * E * H if go == "assign" else 4 * V * F
    return B


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 50 ms during the timed region (the
    sampler's first row is awaited before the region starts, so short regions still get rows)."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,power.draw,"
         "enforced.power.limit")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.time()
            while not self.rows and self.proc.poll() is None and time.time() - t0 < 5.0:
                time.sleep(0.01)
            self.rows.clear()       # keep only rows sampled inside the timed region
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 8:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i] == "Active"})
        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        pw = [v for v in (num(r[6]) for r in self.rows) if v is not None]
        lim = [v for v in (num(r[7]) for r in self.rows) if v is not None]
        out = {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
               "reasons": reasons, "samples": len(self.rows),
               "power_w_median": round(statistics.median(pw), 1) if pw else None,
               "power_w_max": round(max(pw), 1) if pw else None,
               "enforced_power_limit_w": max(lim) if lim else None}
        if "sw_power_cap" in reasons:
            out["note"] = ("sw_power_cap: the sustained L2-bound kernel draws power_w_max against the "
                           "enforced_power_limit_w; the driver lowers the SM clock (DESIGN.md 'Power')")
        return out


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# ---------------------------------------------------------------------------- CPU oracle
def oracle_sample(cfg_name, op, F, src, dst, V, target_s=15.0, seed=0):
    """Time the oracle (1 core) on a bounded random sample of destination rows; returns
    (GB/s in the same logical-byte metric, rows, edges, seconds)."""
    import oracle
    import ugdata
    eo, go, a, b = OPS[op]
    rng = np.random.default_rng(seed)
    deg = np.bincount(dst, minlength=V)
    mean_deg = max(1.0, float(deg.mean()))
    # calibrate: ~2 ns per (edge x feature) element for the plain oracle, then measure
    n_rows = int(max(16, min(V, target_s / (8e-9 * mean_deg * F))))
    rows = np.sort(rng.choice(V, size=n_rows, replace=False)).astype(np.int64)
    sub = np.nonzero(np.isin(dst, rows))[0]
    X = ugdata.values(V, F, 99, 1)
    w = ugdata.values(len(sub), 1, 99, 2, role="edge") if b == "e" else None
    s_src, s_dst = src[sub], dst[sub]
    t0 = time.perf_counter()
    if go == "assign":
        oracle.op(V, s_src, s_dst, eo, go, A=X, a_type=a, B=X, b_type=b, c_type="e", F=F, H=1)
        Es, Vs = len(sub), 0
    else:
        oracle.op(V, s_src, s_dst, eo, go, A=X, a_type=a, B=w, b_type=b, c_type="v", F=F, H=1, rows=rows)
        Es, Vs = len(sub), len(rows)
    dt = time.perf_counter() - t0
    by = logical_bytes(Vs, Es, F, op)
    return by / dt / 1e9, len(rows), Es, dt


def cores_used():
    """The oracle is single-threaded and this process is pinned to one core while it runs."""
    return 1


def host_info():
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


class PinnedCore:
    """taskset -c 0 for the oracle timings: this process runs on core 0 only."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {min(self.prev)})
        return self

    def __exit__(self, *a):
        os.sched_setaffinity(0, self.prev)


def oracle_per_config(secondary):
    """The oracle (1 pinned core) on every per_op_graph case of C1-C4 over the WHOLE graph, median
    of 3 (SURVEY 8(d) / BASELINE.md 3), beside the GPU latency of the same op."""
    import oracle
    import ugdata
    out = []
    graphs = {}
    for ent in secondary:
        if "schedule" not in ent:
            continue
        cfg = ent["config"]
        spec = next(x for x in SECONDARY if x[0] == cfg and x[1] == ent["op"] and x[7] == ent["F"])
        _, nm, eo, go, a, b, c, F, H, wa, wb = spec
        if cfg not in graphs:
            graphs[cfg] = ugdata.graph(cfg)
        src, dst = graphs[cfg]
        V, E = ugdata.CONFIGS[cfg].V, len(src)
        rows = lambda t: V if t in ("u", "v") else E
        A = ugdata.values(rows(a), wa, 5, 1)
        B = ugdata.values(rows(b), wb, 5, 2, role="den" if eo == "div" else "num") if b else None
        ts = []
        with PinnedCore():
            for _ in range(3):
                t0 = time.perf_counter()
                oracle.op(V, src, dst, eo, go, A=A, a_type=a, B=B, b_type=b, c_type=c, F=F, H=H)
                ts.append(time.perf_counter() - t0)
        med = statistics.median(ts)
        out.append({"config": cfg, "op": nm, "F": F, "H": H, "oracle_ms_median_of_3": round(med * 1e3, 3),
                    "oracle_gbs": round(ent["logical_bytes"] / med / 1e9, 4),
                    "gpu_us_warm": ent["warm"]["latency_us"],
                    "gpu_over_oracle": round(med * 1e6 / ent["warm"]["latency_us"], 1)})
    return out


# Per op x graph latencies on the other BASELINE.json configs (C1-C4): (config, op name,
# edge_op, gather_op, A type, B type, C type, F, H, A width, B width).
SECONDARY = [
    ("C1", "u_mul_e_sum", "mul", "sum", "u", "e", "v", 16, 1, 16, 1),
    ("C2", "u_add_v", "add", "assign", "u", "v", "e", 8, 8, 8, 8),
    ("C2", "copy_e_max", "copy_lhs", "max", "e", None, "v", 8, 8, 8, 0),
    ("C2", "copy_e_sum", "copy_lhs", "sum", "e", None, "v", 8, 8, 8, 0),
    ("C2", "e_sub_v", "sub", "assign", "e", "v", "e", 8, 8, 8, 8),
    ("C2", "e_div_v", "div", "assign", "e", "v", "e", 8, 8, 8, 8),
    ("C2", "u_mul_e_sum", "mul", "sum", "u", "e", "v", 64, 8, 64, 8),
    ("C3", "copy_u_sum", "copy_lhs", "sum", "u", None, "v", 128, 1, 128, 0),
    ("C3", "u_mul_e_sum", "mul", "sum", "u", "e", "v", 128, 1, 128, 1),
    ("C3", "copy_u_sum", "copy_lhs", "sum", "u", None, "v", 32, 1, 32, 0),
    ("C4", "u_dot_v", "dot", "assign", "u", "v", "e", 128, 1, 128, 128),
    ("C4", "u_dot_v", "dot", "assign", "u", "v", "e", 256, 1, 256, 256),
    ("C4", "u_dot_v_H4", "dot", "assign", "u", "v", "e", 128, 4, 128, 128),
]


def headline_graph_ops(ug, torch, g, X, V, E, F, cfg, reps=5, warm=2):
    """The other operators of the headline graph (same C5 graph and X, schedule by the selector):
    weighted aggregation, mean / max, and the SDDMM dot (message creation and its sum) -- device
    latency (CUDA events, median) and effective GB/s of the SURVEY 8(d) logical bytes."""
    import ugdata
    out = []
    w = torch.from_numpy(ugdata.values(E, 1, cfg.seed + 1, 2, role="edge")).to(X.device)
    cases = [("u_mul_e_sum", "mul", "sum", w, "e", "v", F), ("copy_u_mean", "copy_lhs", "mean", None, None, "v", F),
             ("copy_u_max", "copy_lhs", "max", None, None, "v", F), ("u_dot_v", "dot", "assign", X, "v", "e", 1),
             ("u_dot_v_sum", "dot", "sum", X, "v", "v", 1)]
    for nm, eo, go, B, bt, ct, W in cases:
        C = torch.empty(V if ct == "v" else E, W, device=X.device)
        kw = dict(A=X, a_type="u", B=B, b_type=bt, C=C, c_type=ct, F=F, H=1)
        sched = ug.schedule_select(g, eo, go, **kw)
        ts = []
        for i in range(warm + reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ug.op_run(g, eo, go, schedule=sched, **kw)
            e1.record()
            torch.cuda.synchronize()
            if i >= warm:
                ts.append(e0.elapsed_time(e1))
        ms = statistics.median(ts)
        by = 4 * (V + 1) + 4 * E + 4 * E * F + (4 * E if bt == "e" else (4 * V * F if bt == "v" else 0))
        by += 4 * E * W if ct == "e" else 4 * V * W
        out.append({"config": cfg.name if hasattr(cfg, "name") else "C5", "op": nm, "F": F, "schedule": sched,
                    "latency_ms": round(ms, 3), "gbs": round(by / (ms * 1e-3) / 1e9, 1), "logical_bytes": by})
        del C
    return out


def secondary_configs(ug, torch, dev, reps=20, warm=5):
    """Latency (median of `reps` CUDA-event timings after `warm` warm-ups) and effective GB/s,
    warm L2 (back to back) and cold L2 (a 256 MB scrub written between runs), per op x graph.
    Each timed op is queued behind GPU work so the events measure device time, not the host's
    launch latency (which is reported separately as host_launch_us)."""
    import ugdata
    out = []
    scrub = torch.empty(64 * 1024 * 1024, device=dev)     # 256 MB > 2 x L2
    graphs = {}
    for (cfg, nm, eo, go, a, b, c, F, H, wa, wb) in SECONDARY:
        if cfg not in graphs:
            s, d = ugdata.graph(cfg)
            graphs[cfg] = (ug.Graph(ugdata.CONFIGS[cfg].V, s, d), len(s))
        g, E = graphs[cfg]
        V = ugdata.CONFIGS[cfg].V
        rows = lambda t: V if t in ("u", "v") else E
        A = torch.rand(rows(a), wa, device=dev) - 0.5
        B = (torch.rand(rows(b), wb, device=dev) + 0.5) if b else None
        W = H if eo == "dot" else F
        C = torch.empty(V if c == "v" else E, W, device=dev)
        kw = dict(A=A, a_type=a, B=B, b_type=b, C=C, c_type=c, F=F, H=H)
        sched = ug.schedule_select(g, eo, go, **kw)
        by = 4 * (V + 1) + 4 * E
        for t, w in ((a, wa), (b, wb)):
            if t in ("u", "e"):
                by += 4 * E * w
            elif t == "v":
                by += 4 * V * w
        by += 4 * (V if c == "v" else E) * W
        res = {}
        for mode in ("warm", "cold"):
            ts = []
            for i in range(warm + reps):
                if mode == "cold":
                    scrub.fill_(float(i))       # evict L2; also queues the op behind GPU work
                else:
                    torch.cuda._sleep(400_000)  # queue behind a spin kernel: device time only
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record()
                ug.op_run(g, eo, go, schedule=sched, **kw)
                e1.record()
                torch.cuda.synchronize()
                if i >= warm:
                    ts.append(e0.elapsed_time(e1))
            ms = statistics.median(ts)
            res[mode] = {"latency_us": round(ms * 1e3, 2), "gbs": round(by / (ms * 1e-3) / 1e9, 1)}
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(20):
            ug.op_run(g, eo, go, schedule=sched, **kw)
        host_us = (time.perf_counter() - t0) / 20 * 1e6
        torch.cuda.synchronize()
        pop = ug.prepare(g, eo, go, schedule=sched, **kw)     # marshalled once (serving loop)
        t0 = time.perf_counter()
        for _ in range(20):
            pop()
        prep_us = (time.perf_counter() - t0) / 20 * 1e6
        torch.cuda.synchronize()
        out.append({"config": cfg, "op": nm, "F": F, "H": H, "schedule": sched, "logical_bytes": by,
                    "warm": res["warm"], "cold": res["cold"], "host_launch_us": round(host_us, 2),
                    "host_launch_prepared_us": round(prep_us, 2)})
        del A, B, C
    del scrub
    out.append(gat_chain_graph(ug, torch, dev, graphs["C2"][0]))
    out += dot_attention_graphs(ug, torch, dev, graphs)
    return out


def dot_attention_graphs(ug, torch, dev, graphs, reps=20):
    """Fused dot-product attention (ug_dot_attention, f3) on the C2 / C4 shapes: device latency
    (queued behind a spin kernel) and effective GB/s of its logical bytes (row_ptr, col_idx, the
    q row per destination, the k and val rows per edge, the output)."""
    import ugdata
    out = []
    for cfg, H, F in (("C2", 8, 64), ("C4", 8, 128), ("C4", 1, 128)):
        g, E = graphs[cfg]
        V = ugdata.CONFIGS[cfg].V
        z = torch.randn(V, F, device=dev)
        o = torch.empty(V, F, device=dev)
        ts = []
        for i in range(5 + reps):
            torch.cuda._sleep(200_000)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ug.dot_attention(g, z, z, z, H, out=o)
            e1.record()
            torch.cuda.synchronize()
            if i >= 5:
                ts.append(e0.elapsed_time(e1) * 1e3)
        us = statistics.median(ts)
        by = 4 * (V + 1) + 4 * E + 4 * V * F + 2 * 4 * E * F + 4 * V * F
        out.append({"config": cfg, "op": "dot attention (fused SDDMM + softmax + SpMM)", "F": F, "H": H,
                    "latency_us": round(us, 2), "logical_bytes": by, "gbs": round(by / (us * 1e-6) / 1e9, 1)})
    return out


def gat_chain_graph(ug, torch, dev, g, reps=50):
    """C2 GAT attention chain (u_add_v -> e_max -> e_div_v -> e_sum -> e_div_v -> u_mul_e_sum,
    6 graph ops) issued eagerly through PreparedOp vs replayed as one CUDA graph:
    small graphs are launch-bound, a captured chain removes the host cost per op."""
    import ugdata
    c = ugdata.CONFIGS["C2"]
    V, E, H, F = c.V, c.E, 8, 64
    X = torch.rand(V, F, device=dev)
    el, er = torch.rand(V, H, device=dev) + 0.5, torch.rand(V, H, device=dev) + 0.5
    a, s, p = (torch.empty(E, H, device=dev) for _ in range(3))
    m, den = torch.empty(V, H, device=dev), torch.empty(V, H, device=dev)
    Y = torch.empty(V, F, device=dev)
    chain = [ug.prepare(g, "add", "assign", A=el, a_type="u", B=er, b_type="v", C=a, c_type="e", F=H, H=H),
             ug.prepare(g, "copy_lhs", "max", A=a, a_type="e", C=m, c_type="v", F=H, H=H),
             ug.prepare(g, "div", "assign", A=a, a_type="e", B=m, b_type="v", C=s, c_type="e", F=H, H=H),
             ug.prepare(g, "copy_lhs", "sum", A=s, a_type="e", C=den, c_type="v", F=H, H=H),
             ug.prepare(g, "div", "assign", A=s, a_type="e", B=den, b_type="v", C=p, c_type="e", F=H, H=H),
             ug.prepare(g, "mul", "sum", A=X, a_type="u", B=p, b_type="e", C=Y, c_type="v", F=F, H=H)]
    side = torch.cuda.Stream(dev)
    with torch.cuda.stream(side):
        for op in chain:
            op()
    torch.cuda.synchronize()
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg):
        for op in chain:
            op()
    torch.cuda.synchronize()

    def timed(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        fn()
        torch.cuda.synchronize()
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps * 1e3

    eager = timed(lambda: [op() for op in chain])
    graph = timed(cg.replay)
    # the same chain (with the real LeakyReLU / exp) as ONE traversal: ug_gat_attention (f3)
    out, att = torch.empty(V, F, device=dev), torch.empty(E, H, device=dev)
    fused = timed(lambda: ug.gat_attention(g, el, er, X, H, 0.2, out=out))
    fused_attn = timed(lambda: ug.gat_attention(g, el, er, X, H, 0.2, out=out, attn=att))
    dev_ts = []
    for i in range(25):
        torch.cuda._sleep(400_000)          # queued behind a spin kernel: device time only
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ug.gat_attention(g, el, er, X, H, 0.2, out=out)
        e1.record()
        torch.cuda.synchronize()
        if i >= 5:
            dev_ts.append(e0.elapsed_time(e1) * 1e3)
    # algorithmic bytes of the fused traversal: row_ptr, col_idx, el gathers (E x H), er (V x H),
    # z gathers (E x F), out (V x F)
    by = 4 * (V + 1) + 4 * E + 4 * E * H + 4 * V * H + 4 * E * F + 4 * V * F
    dmed = statistics.median(dev_ts)
    return {"config": "C2", "op": "GAT attention chain (6 ops)", "F": F, "H": H,
            "schedules": [op.schedule for op in chain],
            "eager_us_per_chain": round(eager, 2), "cuda_graph_us_per_chain": round(graph, 2),
            "fused_one_kernel_us": round(fused, 2), "fused_with_attention_out_us": round(fused_attn, 2),
            "fused_device_us": round(dmed, 2), "fused_logical_bytes": by,
            "fused_gbs": round(by / (dmed * 1e-6) / 1e9, 1)}


# ---------------------------------------------------------------------------- GPU run
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--op", default="copy_u_sum", choices=sorted(OPS))
    ap.add_argument("--F", type=int, default=None)
    ap.add_argument("--schedule", default=None, help="Table 9 notation; default: ug_schedule_select")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-secondary", action="store_true", help="skip the C1-C4 per op x graph latencies")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world, rank, local = dist_env()
    import ugdata
    cfg = ugdata.CONFIGS[args.config]
    F = args.F or cfg.widths[-1]
    workload = f"{args.config} {cfg.label} synthetic graph ({cfg.V:,} v / {cfg.E:,} e), {args.op}, F={F}"

    if args.impl == "reference":
        run_reference(args, cfg, F, workload, world, rank)
        return

    import torch
    import paper_conf_asplos_0001lslwlgslllw23_b200 as ug
    from paper_conf_asplos_0001lslwlgslllw23_b200.pipeline import StreamedOperator
    from paper_conf_asplos_0001lslwlgslllw23_b200.shard import ShardedOperator, x_block

    dist = None
    # one process per GPU over NCCL; UG_DIST_BACKEND=gloo is a single-GPU dry run of the N > 1
    # path (ranks share cuda:0, the exchange is staged through host memory) -- never a bench number
    backend = os.environ.get("UG_DIST_BACKEND", "nccl")
    dev = torch.device("cuda", local % max(1, torch.cuda.device_count()))
    torch.cuda.set_device(dev)
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    def max_over_ranks(vals):
        t = torch.tensor(vals, dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return [float(x) for x in t]

    src, dst = ugdata.graph(args.config)
    V, E = cfg.V, len(src)
    eo, go, a_t, b_t = OPS[args.op]
    t_ing = time.perf_counter()
    g_full = ug.Graph(V, src, dst)                    # a1: COO -> in-CSR + stats + upload (one-time)
    ingest_ms = (time.perf_counter() - t_ing) * 1e3
    sh = ShardedOperator(g_full, world, rank)
    g = sh.view
    Vl, El = sh.local_rows, sh.e1 - sh.e0

    X_host = ugdata.values(V, F, cfg.seed + 1, 1)
    X_full = torch.empty(sh.blk * world, F, device=dev)
    X_full[:V].copy_(torch.from_numpy(X_host))
    X_local = x_block(X_full[:V], V, world, rank)
    Bt = None
    if b_t == "e":
        Bt = sh.edge_slice(torch.from_numpy(ugdata.values(E, 1, cfg.seed + 1, 2, role="edge")).to(dev))
    elif b_t == "v":
        Bt = sh.dst_slice(X_full)
    c_t = "e" if go == "assign" else "v"
    W = 1 if eo == "dot" else F
    Y = torch.empty(Vl if c_t == "v" else El, W, device=dev)
    kw = dict(A=X_full[:V], a_type=a_t, B=Bt, b_type=b_t, C=Y, c_type=c_t, F=F, H=1)
    chosen = args.schedule or ug.schedule_select(g, eo, go, **kw)
    launches = ug.launch_count(g, eo, go, schedule=chosen, **kw)

    stream = torch.cuda.current_stream(dev)
    ev_k0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev_k1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev_s0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev_s1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    for e in ev_k0 + ev_k1:
        e.record(stream)   # materialise the cudaEvent_t handles
    torch.cuda.synchronize()

    # N > 1, single-operand aggregation (copy_u_*): column-chunked all-gather overlapped with
    # the per-chunk op (ShardedOperator.run_chunked); otherwise gather X, then one op.
    chunked = world > 1 and b_t is None and go != "assign"
    bufs = sh.chunk_buffers(F, 64, dev) if chunked else None
    if chunked:
        launches = sum(ug.launch_count(g, eo, go, A=bufs["full"][c][:V], a_type="u", C=Y[:, c0:c1], c_type="v",
                                       F=c1 - c0, H=1) for c, (c0, c1) in enumerate(bufs["cols"]))

    def step(i=None):
        if chunked:
            if i is not None:
                ev_k0[i].record(stream)
            sh.run_chunked(eo, go, X_local, Y, chunk=64, buffers=bufs)
            if i is not None:
                ev_k1[i].record(stream)
            return
        if world > 1:
            sh.gather_x(X_local, X_full)          # the exchange: NCCL all-gather of X row blocks
        if i is None:
            ug.op_run(g, eo, go, schedule=chosen, **kw)
        else:
            ug.op_run_events(g, eo, go, ev_k0[i], ev_k1[i], schedule=chosen, **kw)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(dev.index) as clocks:
        for i in range(args.steps):
            ev_s0[i].record(stream)
            step(i)
            ev_s1[i].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    tot = sum(ev_s0[i].elapsed_time(ev_s1[i]) for i in range(args.steps))
    ktot = sum(ev_k0[i].elapsed_time(ev_k1[i]) for i in range(args.steps))
    t_p = None
    if world > 1:
        # T_P with and without the all-gather.  The exchange-free step runs the same
        # local op(s) on the X already gathered (same buffers, same schedule), K times, timed the
        # same way (barrier + sync on both sides, max over ranks).
        def local_only():
            if chunked:
                for c, (c0, c1) in enumerate(bufs["cols"]):
                    ug.op_run(g, eo, go, A=bufs["full"][c][:V], a_type="u", C=Y[:, c0:c1], c_type="v",
                              F=c1 - c0, H=1)
            else:
                ug.op_run(g, eo, go, schedule=chosen, **kw)
        local_only()
        torch.cuda.synchronize()
        dist.barrier()
        torch.cuda.synchronize()
        n0 = torch.cuda.Event(enable_timing=True)
        n1 = torch.cuda.Event(enable_timing=True)
        n0.record(stream)
        for _ in range(args.steps):
            local_only()
        n1.record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        torch.cuda.synchronize()
        g0 = torch.cuda.Event(enable_timing=True)
        g1 = torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        for _ in range(args.steps):
            sh.gather_x(X_local, X_full)
        g1.record(stream)
        torch.cuda.synchronize()
        tot, ktot, ntot, gtot = max_over_ranks([tot, ktot, n0.elapsed_time(n1), g0.elapsed_time(g1)])
        t_p = {"with_allgather_ms": round(tot / args.steps, 4),
              "without_allgather_ms": round(ntot / args.steps, 4),
              "allgather_alone_ms": round(gtot / args.steps, 4),
              "allgather_bytes_per_rank": int(sh.blk * (world - 1) * F * 4),
              "how": "max over ranks of K steps, CUDA events on the launching stream; 'with' is the "
                     "timed step (exchange overlapped by column chunks when chunked), 'without' the "
                     "same local op(s) on the already-gathered X, 'alone' the unchunked all-gather"}
    ms = tot / args.steps
    kms = ktot / args.steps
    by = logical_bytes(V, E, F, args.op)
    by_local = logical_bytes(Vl, El, F, args.op)
    value = by / (ms * 1e-3) / 1e9
    peak, peak_src = load_peaks()
    achieved = by_local / (kms * 1e-3) / 1e9

    # e2e through the public API (StreamedOperator): every step copies its X from pinned host
    # memory and reads its Y back; copies of neighbouring steps overlap the operator.
    e2e = None
    if not args.no_e2e:
        Xh = torch.from_numpy(X_host).pin_memory()
        n_e2e = max(3, args.steps)         # K steps, like the device-timed value (pipeline fill amortised alike)
        Yh = [torch.empty(tuple(Y.shape), dtype=torch.float32).pin_memory() for _ in range(2)]
        if world == 1:
            so = StreamedOperator(g, eo, go, a_type=a_t, in_shape=(V, F), out_shape=tuple(Y.shape), c_type=c_t,
                                  schedule=chosen, depth=2, F=F, H=1,
                                  B=Bt if b_t == "e" else None, b_type=b_t)
            bfn = (lambda i, Xd: Xd) if b_t == "v" else None
            so.run([Xh] * 2, Yh, b_fn=bfn)      # warm-up
            so.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(so.s_in)
            so.run([Xh] * n_e2e, [Yh[i % 2] for i in range(n_e2e)], b_fn=bfn)
            so.s_in.wait_stream(so.s_out)
            e1.record(so.s_in)
            so.synchronize()
            e_ms = e0.elapsed_time(e1) / n_e2e
        else:
            Xlh = torch.from_numpy(x_block(torch.from_numpy(X_host), V, world, rank).numpy()).pin_memory()
            Xl = torch.empty_like(X_local)
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            dist.barrier()
            e0.record(stream)
            for i in range(n_e2e):
                Xl.copy_(Xlh, non_blocking=True)
                if chunked:
                    sh.run_chunked(eo, go, Xl, Y, chunk=64, buffers=bufs)
                else:
                    sh.gather_x(Xl, X_full)
                    ug.op_run(g, eo, go, schedule=chosen, **kw)
                Yh[i % 2].copy_(Y, non_blocking=True)
            e1.record(stream)
            torch.cuda.synchronize()
            e_ms = max_over_ranks([e0.elapsed_time(e1) / n_e2e])[0]
        e2e = {"value": round(by / (e_ms * 1e-3) / 1e9, 1), "unit": "GB/s", "ms_per_step": round(e_ms, 3),
               "h2d_bytes_per_step": int((V if world == 1 else sh.blk * world) * F * 4),
               "d2h_bytes_per_step": int(Y.numel() * 4 * world),
               "how": "pinned host X -> device, op, device Y -> pinned host, every step; copies of "
                      "neighbouring steps overlap the op (StreamedOperator)" if world == 1 else
                      "pinned host X block -> device, all-gather, op, Y shard -> host, every step"}

    traffic = None
    l2 = None
    ncu_ent = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            ncu_ent = json.load(open(tp)).get(f"{args.config}:{args.op}:{F}:{chosen}")
            # dram__bytes_read.sum + dram__bytes_write.sum of one launch (ncu --set full)
            traffic = int(ncu_ent["dram_bytes_per_launch"]) if ncu_ent and world == 1 else None
            if ncu_ent and world == 1 and "l2_to_sm_bytes" in ncu_ent:
                # the binding roof of the tile-major schedule is L2 -> SM, not HBM
                l2 = {"l2_to_sm_bytes_per_launch": int(ncu_ent["l2_to_sm_bytes"]),
                      "achieved_gbs": round(ncu_ent["l2_to_sm_bytes"] / (kms * 1e-3) / 1e9, 1),
                      "ncu_lts_throughput_pct": ncu_ent.get("lts_throughput_pct"),
                      "ncu_source": ncu_ent.get("source")}
        except (ValueError, OSError, KeyError, TypeError):
            traffic = None
    # measured L2 -> SM read peak (scripts/probes/peaks.cu on this pool's B200s; the median of the
    # probe's 96 MB runs): the direct denominator of the L2-bound kernel's achieved L2 -> SM bytes
    pk = os.path.join(ROOT, "profiles", "r2", "peaks_r2.json")
    if l2 and os.path.exists(pk):
        try:
            pkd = json.load(open(pk))
            l2["l2_read_peak_gbs"] = pkd["l2_read_gbs_96MB"]
            l2["frac_of_l2_read_peak"] = round(l2["achieved_gbs"] / pkd["l2_read_gbs_96MB"], 4)
            l2["l2_peak_source"] = "profiles/r2/peaks_r2.json (" + pkd.get("how", "") + ")"
        except (ValueError, OSError, KeyError, TypeError):
            pass

    secondary = None
    headline_ops = None
    if rank == 0 and world == 1 and not args.no_secondary:
        headline_ops = headline_graph_ops(ug, torch, g, X_full[:V], V, E, F, cfg)
        secondary = secondary_configs(ug, torch, dev)
        # ncu DRAM bytes / L2 hit rate of the same (op, config, schedule), scripts/ncu_per_op.py
        pp = os.path.join(ROOT, "profiles", "ncu_per_op.json")
        if os.path.exists(pp):
            prof = {(o["config"], o["op"], o["F"], o["schedule"]): o for o in json.load(open(pp))["ops"]}
            for ent in secondary:
                o = prof.get((ent.get("config"), ent.get("op"), ent.get("F"), ent.get("schedule")))
                if o:
                    ent["ncu"] = {"dram_bytes": o["dram_bytes"], "l2_to_sm_bytes": o["l2_to_sm_bytes"],
                                  "l2_hit_rate_pct": o["l2_hit_rate_pct_main_kernel"], "cold_us": o["ncu_us"]}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        with PinnedCore():
            gbs, nr, ne, dt = oracle_sample(args.config, args.op, F, src, dst, V)
        cpu = {"value": round(gbs, 4), "unit": "GB/s", "cores": cores_used(), "kind": "oracle",
               "sample": f"{args.op} on {nr} random dst rows ({ne} in-edges) of {args.config}, {dt:.1f} s, "
                         f"oracle/ug_oracle.c single thread pinned to one core (sched_setaffinity, = taskset -c 0)",
               "host": host_info(),
               "per_config": oracle_per_config(secondary) if secondary else None}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": workload, "op": args.op, "V": V, "E": E, "F": F, "ld": F,
                       "schedule": chosen, "graph": "Chung-Lu lognormal degrees (ugdata), seed %d" % cfg.seed,
                       "l2": "inputs larger than L2 (X %.0f MB, col_idx %.0f MB > 126 MB): no flush"
                             % (V * F * 4 / 1e6, E * 4 / 1e6),
                       "parallelism": f"dst-row sharding x{world}" + (
                           (" + column-chunked NCCL all-gather of X overlapped with the op" if chunked
                            else " + NCCL all-gather of X") if world > 1 else ""),
                       "logical_bytes": by},
            "latency_ms": round(ms, 4),
            **({"t_p": t_p} if t_p else {}),
            "graph_ingest_ms": round(ingest_ms, 1),
            "frac_of_8TBps": round(value / 8000.0, 4),
            "roofline": {"bound": "l2" if l2 else "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "frac_basis": ("logical (algorithmic, SURVEY 8(d)) bytes per live launch / measured HBM copy "
                                        "bandwidth: an EFFECTIVE rate; above 1 because the tile-major SV schedule "
                                        "serves the per-edge row gathers from L2. The binding roof is L2 -> SM: "
                                        "l2_frac; DRAM use: dram_frac") if l2 else "algorithmic bytes / HBM peak",
                         "l2_frac": round(l2["ncu_lts_throughput_pct"] / 100.0, 4)
                                    if l2 and l2.get("ncu_lts_throughput_pct") else None,
                         "dram_frac": round(traffic / (kms * 1e-3) / 1e9 / peak, 4) if traffic else None,
                         "kernel": ("k_split per 64-column chunk, exchange overlapped" if chunked else
                                    "k_split (SV main traversal)" if chosen.startswith("SV") else "main traversal"),
                         "kernel_ms": round(kms, 4), "peak_source": peak_src,
                         "bytes": "algorithmic (SURVEY 8(d)) per launch, this rank's rows",
                         "l2": l2},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches * args.steps,
            "clocks": clocks.summary(),
            **({"dry_run": f"{backend} backend, ranks share one GPU: not a measurement"} if backend != "nccl" else {}),
            "headline_graph_ops": headline_ops,
            "per_op_graph": secondary,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_reference(args, cfg, F, workload, world, rank):
    """This tier's reference arm: the CPU oracle as it stands, 1 core, bounded row samples."""
    if rank != 0:
        return
    import ugdata
    src, dst = ugdata.graph(args.config)
    V = cfg.V
    per_step = 60.0 / max(1, args.steps + args.warmup)
    for i in range(args.warmup):
        oracle_sample(args.config, args.op, F, src, dst, V, target_s=min(per_step, 5.0), seed=100 + i)
    vals, rows, edges, secs = [], 0, 0, 0.0
    for i in range(args.steps):
        gbs, nr, ne, dt = oracle_sample(args.config, args.op, F, src, dst, V, target_s=min(per_step, 10.0), seed=i)
        vals.append(gbs)
        rows += nr
        edges += ne
        secs += dt
    value = float(np.mean(vals))
    sample = f"{args.op} on {args.steps} random samples ({rows} dst rows, {edges} in-edges total) of {args.config}"
    line = {"metric": METRIC, "value": round(value, 4), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(secs / args.steps * 1e3, 2), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic", "impl": "reference",
            "config": {"workload": workload, "op": args.op, "V": V, "E": cfg.E, "F": F},
            "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
