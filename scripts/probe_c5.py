#!/usr/bin/env python
"""Where do the C5 headline kernel's in-bench milliseconds go?  Times the SV main traversal
(CUDA events recorded by ug_op_run_events around that launch) under several step shapes:

  b2b      back-to-back calls, as bench.py's timed loop;
  gap      an idle spin kernel (~0.4 ms) before each call;
  flush    a 256 MB buffer written before each call (L2 holds no X lines);
  aligned  X allocated with ld = 608 (2,432-byte rows), schedule without the pack.

    python scripts/probe_c5.py [--schedule SV_G512_F128_P1] [--reps 8]
"""
import argparse
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--schedule", default="SV_G512_F128_P1")
    ap.add_argument("--reps", type=int, default=8)
    ap.add_argument("--F", type=int, default=602)
    ap.add_argument("--modes", default="b2b,gap,flush,aligned")
    a = ap.parse_args()
    c = ugdata.CONFIGS[a.config]
    src, dst = ugdata.graph(a.config)
    g = ug.Graph(c.V, src, dst)
    F = a.F
    X = torch.rand(c.V, F, device="cuda") - 0.5
    Y = torch.empty(c.V, F, device="cuda")
    Xa = torch.zeros(c.V, 608, device="cuda")[:, :F]
    Xa.copy_(X)
    Ya = torch.empty(c.V, 608, device="cuda")[:, :F]
    junk = torch.empty(64 * 1024 * 1024, device="cuda")
    s = torch.cuda.current_stream()

    def run(mode, sched, A, C):
        ts, tk = [], []
        for i in range(a.reps + 2):
            if mode == "gap":
                torch.cuda._sleep(800_000)
            elif mode == "flush":
                junk.fill_(float(i))
            k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            k0.record(s)    # materialise the cudaEvent_t handles ug_op_run_events records into
            k1.record(s)
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s0.record(s)
            ug.op_run_events(g, "copy_lhs", "sum", k0, k1, A=A, a_type="u", C=C, c_type="v", schedule=sched)
            s1.record(s)
            if mode != "b2b":
                torch.cuda.synchronize()
            ts.append((s0, s1))
            tk.append((k0, k1))
        torch.cuda.synchronize()
        step = [x.elapsed_time(y) for x, y in ts[2:]]
        kern = [x.elapsed_time(y) for x, y in tk[2:]]
        print(f"{mode:8s} {sched:18s} step median {statistics.median(step):8.3f} ms  kernel median "
              f"{statistics.median(kern):8.3f} ms  min {min(kern):8.3f}", flush=True)

    modes = a.modes.split(",")
    from bench import ClockSampler
    for mode in ("b2b", "gap", "flush"):
        if mode in modes:
            with ClockSampler(torch.cuda.current_device()) as cs:
                run(mode, a.schedule, X, Y)
            print("   clocks", cs.summary(), flush=True)
    if "aligned" in modes:
        base = a.schedule.replace("_P1", "")
        for mode in ("b2b", "gap"):
            run(mode, base, Xa, Ya)


if __name__ == "__main__":
    main()
