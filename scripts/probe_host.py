#!/usr/bin/env python
"""Host-side cost of one unified-operator call on small graphs (C1, C2), split into its parts:
stream lookup, ctypes call into ug_op_run (validation + lowering + launches), and the bare
CUDA launch cost for comparison.  Wall-clock means over many back-to-back calls; the GPU is
kept busy behind a spin kernel so the launch queue never throttles the host.

  python scripts/probe_host.py > gpurun_out/probe_host.json
"""
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_0001lslwlgslllw23_b200 as ug  # noqa: E402
import ugdata  # noqa: E402


def per_call_us(fn, n=2000):
    for _ in range(50):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    dt = (time.perf_counter() - t0) / n * 1e6
    torch.cuda.synchronize()
    return round(dt, 3)


def main():
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    out = {"parts": {}, "ops": []}
    p = out["parts"]
    p["torch_current_stream"] = per_call_us(lambda: torch.cuda.current_stream().cuda_stream)
    p["raw_stream_dev0"] = per_call_us(lambda: torch._C._cuda_getCurrentRawStream(0))
    p["raw_stream_current_device"] = per_call_us(
        lambda: torch._C._cuda_getCurrentRawStream(torch.cuda.current_device()))
    p["is_available"] = per_call_us(torch.cuda.is_available)
    x = torch.empty(1, device=dev)
    p["torch_fill_1_elem"] = per_call_us(lambda: x.fill_(1.0))
    for cfg, eo, go, a, b, c, F, H, wa, wb in (("C1", "mul", "sum", "u", "e", "v", 16, 1, 16, 1),
                                              ("C2", "add", "assign", "u", "v", "e", 8, 8, 8, 8),
                                              ("C2", "mul", "sum", "u", "e", "v", 64, 8, 64, 8)):
        s, d = ugdata.graph(cfg)
        V, E = ugdata.CONFIGS[cfg].V, len(s)
        g = ug.Graph(V, s, d)
        rows = lambda t: V if t in ("u", "v") else E
        A = torch.rand(rows(a), wa, device=dev)
        B = torch.rand(rows(b), wb, device=dev) + 0.5
        C = torch.empty(rows(c), H if eo == "dot" else F, device=dev)
        kw = dict(A=A, a_type=a, B=B, b_type=b, C=C, c_type=c, F=F, H=H)
        sched = ug.schedule_select(g, eo, go, **kw)
        pop = ug.prepare(g, eo, go, schedule=sched, **kw)
        st = torch.cuda.current_stream().cuda_stream
        r = {"config": cfg, "op": f"{eo}_{go}_{a}{b}{c}", "F": F, "H": H, "schedule": sched,
             "launches": ug.launch_count(g, eo, go, schedule=sched, **kw)}
        r["op_run_us"] = per_call_us(lambda: ug.op_run(g, eo, go, schedule=sched, **kw))
        r["prepared_us"] = per_call_us(pop)
        r["prepared_given_stream_us"] = per_call_us(lambda: pop(st))
        h, ir, sr, sv = pop._h, pop._iref, pop._sref, ctypes.c_void_p(st)
        r["bare_ctypes_ug_op_run_us"] = per_call_us(lambda: ug.lib.ug_op_run(h, ir, sr, sv))
        out["ops"].append(r)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
