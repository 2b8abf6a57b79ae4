"""Host-to-host streaming of the unified operator over many feature batches (serving path).

For each batch i: copy X_i host->device on a copy stream, run the operator on the compute
stream, copy Y_i device->host on a second copy stream.  With `depth` device buffers the copy
of batch i+1 and the read-back of batch i-1 overlap the operator of batch i (separate copy
engines), so the steady-state cost per batch is max(H2D, op, D2H) instead of their sum.
Every batch still moves all of its inputs and outputs across the host link.  Plumbing only:
torch streams/events + ug_op_run.
"""
from __future__ import annotations

import torch

from . import op_run


class StreamedOperator:
    def __init__(self, graph, edge_op, gather_op, a_type="u", in_shape=None, out_shape=None, c_type="v",
                 schedule=None, depth=2, device=None, F=None, H=None, B=None, b_type=None):
        self.graph = graph
        self.edge_op, self.gather_op = edge_op, gather_op
        self.a_type, self.c_type = a_type, c_type
        self.B, self.b_type = B, b_type
        self.schedule = schedule
        self.F, self.H = F, H
        self.depth = depth
        dev = device or torch.device("cuda", torch.cuda.current_device())
        self.Xd = [torch.empty(in_shape, device=dev) for _ in range(depth)]
        self.Yd = [torch.empty(out_shape, device=dev) for _ in range(depth)]
        self.s_in = torch.cuda.Stream(dev)
        self.s_comp = torch.cuda.Stream(dev)
        self.s_out = torch.cuda.Stream(dev)
        mk = lambda: [torch.cuda.Event() for _ in range(depth)]
        self.ev_in, self.ev_done, self.ev_out = mk(), mk(), mk()
        self.started = [False] * depth

    def run(self, host_inputs, host_outputs, b_fn=None):
        """host_inputs / host_outputs: sequences of pinned CPU tensors (same length).
        b_fn(i, X_dev) optionally returns the B operand for batch i (e.g. Dst_V = X itself)."""
        for i, (xh, yh) in enumerate(zip(host_inputs, host_outputs)):
            k = i % self.depth
            if self.started[k]:
                self.s_in.wait_event(self.ev_done[k])      # compute of batch i-depth finished reading Xd[k]
            with torch.cuda.stream(self.s_in):
                self.Xd[k].copy_(xh, non_blocking=True)
                self.ev_in[k].record(self.s_in)
            self.s_comp.wait_event(self.ev_in[k])
            if self.started[k]:
                self.s_comp.wait_event(self.ev_out[k])     # read-back of batch i-depth finished with Yd[k]
            with torch.cuda.stream(self.s_comp):
                B = b_fn(i, self.Xd[k]) if b_fn else self.B
                op_run(self.graph, self.edge_op, self.gather_op, A=self.Xd[k], a_type=self.a_type, B=B,
                       b_type=self.b_type, C=self.Yd[k], c_type=self.c_type, F=self.F, H=self.H,
                       schedule=self.schedule, stream=self.s_comp.cuda_stream)
                self.ev_done[k].record(self.s_comp)
            self.s_out.wait_event(self.ev_done[k])
            with torch.cuda.stream(self.s_out):
                yh.copy_(self.Yd[k], non_blocking=True)
                self.ev_out[k].record(self.s_out)
            self.started[k] = True
        return host_outputs

    def synchronize(self):
        for s in (self.s_in, self.s_comp, self.s_out):
            s.synchronize()
