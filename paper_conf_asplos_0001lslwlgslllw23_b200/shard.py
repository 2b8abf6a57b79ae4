"""Destination-row sharding of the unified operator across the GPUs of one node (north star
(4)).  Plumbing only: the partition and the zero-copy views come from the C ABI
(ug_graph_partition / ug_graph_view_rows), the exchange is torch.distributed's
all_gather_into_tensor (NCCL over NVLink 5 / NVSwitch on B200), and the compute is ug_op_run.

Layout contract:
  * rank k owns destination rows [splits[k], splits[k+1]) with splits edge-balanced (R21);
  * the Src_V feature matrix X is held as equal row blocks of blk = ceil(V / P) rows (the
    last block zero-padded), so the all-gathered buffer [P * blk, F] IS the full X with no
    remapping; rows >= V are padding and never indexed;
  * Dst_V operands and the output are local row slices; Edge operands are the slice
    [row_ptr[r0], row_ptr[r1]) of a dst-sorted edge tensor.
"""
from __future__ import annotations

import torch


def _all_gather(out: torch.Tensor, inp: torch.Tensor, group=None):
    """all_gather_into_tensor; with a gloo group (CPU dry runs of the N > 1 path) the CUDA
    tensors are staged through host memory."""
    import torch.distributed as dist
    if dist.get_backend(group) == "gloo" and out.is_cuda:
        o = torch.empty(out.shape, dtype=out.dtype)
        dist.all_gather_into_tensor(o, inp.cpu(), group=group)
        out.copy_(o)
    else:
        dist.all_gather_into_tensor(out, inp, group=group)


def block_rows(V: int, world: int) -> int:
    return -(-V // world)


def x_block(X_full_rows: torch.Tensor, V: int, world: int, rank: int) -> torch.Tensor:
    """This rank's row block of X (padded to blk rows), e.g. to seed X_local from a full copy."""
    blk = block_rows(V, world)
    out = X_full_rows.new_zeros((blk,) + tuple(X_full_rows.shape[1:]))
    lo, hi = rank * blk, min(V, (rank + 1) * blk)
    if hi > lo:
        out[: hi - lo].copy_(X_full_rows[lo:hi])
    return out


class ShardedOperator:
    """Per-rank state of one sharded operator over a graph replicated on every rank."""

    def __init__(self, graph, world: int, rank: int, group=None):
        self.graph = graph
        self.world = world
        self.rank = rank
        self.group = group
        st = graph.stats()
        self.V = st["V"]
        self.splits = graph.partition(world)
        self.r0, self.r1 = int(self.splits[rank]), int(self.splits[rank + 1])
        self.view = graph.view_rows(self.r0, self.r1) if world > 1 else graph
        rp = graph.row_ptr()
        self.e0, self.e1 = int(rp[self.r0]), int(rp[self.r1])
        self.blk = block_rows(self.V, world)

    @property
    def local_rows(self) -> int:
        return self.r1 - self.r0

    def gather_x(self, X_local: torch.Tensor, X_full: torch.Tensor | None = None) -> torch.Tensor:
        """All-gather the row blocks of X into the full [P * blk, F] buffer (the exchange step)."""
        import torch.distributed as dist
        if X_full is None:
            X_full = X_local.new_empty((self.blk * self.world,) + tuple(X_local.shape[1:]))
        if self.world == 1:
            X_full.copy_(X_local)
        else:
            _all_gather(X_full, X_local.contiguous(), group=self.group)
        return X_full

    def edge_slice(self, T: torch.Tensor) -> torch.Tensor:
        return T[self.e0:self.e1]

    def dst_slice(self, T: torch.Tensor) -> torch.Tensor:
        return T[self.r0:self.r1]

    def run(self, edge_op, gather_op, X_local, C_local, B=None, b_type=None, X_full=None, schedule=None,
            F=None, H=None):
        """One sharded step: all-gather X, then the local op on this rank's rows.  A is the
        gathered X as Src_V; B (optional) is this rank's Dst_V / Edge slice."""
        from . import op_run
        X_full = self.gather_x(X_local, X_full)
        op_run(self.view, edge_op, gather_op, A=X_full[: self.V], a_type="u", B=B, b_type=b_type, C=C_local,
               c_type="v", F=F, H=H, schedule=schedule)
        return C_local

    def run_chunked(self, edge_op, gather_op, X_local, C_local, chunk=64, schedule=None, buffers=None):
        """Sharded step with the exchange overlapped (SURVEY 8(e) overlap option): X is
        all-gathered in column chunks (the paper's feature-tiling axis) on a side
        stream while the operator runs on the previous chunk; every chunk's op writes its own
        columns of C_local.  Only ops whose sole feature operand is the Src_V X (copy_u_*) are
        column-separable this way.  `buffers` (from chunk_buffers) are reused across steps."""
        import torch.distributed as dist
        from . import op_run
        F = X_local.shape[1]
        bufs = buffers or self.chunk_buffers(F, chunk, X_local.device)
        main = torch.cuda.current_stream(X_local.device)
        side = bufs["stream"]
        side.wait_stream(main)                       # X_local is ready
        for c, (c0, c1) in enumerate(bufs["cols"]):
            with torch.cuda.stream(side):
                bufs["send"][c].copy_(X_local[:, c0:c1])
                if self.world == 1:
                    bufs["full"][c].copy_(bufs["send"][c])
                else:
                    _all_gather(bufs["full"][c], bufs["send"][c], group=self.group)
                bufs["ready"][c].record(side)
        for c, (c0, c1) in enumerate(bufs["cols"]):
            main.wait_event(bufs["ready"][c])
            op_run(self.view, edge_op, gather_op, A=bufs["full"][c][: self.V], a_type="u",
                   C=C_local[:, c0:c1], c_type="v", F=c1 - c0, H=1, schedule=schedule)
        return C_local

    def chunk_buffers(self, F, chunk, device):
        cols = [(c0, min(F, c0 + chunk)) for c0 in range(0, F, chunk)]
        return {"cols": cols, "stream": torch.cuda.Stream(device),
                "send": [torch.empty(self.blk, c1 - c0, device=device) for c0, c1 in cols],
                "full": [torch.empty(self.blk * self.world, c1 - c0, device=device) for c0, c1 in cols],
                "ready": [torch.cuda.Event() for _ in cols]}

    def gather_rows(self, Y_local: torch.Tensor) -> torch.Tensor:
        """Reassemble the row-sharded output on every rank (verification / next-layer input)."""
        import torch.distributed as dist
        if self.world == 1:
            return Y_local
        sizes = [int(self.splits[k + 1] - self.splits[k]) for k in range(self.world)]
        m = max(sizes)
        pad = Y_local.new_zeros((m,) + tuple(Y_local.shape[1:]))
        pad[: Y_local.shape[0]].copy_(Y_local)
        allp = Y_local.new_empty((m * self.world,) + tuple(Y_local.shape[1:]))
        _all_gather(allp, pad, group=self.group)
        return torch.cat([allp[k * m: k * m + sizes[k]] for k in range(self.world)])
