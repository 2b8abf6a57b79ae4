"""N > 1 path on CPU: world_size-2 gloo run of the sharded operator's host logic.

Each rank builds the (host-only) graph, takes its edge-balanced row view, all-gathers the row
blocks of X with torch.distributed (gloo here, NCCL on B200), computes its rows, and the
row shards are gathered back.  The per-rank compute here is the CPU oracle applied to the
rank's VIEW (its local CSR from the C ABI) -- a stand-in for ug_op_run, which needs a GPU --
so the test pins the partition, the view CSR, the X block layout and the output reassembly
against the unsharded oracle, bit-for-bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        import oracle
        import paper_conf_asplos_0001lslwlgslllw23_b200 as ug
        from paper_conf_asplos_0001lslwlgslllw23_b200.shard import ShardedOperator, x_block
        import ugdata

        c = ugdata.CONFIGS["C2"]
        src, dst = ugdata.graph("C2")
        V, E = c.V, len(src)
        g = ug.Graph(V, src, dst, host_only=True)
        sh = ShardedOperator(g, world, rank)
        F = 16
        X = ugdata.values(V, F, 5, 1)
        w = ugdata.values(E, 1, 5, 2, role="edge")
        X_local = x_block(torch.from_numpy(X), V, world, rank)
        X_full = sh.gather_x(X_local)
        assert torch.equal(X_full[:V], torch.from_numpy(X))

        # the rank's view, as the C ABI exposes it
        rp, col, eid = sh.view.csr()
        Vl = sh.local_rows
        assert len(rp) == Vl + 1 and rp[-1] == sh.e1 - sh.e0
        dst_local = np.repeat(np.arange(Vl, dtype=np.int32), np.diff(rp))
        Xg = X_full[:V].numpy()
        outs = {}
        for name, eo, b, bt in (("copy_u_sum", "copy_lhs", None, None),
                                ("u_mul_e_max", "mul", sh.edge_slice(torch.from_numpy(w)).numpy(), "e"),
                                ("u_sub_v_mean", "sub", sh.dst_slice(torch.from_numpy(X)).numpy(), "v")):
            gop = name.rsplit("_", 1)[1]
            Yl = oracle.op(V, col, dst_local, eo, gop, A=Xg, a_type="u", B=b, b_type=bt, c_type="v", F=F,
                           rows=np.arange(Vl, dtype=np.int64))
            Y = sh.gather_rows(torch.from_numpy(Yl))
            full = oracle.op(V, src, dst, eo, gop, A=X, a_type="u",
                             B={"e": w, "v": X, None: None}[bt], b_type=bt, c_type="v", F=F)
            outs[name] = bool(np.array_equal(Y.numpy().view(np.uint32), full.view(np.uint32)))
        q.put((rank, outs, int(sh.r0), int(sh.r1)))
        dist.destroy_process_group()
    except Exception as e:  # surface failures to the parent
        q.put((rank, repr(e), -1, -1))
        raise


@pytest.mark.parametrize("world", [2])
def test_sharded_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    res.sort()
    ranges = []
    for rank, outs, r0, r1 in res:
        assert isinstance(outs, dict), outs
        assert all(outs.values()), outs
        ranges.append((r0, r1))
    assert ranges[0][0] == 0 and ranges[-1][1] == 19717
    assert all(ranges[i][1] == ranges[i + 1][0] for i in range(world - 1))
