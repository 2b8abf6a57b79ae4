"""Re-entrancy of the fused single-launch kernels across streams, and CUDA-graph capture of the
very first call on a graph (include/ug.h: "re-entrant across streams").

ug_gat_attention and ug_op_run_arg merge the partials of split rows by a last-arriver count per
(split row, column tile).  The counters are scratch of each call (allocated and zeroed on the
call's stream), so calls on different streams over ONE graph must not disturb each other: many
calls are queued alternately on two streams with different inputs, and every output must equal
the same call run alone (bit-exact: the merge order is the chunk order, fixed per call).
"""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def _hub_graph():
    V = 3001                          # a hub of in-degree 3000 (split into ~94 chunks) + a ring
    s = np.concatenate([np.arange(1, V), np.arange(V)]).astype(np.int32)
    d = np.concatenate([np.zeros(V - 1, np.int32), (np.arange(V) + 1) % V]).astype(np.int32)
    return V, s, d


def test_gat_two_streams_one_graph():
    V, src, dst = _hub_graph()
    g = ug.Graph(V, src, dst)
    H, F, n = 4, 64, 6
    ins = []
    for i in range(n):
        ins.append(tuple(torch.from_numpy(ugdata.values(V, w, 100 + i, t)).cuda() for w, t in ((H, 1), (H, 2), (F, 3))))
    alone = []
    for el, er, z in ins:
        alone.append(ug.gat_attention(g, el, er, z, H, 0.2).clone())
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    outs = [torch.empty(V, F, device="cuda") for _ in range(n)]
    for rep in range(5):
        for i, (el, er, z) in enumerate(ins):
            with torch.cuda.stream(streams[i % 2]):
                ug.gat_attention(g, el, er, z, H, 0.2, out=outs[i])
        torch.cuda.synchronize()
        for i in range(n):
            assert torch.equal(outs[i].view(torch.int32), alone[i].view(torch.int32)), (rep, i)
    # and the single call agrees with the definition
    el, er, z = (t.cpu().numpy() for t in ins[0])
    ref, _, bnd = oracle.gat(V, src, dst, el, er, z, H, 0.2, bound=True)
    err = np.abs(alone[0].cpu().numpy().astype(np.float64) - ref)
    assert (err <= 1e-5 * bnd).all()


def test_arg_two_streams_one_graph():
    V, src, dst = _hub_graph()
    g = ug.Graph(V, src, dst)
    F, n = 40, 6
    Xs = [torch.from_numpy(ugdata.values(V, F, 200 + i, 1)).cuda() for i in range(n)]
    alone = []
    for X in Xs:
        C = torch.empty(V, F, device="cuda")
        a = ug.op_run_arg(g, "copy_lhs", "max", A=X, a_type="u", C=C, F=F)
        alone.append((C.clone(), a.clone()))
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    Cs = [torch.empty(V, F, device="cuda") for _ in range(n)]
    As = [torch.empty(V, F, device="cuda", dtype=torch.int32) for _ in range(n)]
    for rep in range(5):
        for i, X in enumerate(Xs):
            with torch.cuda.stream(streams[i % 2]):
                ug.op_run_arg(g, "copy_lhs", "max", A=X, a_type="u", C=Cs[i], F=F, arg=As[i])
        torch.cuda.synchronize()
        for i in range(n):
            assert torch.equal(Cs[i].view(torch.int32), alone[i][0].view(torch.int32)), (rep, i)
            assert torch.equal(As[i], alone[i][1]), (rep, i)
    C0, a0 = oracle.op_arg(V, src, dst, "copy_lhs", "max", A=Xs[0].cpu().numpy(), a_type="u", F=F)
    np.testing.assert_array_equal(alone[0][0].cpu().numpy().view(np.uint32), C0.view(np.uint32))
    np.testing.assert_array_equal(alone[0][1].cpu().numpy(), a0)


@pytest.mark.parametrize("sched", ["SV_G64", "SV_G64_F32_A1", "SV_G64_M1"])
def test_first_call_inside_cuda_graph_capture(sched):
    """The one-time SV plan upload of a fresh graph may happen during stream capture."""
    V, src, dst = _hub_graph()
    order = np.argsort(dst, kind="stable")
    src, dst = src[order], dst[order]
    g = ug.Graph(V, src, dst)               # no call on g yet: its plans are not built
    F = 64
    X = torch.from_numpy(ugdata.values(V, F, 5, 1, mode="int", k=4)).cuda()
    Y = torch.empty(V, F, device="cuda")
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg, stream=side):
        ug.op_run(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v", schedule=sched)
    Y.fill_(float("nan"))
    cg.replay()
    torch.cuda.synchronize()
    ref = oracle.op(V, src, dst, "copy_lhs", "sum", A=X.cpu().numpy(), a_type="u", c_type="v", F=F)
    np.testing.assert_array_equal(Y.cpu().numpy().view(np.uint32), ref.view(np.uint32))
